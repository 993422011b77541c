"""C4 loop time under shared-memory placement variants (allocation bitmap
early / late).  With DTS_PROFILE=1 also cycles per scan by phase.  Needs a B200."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import gen  # noqa: E402
import paper_conf_ipps_gonthiermt22_b200 as dts  # noqa: E402

NAMES = ["pop", "argmax", "plan", "serve_loads", "luf", "evict", "seg_load", "other"]
for cfg in (sys.argv[1:] or ["C4a", "C4b"]):
    inst = gen.config_instances(cfg)[0]
    for late in ("0", "1"):
        os.environ["DTS_AL_LATE"] = late
        g = dts.schedule(inst)
        print(f"{cfg} al_late={late}: loop {g.loop_ms:.1f} ms, {g.n_scans} scans ({g.n_fallback2} fb2, "
              f"{g.n_fallback_first} fbf), {1e6 * g.loop_ms / g.n_served:.0f} ns/dec", flush=True)
        if os.environ.get("DTS_PROFILE") == "1":
            print("   cycles/scan: " + ", ".join(
                f"{n}={c / max(g.n_scans, 1):.0f}" for n, c in zip(NAMES, g.prof_cycles)), flush=True)

"""Per-phase cycle split of the C4 decision loops, cluster mode vs one CTA
(DTS_F_NOCLUSTER), profiling build.  python tools/prof_c4.py [C4a C4b]"""
import os
os.environ.setdefault("DTS_PROFILE", "1")
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import gen  # noqa: E402
import paper_conf_ipps_gonthiermt22_b200 as dts  # noqa: E402

NAMES = ["pop", "argmax", "plan", "serve_loads", "luf", "evict", "seg_load", "other"]
for cfg in (sys.argv[1:] or ["C4a", "C4b"]):
    inst = gen.config_instances(cfg)[0]
    for name, fl in (("cluster", 1), ("one-CTA", 1 | dts.DTS_F_NOCLUSTER)):
        g = dts.schedule(inst, flags=fl)
        print(f"{cfg} {name}: loop {g.loop_ms:.0f} ms, {g.n_scans} scans, "
              f"{1e6 * g.loop_ms / max(g.n_served, 1):.0f} ns/dec; cycles/scan: " +
              ", ".join(f"{n}={c / max(g.n_scans, 1):.0f}" for n, c in zip(NAMES, g.prof_cycles)), flush=True)

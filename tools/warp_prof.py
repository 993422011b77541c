"""Per-phase cycle split of the one-warp loop (dts_warp.cu probes, profiling
build lib/libdts_prof.so).  Needs a B200.   python tools/warp_prof.py"""
import os
os.environ.setdefault("DTS_PROFILE", "1")
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import gen  # noqa: E402
import paper_conf_ipps_gonthiermt22_b200 as dts  # noqa: E402

NAMES = ["pop", "argmax", "planwalk", "planpool", "fallback", "luf", "evict", "seg_ev", "load", "finish",
         "build", "assemble"]
for inst in (gen.sweep_instance(160, 4, 1), gen.sweep_instance(160, 4, 7), gen.sweep_instance(160, 128, 8), gen.config_instances("C2")[19],
             gen.matmul2d(10, M=6, K=1)):
    dts.schedule(inst)
    g = dts.schedule(inst)
    cyc = g.prof_cycles
    tot = sum(cyc[:12])
    print(f"{inst.name}: loop {g.loop_ms:.3f} ms, {g.n_served} dec, {g.n_scans} scans ({g.n_fallback2} fb2, "
          f"{g.n_fallback_first} fbf), {g.n_loads} loads, {g.n_evictions} evictions, "
          f"{1e6 * g.loop_ms / max(g.n_served, 1):.0f} ns/dec; cycles total {tot / 1e6:.2f} M")
    print("   cycles/scan: " + ", ".join(f"{n}={c / max(g.n_scans, 1):.0f}" for n, c in zip(NAMES, cyc)))

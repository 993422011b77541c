"""Per-scan cycle split of the decision loop (dts_result_view.prof_cycles) for
a few instances.  python tools/prof_fine.py [c2|c3|c5long]...  Needs a B200."""
import os
os.environ.setdefault("DTS_PROFILE", "1")
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import gen  # noqa: E402
import paper_conf_ipps_gonthiermt22_b200 as dts  # noqa: E402

NAMES = ["pop", "argmax", "plan", "serve_loads", "luf", "evict", "seg_load", "other", "bw0", "bd",
         "nb", "np", "x1", "x2", "x3", "x4"]
SETS = {"c2": [gen.config_instances("C2")[19], gen.config_instances("C2")[18]],
        "c3": [gen.config_instances("C3")[0]],
        "c5long": [gen.sweep_instance(160, 4, 7), gen.sweep_instance(160, 4, 1)]}
for name in (sys.argv[1:] or ["c2", "c3"]):
    for inst in SETS[name]:
        dts.schedule(inst)
        g = dts.schedule(inst)
        print(inst.name, f"K={inst.K} loop {g.loop_ms:.2f} ms scans {g.n_scans} (fb2 {g.n_fallback2}) "
              f"loads {g.n_loads} ev {g.n_evictions} served {g.n_served}")
        print("  per scan: " + ", ".join(f"{n}={c / max(g.n_scans, 1):.0f}" for n, c in zip(NAMES, g.prof_cycles)))

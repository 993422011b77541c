import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import gen
import paper_conf_ipps_gonthiermt22_b200 as dts
NAMES = ["pop", "argmax", "plan", "serve_loads", "luf", "evict", "seg_load", "other", "bw0", "bd", "nb", "np", "x1", "x2", "x3", "x4"]
for inst in [gen.config_instances("C2")[19], gen.config_instances("C2")[18], gen.config_instances("C3")[0]]:
    dts.schedule(inst)
    g = dts.schedule(inst)
    print(inst.name, f"loop {g.loop_ms:.2f} ms scans {g.n_scans} loads {g.n_loads} ev {g.n_evictions} served {g.n_served}")
    print("  per scan: " + ", ".join(f"{n}={c / max(g.n_scans, 1):.0f}" for n, c in zip(NAMES, g.prof_cycles)))

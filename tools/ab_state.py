"""A/B of the two state modes of the decision loop: row-derived (default for
rows <= 3 inputs) vs the packed per-(GPU, task) words (DTS_F_PACKED).
Prints loop time per instance and, with DTS_PROFILE=1, cycles per scan by
phase.  python tools/ab_state.py [c2 c3 c5long c4]...  Needs a B200."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import gen  # noqa: E402
import paper_conf_ipps_gonthiermt22_b200 as dts  # noqa: E402

NAMES = ["pop", "argmax", "plan", "serve_loads", "luf", "evict", "seg_load", "other"]
SETS = {"c2": lambda: [gen.config_instances("C2")[19], gen.config_instances("C2")[18]],
        "c3": lambda: [gen.config_instances("C3")[0]],
        "c5long": lambda: [gen.sweep_instance(160, 4, 7), gen.sweep_instance(160, 6, 6),
                           gen.sweep_instance(160, 4, 1)],
        "c4": lambda: [gen.config_instances("C4a")[0], gen.config_instances("C4b")[0]]}
prof = os.environ.get("DTS_PROFILE") == "1"
for name in (sys.argv[1:] or ["c2", "c3", "c5long"]):
    for inst in SETS[name]():
        for label, fl in (("packed", dts.DTS_F_FALLBACK2 | dts.DTS_F_PACKED), ("row", dts.DTS_F_FALLBACK2)):
            dts.schedule(inst, flags=fl)
            g = dts.schedule(inst, flags=fl)
            print(f"{inst.name:28s} {label:6s} loop {g.loop_ms:9.2f} ms  {g.n_served} dec  {g.n_scans} scans  "
                  f"{1e6 * g.loop_ms / max(g.n_served, 1):.0f} ns/dec", flush=True)
            if prof:
                print("   cycles/scan: " + ", ".join(
                    f"{n}={c / max(g.n_scans, 1):.0f}" for n, c in zip(NAMES, g.prof_cycles)), flush=True)

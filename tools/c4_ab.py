"""A/B of the C4 decision loops (production build): cluster mode vs one CTA
(DTS_F_NOCLUSTER), loop kernel time from the library's events, best of 2.
python tools/c4_ab.py [C4a C4b]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import gen  # noqa: E402
import paper_conf_ipps_gonthiermt22_b200 as dts  # noqa: E402

for cfg in (sys.argv[1:] or ["C4a", "C4b"]):
    inst = gen.config_instances(cfg)[0]
    h = dts.create(inst)
    for name, fl in (("cluster", 1), ("one-CTA", 1 | dts.DTS_F_NOCLUSTER)):
        ms = []
        for _ in range(2):
            dts.dts_run(h, dts.DTS_POLICY_DARTS_LUF, dts.dts_run_opts_default(flags=fl))
            ms.append(dts.dts_run_times(h)[0])
        g = dts.dts_result(h)
        print(f"{cfg} {name}: loop {min(ms):.0f} ms ({ms}), {g.n_served} decisions, "
              f"{1e6 * min(ms) / g.n_served:.0f} ns/decision", flush=True)

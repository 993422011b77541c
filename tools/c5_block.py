"""C5 sweep loop time vs the CTA-size policy (default split launches vs one
launch with forced 64 / 128 / 256-thread CTAs).  Needs a B200."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import gen  # noqa: E402
import paper_conf_ipps_gonthiermt22_b200 as dts  # noqa: E402

hs = [dts.create(i) for i in gen.config_instances("C5")]
for b in (128, 96, 160, 128):
    t = []
    for _ in range(3):
        dts.dts_sweep_run(hs, dts.DTS_POLICY_DARTS_LUF, dts.dts_run_opts_default(block_threads=b))
        t.append(dts.dts_run_times(hs[0])[0])
    print(f"block {b}: loop {min(t):.1f} ms ({[round(x, 1) for x in t]})", flush=True)

"""C4 loop time per CTA size (DTS_BLOCK read at each run).  Needs a B200."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import gen  # noqa: E402
import paper_conf_ipps_gonthiermt22_b200 as dts  # noqa: E402

for cfg in (sys.argv[1:] or ["C4a", "C4b"]):
    h = dts.create(gen.config_instances(cfg)[0])
    for b in (512, 384, 256):
        o = dts.dts_run_opts_default(block_threads=b)
        dts.dts_run(h, dts.DTS_POLICY_DARTS_LUF, o)
        g = dts.dts_result(h)
        print(f"{cfg} block {b}: loop {g.loop_ms:.1f} ms", flush=True)

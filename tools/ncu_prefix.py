"""One C4 decision-loop launch stopped after a prefix of served requests (a
short launch of the same kernel for ncu --set full, which replays it ~40
times): python tools/ncu_prefix.py C4b 20000."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import gen  # noqa: E402
import paper_conf_ipps_gonthiermt22_b200 as dts  # noqa: E402

cfg, n = sys.argv[1], int(sys.argv[2])
g = dts.schedule(gen.config_instances(cfg)[0], max_served=n)
print(cfg, g.n_served, "served", g.n_scans, "scans", f"{g.loop_ms:.1f} ms")

"""Run one named instance once (after a warm-up) for profiling: python tools/one_instance.py C2 19"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import gen  # noqa: E402
import paper_conf_ipps_gonthiermt22_b200 as dts  # noqa: E402

cfg, idx = sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else 0
inst = gen.config_instances(cfg)[idx]
dts.schedule(inst)
r = dts.schedule(inst)
print(inst.name, r.n_served, r.loop_ms)

"""Run one instance twice through the C ABI (for ncu captures of the loop kernel).
usage: python tools/one.py C2big|C3|C4a|C4b|C5big"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import gen  # noqa: E402
import paper_conf_ipps_gonthiermt22_b200 as dts  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "C2big"
inst = {"C2big": lambda: gen.matmul2d(100, M=35, K=4), "C3": lambda: gen.config_instances("C3")[0],
        "C4a": lambda: gen.config_instances("C4a")[0], "C4b": lambda: gen.config_instances("C4b")[0],
        "C5big": lambda: gen.matmul2d(160, M=16, K=8)}[name]()
for _ in range(2):
    g = dts.schedule(inst)
print(name, g.n_served, g.n_scans, g.loop_ms)

"""Run one instance through the default (one-warp) path a few times (for ncu)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import gen  # noqa: E402
import paper_conf_ipps_gonthiermt22_b200 as dts  # noqa: E402

N, M, K = (int(x) for x in (sys.argv[1:4] if len(sys.argv) > 3 else (160, 4, 1)))
inst = gen.sweep_instance(N, M, K)
for _ in range(3):
    r = dts.schedule(inst)
print(inst.name, r.loop_ms, "ms")

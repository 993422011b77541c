"""Loop-kernel device time of a few instances (production build unless DTS_PROFILE=1)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import gen  # noqa: E402
import paper_conf_ipps_gonthiermt22_b200 as dts  # noqa: E402

insts = [gen.config_instances("C2")[19], gen.config_instances("C3")[0], gen.sweep_instance(160, 4, 7)]
print("lib", os.path.basename(dts.LIB_PATH))
for inst in insts:
    dts.schedule(inst)
    ms = min(dts.schedule(inst).loop_ms for _ in range(3))
    print(f"  {inst.name}: loop {ms:.2f} ms")

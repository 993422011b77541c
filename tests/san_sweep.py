"""compute-sanitizer target: a batched sweep over a sample of C5 instances
(every 64th), checked against the oracle.  Needs a B200."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
import gen  # noqa: E402
import oracle  # noqa: E402
import paper_conf_ipps_gonthiermt22_b200 as dts  # noqa: E402
from parity import assert_parity  # noqa: E402

insts = [i for i in gen.config_instances("C5")[::64] if i.m <= 4000]
gs = dts.schedule_batch(insts)
for inst, g in zip(insts, gs):
    assert_parity(g, oracle.run(inst))
print("sweep sample ok:", len(insts), "instances")

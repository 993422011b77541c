"""The shape of the paper's transfer-volume experiment (Fig. 4, PAPER.md:976-1060,
1213-1230) on the simulator: 2D matmul N = 5..140 (working set 140..7,875 MiB),
memory = 500 MiB (M = 35 data), K = 1 and 2 simulated GPUs; bytes loaded by
DARTS+LUF, DARTS+LRU and EAGER+LRU, each policy's whole sweep in one batched
launch on the B200.  Prints a table (MiB loaded) and writes JSON.

usage: python tools/transfer_volumes.py [out.json]"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import gen  # noqa: E402
import paper_conf_ipps_gonthiermt22_b200 as dts  # noqa: E402

NS = [5, 10, 20, 30, 40, 50, 60, 70, 80, 90, 100, 110, 120, 130, 140]
POL = {"DARTS+LUF": dts.DTS_POLICY_DARTS_LUF, "DARTS+LRU": dts.DTS_POLICY_DARTS_LRU,
       "EAGER+LRU": dts.DTS_POLICY_EAGER_LRU}
out = {"N": NS, "working_set_MiB": [2 * N * gen.DATUM_2D_BYTES / 2 ** 20 for N in NS], "runs": {}}
for K in (1, 2):
    insts = [gen.matmul2d(N, M=35, K=K) for N in NS]
    for name, pol in POL.items():
        t0 = time.perf_counter()
        rs = dts.schedule_batch(insts, policy=pol)
        dt = time.perf_counter() - t0
        out["runs"][f"{name} K={K}"] = {"MiB_loaded": [r.bytes_loaded / 2 ** 20 for r in rs],
                                        "makespan_s": [r.makespan_s for r in rs],
                                        "decisions": sum(r.n_served for r in rs), "wall_s": dt}
print("MiB loaded (2D matmul, M = 35 data = 500 MiB per simulated GPU)")
print("N     WS_MiB " + " ".join(f"{k:>16s}" for k in out["runs"]))
for i, N in enumerate(NS):
    print(f"{N:<5d} {out['working_set_MiB'][i]:7.0f} " +
          " ".join(f"{v['MiB_loaded'][i]:16.0f}" for v in out["runs"].values()))
if len(sys.argv) > 1:
    json.dump(out, open(sys.argv[1], "w"), indent=1)

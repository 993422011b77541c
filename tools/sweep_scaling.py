"""Estimate C5 multi-GPU scaling on ONE B200: run each rank's LPT shard of the
4,096-instance sweep (as bench.py --gpus G would) one after another and
report the per-rank device times; max over ranks = the G-GPU step time.
Also times every instance alone to show the longest chain.  Needs a B200."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_ipps_gonthiermt22_b200 as dts  # noqa: E402
from paper_conf_ipps_gonthiermt22_b200.shard import instance_cost, shard  # noqa: E402

params = gen.sweep_params()
insts = [gen.sweep_instance(*p) for p in params]
hs = [dts.create(i) for i in insts]
st = torch.cuda.current_stream()
o = dts.dts_run_opts_default(cuda_stream=st.cuda_stream)
for h in hs:
    dts.dts_instance_upload(h, 0, st.cuda_stream)
torch.cuda.synchronize()


def timed(sub, reps=3):
    best = 1e30
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(st)
        dts.dts_sweep_run(sub, dts.DTS_POLICY_DARTS_LUF, o)
        b.record(st)
        b.synchronize()
        best = min(best, a.elapsed_time(b))
    return best


full = timed(hs)
print(f"G=1: {full:.1f} ms", flush=True)
# longest single chains
big = sorted(range(len(insts)), key=lambda i: -insts[i].m)[:64]
solo = sorted(((timed([hs[i]], 1), params[i]) for i in big), reverse=True)[:8]
print("longest single instances (ms, (N, M, K)):", [(round(t, 1), p) for t, p in solo], flush=True)
costs_env = os.environ.get("COST", "default")
for G in (2, 4, 8):
    costs = [instance_cost(N * N, 2 * N) for (N, M, K) in params]
    ts = [timed([hs[i] for i in shard(costs, r, G)], 2) for r in range(G)]
    print(f"G={G}: per-rank ms {[round(t, 1) for t in ts]} -> step {max(ts):.1f} ms, "
          f"scaling {full / max(ts):.2f}x", flush=True)

"""Small instances through the one-warp loop, for compute-sanitizer
(memcheck / racecheck / synccheck): each schedule is compared with the
per-CTA loop's (DTS_F_CTA) digest.  Needs a B200:
    compute-sanitizer --tool racecheck python tools/san_warp.py"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
import numpy as np  # noqa: E402

import gen  # noqa: E402
import paper_conf_ipps_gonthiermt22_b200 as dts  # noqa: E402
from digest import digest  # noqa: E402


def dg(r):
    return digest(r.serve_gpu, r.serve_task, r.task_start, r.task_end, r.events)


rng = np.random.default_rng(1)
rows = [tuple(int(x) for x in rng.choice(40, 1 + (i % 3 > 0), replace=False)) for i in range(400)]
ptr = np.zeros(len(rows) + 1, np.int64)
ptr[1:] = np.cumsum([len(r) for r in rows])
mixed = gen.Instance("mixed", ptr, np.asarray([d for r in rows for d in r], np.int32),
                     np.full(40, 1000, np.uint64), None, 9, 5 * 1000, 3)
insts = [gen.fig1(), gen.matmul2d(10, M=6, K=1), gen.matmul2d(30, M=5, K=4),
         gen.matmul2d(20, M=8, K=7, order="random", seed=2), gen.matmul2d(12, M=3, K=32), mixed]
ok = True
for inst in insts:
    g = dts.schedule(inst)
    c = dts.schedule(inst, flags=dts.DTS_F_FALLBACK2 | dts.DTS_F_CTA)
    same = g.loop_kind == dts.LOOP_WARP and dg(g) == dg(c) and g.n_served == inst.m
    ok &= same
    print(inst.name, "same" if same else "DIFFERENT", flush=True)
gs = dts.schedule_batch(insts[1:])
for inst, g in zip(insts[1:], gs):
    ok &= g.n_served == inst.m and g.loop_kind == dts.LOOP_WARP
print("ALL OK" if ok else "MISMATCH")

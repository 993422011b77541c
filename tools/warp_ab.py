"""One-warp loop (dts_warp.cu, default for small 2-input instances) against
the per-CTA loop (DTS_F_CTA): same schedule (digests) and loop-kernel device
time, single instances and batched launches.  Needs a B200.
    python tools/warp_ab.py [reps]"""
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
import gen  # noqa: E402
import paper_conf_ipps_gonthiermt22_b200 as dts  # noqa: E402
from digest import digest  # noqa: E402

reps = int(sys.argv[1]) if len(sys.argv) > 1 else 5
F = dts.DTS_F_FALLBACK2
CTA = F | dts.DTS_F_CTA


def dg(r):
    return digest(r.serve_gpu, r.serve_task, r.task_start, r.task_end, r.events)


def one(inst):
    out = {}
    for name, fl in (("warp", F), ("cta", CTA)):
        rs = [dts.schedule(inst, flags=fl) for _ in range(reps)]
        out[name] = (statistics.median(r.loop_ms for r in rs), dg(rs[0]), rs[0].n_served)
    same = out["warp"][1] == out["cta"][1]
    print(f"{inst.name:28s} warp {out['warp'][0]:9.3f} ms  cta {out['cta'][0]:9.3f} ms  "
          f"x{out['cta'][0] / max(out['warp'][0], 1e-9):5.2f}  same={same}  served={out['warp'][2]}", flush=True)
    return same


def batch(name, insts):
    hs = [dts.create(i) for i in insts]
    res = {}
    for nm, fl in (("warp", F), ("cta", CTA)):
        o = dts.dts_run_opts_default(flags=fl)
        ts = []
        for _ in range(reps):
            dts.dts_sweep_run(hs, dts.DTS_POLICY_DARTS_LUF, o)
            dts.dts_fetch_results(hs)
            ts.append(dts.dts_run_times(hs[0])[0])
        res[nm] = (statistics.median(ts), [dg(dts.dts_result(h)) for h in hs])
    same = sum(a == b for a, b in zip(res["warp"][1], res["cta"][1]))
    print(f"{name:28s} warp {res['warp'][0]:9.3f} ms  cta {res['cta'][0]:9.3f} ms  "
          f"x{res['cta'][0] / max(res['warp'][0], 1e-9):5.2f}  same={same}/{len(insts)}", flush=True)
    return same == len(insts)


ok = True
for inst in (gen.fig1(), gen.matmul2d(10, M=6, K=1), gen.config_instances("C2")[19],
             gen.config_instances("C2")[9], gen.sweep_instance(160, 4, 1), gen.sweep_instance(160, 4, 7),
             gen.sweep_instance(160, 128, 8), gen.matmul2d(30, M=8, K=3, order="random"),
             gen.random_shared(3000, 256, 2, M=12, K=5, seed=7)):
    ok &= one(inst)
ok &= batch("C2 batch", gen.config_instances("C2"))
gc = __import__("gc")
gc.disable()
ok &= batch("C5 sweep", gen.config_instances("C5"))
print("ALL SAME" if ok else "MISMATCH")

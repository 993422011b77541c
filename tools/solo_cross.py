"""Lone instances: one-warp loop vs per-CTA loop (DTS_F_CTA), loop ms (best of 2),
to place the lone-instance threshold (dts_api.cu WARP_SOLO_MAX).
    python tools/solo_cross.py LIB.so   (a build with a high threshold)"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ipps_gonthiermt22_b200 as dts  # noqa: E402

dts.load_library(sys.argv[1])
import gen  # noqa: E402

F = dts.DTS_F_FALLBACK2
cases = [gen.matmul3d(40, M=142, K=4), gen.matmul3d(30, M=60, K=8), gen.matmul2d(250, M=35, K=4),
         gen.random_shared(60000, 2048, 2, M=64, K=4, seed=1), gen.random_shared(60000, 4096, 2, M=64, K=4, seed=1),
         gen.random_shared(60000, 8192, 2, M=128, K=4, seed=1), gen.random_shared(60000, 4096, 2, M=512, K=8, seed=2)]
for inst in cases:
    out = []
    for fl in (F, F | dts.DTS_F_CTA):
        h = dts.create(inst)
        o = dts.dts_run_opts_default(flags=fl)
        t, kind = [], 0
        for _ in range(2):
            dts.dts_run(h, dts.DTS_POLICY_DARTS_LUF, o)
            r = dts.dts_result(h)
            t.append(r.loop_ms)
            kind = r.loop_kind
        out.append(f"kind{kind} {min(t):8.2f} ms")
    print(f"{inst.name:32s} n={inst.n:6d} " + "  ".join(out), flush=True)

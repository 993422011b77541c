"""Write golden per-instance digests for the whole config-5 sweep (4,096 2D
instances) by running the plain CPU oracle on every
instance, in parallel over the host cores.

Calls only oracle/ and gen/ (never the CUDA path).  Output:
tests/golden/digests_C5.json: for each instance (in gen.sweep_params() order)
its (N, M, K), the counters and the SHA-256 of tests/digest.py over the
full schedule (service order, task start/end, every trace event).

usage: python tests/golden/make_c5_digests.py [n_procs]
"""
import json
import multiprocessing as mp
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))

import gen  # noqa: E402
import oracle  # noqa: E402
from digest import digest  # noqa: E402


def one(i):
    N, M, K = gen.sweep_params()[i]
    inst = gen.sweep_instance(N, M, K)
    r = oracle.run(inst)
    return dict(i=i, N=N, M=M, K=K, m=inst.m, n_served=r.n_served, n_loads=r.n_loads,
                n_evictions=r.n_evictions, n_scans=r.n_scans, n_fallback2=r.n_fallback2,
                n_fallback_first=r.n_fallback_first, n_idle_requests=r.n_idle_requests,
                bytes_loaded=int(r.bytes_loaded), makespan=int(r.makespan),
                sha256=digest(r.serve_gpu, r.serve_task, r.task_start, r.task_end, r.events))


def main(nproc):
    oracle.build()
    params = gen.sweep_params()
    # longest instances first so the pool's tail is short
    order = sorted(range(len(params)), key=lambda i: -params[i][0] ** 3)
    t0 = time.time()
    with mp.Pool(nproc) as pool:
        rows = pool.map(one, order, chunksize=1)
    rows.sort(key=lambda r: r["i"])
    out = dict(config="C5", n_instances=len(rows), W=0, flags=oracle.F_FALLBACK2,
               bus_bps=oracle.DEFAULT_BUS_BPS, oracle_seconds=round(time.time() - t0, 1),
               processes=nproc, produced_by="tests/golden/make_c5_digests.py (oracle/ only)",
               instances=rows)
    path = os.path.join(os.path.dirname(os.path.abspath(__file__)), "digests_C5.json")
    with open(path, "w") as f:
        json.dump(out, f, separators=(",", ":"))
    print("wrote", path, len(rows), "instances in", out["oracle_seconds"], "s")


if __name__ == "__main__":
    main(int(sys.argv[1]) if len(sys.argv) > 1 else os.cpu_count())

"""Write golden full-run digests for the large configs (C4a, C4b) by running
the plain CPU oracle once, offline (hours of CPU: O(E) per scan).

Calls only oracle/ and gen/ (never the CUDA path).  Output:
tests/golden/digests_<cfg>.json with the counters and a SHA-256 over the
canonical little-endian bytes of (serve_gpu int32, serve_task int32,
task_start int64, task_end int64, events 32-byte records) -- see
tests/digest.py.

usage: python tests/golden/make_digests.py C4a [C4b ...]
"""
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))

import gen  # noqa: E402
import oracle  # noqa: E402
from digest import digest  # noqa: E402


def main(cfgs):
    for cfg in cfgs:
        inst = gen.config_instances(cfg)[0]
        t0 = time.time()
        r = oracle.run(inst)
        dt = time.time() - t0
        out = dict(config=cfg, instance=inst.name, m=inst.m, n=inst.n, E=inst.E, K=inst.K,
                   mem_capacity=int(inst.mem_capacity), W=0, flags=oracle.F_FALLBACK2,
                   bus_bps=oracle.DEFAULT_BUS_BPS,
                   n_served=r.n_served, n_loads=r.n_loads, n_evictions=r.n_evictions,
                   n_scans=r.n_scans, n_fallback2=r.n_fallback2,
                   n_fallback_first=r.n_fallback_first, n_idle_requests=r.n_idle_requests,
                   bytes_loaded=int(r.bytes_loaded), makespan=int(r.makespan),
                   sha256=digest(r.serve_gpu, r.serve_task, r.task_start, r.task_end, r.events),
                   oracle_seconds=round(dt, 1),
                   produced_by="tests/golden/make_digests.py (oracle/ only)")
        path = os.path.join(os.path.dirname(os.path.abspath(__file__)), f"digests_{cfg}.json")
        with open(path, "w") as f:
            json.dump(out, f, indent=1)
        print(cfg, out, flush=True)


if __name__ == "__main__":
    main(sys.argv[1:] or ["C4a", "C4b"])

"""Multi-GPU plumbing for independent instances.

Instances of a sweep are independent problems (BASELINE config 5), so they
shard across ranks -- one process per B200 -- with no data-path collective:
each rank schedules its own shard in one batched launch (``dts_sweep_run``).
The only collectives are the timing ones ``bench.py`` needs (a barrier and the
max / sum over ranks), done here through ``torch.distributed`` (NCCL on the
GPU box, gloo in the CPU tests).

Assignment is LPT (longest processing time first): instances sorted by a
cost estimate, each given to the currently least-loaded rank.  The cost of a
2D instance with N x N tasks is ~N^3 (N^2 decisions, scans over segments of
~N tasks), which is what makes the last few N=160 instances dominate the
sweep; LPT keeps the per-rank maxima within one instance of each other.
"""
from __future__ import annotations

import heapq
from typing import Sequence


def instance_cost(m: int, n: int) -> float:
    """Cost estimate of one instance: decisions x segment length ~ m * (E / n)."""
    return float(m) * max(1.0, 2.0 * m / max(n, 1))


def lpt_assign(costs: Sequence[float], world: int) -> list[list[int]]:
    """Deterministic LPT: ties broken by lower index, then lower rank.
    Returns, per rank, the ascending list of instance indices it owns."""
    if world < 1:
        raise ValueError("world must be >= 1")
    order = sorted(range(len(costs)), key=lambda i: (-float(costs[i]), i))
    heap = [(0.0, r) for r in range(world)]
    heapq.heapify(heap)
    out: list[list[int]] = [[] for _ in range(world)]
    for i in order:
        load, r = heapq.heappop(heap)
        out[r].append(i)
        heapq.heappush(heap, (load + float(costs[i]), r))
    return [sorted(x) for x in out]


def shard(costs: Sequence[float], rank: int, world: int) -> list[int]:
    """Indices owned by ``rank``."""
    return lpt_assign(costs, world)[rank]


def reduce_over_ranks(values, op: str = "max", device=None):
    """All-reduce a list of floats over the default process group (identity
    without one).  Returns a list of Python floats."""
    import torch
    import torch.distributed as dist

    vals = [float(v) for v in values]
    if not (dist.is_available() and dist.is_initialized()) or dist.get_world_size() == 1:
        return vals
    t = torch.tensor(vals, dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX if op == "max" else dist.ReduceOp.SUM)
    return [float(x) for x in t.tolist()]

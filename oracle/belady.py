"""Belady replay and brute force.  TEST INFRASTRUCTURE ONLY (see oracle/__init__).

* :func:`belady_loads` -- for a FIXED schedule sigma (a task order per GPU),
  the number of loads when every GPU evicts by Belady's rule, "always evict
  the data whose next usage is the furthest in the future", which is optimal
  for a fixed sigma with unit-size data (§III).  Loads are
  counted as in Obj. 2: #Loads_k = sum_i |D(T_sigma(k,i)) \\ L(k,i-1)|
  (PAPER.md:402-407), with V(k,i) disjoint from D(T_sigma(k,i)) (397-399)
  and |L(k,i)| <= M (377).
* :func:`brute_force_opt` -- min over every sigma of belady_loads, for tiny
  instances (the problem is NP-complete, Thm. 1).
"""
from __future__ import annotations

import itertools


def belady_loads_one(order, dsets, M):
    """Loads on one GPU processing tasks ``order`` with memory M (unit sizes)."""
    mem = set()
    loads = 0
    for i, T in enumerate(order):
        need = dsets[T]
        assert len(need) <= M
        for D in sorted(need - mem):
            if len(mem) >= M:
                # candidates: resident data not needed by the current task
                def next_use(x):
                    for j in range(i + 1, len(order)):
                        if x in dsets[order[j]]:
                            return j
                    return len(order) + 1  # never used again: furthest
                cands = sorted(mem - need)
                far = max(next_use(x) for x in cands)
                victim = min(x for x in cands if next_use(x) == far)
                mem.remove(victim)
            mem.add(D)
            loads += 1
    return loads


def belady_loads(orders, dsets, M):
    return sum(belady_loads_one(list(o), dsets, M) for o in orders)


def brute_force_opt(dsets, M, K=1):
    """Minimum total loads over all schedules (partition into K ordered
    sequences) of the tasks; exponential, tiny inputs only."""
    m = len(dsets)
    best = None
    tasks = list(range(m))
    if K == 1:
        for perm in itertools.permutations(tasks):
            v = belady_loads_one(list(perm), dsets, M)
            best = v if best is None or v < best else best
        return best
    for assign in itertools.product(range(K), repeat=m):
        groups = [[t for t in tasks if assign[t] == k] for k in range(K)]
        tot = 0
        for g in groups:
            tot += min(belady_loads_one(list(p), dsets, M) for p in itertools.permutations(g)) if g else 0
            if best is not None and tot >= best:
                break
        best = tot if best is None or tot < best else best
    return best


def dsets_of(inst):
    """D(T) as Python sets (de-duplicated: D(T) is a set)."""
    tp, td = inst.task_ptr, inst.task_data
    return [frozenset(int(x) for x in td[tp[t]:tp[t + 1]]) for t in range(inst.m)]

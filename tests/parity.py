"""Element-by-element comparison of a libdts result with the oracle's
(bit-exact: the schedule is integer, R22)."""
import numpy as np


def assert_parity(g, o, complete=True):
    assert g.n_served == o.n_served, (g.n_served, o.n_served)
    assert np.array_equal(g.serve_gpu, o.serve_gpu), "service order: GPU differs"
    assert np.array_equal(g.serve_task, o.serve_task), "service order: task differs"
    for f in ("t", "t_end", "gpu", "data", "task", "op"):
        assert len(g.events) == len(o.events), (len(g.events), len(o.events))
        if not np.array_equal(g.events[f], o.events[f]):
            i = int(np.nonzero(g.events[f] != o.events[f])[0][0])
            raise AssertionError(f"event {i} field {f}: gpu {g.events[i]} oracle {o.events[i]}")
    assert np.array_equal(g.task_start, o.task_start)
    assert np.array_equal(g.task_end, o.task_end)
    assert g.bytes_loaded == o.bytes_loaded
    assert g.n_loads == o.n_loads and g.n_evictions == o.n_evictions
    assert g.makespan == o.makespan
    assert g.n_scans == o.n_scans
    assert g.n_fallback2 == o.n_fallback2 and g.n_fallback_first == o.n_fallback_first
    assert g.n_belady == o.n_belady
    # SURVEY §8(d) byte-model counters (measurement)
    assert g.sum_avail_at_scans == o.sum_avail_at_scans, (g.sum_avail_at_scans, o.sum_avail_at_scans)
    assert g.n_allocations == o.n_allocations, (g.n_allocations, o.n_allocations)
    if complete:
        assert g.n_idle_requests == o.n_idle_requests
    # per-GPU orders (a8) agree with the service sequence
    for k, ok in enumerate(o.orders()):
        assert np.array_equal(g.orders()[k], ok)


def deg_sum_of_events(inst, events):
    """sum of deg(D) (#tasks using D, rows de-duplicated) over LOAD and EVICT
    events -- the oracle-side value of dts_result's sum_deg_loads_evictions."""
    deg = np.zeros(inst.n, np.int64)
    for T in range(inst.m):
        for D in set(inst.task_data[inst.task_ptr[T]:inst.task_ptr[T + 1]].tolist()):
            deg[D] += 1
    return int(deg[np.asarray(events["data"], dtype=np.int64)].sum()) if len(events) else 0

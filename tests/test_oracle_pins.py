"""Pins of the CPU oracle against what the paper and the mathematics fix
(DESIGN.md "Oracle pins").  CPU only."""
import json
import os
import random

import numpy as np
import pytest

import gen
import oracle
from oracle.belady import belady_loads, belady_loads_one, brute_force_opt, dsets_of
from conftest import GOLDEN
from validate import validate


def _golden(name):
    with open(os.path.join(GOLDEN, name)) as f:
        return json.load(f)


def _unit(inst):
    """Unit sizes / unit task time: capacity in data counts, delta = tau = 1 tick
    with a 1e9 B/s bus."""
    M = int(inst.mem_capacity // int(inst.data_size[0]))
    return inst.with_(data_size=np.ones(inst.n, dtype=np.uint64), mem_capacity=M,
                      default_task_ns=1, task_ns=None)


def _check(inst, r, W=0, bus=oracle.DEFAULT_BUS_BPS, complete=True):
    return validate(inst, r.serve_gpu, r.serve_task, r.events, r.task_start, r.task_end,
                    W=W, bus_bps=bus, complete=complete)


# ---------------------------------------------------------------- P1 (paper)
def test_p1_fig1_paper_schedule_belady_11_loads():
    g = _golden("fig1_paper_schedule.json")
    ds = dsets_of(gen.fig1())
    per = [belady_loads_one(o, ds, g["M"]) for o in g["sigma"]]
    assert per == g["per_gpu_loads_by_hand"]
    assert sum(per) == g["paper_total_loads"] == 11


# ---------------------------------------------------------------- P2 (hand)
@pytest.mark.parametrize("flags", [oracle.F_FALLBACK2, 0])
def test_p2_fig1_darts_luf_hand_trace(flags):
    g = _golden("fig1_darts_luf_hand.json")
    inst = gen.fig1(K=g["K"], M=g["M"])
    r = oracle.run(inst, bus_bps=10 ** 9, flags=flags)
    assert [list(map(int, o)) for o in r.orders()] == g["orders"]
    loads = [[int(e["gpu"]), int(e["data"])] for e in r.events if e["op"] == 0]
    evs = [[int(e["gpu"]), int(e["data"])] for e in r.events if e["op"] == 1]
    assert loads == g["loads_in_event_order"]
    assert evs == g["evictions_in_event_order"]
    assert (r.n_loads, r.n_evictions, r.makespan) == (g["n_loads"], g["n_evictions"], g["makespan"])
    if flags:
        assert r.n_fallback2 == g["n_fallback2"]
    _check(inst, r, bus=10 ** 9)


# ---------------------------------------------------------------- H0
def test_h0_2d_N2_equals_brute_force():
    g = _golden("h0_2d_N2.json")
    inst = _unit(gen.matmul2d(2, M=2, K=1))
    r = oracle.run(inst, bus_bps=10 ** 9)
    assert list(map(int, r.orders()[0])) == g["order"]
    assert r.n_loads == g["n_loads"]
    assert brute_force_opt(dsets_of(inst), 2) == g["brute_force_opt"] == r.n_loads


# ---------------------------------------------------------------- P3 / H1
def test_p3_h1_config1_hand_trace():
    g = _golden("h1_2d_N10_M6.json")
    inst = _unit(gen.matmul2d(10, M=6, K=1))
    r = oracle.run(inst, bus_bps=10 ** 9)
    name = lambda d: f"A{d}" if d < 10 else f"B{d - 10}"
    seq = [name(int(e["data"])) for e in r.events if e["op"] == 0]
    assert seq == g["load_sequence"]
    assert r.n_loads == g["n_loads"] and r.n_evictions == g["n_evictions"]
    assert r.n_scans == g["n_scans"] and r.n_fallback2 == g["n_fallback2"]
    assert r.n_fallback_first == g["n_fallback_first"]
    assert r.n_idle_requests == g["n_idle_requests"]
    assert r.n_served - r.n_scans == g["pops"]
    assert r.makespan == 43 * 1 + 100 * 1
    _check(inst, r, bus=10 ** 9)


def test_config1_real_units_makespan_closed_form():
    """K=1, W=0: the GPU requests at the end of its task and the bus is idle
    then, so makespan = sum of transfer times + sum of task times exactly."""
    inst = gen.config_instances("C1")[0]
    r = oracle.run(inst)
    d = -(-gen.DATUM_2D_BYTES * 10 ** 9 // gen.DEFAULT_BUS_BPS)
    assert d == 1_228_800
    assert r.n_loads == 43
    assert r.makespan == 43 * d + 100 * gen.TAU_2D_NS
    assert r.bytes_loaded == 43 * gen.DATUM_2D_BYTES
    _check(inst, r)


# ---------------------------------------------------------------- P4
def _small_instances():
    out = [gen.matmul2d(6, M=4, K=1), gen.matmul2d(7, M=5, K=2, order="random", seed=3),
           gen.matmul3d(4, M=6, K=2), gen.matmul3d(3, M=9, K=3, with_c=True),
           gen.cholesky(6, M=5, K=2), gen.random_shared(300, 64, 3, M=8, K=3, seed=7),
           gen.random_shared(200, 32, 2, M=3, K=1, seed=9),
           gen.matmul2d(20, M=6, K=4, keep_frac=0.1, seed=5)]
    return out


@pytest.mark.parametrize("idx", range(8))
def test_p4_ample_memory_each_datum_loaded_once(idx):
    inst = _small_instances()[idx]
    big = inst.with_(mem_capacity=int(inst.data_size.sum()))
    r = oracle.run(big)
    _check(big, r)
    used = np.unique(inst.task_data)
    loads = [(int(e["gpu"]), int(e["data"])) for e in r.events if e["op"] == 0]
    assert len(loads) == len(set(loads)), "a GPU loaded a datum twice with ample memory"
    assert r.n_evictions == 0
    if inst.K == 1:
        assert r.n_loads == len(used)
        assert r.bytes_loaded == int(inst.data_size[used].sum())


@pytest.mark.parametrize("N", [3, 5, 8])
def test_p4_2d_memory_2N_loads_2N(N):
    inst = gen.matmul2d(N, M=2 * N, K=1)
    r = oracle.run(inst)
    assert r.n_loads == 2 * N and r.n_evictions == 0


# ---------------------------------------------------------------- P5
@pytest.mark.parametrize("idx", range(8))
@pytest.mark.parametrize("W", [0, 1])
def test_p5_invariants(idx, W):
    inst = _small_instances()[idx]
    if W == 1:
        inst = inst.with_(mem_capacity=int(inst.mem_capacity) + int(inst.data_size.max()) * 3)
    r = oracle.run(inst, W=W)
    chk = _check(inst, r, W=W)
    assert chk["n_loads"] == r.n_loads and chk["n_evictions"] == r.n_evictions
    assert chk["bytes_loaded"] == r.bytes_loaded and chk["makespan"] == r.makespan
    assert r.n_belady == 0  # unreachable with the capacity check (reading R7)
    assert r.n_wakes == 0   # unreachable (reading R18)
    assert sum(len(o) for o in r.orders()) == inst.m


def test_p5_heterogeneous_sizes():
    rng = np.random.default_rng(4)
    base = gen.random_shared(400, 64, 3, M=8, K=3, seed=11)
    sizes = rng.integers(1, 5, size=64).astype(np.uint64) * 1_000_000
    inst = base.with_(data_size=sizes, mem_capacity=int(sizes.max()) * 7)
    r = oracle.run(inst)
    _check(inst, r)


def test_prefix_is_prefix_of_full_run():
    inst = gen.random_shared(500, 64, 3, M=6, K=4, seed=5)
    full = oracle.run(inst)
    pre = oracle.run(inst, max_served=123)
    assert pre.n_served == 123
    assert np.array_equal(pre.serve_task, full.serve_task[:123])
    assert np.array_equal(pre.events, full.events[:len(pre.events)])
    _check(inst, pre, complete=False)


# ---------------------------------------------------------------- P6
def _tiny(seed, m, n, K, M):
    rnd = random.Random(seed)
    rows = [sorted(rnd.sample(range(n), rnd.choice([1, 2, 2, 3]))) for _ in range(m)]
    tp = np.zeros(m + 1, np.int64)
    tp[1:] = np.cumsum([len(r) for r in rows])
    td = np.array([d for r in rows for d in r], np.int32)
    return gen.Instance(f"tiny{seed}", tp, td, np.ones(n, np.uint64), None, 1, M, K)


@pytest.mark.parametrize("seed", range(12))
def test_p6_brute_force_k1(seed):
    inst = _tiny(seed, m=6 + seed % 2, n=5, K=1, M=3)
    r = oracle.run(inst, bus_bps=10 ** 9)
    ds = dsets_of(inst)
    opt = brute_force_opt(ds, 3)
    bel = belady_loads(r.orders(), ds, 3)
    assert opt <= bel <= r.n_loads


@pytest.mark.parametrize("seed", range(6))
def test_p6_brute_force_k2(seed):
    inst = _tiny(100 + seed, m=5, n=5, K=2, M=3)
    r = oracle.run(inst, bus_bps=10 ** 9)
    ds = dsets_of(inst)
    opt = brute_force_opt(ds, 3, K=2)
    bel = belady_loads(r.orders(), ds, 3)
    assert opt <= bel <= r.n_loads
    _check(inst, r, bus=10 ** 9)


# ---------------------------------------------------------------- OPTI (§V-F)
@pytest.mark.parametrize("N", [4, 6])
def test_opti_2d_ample_memory_column_major(N):
    """Hand-derived: 2D N x N, K=1, M=2N (everything fits).  The first request
    falls back to T(0,0) (loads A0, B0).  Then A_i frees only T(i,0) and B_j
    frees T(0,j) and the rows already loaded, so OPTI (first datum with
    n(D) >= 1 in id order, reading R28) loads A1..A_{N-1}
    one by one, then each B_j plans the whole column j: column-major order,
    2N loads.  Plain DARTS prefers B1 (n=2) after A1 and differs."""
    inst = _unit(gen.matmul2d(N, M=2 * N, K=1))
    r = oracle.run(inst, bus_bps=10 ** 9, flags=oracle.F_FALLBACK2 | oracle.F_OPTI)
    col_major = [i * N + j for j in range(N) for i in range(N)]
    assert list(map(int, r.orders()[0])) == col_major
    assert r.n_loads == 2 * N and r.n_evictions == 0
    plain = oracle.run(inst, bus_bps=10 ** 9)
    assert list(map(int, plain.orders()[0])) != col_major
    _check(inst, r, bus=10 ** 9)


@pytest.mark.parametrize("idx", range(8))
def test_opti_invariants(idx):
    inst = _small_instances()[idx]
    r = oracle.run(inst, flags=oracle.F_FALLBACK2 | oracle.F_OPTI)
    chk = _check(inst, r)
    assert chk["n_loads"] == r.n_loads and chk["makespan"] == r.makespan


# ---------------------------------------------------- EAGER / LRU (§8(f)2)
def lru_replay_one(order, dsets, M):
    """Independent LRU replay of a FIXED per-GPU order with unit sizes: before
    each task, load its missing inputs in ascending id, evicting the resident
    datum (not an input of the task) whose last use is the oldest, lowest id on
    ties; then every input is 'used' by this task.  Returns (loads, evicts)
    as lists of data ids in event order."""
    mem, last, loads, evicts = set(), {}, [], []
    for idx, T in enumerate(order):
        need = dsets[T]
        for D in sorted(need - mem):
            if len(mem) >= M:
                cand = sorted(mem - need)
                V = min(cand, key=lambda x: (last[x], x))
                mem.remove(V)
                evicts.append(V)
            mem.add(D)
            loads.append(D)
        for D in need:
            last[D] = idx
    return loads, evicts


def test_eager_lru_2d_hand_trace():
    """Hand trace (EAGER = shared FIFO in submission order, PAPER.md:819-825;
    LRU eviction): 2D N=3, K=1, M=4.  Loads A0 B0 B1 B2 A1 B1 A2 B1, evictions
    B1 A0 B1 A1 (ids: A_i = i, B_j = 3 + j); 8 loads."""
    inst = _unit(gen.matmul2d(3, M=4, K=1))
    r = oracle.run(inst, bus_bps=10 ** 9, flags=oracle.POLICY_FLAGS["eager_lru"])
    assert list(map(int, r.orders()[0])) == list(range(9))
    assert [int(e["data"]) for e in r.events if e["op"] == 0] == [0, 3, 4, 5, 1, 4, 2, 4]
    assert [int(e["data"]) for e in r.events if e["op"] == 1] == [4, 0, 4, 1]
    assert r.n_scans == 0
    _check(inst, r, bus=10 ** 9)


@pytest.mark.parametrize("policy", ["eager_lru", "darts_lru"])
@pytest.mark.parametrize("idx", range(8))
def test_lru_matches_independent_replay(policy, idx):
    """Every GPU's load/evict sequence equals an independent LRU replay of its
    task order (LRU decisions depend only on the GPU's own order)."""
    inst = _unit(_small_instances()[idx])
    M = int(inst.mem_capacity)
    r = oracle.run(inst, bus_bps=10 ** 9, flags=oracle.F_FALLBACK2 | oracle.POLICY_FLAGS[policy])
    _check(inst, r, bus=10 ** 9)
    ds = dsets_of(inst)
    for k, order in enumerate(r.orders()):
        loads, evicts = lru_replay_one(list(map(int, order)), ds, M)
        ev = r.events[r.events["gpu"] == k]
        assert [int(e["data"]) for e in ev if e["op"] == 0] == loads
        assert [int(e["data"]) for e in ev if e["op"] == 1] == evicts
    if policy == "eager_lru" and inst.K == 1:
        assert list(map(int, r.orders()[0])) == list(range(inst.m))


def test_eager_lru_collapse_when_one_matrix_fits():
    """EAGER+LRU collapses once only one matrix fits:
    2D N=20 with M = N+1 reloads far more than DARTS+LUF."""
    inst = gen.matmul2d(20, M=21, K=1)
    eager = oracle.run(inst, flags=oracle.POLICY_FLAGS["eager_lru"])
    darts = oracle.run(inst)
    assert eager.n_loads > 2 * darts.n_loads


# ------------------------------------------------ F1: the 3inputs fallback (§V-E)
def f1_instance(g=None):
    """The hand-traced fallback instance of tests/golden/f1_fallback2_hand.json
    (unit sizes, delta = tau = 1 tick)."""
    g = g or _golden("f1_fallback2_hand.json")
    rows = g["rows"]
    tp = np.zeros(len(rows) + 1, np.int64)
    tp[1:] = np.cumsum([len(r) for r in rows])
    td = np.array([d for r in rows for d in r], np.int32)
    return gen.Instance("f1_fallback2", tp, td, np.ones(g["data"], np.uint64), None, g["tau"],
                        g["M"], g["K"])


def test_f1_fallback2_hand_trace():
    """Pins the 3inputs scoring (readings R6, R24): n2
    credits both missing inputs, the key is (n2, u, -id), the task is the
    lowest-id one with D2 and one other input missing.  Each plausible
    mistake changes the first pick (see the golden's derivation)."""
    g = _golden("f1_fallback2_hand.json")
    inst = f1_instance(g)
    r = oracle.run(inst, bus_bps=10 ** 9)
    assert list(map(int, r.orders()[0])) == g["order"]
    ev = [["L" if e["op"] == 0 else "E", int(e["data"]), int(e["task"]), int(e["t"]), int(e["t_end"])]
          for e in r.events]
    assert ev == g["events"]
    assert (r.n_loads, r.n_evictions, r.n_scans) == (g["n_loads"], g["n_evictions"], g["n_scans"])
    assert (r.n_fallback2, r.n_fallback_first) == (g["n_fallback2"], g["n_fallback_first"])
    assert r.n_idle_requests == g["n_idle_requests"] and r.n_served - r.n_scans == g["pops"]
    assert r.makespan == g["makespan"]
    _check(inst, r, bus=10 ** 9)
    c = g["measurement_counters"]
    rc = oracle.run(inst, bus_bps=10 ** 9, flags=oracle.F_FALLBACK2 | oracle.F_COUNT_DEG)
    assert (rc.n_allocations, rc.sum_avail_at_scans, rc.sum_deg) == (
        c["n_allocations"], c["sum_avail_at_scans"], c["sum_deg"])


def test_measurement_counters_closed_form():
    """SURVEY §8(d) counters: K=1 with ample memory loads every used datum
    once and never evicts or returns a task, so n_allocations = m and the
    deg(D) sum over loads = E (each edge counted once)."""
    for inst in _small_instances():
        big = inst.with_(mem_capacity=int(inst.data_size.sum()), K=1)
        r = oracle.run(big, flags=oracle.F_FALLBACK2 | oracle.F_COUNT_DEG)
        E = sum(len(set(big.task_data[big.task_ptr[T]:big.task_ptr[T + 1]])) for T in range(big.m))
        assert r.n_allocations == big.m and r.sum_deg == E and r.n_evictions == 0
        assert r.sum_avail_at_scans >= big.m  # the first scan alone sees all m


def test_f1_fallback_off_takes_lowest_id_task():
    """Without the 3inputs variant the first request falls to Alg. 5 l.13
    (R5): the lowest-id available task, T0, which does not use D2 = D5."""
    inst = f1_instance()
    r = oracle.run(inst, bus_bps=10 ** 9, flags=0)
    assert int(r.serve_task[0]) == 0 and r.n_fallback_first >= 1 and r.n_fallback2 == 0
    _check(inst, r, bus=10 ** 9)


@pytest.mark.parametrize("seed", range(40))
def test_r18_idle_wake_never_fires(seed):
    """Reading R18 (wake idle GPUs when LUF returns planned tasks, Alg. 6
    l.8) is unreachable: a return happens while serving the first task of a
    plan made at the same request out of a non-empty pool, an idle GPU saw
    an empty pool, and the pool refills only by returns.  Checked here on
    small random instances with K = 2..4 and tight memory (many returns)."""
    K = 2 + seed % 3
    inst = _tiny(2000 + seed, m=40 + seed, n=12, K=K, M=3 + seed % 2)
    for W in (0, 1):
        if W and inst.mem_capacity < 6:
            continue
        for flags in (oracle.F_FALLBACK2, 0, oracle.F_FALLBACK2 | oracle.F_OPTI):
            r = oracle.run(inst, W=W, bus_bps=10 ** 9, flags=flags)
            assert r.n_wakes == 0 and r.n_served == inst.m


# -------------------------------------- Belady (Alg. 6 l.6-7) and W >= 2 (R29)
def belady_instance(g):
    if "rows" in g:
        rows = g["rows"]
        tp = np.zeros(len(rows) + 1, np.int64)
        tp[1:] = np.cumsum([len(r) for r in rows])
        td = np.array([d for r in rows for d in r], np.int32)
        return gen.Instance("belady_rows", tp, td, np.ones(g["data"], np.uint64), None, g["tau"],
                            g["M"], g["K"])
    return _unit(gen.matmul2d(g["N"], M=g["M"], K=g["K"]))


BELADY_GOLDENS = ["belady_w1_2d_N2.json", "belady_w2_2d_N3.json", "belady_w1_disjoint.json"]


@pytest.mark.parametrize("name", BELADY_GOLDENS)
def test_belady_hand_traces(name):
    """Alg. 6's Belady branch made reachable by a
    capacity of max(1, W) tasks' inputs, and a W+1-task taskBuffer
    (PAPER.md:742-746), under reading R29 -- hand traces."""
    g = _golden(name)
    inst = belady_instance(g)
    r = oracle.run(inst, W=g["W"], bus_bps=10 ** 9)
    assert list(map(int, r.orders()[0])) == g["order"]
    ev = [["L" if e["op"] == 0 else "E", int(e["data"]), int(e["task"]), int(e["t"]), int(e["t_end"])]
          for e in r.events]
    assert ev == g["events"]
    assert (r.n_loads, r.n_evictions, r.n_belady) == (g["n_loads"], g["n_evictions"], g["n_belady"])
    assert (r.n_scans, r.n_fallback2, r.n_idle_requests) == (g["n_scans"], g["n_fallback2"], g["n_idle_requests"])
    assert r.makespan == g["makespan"]
    _check(inst, r, W=g["W"], bus=10 ** 9)


@pytest.mark.parametrize("W", [1, 2, 3, 5])
@pytest.mark.parametrize("idx", range(8))
def test_w_tight_capacity_invariants(W, idx):
    """Any W with the capacity the library accepts for DARTS+LUF (max(1, W)
    tasks' inputs): the schedule passes the independent validator (which
    checks R29's Belady conditions and request times), every task runs."""
    inst = _small_instances()[idx]
    row = max(int(inst.data_size[inst.task_data[inst.task_ptr[T]:inst.task_ptr[T + 1]]].sum())
              for T in range(inst.m))
    inst = inst.with_(mem_capacity=max(1, W) * row)
    r = oracle.run(inst, W=W)
    chk = _check(inst, r, W=W)
    assert chk["n_loads"] == r.n_loads and chk["makespan"] == r.makespan
    assert r.n_served == inst.m and r.n_wakes == 0


def test_belady_fires_on_random_tight_instances():
    """The branch is reachable: with W = 2 and 2 tasks' inputs of memory the
    random shared-input instances trigger it."""
    tot = 0
    for seed in range(6):
        inst = gen.random_shared(400, 64, 3, M=6, K=2, seed=seed)
        r = oracle.run(inst, W=2)
        _check(inst, r, W=2)
        tot += r.n_belady
    assert tot > 0

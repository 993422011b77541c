"""GPU parity: libdts (sm_100a kernels, through the C ABI) vs the plain CPU
oracle, element by element, bit-exact (integer schedule, reading R22).
Needs a B200."""
import json
import os

import numpy as np
import pytest

import gen
import oracle
import paper_conf_ipps_gonthiermt22_b200 as dts
from conftest import GOLDEN
from digest import digest
from parity import assert_parity, deg_sum_of_events
from validate import validate

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module", autouse=True)
def _need_gpu():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    dts.load_library()


def _unit(inst):
    M = int(inst.mem_capacity // int(inst.data_size[0]))
    return inst.with_(data_size=np.ones(inst.n, dtype=np.uint64), mem_capacity=M,
                      default_task_ns=1, task_ns=None)


def _both(inst, bus=oracle.DEFAULT_BUS_BPS, block=0, smem=0, flags=1, max_served=-1):
    g = dts.schedule(inst, bus_bps=bus, block_threads=block, smem_budget=smem, flags=flags,
                     max_served=max_served)
    o = oracle.run(inst, bus_bps=bus, flags=flags, max_served=max_served)
    if inst.E <= 200_000:
        assert g.sum_deg_loads_evictions == deg_sum_of_events(inst, o.events)
    return g, o


# ------------------------------------------------------------ hand traces
@pytest.mark.parametrize("flags", [1, 0])
def test_fig1(flags):
    inst = gen.fig1()
    g, o = _both(inst, bus=10 ** 9, flags=flags)
    assert_parity(g, o)
    gold = json.load(open(os.path.join(GOLDEN, "fig1_darts_luf_hand.json")))
    assert [list(map(int, x)) for x in g.orders()] == gold["orders"]
    assert g.n_loads == 11 and g.makespan == 12


def test_f1_fallback2_hand():
    """The hand-traced 3inputs instance (tests/golden/f1_fallback2_hand.json)."""
    from test_oracle_pins import f1_instance
    gold = json.load(open(os.path.join(GOLDEN, "f1_fallback2_hand.json")))
    for flags in (1, 0):
        g, o = _both(f1_instance(), bus=10 ** 9, flags=flags)
        assert_parity(g, o)
    g, _ = _both(f1_instance(), bus=10 ** 9)
    assert list(map(int, g.orders()[0])) == gold["order"] and g.n_fallback2 == gold["n_fallback2"]


def test_h1_config1_unit():
    inst = _unit(gen.matmul2d(10, M=6, K=1))
    g, o = _both(inst, bus=10 ** 9)
    assert_parity(g, o)
    assert g.n_loads == 43 and g.n_evictions == 37


def test_config1():
    inst = gen.config_instances("C1")[0]
    g, o = _both(inst)
    assert_parity(g, o)


@pytest.mark.parametrize("idx", range(20))
def test_config2(idx):
    inst = gen.config_instances("C2")[idx]
    g, o = _both(inst)
    assert_parity(g, o)


# ------------------------------------------------------------ varied shapes
def _shapes():
    return [gen.matmul2d(6, M=4, K=1), gen.matmul2d(7, M=5, K=2, order="random", seed=3),
            gen.matmul3d(4, M=6, K=2), gen.matmul3d(3, M=9, K=3, with_c=True),
            gen.cholesky(6, M=5, K=2), gen.random_shared(300, 64, 3, M=8, K=3, seed=7),
            gen.random_shared(200, 32, 2, M=3, K=1, seed=9),
            gen.matmul2d(20, M=6, K=4, keep_frac=0.1, seed=5),
            gen.random_shared(5000, 256, 3, M=20, K=8, seed=1),
            gen.cholesky(20, M=30, K=4), gen.matmul3d(10, M=25, K=4),
            gen.matmul2d(30, M=12, K=3, order="random", seed=8)]


# block sizes x shared-memory placements: 0 = all that fits, -1 = every array
# in its global home, 3000 B = a partial placement
@pytest.mark.parametrize("idx", range(12))
@pytest.mark.parametrize("block,smem", [(0, 0), (32, 0), (512, 0), (64, -1), (128, 3000)])
def test_shapes_block_and_placement(idx, block, smem):
    inst = _shapes()[idx]
    g, o = _both(inst, block=block, smem=smem)
    assert_parity(g, o)
    validate(inst, g.serve_gpu, g.serve_task, g.events, g.task_start, g.task_end)


def test_heterogeneous_sizes():
    rng = np.random.default_rng(4)
    base = gen.random_shared(2000, 128, 3, M=8, K=4, seed=11)
    sizes = rng.integers(1, 5, size=128).astype(np.uint64) * 1_000_000
    inst = base.with_(data_size=sizes, mem_capacity=int(sizes.max()) * 9)
    for smem in (0, -1):
        g, o = _both(inst, smem=smem)
        assert_parity(g, o)


def test_ample_memory_and_duplicates():
    inst = gen.random_shared(3000, 128, 3, M=8, K=2, seed=2)
    # duplicated ids inside rows are removed (D(T) is a set, R27)
    td = inst.task_data.copy()
    td[1::3] = td[0::3]
    dup = inst.with_(task_data=td)
    g, o = _both(dup)
    assert_parity(g, o)
    big = inst.with_(mem_capacity=int(inst.data_size.sum()))
    g, o = _both(big, smem=-1)
    assert_parity(g, o)
    assert g.n_evictions == 0


def test_empty_and_degenerate():
    # tasks without inputs, an unused datum, a single task
    tp = np.array([0, 0, 2, 2, 3], np.int64)
    td = np.array([0, 2, 2], np.int32)
    inst = gen.Instance("degen", tp, td, np.ones(4, np.uint64), None, 5, 2, 2)
    g, o = _both(inst, bus=10 ** 9)
    assert_parity(g, o)
    one = gen.Instance("one", np.array([0, 1], np.int64), np.array([0], np.int32),
                       np.ones(1, np.uint64), None, 3, 1, 3)
    g, o = _both(one, bus=10 ** 9)
    assert_parity(g, o)
    empty = gen.Instance("empty", np.array([0], np.int64), np.zeros(0, np.int32),
                         np.ones(2, np.uint64), None, 3, 1, 2)
    g = dts.schedule(empty)
    assert g.n_served == 0 and len(g.events) == 0


def test_ragged_tail_sizes():
    # m not a multiple of 4 (uint4 scan tail) and of the CTA size
    for m in (1, 2, 3, 5, 4097, 10001):
        inst = gen.random_shared(m, 64, 3, M=6, K=2, seed=m)
        g, o = _both(inst, block=64)
        assert_parity(g, o)


@pytest.mark.parametrize("idx", [0, 2, 4, 5, 6, 8, 9])
@pytest.mark.parametrize("smem", [0, -1])
def test_verify_incremental_scores(idx, smem):
    """P9: at every scan the incremental scores n_k(D), n2_k(D), u(D) and every
    task's (cnt, xor) equal a from-scratch recomputation."""
    inst = _shapes()[idx]
    g = dts.schedule(inst, flags=dts.DTS_F_FALLBACK2 | dts.DTS_F_VERIFY, smem_budget=smem)
    assert g.n_verify_err == 0
    assert_parity(g, oracle.run(inst))


def test_long_rows():
    """Tasks with more than 3 inputs (the plan entry caches 3) and 1-input tasks."""
    rng = np.random.default_rng(12)
    rows = [sorted(rng.choice(40, size=int(rng.integers(1, 7)), replace=False)) for _ in range(600)]
    tp = np.zeros(601, np.int64)
    tp[1:] = np.cumsum([len(r) for r in rows])
    td = np.concatenate(rows).astype(np.int32)
    inst = gen.Instance("long", tp, td, np.ones(40, np.uint64), None, 3, 9, 3)
    for smem in (0, -1):
        g = dts.schedule(inst, bus_bps=10 ** 9, smem_budget=smem,
                         flags=dts.DTS_F_FALLBACK2 | dts.DTS_F_VERIFY)
        assert g.n_verify_err == 0
        assert_parity(g, oracle.run(inst, bus_bps=10 ** 9))


# ------------------------------------------------------------ state modes
# Rows of <= 3 inputs run in the row-derived state mode by default (no
# per-(GPU, task) words: missing inputs read off the row and the residency
# bitmaps); DTS_F_PACKED keeps the packed cnt:7|xor:24 words.  Both must give
# the oracle's schedule.
PACKED = dts.DTS_F_FALLBACK2 | dts.DTS_F_PACKED


@pytest.mark.parametrize("idx", range(12))
@pytest.mark.parametrize("smem", [0, -1])
def test_packed_state_mode_shapes(idx, smem):
    inst = _shapes()[idx]
    g = dts.schedule(inst, flags=PACKED | dts.DTS_F_VERIFY, smem_budget=smem)
    assert g.n_verify_err == 0
    assert_parity(g, oracle.run(inst))


@pytest.mark.parametrize("name", ["darts_luf", "darts_lru", "eager_lru"])
@pytest.mark.parametrize("W", [0, 1])
def test_packed_state_mode_policies(name, W):
    pol, of = {"darts_luf": (dts.DTS_POLICY_DARTS_LUF, 0),
               "darts_lru": (dts.DTS_POLICY_DARTS_LRU, oracle.F_LRU),
               "eager_lru": (dts.DTS_POLICY_EAGER_LRU, oracle.F_EAGER | oracle.F_LRU)}[name]
    for inst in (_shapes()[5], _shapes()[9]):
        o = oracle.run(inst, W=W, flags=oracle.F_FALLBACK2 | of)
        assert_parity(dts.schedule(inst, policy=pol, W=W, flags=PACKED), o)
        assert_parity(dts.schedule(inst, policy=pol, W=W), o)  # row-derived


def test_packed_state_mode_config3_and_4_prefix():
    inst = gen.config_instances("C3")[0]
    assert_parity(dts.schedule(inst, flags=PACKED), oracle.run(inst))
    for cfg in ("C4a", "C4b"):
        inst = gen.config_instances(cfg)[0]
        g = dts.schedule(inst, flags=PACKED, max_served=800)
        assert_parity(g, oracle.run(inst, max_served=800), complete=False)


def test_row_derived_verify_partial_placement():
    """P9 in the row-derived mode with the allocation bitmap in HBM / partly placed."""
    for inst in (_shapes()[8], _shapes()[10]):
        for smem in (-1, 2000, 0):
            g = dts.schedule(inst, flags=dts.DTS_F_FALLBACK2 | dts.DTS_F_VERIFY, smem_budget=smem)
            assert g.n_verify_err == 0
            assert_parity(g, oracle.run(inst))


def test_row_derived_mode_row_widths():
    """Row-derived mode on rows of 1, 2 and 3 inputs and on ids wider than 32
    bits in total (T and two other inputs), each against the oracle with P9
    on, state placed and unplaced, alone and batched."""
    cases = [gen.matmul2d(40, M=10, K=3),                       # rows of 2
             gen.random_shared(5000, 256, 3, M=20, K=4, seed=21),  # rows of 3
             gen.random_shared(6000, 1024, 3, M=24, K=2, seed=22),  # 13 + 2 * 11 id bits
             gen.cholesky(12, M=20, K=3)]                        # rows of 1..3 inputs
    for inst in cases:
        o = oracle.run(inst)
        for smem in (0, -1):
            g = dts.schedule(inst, flags=dts.DTS_F_FALLBACK2 | dts.DTS_F_VERIFY, smem_budget=smem)
            assert g.n_verify_err == 0
            assert_parity(g, o)
    gs = dts.schedule_batch(cases)
    for inst, g in zip(cases, gs):
        assert_parity(g, oracle.run(inst))


# ------------------------------------------------------------ larger configs
def test_config3():
    inst = gen.config_instances("C3")[0]
    g, o = _both(inst)
    assert_parity(g, o)


@pytest.mark.parametrize("cfg", ["C4a", "C4b"])
def test_config4_prefix(cfg):
    """Full-size config 4 in the bench's launch configuration, prefix of 1,500
    served requests (the plain oracle costs O(E) per scan)."""
    inst = gen.config_instances(cfg)[0]
    g, o = _both(inst, max_served=1500)
    assert_parity(g, o, complete=False)


@pytest.mark.parametrize("cfg", ["C4a", "C4b"])
def test_config4_full_digest(cfg):
    path = os.path.join(GOLDEN, f"digests_{cfg}.json")
    if not os.path.exists(path):
        pytest.skip("golden digest not produced yet (tests/golden/make_digests.py)")
    gold = json.load(open(path))
    inst = gen.config_instances(cfg)[0]
    g = dts.schedule(inst)
    for k in ("n_served", "n_loads", "n_evictions", "n_scans", "n_fallback2", "n_fallback_first",
              "bytes_loaded", "makespan"):
        assert getattr(g, k) == gold[k], k
    assert digest(g.serve_gpu, g.serve_task, g.task_start, g.task_end, g.events) == gold["sha256"]


# ------------------------------------------------------------ batched sweep
def test_sweep_batch_config2():
    """dts_sweep_run (one CTA per instance, one launch) on the 20 C2 instances:
    every instance bit-exact against its own oracle run."""
    insts = gen.config_instances("C2")
    gs = dts.schedule_batch(insts)
    for inst, g in zip(insts, gs):
        assert_parity(g, oracle.run(inst))


def test_sweep_batch_mixed_shapes():
    insts = _shapes() + [gen.fig1(), _unit(gen.matmul2d(10, M=6, K=1))]
    buses = [oracle.DEFAULT_BUS_BPS] * len(insts)
    gs = dts.schedule_batch(insts)
    for inst, g, b in zip(insts, gs, buses):
        assert_parity(g, oracle.run(inst, bus_bps=b))


def test_sweep_sample_config5():
    """A seeded sample of the 4,096 config-5 instances in one batched launch."""
    params = gen.sweep_params()
    rng = np.random.default_rng(5)
    pick = sorted(rng.choice(len(params), size=48, replace=False))
    insts = [gen.sweep_instance(*params[i]) for i in pick]
    gs = dts.schedule_batch(insts)
    for inst, g in zip(insts, gs):
        assert_parity(g, oracle.run(inst))


def test_sweep_split_launch():
    """A batch of >= 2 x 148 instances runs as one launch of <= 128-thread CTAs
    (several chains per SM, longest first): every instance must match the
    oracle, including the wide-segment ones."""
    params = [(N, M, K) for N in (5, 10, 15) for M in (4, 6, 8, 12) for K in (1, 2, 3, 4)]
    insts = [gen.sweep_instance(*p) for p in params] * 7                 # 336 narrow
    insts += [gen.sweep_instance(70, 8, 2), gen.sweep_instance(140, 12, 3)]  # 128 (B), 256 (A)
    gs = dts.schedule_batch(insts)
    cache = {}
    for inst, g in zip(insts, gs):
        if inst.name not in cache:
            cache[inst.name] = oracle.run(inst)
        assert_parity(g, cache[inst.name])


def test_sweep_config5_full_digests():
    """Full config-5 parity: all 4,096 instances of the sweep in the bench's
    launch configuration (dts_sweep_run, default options: two concurrent
    batched launches), every instance's whole schedule (service order, task
    start/end, every trace event) compared with the oracle through the
    SHA-256 digests written by tests/golden/make_c5_digests.py (oracle only)
    -- plus the counters, so a mismatch names the instance."""
    gold = json.load(open(os.path.join(GOLDEN, "digests_C5.json")))
    params = gen.sweep_params()
    assert gold["n_instances"] == len(params) == 4096
    insts = gen.config_instances("C5")
    hs = [dts.create(i) for i in insts]
    dts.dts_sweep_run(hs, dts.DTS_POLICY_DARTS_LUF, dts.dts_run_opts_default(flags=dts.DTS_F_FALLBACK2))
    dts.dts_fetch_results(hs)
    bad = []
    for i, (h, row) in enumerate(zip(hs, gold["instances"])):
        assert (row["N"], row["M"], row["K"]) == tuple(params[i])
        g = dts.dts_result(h, copy=False)
        got = (g.n_served, g.n_loads, g.n_evictions, g.n_scans, g.n_fallback2, g.n_fallback_first,
               g.n_idle_requests, int(g.bytes_loaded), int(g.makespan),
               digest(g.serve_gpu, g.serve_task, g.task_start, g.task_end, g.events))
        want = (row["n_served"], row["n_loads"], row["n_evictions"], row["n_scans"], row["n_fallback2"],
                row["n_fallback_first"], row["n_idle_requests"], row["bytes_loaded"], row["makespan"],
                row["sha256"])
        if got != want:
            bad.append((params[i], got[:-1], want[:-1]))
    assert not bad, f"{len(bad)} of 4096 instances differ, first: {bad[:3]}"


@pytest.mark.parametrize("block", [0, 128])
def test_sweep_config5_repeated(block):
    """The full 4,096-instance sweep (bench launch configuration, and forced
    128-thread CTAs) three times: every repetition schedules every task and
    gives the same schedules (guards the block-level pop-batch race), and a
    sample matches the oracle."""
    insts = gen.config_instances("C5")
    hs = [dts.create(i) for i in insts]
    o = dts.dts_run_opts_default(flags=dts.DTS_F_FALLBACK2, block_threads=block)
    ref = None
    for _ in range(3):
        dts.dts_sweep_run(hs, dts.DTS_POLICY_DARTS_LUF, o)
        res = [dts.dts_result(h) for h in hs]
        assert all(g.n_served == i.m for g, i in zip(res, insts))
        sig = [(g.n_loads, g.n_evictions, g.makespan, g.n_scans) for g in res]
        ref = ref or sig
        assert sig == ref
    for i in range(0, len(insts), 409):
        if insts[i].m <= 12000:
            assert_parity(res[i], oracle.run(insts[i]))


@pytest.mark.parametrize("K", [5, 9, 16, 64])
def test_many_simulated_gpus(K):
    """K beyond the register-resident pop path (K <= 8) and up to MAX_K = 64."""
    inst = gen.random_shared(6000, 512, 3, M=24, K=K, seed=K)
    g, o = _both(inst)
    assert_parity(g, o)
    inst2 = gen.matmul2d(40, M=10, K=K)
    g, o = _both(inst2, smem=-1)
    assert_parity(g, o)


def test_hub_datum_64bit_argmax_keys():
    """A datum used by >= 2^15 tasks disables the packed 32-bit argmax keys
    (I.key32): the 64-bit (score, u, ~D) path must give the same schedule."""
    m = 40000
    rng = np.random.default_rng(3)
    other = rng.integers(1, 300, size=m)
    tp = np.arange(0, 2 * m + 1, 2, dtype=np.int64)
    td = np.empty(2 * m, np.int32)
    td[0::2] = 0
    td[1::2] = other
    inst = gen.Instance("hub", tp, td, np.ones(300, np.uint64), None, 5, 12, 3)
    g, o = _both(inst, bus=10 ** 9)
    assert_parity(g, o)


@pytest.mark.parametrize("idx", range(12))
def test_fused_and_separate_csr_build(idx):
    """Small instances build their CSR and initial state inside the loop CTA
    (one launch); DTS_F_NOFUSE forces the separate grid-wide kernels.  Both
    must give the oracle's schedule, with and without shared-memory state."""
    inst = _shapes()[idx]
    o = oracle.run(inst)
    for flags in (dts.DTS_F_FALLBACK2, dts.DTS_F_FALLBACK2 | dts.DTS_F_NOFUSE):
        for smem in (0, -1):
            g = dts.schedule(inst, flags=flags, smem_budget=smem)
            assert_parity(g, o)


# ------------------------------------------------------------ OPTI (§V-F)
@pytest.mark.parametrize("idx", range(12))
@pytest.mark.parametrize("fb2", [1, 0])
def test_opti_shapes(idx, fb2):
    inst = _shapes()[idx]
    flags = dts.DTS_F_OPTI | (dts.DTS_F_FALLBACK2 if fb2 else 0)
    g, o = _both(inst, flags=flags)
    assert_parity(g, o)


@pytest.mark.parametrize("N", [4, 6])
def test_opti_2d_column_major(N):
    inst = _unit(gen.matmul2d(N, M=2 * N, K=1))
    g = dts.schedule(inst, bus_bps=10 ** 9, flags=dts.DTS_F_FALLBACK2 | dts.DTS_F_OPTI)
    assert [int(x) for x in g.orders()[0]] == [i * N + j for j in range(N) for i in range(N)]


@pytest.mark.parametrize("cfg", ["C4a", "C4b"])
def test_opti_config4_prefix(cfg):
    """DARTS+LUF+OPTI-3inputs (the paper's Cholesky setting, Fig. 11) at full size, prefix."""
    inst = gen.config_instances(cfg)[0]
    g, o = _both(inst, flags=dts.DTS_F_FALLBACK2 | dts.DTS_F_OPTI, max_served=1500)
    assert_parity(g, o, complete=False)


def test_opti_config2_batch():
    insts = gen.config_instances("C2")
    gs = dts.schedule_batch(insts, flags=dts.DTS_F_FALLBACK2 | dts.DTS_F_OPTI)
    for inst, g in zip(insts, gs):
        assert_parity(g, oracle.run(inst, flags=oracle.F_FALLBACK2 | oracle.F_OPTI))


# ------------------------------------------------------------ workload variants (§8(f)3)
def _variants():
    return [gen.matmul2d(50, M=35, K=2, order="random", seed=11),    # PAPER.md:800, Fig. 9
            gen.matmul2d(100, M=35, K=4, keep_frac=0.02, seed=12),  # sparse 2D
            gen.matmul2d(60, M=35, K=4, keep_frac=0.3, seed=13),
            gen.matmul3d(20, M=142, K=4, with_c=True)]              # 3D with C_ij (reading R12)


@pytest.mark.parametrize("idx", range(4))
@pytest.mark.parametrize("flags", [1, 1 | 8])
def test_workload_variants(idx, flags):
    inst = _variants()[idx]
    g, o = _both(inst, flags=flags)
    assert_parity(g, o)
    validate(inst, g.serve_gpu, g.serve_task, g.events, g.task_start, g.task_end)


# ------------------------------------------------------------ DARTS+LRU, EAGER+LRU (§8(f)2)
_POL = {"darts_lru": (dts.DTS_POLICY_DARTS_LRU, oracle.F_LRU),
        "eager_lru": (dts.DTS_POLICY_EAGER_LRU, oracle.F_EAGER | oracle.F_LRU)}


def _both_policy(inst, name, bus=oracle.DEFAULT_BUS_BPS, flags=1, smem=0, max_served=-1):
    pol, of = _POL[name]
    g = dts.schedule(inst, policy=pol, bus_bps=bus, flags=flags, smem_budget=smem,
                     max_served=max_served)
    o = oracle.run(inst, bus_bps=bus, flags=flags | of, max_served=max_served)
    return g, o


@pytest.mark.parametrize("name", ["darts_lru", "eager_lru"])
@pytest.mark.parametrize("idx", range(12))
def test_lru_policies_shapes(name, idx):
    inst = _shapes()[idx]
    for smem in (0, -1):
        g, o = _both_policy(inst, name, smem=smem)
        assert_parity(g, o)
        validate(inst, g.serve_gpu, g.serve_task, g.events, g.task_start, g.task_end)


def test_eager_lru_hand_trace_gpu():
    inst = _unit(gen.matmul2d(3, M=4, K=1))
    g = dts.schedule(inst, policy=dts.DTS_POLICY_EAGER_LRU, bus_bps=10 ** 9)
    assert [int(e["data"]) for e in g.events if e["op"] == 0] == [0, 3, 4, 5, 1, 4, 2, 4]
    assert [int(e["data"]) for e in g.events if e["op"] == 1] == [4, 0, 4, 1]


@pytest.mark.parametrize("name", ["darts_lru", "eager_lru"])
def test_lru_policies_config2_batch(name):
    pol, of = _POL[name]
    insts = gen.config_instances("C2")
    gs = dts.schedule_batch(insts, policy=pol)
    for inst, g in zip(insts, gs):
        assert_parity(g, oracle.run(inst, flags=1 | of))


@pytest.mark.parametrize("name", ["darts_lru", "eager_lru"])
def test_lru_policies_config3(name):
    g, o = _both_policy(gen.config_instances("C3")[0], name)
    assert_parity(g, o)


@pytest.mark.parametrize("name", ["darts_lru", "eager_lru"])
@pytest.mark.parametrize("cfg", ["C4a", "C4b"])
def test_lru_policies_config4_prefix(name, cfg):
    g, o = _both_policy(gen.config_instances(cfg)[0], name, max_served=1500)
    assert_parity(g, o, complete=False)


# ------------------------------------------------------------ W = 1 prefetch window (§8(f)4)
def _w1(inst):
    """Room for two tasks' inputs (the capacity check for W = 1)."""
    return inst.with_(mem_capacity=int(inst.mem_capacity) + 3 * int(inst.data_size.max()))


@pytest.mark.parametrize("idx", range(12))
@pytest.mark.parametrize("name", ["darts_luf", "darts_lru", "eager_lru"])
def test_w1_shapes(idx, name):
    inst = _w1(_shapes()[idx])
    pol = {"darts_luf": (dts.DTS_POLICY_DARTS_LUF, 0), **_POL}[name]
    g = dts.schedule(inst, policy=pol[0], W=1)
    o = oracle.run(inst, W=1, flags=1 | pol[1])
    assert_parity(g, o)
    validate(inst, g.serve_gpu, g.serve_task, g.events, g.task_start, g.task_end, W=1)


def test_w1_config2_and_3():
    for inst in gen.config_instances("C2")[::3] + gen.config_instances("C3"):
        g = dts.schedule(inst, W=1)
        o = oracle.run(inst, W=1)
        assert_parity(g, o)


@pytest.mark.parametrize("cfg", ["C4a", "C4b"])
def test_w1_config4_prefix(cfg):
    inst = gen.config_instances(cfg)[0]
    g = dts.schedule(inst, W=1, max_served=1500)
    o = oracle.run(inst, W=1, max_served=1500)
    assert_parity(g, o, complete=False)


def test_fetch_results_matches_per_instance_result():
    """dts_fetch_results (batched copies, two waits) returns what dts_result
    alone would, for a sweep and for separately run instances."""
    insts = gen.config_instances("C2")[:6]
    a = dts.schedule_batch(insts)  # fetch + result
    hs = [dts.create(i) for i in insts]
    for h in hs:
        dts.dts_run(h, dts.DTS_POLICY_DARTS_LUF, dts.dts_run_opts_default())
    b = [dts.dts_result(h) for h in hs]  # one at a time
    for x, y, inst in zip(a, b, insts):
        assert np.array_equal(x.serve_task, y.serve_task) and np.array_equal(x.events, y.events)
        assert_parity(x, oracle.run(inst))



def test_result_views_without_copy():
    """dts_result(copy=False): read-only views of the pinned result buffers,
    equal to the copies, valid until the instance runs again."""
    insts = gen.config_instances("C2")[:4]
    hs = [dts.create(i) for i in insts]
    dts.dts_sweep_run(hs, dts.DTS_POLICY_DARTS_LUF, dts.dts_run_opts_default())
    dts.dts_fetch_results(hs)
    for h, inst in zip(hs, insts):
        v = dts.dts_result(h, copy=False)
        c = dts.dts_result(h)
        assert not v.serve_task.flags.writeable
        assert np.array_equal(v.serve_task, c.serve_task) and np.array_equal(v.events, c.events)
        assert_parity(v, oracle.run(inst))


def test_sweep_devices_list():
    """include/dts.h dts_sweep_run with a device list:
    devices = [0, 0] splits the batch by LPT into two concurrent launches on
    device 0 (the caller's stream and a library stream joined back into it);
    every instance matches the oracle."""
    insts = gen.config_instances("C2") + [gen.sweep_instance(N, M, K) for (N, M, K) in
                                          [(40, 6, 3), (25, 4, 1), (60, 12, 8), (15, 35, 2)]]
    hs = [dts.create(i) for i in insts]
    dts.dts_sweep_run(hs, dts.DTS_POLICY_DARTS_LUF, dts.dts_run_opts_default(), devices=[0, 0])
    dts.dts_fetch_results(hs)
    for inst, h in zip(insts, hs):
        assert_parity(dts.dts_result(h), oracle.run(inst))


def test_concurrent_sweeps_on_two_streams():
    """Two batched launches in flight at once on different streams (each
    launch has its own descriptor buffer and instance counters):
    both batches match the oracle."""
    import torch
    a = [gen.sweep_instance(N, M, K) for (N, M, K) in [(30, 5, 2), (45, 8, 4), (20, 4, 1)]]
    b = [gen.sweep_instance(N, M, K) for (N, M, K) in [(35, 6, 3), (50, 10, 5), (10, 4, 2)]]
    ha, hb = [dts.create(i) for i in a], [dts.create(i) for i in b]
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
    for _ in range(3):
        dts.dts_sweep_run(ha, dts.DTS_POLICY_DARTS_LUF, dts.dts_run_opts_default(cuda_stream=s1.cuda_stream))
        dts.dts_sweep_run(hb, dts.DTS_POLICY_DARTS_LUF, dts.dts_run_opts_default(cuda_stream=s2.cuda_stream))
        dts.dts_fetch_results(ha + hb)
        for inst, h in zip(a + b, ha + hb):
            assert_parity(dts.dts_result(h), oracle.run(inst))


# ---------------------------------------- W >= 2 and Alg. 6's Belady branch (R29)
def _tight(inst, W):
    """The least capacity the library accepts for DARTS+LUF with window W:
    max(1, W) tasks' inputs (Belady fires, reading R29)."""
    row = max(int(inst.data_size[inst.task_data[inst.task_ptr[T]:inst.task_ptr[T + 1]]].sum())
              for T in range(inst.m))
    return inst.with_(mem_capacity=max(1, W) * row)


@pytest.mark.parametrize("name", ["belady_w1_2d_N2.json", "belady_w2_2d_N3.json", "belady_w1_disjoint.json"])
def test_belady_hand_traces_gpu(name):
    from test_oracle_pins import belady_instance
    gold = json.load(open(os.path.join(GOLDEN, name)))
    inst = belady_instance(gold)
    g = dts.schedule(inst, W=gold["W"], bus_bps=10 ** 9)
    o = oracle.run(inst, W=gold["W"], bus_bps=10 ** 9)
    assert_parity(g, o)
    assert g.n_belady == gold["n_belady"] > 0
    assert list(map(int, g.orders()[0])) == gold["order"]


@pytest.mark.parametrize("W", [1, 2, 3, 5, 8])
@pytest.mark.parametrize("idx", range(12))
def test_w_tight_shapes(W, idx):
    inst = _tight(_shapes()[idx], W)
    if W * max(inst.task_ptr[1:] - inst.task_ptr[:-1]) > 128:
        pytest.skip("W * inputs per task > 128 (UNSUPPORTED by design)")
    g, o = dts.schedule(inst, W=W), oracle.run(inst, W=W)
    assert_parity(g, o)
    validate(inst, g.serve_gpu, g.serve_task, g.events, g.task_start, g.task_end, W=W)


@pytest.mark.parametrize("W", [2, 4])
@pytest.mark.parametrize("name", ["darts_lru", "eager_lru"])
def test_w_lru_policies(W, name):
    """LRU policies with W >= 2 (their capacity check keeps (W+1) tasks)."""
    for inst in _shapes()[:6]:
        inst = inst.with_(mem_capacity=int(inst.mem_capacity) + (W + 1) * 3 * int(inst.data_size.max()))
        pol = _POL[name]
        g = dts.schedule(inst, policy=pol[0], W=W)
        o = oracle.run(inst, W=W, flags=1 | pol[1])
        assert_parity(g, o)


def test_w2_configs_tight():
    """Paper-scale shapes with W = 2 and the tight capacity: C2's largest
    instances, C3, and a C4a / C4b prefix; Belady fires."""
    bel = 0
    for inst in gen.config_instances("C2")[8:10] + gen.config_instances("C3"):
        inst = _tight(inst, 2)
        g, o = dts.schedule(inst, W=2), oracle.run(inst, W=2)
        assert_parity(g, o)
        bel += g.n_belady
    for cfg in ("C4a", "C4b"):
        inst = _tight(gen.config_instances(cfg)[0], 2)
        g = dts.schedule(inst, W=2, max_served=1500)
        o = oracle.run(inst, W=2, max_served=1500)
        assert_parity(g, o, complete=False)
    assert bel > 0


def test_capacity_check_by_policy():
    """DARTS+LUF accepts max(1, W) tasks' inputs, the LRU policies (W+1)."""
    inst = _tight(gen.matmul2d(6, M=4, K=1), 2)
    h = dts.create(inst)
    dts.dts_run(h, dts.DTS_POLICY_DARTS_LUF, dts.dts_run_opts_default(lookahead_W=2))
    dts.dts_result(h)
    with pytest.raises(dts.DtsError) as e:
        dts.dts_run(h, dts.DTS_POLICY_DARTS_LRU, dts.dts_run_opts_default(lookahead_W=2))
    assert e.value.status == -2
    with pytest.raises(dts.DtsError) as e:
        dts.dts_run(h, dts.DTS_POLICY_DARTS_LUF, dts.dts_run_opts_default(lookahead_W=9))
    assert e.value.status == -6


# ------------------------------------------------ large-n shapes (n >= 4096 data)
def _large_n_shapes():
    """Random shared-input instances with 4,096-16,384 data and K up to 16:
    the score arrays live in HBM (L2), not shared memory."""
    return [gen.random_shared(20_000, 8192, 3, M=64, K=4, seed=11),
            gen.random_shared(16_000, 4096, 2, M=40, K=8, seed=12),
            gen.random_shared(12_000, 16384, 3, M=96, K=3, seed=13),
            gen.random_shared(8_000, 4096, 3, M=24, K=16, seed=14)]


@pytest.mark.parametrize("idx", range(4))
@pytest.mark.parametrize("flags", [dts.DTS_F_FALLBACK2, 0, dts.DTS_F_FALLBACK2 | dts.DTS_F_OPTI])
def test_large_n_full_parity(idx, flags):
    inst = _large_n_shapes()[idx]
    g, o = _both(inst, flags=flags)
    assert_parity(g, o)


def test_large_n_lru_policy():
    g, o = _both_policy(_large_n_shapes()[0], "darts_lru")
    assert_parity(g, o)


def test_large_n_in_mixed_sweep():
    insts = _large_n_shapes()[:2] + gen.config_instances("C2")[:6]
    gs = dts.schedule_batch(insts)
    for inst, g in zip(insts, gs):
        assert_parity(g, oracle.run(inst))


def test_large_n_w1_and_belady():
    inst = _tight(_large_n_shapes()[1], 1)
    g, o = dts.schedule(inst, W=1), oracle.run(inst, W=1)
    assert_parity(g, o)


# ------------------------------- the generic loop vs the specialised one
@pytest.mark.parametrize("idx", range(12))
def test_generic_loop_on_shapes(idx):
    """DTS_F_GENERIC forces the run-time-moded loop where the compile-time
    specialised one (row-derived, one shard, W = 0, DARTS+LUF) would run; both
    must give the oracle's schedule."""
    inst = _shapes()[idx]
    for fl in (dts.DTS_F_FALLBACK2 | dts.DTS_F_GENERIC, dts.DTS_F_FALLBACK2):
        g = dts.schedule(inst, flags=fl)
        assert_parity(g, oracle.run(inst))


def test_generic_loop_batch_and_config4_prefix():
    insts = gen.config_instances("C2")[::4] + [gen.sweep_instance(N, M, K) for (N, M, K) in
                                               [(60, 5, 3), (35, 12, 8), (100, 6, 1)]]
    gs = dts.schedule_batch(insts, flags=dts.DTS_F_FALLBACK2 | dts.DTS_F_GENERIC)
    for inst, g in zip(insts, gs):
        assert_parity(g, oracle.run(inst))
    for cfg in ("C4a", "C4b"):
        inst = gen.config_instances(cfg)[0]
        g = dts.schedule(inst, flags=dts.DTS_F_FALLBACK2 | dts.DTS_F_GENERIC, max_served=1500)
        assert_parity(g, oracle.run(inst, max_served=1500), complete=False)

"""The one-warp-per-instance decision loop (csrc/dts_warp.cu):
which loop runs (dts_result_view.loop_kind), parity with the oracle on the
cases specific to that loop (1- and 2-input rows, duplicate inputs, tasks
without inputs, per-task times, K = 1 and K = 32, 16-bit id limits, prefix
runs, batches), and the per-CTA loop kept parity-green on the configurations
the warp loop now serves by default (DTS_F_CTA).  Needs a B200."""
import numpy as np
import pytest

import gen
import oracle
import paper_conf_ipps_gonthiermt22_b200 as dts
from parity import assert_parity
from validate import validate

pytestmark = pytest.mark.gpu

F = dts.DTS_F_FALLBACK2
CTA = F | dts.DTS_F_CTA


@pytest.fixture(scope="module", autouse=True)
def _need_gpu():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    dts.load_library()


def _rows_instance(rows, n, M, K, size=1000, tau=None, default_ns=7, name="rows"):
    ptr = np.zeros(len(rows) + 1, np.int64)
    ptr[1:] = np.cumsum([len(r) for r in rows])
    dat = np.asarray([d for r in rows for d in r], np.int32)
    return gen.Instance(name, ptr, dat, np.full(n, size, np.uint64),
                        None if tau is None else np.asarray(tau, np.int64), default_ns, M * size, K)


def _random_rows(m, n, seed, one_frac=0.2, dup_frac=0.1, empty_frac=0.0):
    """Rows of 1 or 2 inputs, some given twice ([a, a], R27), some empty."""
    rng = np.random.default_rng(seed)
    rows = []
    for _ in range(m):
        x = rng.random()
        if x < empty_frac:
            rows.append(())
        elif x < empty_frac + one_frac:
            rows.append((int(rng.integers(n)),))
        elif x < empty_frac + one_frac + dup_frac:
            a = int(rng.integers(n))
            rows.append((a, a, a) if rng.random() < 0.3 else (a, a))
        else:
            a, b = rng.choice(n, 2, replace=False)
            rows.append((int(a), int(b)) if rng.random() < 0.5 else (int(b), int(a)))
    return rows


def _check(inst, flags=F, max_served=-1, kind=dts.LOOP_WARP, bus=oracle.DEFAULT_BUS_BPS):
    g = dts.schedule(inst, flags=flags, max_served=max_served, bus_bps=bus)
    assert g.loop_kind == kind, (g.loop_kind, kind)
    o = oracle.run(inst, flags=flags & (dts.DTS_F_FALLBACK2 | dts.DTS_F_OPTI), max_served=max_served,
                   bus_bps=bus)
    assert_parity(g, o, complete=max_served < 0)
    if max_served < 0:
        validate(inst, g.serve_gpu, g.serve_task, g.events, g.task_start, g.task_end)
    return g


# ------------------------------------------------------------- which loop runs
def test_loop_kind_selection():
    c1 = gen.config_instances("C1")[0]
    assert dts.schedule(c1).loop_kind == dts.LOOP_WARP
    assert dts.schedule(c1, flags=CTA).loop_kind == dts.LOOP_CTA_FAST
    assert dts.schedule(c1, flags=F | dts.DTS_F_GENERIC).loop_kind == dts.LOOP_GENERIC
    assert dts.schedule(c1, W=1).loop_kind == dts.LOOP_GENERIC            # W >= 1: generic loop
    assert dts.schedule(c1, block_threads=64).loop_kind == dts.LOOP_CTA_FAST  # forced CTA shape
    assert dts.schedule(c1, smem_budget=-1).loop_kind == dts.LOOP_CTA_FAST    # no shared memory
    assert dts.schedule(c1, flags=F | dts.DTS_F_OPTI).loop_kind == dts.LOOP_GENERIC
    three = gen.random_shared(300, 64, 3, M=8, K=3, seed=7)                   # 3-input rows
    assert dts.schedule(three).loop_kind == dts.LOOP_CTA_FAST
    assert dts.schedule(gen.matmul3d(40, M=142, K=4), max_served=50).loop_kind == dts.LOOP_WARP  # C3
    wide = gen.random_shared(20000, 8, 2, M=3, K=2, seed=3)                   # segments of ~5,000 tasks
    assert dts.schedule(wide, max_served=20).loop_kind == dts.LOOP_CTA_FAST
    big = gen.random_shared(60000, 8192, 2, M=128, K=4, seed=1)               # slice > shared memory
    assert dts.schedule(big, max_served=20).loop_kind == dts.LOOP_CTA_FAST
    k33 = gen.matmul2d(8, M=4, K=33)                                          # K > 32
    assert dts.schedule(k33).loop_kind == dts.LOOP_CTA_FAST
    for g in dts.schedule_batch(gen.config_instances("C2")):
        assert g.loop_kind == dts.LOOP_WARP


def test_task_id_limit_16_bits():
    """Edge words hold T in 16 bits: m = 65,535 runs on the warp loop, 65,536
    on a CTA; both prefixes match the oracle."""
    for m, kind in ((65535, dts.LOOP_WARP), (65536, dts.LOOP_CTA_FAST)):
        inst = gen.random_shared(m, 1024, 2, M=24, K=2, seed=11)
        _check(inst, max_served=1200, kind=kind)


# ------------------------------------------------------------- warp-loop cases
@pytest.mark.parametrize("seed", range(6))
def test_one_and_two_input_rows_duplicates(seed):
    n = [12, 40, 97, 200, 33, 64][seed]
    K = [1, 2, 3, 4, 7, 5][seed]
    rows = _random_rows([150, 900, 2000, 4000, 700, 3000][seed], n, seed)
    inst = _rows_instance(rows, n, M=[3, 5, 8, 16, 4, 6][seed], K=K)
    _check(inst)


def test_tasks_without_inputs():
    rows = _random_rows(800, 50, 3, empty_frac=0.15)
    _check(_rows_instance(rows, 50, M=6, K=3))
    _check(_rows_instance([(), (), ()], 4, M=2, K=2))        # no data used at all
    _check(_rows_instance([(), (1, 2), ()], 4, M=2, K=1))


def test_per_task_times():
    rows = _random_rows(1500, 60, 4)
    tau = np.random.default_rng(9).integers(1, 5000, len(rows))
    _check(_rows_instance(rows, 60, M=7, K=4, tau=tau))
    two_d = gen.matmul2d(25, M=8, K=3)
    _check(two_d.with_(task_ns=np.random.default_rng(2).integers(1000, 900000, two_d.m)))
    _check(two_d.with_(task_ns=np.zeros(two_d.m, np.int64)))  # zero-length tasks


@pytest.mark.parametrize("K", [1, 2, 31, 32])
def test_k_range(K):
    _check(gen.matmul2d(40, M=6, K=K))
    _check(gen.matmul2d(12, M=3, K=K, order="random", seed=4))


def test_uniform_time_ties_between_gpus():
    """Unit tasks and unit loads: many GPUs request at the same instant, so the
    batched pops order them by (time, GPU id) inside every round (R8)."""
    for inst in (gen.matmul2d(30, M=6, K=8), gen.matmul2d(20, M=40, K=16)):
        unit = inst.with_(data_size=np.ones(inst.n, np.uint64), mem_capacity=int(inst.mem_capacity //
                          int(inst.data_size[0])), default_task_ns=1, task_ns=None)
        _check(unit, bus=10 ** 9)


def test_fallback_and_lowest_id_picks():
    _check(gen.matmul2d(30, M=8, K=3), flags=0)       # 3inputs off: lowest-id picks
    _check(gen.matmul2d(20, M=4, K=2, keep_frac=0.3, seed=6))
    _check(gen.random_shared(4000, 512, 2, M=4, K=6, seed=3))


@pytest.mark.parametrize("ms", [1, 7, 100, 999])
def test_prefix_runs(ms):
    _check(gen.matmul2d(40, M=6, K=4), max_served=ms)
    _check(gen.matmul2d(60, M=35, K=2), max_served=ms)


def test_wide_segments_several_batches():
    """Data used by more than 32 x (edges per lane) tasks: segment walks take
    several register batches (and Dopt's load the general walk)."""
    _check(gen.random_shared(20000, 32, 2, M=6, K=3, seed=5))
    _check(gen.matmul2d(200, M=10, K=2), max_served=3000)


def test_config3_on_the_warp_loop():
    """C3 (one 64,000-task instance, n = 3,200) runs on one warp: full parity."""
    inst = gen.config_instances("C3")[0]
    _check(inst)
    _check(inst, flags=CTA, kind=dts.LOOP_CTA_FAST)


def test_batch_of_mixed_warp_instances():
    insts = [gen.matmul2d(N, M=M, K=K) for N, M, K in ((5, 4, 1), (33, 6, 3), (90, 35, 4), (12, 3, 8))]
    insts += [_rows_instance(_random_rows(500, 40, s), 40, M=5, K=2) for s in range(3)]
    gs = dts.schedule_batch(insts)
    for inst, g in zip(insts, gs):
        assert g.loop_kind == dts.LOOP_WARP
        assert_parity(g, oracle.run(inst))


# ------------------------------------- the per-CTA loop on the warp loop's configs
def test_cta_loop_config1_and_config2():
    c1 = gen.config_instances("C1")[0]
    _check(c1, flags=CTA, kind=dts.LOOP_CTA_FAST)
    insts = gen.config_instances("C2")
    gs = dts.schedule_batch(insts, flags=CTA)
    for inst, g in zip(insts, gs):
        assert g.loop_kind == dts.LOOP_CTA_FAST
        assert_parity(g, oracle.run(inst))


def test_cta_loop_config5_sample():
    params = gen.sweep_params()
    rng = np.random.default_rng(8)
    pick = sorted(rng.choice(len(params), size=40, replace=False))
    insts = [gen.sweep_instance(*params[i]) for i in pick]
    gs = dts.schedule_batch(insts, flags=CTA)
    for inst, g in zip(insts, gs):
        assert g.loop_kind == dts.LOOP_CTA_FAST
        assert_parity(g, oracle.run(inst))

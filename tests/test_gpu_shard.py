"""GPU parity of the task-sharded single instance (second
mode; include/dts.h "Task-sharded single instance"): one instance, its tasks
split over G shards that exchange partial scores / plan parts inside the
kernel.  The schedule must be the oracle's, bit for bit, on every shard
(reading R22: under R1-R28 it is unique), for every G -- sharding changes
where n_k(D), n2_k(D), u(D) are counted, never what is decided.

Single device: dts_shard_group_run (G co-resident CTAs).  The multi-process
path (CUDA IPC handles, one process per shard) is exercised with two
processes on the same B200.  Needs a B200."""
import json
import os
import subprocess
import sys

import numpy as np
import pytest

import gen
import oracle
import paper_conf_ipps_gonthiermt22_b200 as dts
from conftest import GOLDEN, ROOT
from digest import digest
from parity import assert_parity
from validate import validate

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module", autouse=True)
def _need_gpu():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    dts.load_library()


def _same(rs):
    for r in rs[1:]:
        assert np.array_equal(r.serve_gpu, rs[0].serve_gpu) and np.array_equal(r.serve_task, rs[0].serve_task)
        assert np.array_equal(r.events, rs[0].events)
        assert np.array_equal(r.task_start, rs[0].task_start)


def _check(inst, G, flags=1, policy=dts.DTS_POLICY_DARTS_LUF, oflags=0, W=0, max_served=-1, **kw):
    rs = dts.schedule_sharded(inst, G, policy=policy, flags=flags, W=W, max_served=max_served, **kw)
    o = oracle.run(inst, W=W, flags=flags | oflags, max_served=max_served)
    _same(rs)
    for r in rs:
        assert_parity(r, o, complete=max_served < 0)
    return rs, o


def _shapes():
    return [gen.fig1(), gen.matmul2d(6, M=4, K=1), gen.matmul2d(7, M=5, K=2, order="random", seed=3),
            gen.matmul3d(4, M=6, K=2), gen.matmul3d(3, M=9, K=3, with_c=True),
            gen.cholesky(6, M=5, K=2), gen.random_shared(300, 64, 3, M=8, K=3, seed=7),
            gen.matmul2d(20, M=6, K=4, keep_frac=0.1, seed=5),
            gen.random_shared(5000, 256, 3, M=20, K=8, seed=1),
            gen.cholesky(20, M=30, K=4), gen.matmul3d(10, M=25, K=4)]


@pytest.mark.parametrize("idx", range(11))
@pytest.mark.parametrize("G", [1, 2, 3, 8])
def test_shard_shapes(idx, G):
    inst = _shapes()[idx]
    rs, _ = _check(inst, G)
    validate(inst, rs[0].serve_gpu, rs[0].serve_task, rs[0].events, rs[0].task_start, rs[0].task_end)


@pytest.mark.parametrize("G", [2, 4, 16])
def test_shard_config1_and_more_shards_than_tasks(G):
    _check(gen.config_instances("C1")[0], G)
    _check(gen.fig1(), 16)  # 9 tasks over 16 shards: empty shards


@pytest.mark.parametrize("idx", [0, 9, 10, 19])
@pytest.mark.parametrize("G", [2, 4])
def test_shard_config2(idx, G):
    _check(gen.config_instances("C2")[idx], G)


def test_shard_config3():
    _check(gen.config_instances("C3")[0], 4)


@pytest.mark.parametrize("cfg", ["C4a", "C4b"])
def test_shard_config4_prefix(cfg):
    _check(gen.config_instances(cfg)[0], 8, max_served=1500)


@pytest.mark.parametrize("fb2", [1, 0])
@pytest.mark.parametrize("idx", [1, 5, 8, 9])
def test_shard_opti_and_no_fallback(idx, fb2):
    _check(_shapes()[idx], 3, flags=fb2 | dts.DTS_F_OPTI)
    _check(_shapes()[idx], 2, flags=fb2)


@pytest.mark.parametrize("name", ["darts_lru", "eager_lru"])
@pytest.mark.parametrize("idx", [1, 3, 6, 8, 9])
def test_shard_lru_policies(name, idx):
    pol, of = {"darts_lru": (dts.DTS_POLICY_DARTS_LRU, oracle.F_LRU),
               "eager_lru": (dts.DTS_POLICY_EAGER_LRU, oracle.F_EAGER | oracle.F_LRU)}[name]
    _check(_shapes()[idx], 4, policy=pol, oflags=of)


@pytest.mark.parametrize("idx", [2, 6, 8])
def test_shard_w1(idx):
    inst = _shapes()[idx]
    inst = inst.with_(mem_capacity=int(inst.mem_capacity) + 3 * int(inst.data_size.max()))
    _check(inst, 3, W=1)


@pytest.mark.parametrize("smem", [0, -1])
def test_shard_verify_partial_scores(smem):
    """DTS_F_VERIFY (P9) on shards: each shard's partial n_k, n2_k, u and its
    tasks' (cnt, xor) equal a from-scratch recount over its own tasks."""
    inst = gen.random_shared(5000, 256, 3, M=20, K=8, seed=1)
    rs, _ = _check(inst, 4, flags=1 | dts.DTS_F_VERIFY, smem_budget=smem)
    assert all(r.n_verify_err == 0 for r in rs)


def test_shard_heterogeneous_sizes_and_times():
    rng = np.random.default_rng(4)
    base = gen.random_shared(2000, 128, 3, M=8, K=4, seed=11)
    sizes = rng.integers(1, 5, size=128).astype(np.uint64) * 1_000_000
    tau = rng.integers(1000, 100000, size=base.m).astype(np.int64)
    inst = base.with_(data_size=sizes, mem_capacity=int(sizes.max()) * 9, task_ns=tau)
    _check(inst, 3)


def test_shard_repeated_runs():
    """Exchange numbers move to a new range every run: reruns of the same
    shards (and a change of G) give the same schedule."""
    inst = gen.config_instances("C2")[5]
    hs = [dts.create(inst) for _ in range(4)]
    o = oracle.run(inst)
    for G in (4, 4, 2, 4):
        dts.dts_shard_group_run(hs[:G])
        for h in hs[:G]:
            assert_parity(dts.dts_result(h), o)


@pytest.mark.parametrize("cfg", ["C4b"])
def test_shard_config4_full_digest(cfg):
    """Full-size C4b sharded over 8 CTAs against the oracle's golden digest."""
    gold = json.load(open(os.path.join(GOLDEN, f"digests_{cfg}.json")))
    inst = gen.config_instances(cfg)[0]
    r = dts.schedule_sharded(inst, 8)[0]
    for k in ("n_served", "n_loads", "n_evictions", "n_scans", "n_fallback2", "n_fallback_first",
              "bytes_loaded", "makespan"):
        assert getattr(r, k) == gold[k], k
    assert digest(r.serve_gpu, r.serve_task, r.task_start, r.task_end, r.events) == gold["sha256"]


def test_shard_ipc_two_processes():
    """The multi-GPU path (dts_shard_export / connect, CUDA IPC, one process
    per shard) with both processes on this one B200."""
    script = os.path.join(ROOT, "tests", "shard_ipc_worker.py")
    env = dict(os.environ, MASTER_ADDR="127.0.0.1", MASTER_PORT="29731", WORLD_SIZE="2")
    procs = [subprocess.Popen([sys.executable, script], env=dict(env, RANK=str(r)),
                              stdout=subprocess.PIPE, stderr=subprocess.STDOUT, text=True)
             for r in range(2)]
    outs = []
    for p in procs:
        try:
            out, _ = p.communicate(timeout=240)
        except subprocess.TimeoutExpired:
            p.kill()
            out, _ = p.communicate()
        outs.append(out)
    for p, out in zip(procs, outs):
        assert p.returncode == 0, out
        assert "PARITY OK" in out, out


# ------------------------------------------- dts_run_opts.n_devices
@pytest.mark.parametrize("G", [2, 3, 4])
def test_run_n_devices_matches_oracle(G):
    """dts_run with n_devices = G: the instance task-sharded over G shards in
    this process (on a one-GPU machine all on device 0, separate launches
    exchanging through each other's memory) gives the oracle's schedule."""
    for inst in (gen.matmul2d(30, M=8, K=3), gen.random_shared(5000, 512, 3, M=20, K=4, seed=G),
                 gen.matmul3d(8, M=12, K=2)):
        g = dts.schedule(inst, n_devices=G)
        assert_parity(g, oracle.run(inst))


def test_run_n_devices_then_one_device_again():
    inst = gen.config_instances("C2")[5]
    h = dts.create(inst)
    o = oracle.run(inst)
    for G in (2, 1, 3, 3, 0):
        dts.dts_run(h, dts.DTS_POLICY_DARTS_LUF, dts.dts_run_opts_default(n_devices=G))
        assert_parity(dts.dts_result(h), o)


@pytest.mark.parametrize("policy,flag", [(dts.DTS_POLICY_DARTS_LRU, oracle.F_LRU),
                                         (dts.DTS_POLICY_EAGER_LRU, oracle.F_EAGER | oracle.F_LRU)])
def test_run_n_devices_lru_policies(policy, flag):
    inst = gen.matmul2d(24, M=10, K=3)
    g = dts.schedule(inst, policy=policy, n_devices=2)
    assert_parity(g, oracle.run(inst, flags=1 | flag))


@pytest.mark.parametrize("W", [1, 2])
def test_run_n_devices_window(W):
    """Task-sharded runs with a prefetch window and the tight capacity (Belady, R29)."""
    inst = gen.random_shared(3000, 256, 3, M=8, K=3, seed=W)
    row = 3 * int(inst.data_size[0])
    inst = inst.with_(mem_capacity=max(1, W) * row)
    g = dts.schedule(inst, W=W, n_devices=3)
    o = oracle.run(inst, W=W)
    assert_parity(g, o)

"""Multi-process (world size 2, gloo, CPU) tests of the multi-GPU host logic:
LPT sharding of independent instances and the max/sum-over-ranks timing
reductions bench.py uses.  No GPU needed."""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

import gen
from paper_conf_ipps_gonthiermt22_b200.shard import instance_cost, lpt_assign, shard


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, costs, q):
    import torch.distributed as dist
    from paper_conf_ipps_gonthiermt22_b200.shard import reduce_over_ranks, shard as shard_fn
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    mine = shard_fn(costs, rank, world)
    got = [None] * world
    dist.all_gather_object(got, mine)
    load = sum(costs[i] for i in mine)
    mx, = reduce_over_ranks([load], "max")
    tot, = reduce_over_ranks([load], "sum")
    dist.barrier()
    dist.destroy_process_group()
    q.put((rank, got, load, mx, tot))


def _sweep_costs():
    costs = []
    for (N, M, K) in gen.sweep_params():
        costs.append(instance_cost(N * N, 2 * N))
    return costs


def test_lpt_single_process_properties():
    costs = _sweep_costs()
    assert len(costs) == 4096
    for world in (1, 2, 4, 8):
        parts = lpt_assign(costs, world)
        flat = sorted(i for p in parts for i in p)
        assert flat == list(range(len(costs))), "every instance exactly once"
        loads = [sum(costs[i] for i in p) for p in parts]
        # LPT bound: max - min <= the largest single cost
        assert max(loads) - min(loads) <= max(costs) + 1e-6
        assert max(loads) <= sum(costs) / world + max(costs)
    assert lpt_assign(costs, 8) == lpt_assign(list(costs), 8), "deterministic"


def test_shard_two_ranks_gloo():
    costs = _sweep_costs()
    port = _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, costs, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = sorted(q.get(timeout=120) for _ in procs)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    (_, got0, load0, mx0, tot0), (_, got1, load1, mx1, tot1) = res
    assert got0 == got1
    a, b = got0
    assert not set(a) & set(b), "shards are disjoint"
    assert sorted(a + b) == list(range(len(costs))), "shards cover the sweep"
    assert a == shard(costs, 0, 2) and b == shard(costs, 1, 2)
    assert mx0 == mx1 == max(load0, load1)
    assert tot0 == pytest.approx(load0 + load1)


# ---- task-sharded single instance (§8(e) second mode): host logic
def _shard_worker(rank, world, port, q):
    import torch.distributed as dist
    import paper_conf_ipps_gonthiermt22_b200 as dts
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    inst = gen.config_instances("C4b")[0]
    h = dts.create(inst)
    dts.dts_shard_set(h, world, rank)
    rng = dts.dts_shard_range(h)
    got = [None] * world
    dist.all_gather_object(got, rng)
    # the handle exchange the multi-GPU path uses (tests/shard_ipc_worker.py):
    # fixed-size blobs gathered in rank order; without a GPU export must fail loudly
    try:
        blob = dts.dts_shard_export(h, 0)
        err = None
    except dts.DtsError as e:
        blob, err = bytes([rank]) * dts.DTS_SHARD_HANDLE_BYTES, e.status
    blobs = [None] * world
    dist.all_gather_object(blobs, blob)
    dist.barrier()
    dist.destroy_process_group()
    q.put((rank, got, err, [b[:1] for b in blobs], len(blobs[0])))


def test_task_shard_ranges_two_ranks_gloo():
    port = _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_shard_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = sorted(q.get(timeout=180) for _ in procs)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    (_, g0, e0, b0, n0), (_, g1, e1, b1, n1) = res
    assert g0 == g1
    (lo0, hi0), (lo1, hi1) = g0
    m = 1 << 20
    assert lo0 == 0 and hi0 == lo1 and hi1 == m, "consecutive ranges covering every task"
    assert abs(hi0 - m // 2) <= 1, "about E/G edges each (3 inputs per task)"
    import torch
    if not torch.cuda.is_available():
        assert e0 == e1 == -4, "no GPU: dts_shard_export reports DTS_E_CUDA"
        assert b0 == b1 == [bytes([0]), bytes([1])] and n0 == n1 == 128


def test_task_shard_ranges_single_process():
    import paper_conf_ipps_gonthiermt22_b200 as dts
    for inst in (gen.config_instances("C4a")[0], gen.fig1(), gen.matmul2d(10, M=6, K=1)):
        h = dts.create(inst)
        for G in (1, 2, 3, 8, 16):
            rs = []
            for g in range(G):
                dts.dts_shard_set(h, G, g)
                rs.append(dts.dts_shard_range(h))
            assert rs[0][0] == 0 and rs[-1][1] == inst.m
            assert all(rs[i][1] == rs[i + 1][0] for i in range(G - 1))
            assert all(lo <= hi for lo, hi in rs)
            E = int(inst.task_ptr[-1])
            tp = np.asarray(inst.task_ptr)
            if G > 1 and E >= 100 * G:
                loads = [int(tp[hi] - tp[lo]) for lo, hi in rs]
                assert max(loads) - min(loads) <= 2 * int(np.diff(tp).max()) + 1
        with pytest.raises(dts.DtsError):
            dts.dts_shard_set(h, 0, 0)
        with pytest.raises(dts.DtsError):
            dts.dts_shard_set(h, 4, 4)

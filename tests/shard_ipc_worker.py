"""One rank of a task-sharded single instance (second mode),
one process per shard: dts_shard_set / dts_shard_export, an all-gather of the
IPC handles over torch.distributed (gloo: the handles are 128-byte host
blobs), dts_shard_connect, then dts_run on every rank at once -- the kernels
exchange through each other's memory (NVLink peer memory on an 8xB200 box;
the same B200 when the ranks share one device, as in tests/test_gpu_shard.py).

    RANK=r WORLD_SIZE=G MASTER_ADDR=127.0.0.1 MASTER_PORT=p python tests/shard_ipc_worker.py

Each rank checks its (replicated) schedule against the CPU oracle and prints
"PARITY OK".
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))

import torch  # noqa: E402
import torch.distributed as dist  # noqa: E402

import gen  # noqa: E402
import oracle  # noqa: E402
import paper_conf_ipps_gonthiermt22_b200 as dts  # noqa: E402
from parity import assert_parity  # noqa: E402


def main():
    rank, world = int(os.environ["RANK"]), int(os.environ["WORLD_SIZE"])
    dist.init_process_group("gloo", rank=rank, world_size=world)
    device = int(os.environ.get("LOCAL_RANK", rank)) % max(1, torch.cuda.device_count())
    cases = [gen.config_instances("C1")[0], gen.random_shared(300, 64, 3, M=8, K=3, seed=7),
             gen.matmul2d(12, M=8, K=2)]
    for inst in cases:
        h = dts.create(inst)
        dts.dts_shard_set(h, world, rank)
        mine = dts.dts_shard_export(h, device)
        allh = [None] * world
        dist.all_gather_object(allh, mine)
        dts.dts_shard_connect(h, allh)
        dist.barrier()  # every peer mapped before any kernel exchanges
        o = dts.dts_run_opts_default(device=device)
        for _ in range(2):  # twice: exchange numbers of the next run start above the last
            dts.dts_run(h, dts.DTS_POLICY_DARTS_LUF, o)
            r = dts.dts_result(h)
            assert_parity(r, oracle.run(inst))
        lo, hi = dts.dts_shard_range(h)
        print(f"rank {rank}/{world} device {device}: {inst.name} tasks [{lo}, {hi}) PARITY OK", flush=True)
        dist.barrier()  # nobody unmaps (destroys) while a peer still runs
        del h
    dist.destroy_process_group()


if __name__ == "__main__":
    main()

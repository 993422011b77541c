#!/usr/bin/env python
"""bench.py -- DARTS+LUF scheduling throughput on B200 (driver contract).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
                    [--workload C2|C1|C3|C4a|C4b|C5]

A *step* is one pass of the whole hot path (device CSR
build, state init, the device-resident DARTS+LUF decision loop, result
assembly) over one batch of synthetic instances.  Default workload = BASELINE
config 4, the largest single-GPU configuration: the Cholesky task set (C4a,
1,004,731 tasks) and the random shared-input task set (C4b, 2^20 tasks x 3
inputs), K = 8 simulated GPUs, both scheduled by ONE batched launch of the
decision loop (one CTA each, dts_sweep_run).  C1, C2, C3, C4a, C4b and C5
are available with --workload.

Multi-GPU (torchrun, one process per B200): independent instances need no
communication; C4, C2 and the single-instance workloads
run one copy per rank ("weak": replicas only -- one instance's decisions are
a sequential chain), C5 (the 4,096-instance sweep) is sharded across ranks
by LPT ("strong").  Time = max over ranks of the device time (CUDA events).

value = decisions/s (served requests, reading R21) over all ranks, inputs
resident in HBM.  e2e = the same through the public API from the caller's
host arrays: dts_instance_create (validation + copy), upload, run, the
device->host read of every result and dts_instance_destroy inside the timed
region (C5: instances created once, see e2e.scope).  roofline = SURVEY.md
§8(d)'s algorithmic bytes of the loop kernel (from the kernel's counters,
DESIGN.md "Roofline") / its device time.  --impl reference times the plain
CPU oracle (oracle/) on the host cores instead (the reference arm).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time
from concurrent.futures import ThreadPoolExecutor

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import gen  # noqa: E402

METRIC = "DARTS+LUF scheduling decisions/sec and HBM GB/s at 1/2/4/8 B200; bytes loaded"
UNIT = "decisions/s"

WORKLOADS = {
    "C1": "2D tiled matmul 10x10 tiles (100 tasks, 20 data), K=1, M=6 data",
    "C2": "2D tiled matmul N=10..100 (step 10) x K in {2,4}, M=35 data (500 MiB) per simulated GPU",
    "C3": "3D tiled matmul N=40 (64,000 tasks, 3,200 tiles), K=4, M=142 tiles (500 MiB)",
    "C4a": "Cholesky task set N=181 tiles (1,004,731 tasks, 16,471 tiles), K=8, M=142",
    "C4b": "random shared-input tasks (2^20 tasks x 3 inputs over 2^14 data), K=8, M=1024",
    "C4": "config 4: Cholesky task set N=181 (C4a, 1,004,731 tasks, M=142) + random shared-input "
          "tasks (C4b, 2^20 x 3 inputs, M=1024), K=8, one batched launch",
    "C5": "sweep of 4,096 2D instances (N 5..160 x M 4..128 x K 1..8), sharded over ranks",
}


def _peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured"
    except Exception:
        return 6650.0, "fallback"


def _traffic(workload):
    """Per-launch DRAM bytes (dram__bytes_read.sum + dram__bytes_write.sum) of
    the loop kernel from the committed ncu --set full summary of this round's
    build (profiles/ncu_full_<workload>.json, tools/ncu_summary.py), else None."""
    p = os.path.join(ROOT, "profiles", f"ncu_full_{workload}.json")
    try:
        d = json.load(open(p))
        return int(d["dram_bytes_per_launch"])
    except Exception:
        return None


def bytes_8d(r, inst):
    """SURVEY.md §8(d) algorithmic bytes of one instance's decision loop
    (DESIGN.md "Roofline"): per scan 4 m_avail + 4.125 n, per load / evict of
    D 12 deg(D), per allocated task 4 K + 8 E/m -- from the kernel's counters
    (parity-tested against the oracle's)."""
    abar = inst.E / max(inst.m, 1)
    return (4.0 * r.sum_avail_at_scans + 4.125 * inst.n * r.n_scans
            + 12.0 * r.sum_deg_loads_evictions + (4.0 * inst.K + 8.0 * abar) * r.n_allocations)


class Clocks:
    """nvidia-smi sampler running during the timed region."""
    Q = ("clocks.sm,clocks.max.sm,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap,utilization.gpu")

    def __init__(self, dev):
        self.dev = dev
        self.proc = None
        self.lines = []

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.dev), f"--query-gpu={self.Q}",
                 "--format=csv,noheader,nounits", "-lms", "100"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
            t0 = time.time()  # nvidia-smi's first sample before the region starts
            while not self.lines and time.time() - t0 < 3.0:
                time.sleep(0.01)
        except Exception:
            self.proc = None
        self.n0 = len(self.lines)
        return self

    def _read(self):
        for ln in self.proc.stdout:
            self.lines.append(ln.strip())

    def __exit__(self, *a):
        if self.proc is not None:
            t0 = time.time()  # a region shorter than the 100 ms period: the sample that closes it
            while len(self.lines) <= self.n0 and time.time() - t0 < 1.0:
                time.sleep(0.005)
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()
            self.t.join(timeout=2)

    def summary(self):
        sm, mx, reasons = [], None, set()
        for ln in self.lines:
            f = [x.strip() for x in ln.split(",")]
            if len(f) < 8:
                continue
            try:
                s, m_, util = float(f[0]), float(f[1]), float(f[7])
            except ValueError:
                continue
            mx = m_
            if util > 0:
                sm.append(s)
            for name, v in zip(("hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown",
                                "sw_power_cap"), f[3:7]):
                if v.lower() == "active":
                    reasons.add(name)
        if not sm:
            sm = [float(ln.split(",")[0]) for ln in self.lines
                  if ln and ln.split(",")[0].strip().replace(".", "").isdigit()]
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": mx,
                "reasons": sorted(reasons), "samples": len(self.lines)}


def workload_instances(name, rank, world):
    if name == "C4":
        return gen.config_instances("C4a") + gen.config_instances("C4b"), "weak"
    if name == "C5":
        from paper_conf_ipps_gonthiermt22_b200.shard import instance_cost, shard
        params = gen.sweep_params()
        # strong scaling: the 4,096 independent instances are sharded by LPT on
        # a cost estimate; no data-path collective
        costs = [instance_cost(N * N, 2 * N) for (N, M, K) in params]
        return [gen.sweep_instance(*params[i]) for i in shard(costs, rank, world)], "strong"
    return gen.config_instances(name), "weak"


# ------------------------------------------------------------------ oracle
ORACLE_FLAGS = 1  # set in main(): FALLBACK2 | policy | OPTI


def oracle_sample(insts, budget_s, threads):
    """Time the plain CPU oracle (as it stands) over the batch, repeated until
    budget_s elapsed; one instance per thread (ctypes releases the GIL)."""
    import oracle
    oracle._load()
    done_dec = 0
    n_batches = 0
    t0 = time.perf_counter()
    with ThreadPoolExecutor(max_workers=threads) as ex:
        while True:
            # biggest instances first so the pool stays busy
            order = sorted(insts, key=lambda i: -i.E)
            rs = list(ex.map(lambda i: oracle.run(i, flags=ORACLE_FLAGS), order))
            done_dec += sum(r.n_served for r in rs)
            n_batches += 1
            if time.perf_counter() - t0 >= budget_s:
                break
    dt = time.perf_counter() - t0
    return done_dec / dt, dt, n_batches, done_dec


def oracle_prefix_sample(inst, budget_s):
    """Large single instances: the oracle on a prefix of served requests sized
    to ~budget_s (the plain oracle costs O(E) per scan)."""
    import oracle
    n = 200
    while True:
        t0 = time.perf_counter()
        r = oracle.run(inst, max_served=n, flags=ORACLE_FLAGS)
        dt = time.perf_counter() - t0
        if dt >= budget_s / 4 or n >= inst.m:
            return r.n_served / dt, dt, r.n_served
        n = min(inst.m, int(n * max(2.0, budget_s / 4 / max(dt, 1e-3))))


def run_reference(args, rank, world):
    if rank != 0:
        return
    insts, scaling = workload_instances(args.workload, 0, 1)
    cores = os.cpu_count() or 1
    big = args.workload in ("C4a", "C4b", "C4")
    for _ in range(args.warmup):
        if big:
            oracle_prefix_sample(insts[0], 2.0)
        else:
            oracle_sample(insts[:min(len(insts), 64)], 0.0, cores)
    times, decs = [], []
    for _ in range(args.steps):
        if big:
            dt = nd = 0
            parts = []
            for inst in insts:  # C4: a prefix of each instance
                _, dti, ndi = oracle_prefix_sample(inst, 8.0 / len(insts))
                dt += dti
                nd += ndi
                parts.append(f"{ndi} of {inst.name}")
            sample = "prefix of the served requests (" + ", ".join(parts) + "), 1 thread"
            thr = 1
        else:
            sub = insts if args.workload != "C5" else insts[::16]
            rate, dt, nb, nd = oracle_sample(sub, 0.0, cores)
            sample = (f"{len(sub)} instances of {args.workload} (the whole batch)" if args.workload != "C5"
                      else f"{len(sub)} of the 4,096 C5 instances (every 16th)") + f", {cores} threads"
            thr = cores
        times.append(dt)
        decs.append(nd)
    value = sum(decs) / sum(times)
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": 1e3 * sum(times) / len(times), "higher_is_better": True,
            "scaling": scaling, "vs_baseline": None, "dtype": "int64", "data": "synthetic",
            "config": {"workload": f"{args.workload}: {WORKLOADS[args.workload]}",
                       "policy": args.policy + ("+opti" if args.opti else "") + " (3inputs fallback on)"},
            "cpu_baseline": {"value": value, "unit": UNIT, "cores": thr, "kind": "oracle",
                             "sample": sample},
            "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ------------------------------------------------------------------ ours
def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--workload", default="C4", choices=list(WORKLOADS))
    ap.add_argument("--policy", default="darts_luf", choices=["darts_luf", "darts_lru", "eager_lru"],
                    help="DARTS+LUF (the method) or a comparison policy of the paper")
    ap.add_argument("--opti", action="store_true", help="OPTI variant (PAPER.md:2121-2124)")
    ap.add_argument("--cpu-budget", type=float, default=10.0,
                    help="seconds of oracle time for cpu_baseline (rank 0, N=1)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--mode", default="replica", choices=["replica", "shard"],
                    help="N>1 with a single-instance workload (C3/C4): 'replica' = every rank "
                         "schedules its own copy (weak); 'shard' = ONE instance task-sharded over "
                         "the ranks, exchanging through NVLink peer memory (strong, SURVEY §8(e))")
    ap.add_argument("--shards", type=int, default=1,
                    help="single-instance workloads at N=1: task shards as co-resident CTAs of "
                         "one B200 (dts_shard_group_run)")
    args = ap.parse_args()

    global ORACLE_FLAGS
    ORACLE_FLAGS = 1 | {"darts_luf": 0, "darts_lru": 16, "eager_lru": 48}[args.policy] | (8 if args.opti else 0)
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))

    if args.impl == "reference":
        run_reference(args, rank, world)
        return

    import torch
    import torch.distributed as dist
    import paper_conf_ipps_gonthiermt22_b200 as dts

    if not torch.cuda.is_available():
        raise SystemExit("bench.py: no CUDA device (libdts has no CPU path)")
    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    dts.load_library()
    dev = local
    stream = torch.cuda.current_stream()
    sptr = stream.cuda_stream

    insts, scaling = workload_instances(args.workload, rank, world)
    single = args.workload in ("C3", "C4a", "C4b")  # one large instance
    xsh = single and world > 1 and args.mode == "shard"  # one instance over the ranks
    gsh = single and not xsh and args.shards > 1          # one instance over CTAs of this GPU
    if gsh:
        handles = [dts.create(insts[0]) for _ in range(args.shards)]
    else:
        handles = [dts.create(i) for i in insts]
    if xsh:
        scaling = "strong"
    policy = {"darts_luf": dts.DTS_POLICY_DARTS_LUF, "darts_lru": dts.DTS_POLICY_DARTS_LRU,
              "eager_lru": dts.DTS_POLICY_EAGER_LRU}[args.policy]
    opts = dts.dts_run_opts_default(device=dev, cuda_stream=sptr,
                                    flags=dts.DTS_F_FALLBACK2 | (dts.DTS_F_OPTI if args.opti else 0))
    if xsh:  # map the peers' shard state (CUDA IPC over NVLink); handles are host blobs
        dts.dts_shard_set(handles[0], world, rank)
        blobs = [None] * world
        dist.all_gather_object(blobs, dts.dts_shard_export(handles[0], dev))
        dts.dts_shard_connect(handles[0], blobs)
        dist.barrier()
    for h in handles:
        dts.dts_instance_upload(h, dev, sptr)
    torch.cuda.synchronize()

    def step():
        if gsh:
            dts.dts_shard_group_run(handles, policy, opts)
        elif single:
            for h in handles:
                dts.dts_run(h, policy, opts)
        else:
            dts.dts_sweep_run(handles, policy, opts)

    flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.int32, device="cuda")  # > 126 MB L2

    def barrier():
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()

    for _ in range(max(args.warmup, 0)):
        step()
    barrier()
    res0 = [dts.dts_result(h) for h in handles]
    decisions = sum(r.n_served for r in res0)
    if gsh or xsh:  # every shard holds the (same) whole schedule: count it once
        decisions = res0[0].n_served if (gsh or rank == 0) else 0
    assert decisions == sum(i.m for i in insts) or (xsh and rank > 0), "not every task scheduled"

    # ---- device-resident timed region (Python's cyclic GC paused, as timeit does:
    # a full collection over the thousands of handle objects of a C5 batch
    # stalled the host for ~100 ms inside some steps, profiles/r02v_host_c5.txt)
    import gc
    gc.collect()
    gc.disable()
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
           for _ in range(args.steps)]
    loop_ms_steps = []
    barrier()
    with Clocks(dev) as clk:
        l0 = dts.dts_kernel_launches()
        enq = []
        for i in range(args.steps):
            flush.zero_()  # L2 flush between timed steps (outside the events)
            evs[i][0].record(stream)
            t_enq = time.perf_counter()
            step()
            enq.append(time.perf_counter() - t_enq)
            evs[i][1].record(stream)
            # the loop kernel's own launch time (library events on the same
            # stream); waits for this step, so the next step's enqueue starts
            # after it -- outside both events
            loop_ms_steps.append(max(dts.dts_run_times(h)[0] for h in handles))
        barrier()
        launches = dts.dts_kernel_launches() - l0
    step_ms = [a.elapsed_time(b) for a, b in evs]
    if os.environ.get("DTS_BENCH_DEBUG"):
        print("host enqueue ms", [round(1e3 * x, 2) for x in enq], "step ms", [round(x, 2) for x in step_ms],
              "loop ms", [round(x, 2) for x in loop_ms_steps], file=sys.stderr, flush=True)
    rs = [dts.dts_result(h) for h in handles]  # last step's results (after the region)
    loop_ms = sum(loop_ms_steps) / len(loop_ms_steps)
    alg = sum(r.alg_bytes for r in rs)
    # §8(d) bytes of one launch (a task-sharded group counts the instance once)
    b8d = sum(bytes_8d(r, i) for r, i in zip(rs, insts if not (gsh or xsh) else insts[:1]))
    bytes_loaded = sum(r.bytes_loaded for r in rs)
    n_loads = sum(r.n_loads for r in rs)
    n_scans = sum(r.n_scans for r in rs)
    ms = sum(step_ms) / len(step_ms)

    # ---- e2e: the public API from the caller's host arrays, every step
    e2e_ms = []
    create_each_step = args.workload != "C5" and not (gsh or xsh)
    h2d = sum(8 * (i.m + 1) + 4 * i.E + 8 * i.n + (8 * i.m if i.task_ns is not None else 0)
              for i in insts) * (args.shards if gsh else 1)
    d2h = 0
    barrier()
    n_e2e = max(2, args.steps // 2)
    for i in range(n_e2e + 1):  # the first pass is an untimed warm-up (the library's pools)
        t0 = torch.cuda.Event(enable_timing=True)
        t1 = torch.cuda.Event(enable_timing=True)
        flush.zero_()
        t0.record(stream)
        if create_each_step:  # create (host validation + copy) .. destroy, all timed
            hs = [dts.create(x) for x in insts]
            for h in hs:
                dts.dts_instance_upload(h, dev, sptr)
            if single:
                for h in hs:
                    dts.dts_run(h, policy, opts)
            else:
                dts.dts_sweep_run(hs, policy, opts)
        else:
            hs = handles
            for h in hs:
                dts.dts_instance_upload(h, dev, sptr)
            step()
        dts.dts_fetch_results(hs)  # all instances' results to host, two waits
        out = [dts.dts_result(h, copy=False) for h in hs]  # views of the pinned result buffers
        d2h = sum(8 * (r.K + 1) + 4 * r.n_served * 3 + 16 * len(r.task_start) + 32 * len(r.events)
                  + 128 for r in out)
        assert sum(r.n_served for r in out) == decisions or xsh or gsh
        del out
        if create_each_step:
            del hs  # dts_instance_destroy (inside the timed region)
        t1.record(stream)
        t1.synchronize()
        if i > 0:
            e2e_ms.append(t0.elapsed_time(t1))
    e2e_avg = sum(e2e_ms) / len(e2e_ms)
    if os.environ.get("DTS_BENCH_DEBUG"):
        print("e2e ms", [round(x, 2) for x in e2e_ms], file=sys.stderr, flush=True)
    gc.enable()

    # ---- max over ranks (device times), sum of the work
    from paper_conf_ipps_gonthiermt22_b200.shard import reduce_over_ranks
    ms, e2e_avg, loop_ms_max = reduce_over_ranks([ms, e2e_avg, loop_ms], "max", device="cuda")
    all_dec, all_alg = reduce_over_ranks([decisions, alg], "sum", device="cuda")

    if rank == 0:
        peak, peak_src = _peaks()
        achieved = (b8d / 1e9) / (loop_ms / 1e3) if loop_ms > 0 else 0.0  # GB/s, this rank's launch
        cpu = None
        if world == 1 and not args.no_cpu_baseline:
            cores = os.cpu_count() or 1
            if args.workload in ("C4a", "C4b", "C3", "C4"):
                nd, dt, parts = 0, 0.0, []
                for inst in insts:
                    _, dti, ndi = oracle_prefix_sample(inst, args.cpu_budget / len(insts))
                    nd += ndi
                    dt += dti
                    parts.append(f"{ndi} of {inst.name}")
                cpu = {"value": nd / dt, "unit": UNIT, "cores": 1, "kind": "oracle",
                       "sample": "prefix of the served requests (" + ", ".join(parts)
                                 + f"; {dt:.1f} s, 1 thread)"}
            else:
                sub = insts if args.workload != "C5" else insts[::16]
                rate, dt, nb, nd = oracle_sample(sub, args.cpu_budget, cores)
                cpu = {"value": rate, "unit": UNIT, "cores": cores, "kind": "oracle",
                       "sample": f"{nb} passes over {len(sub)} instances of {args.workload}"
                                 f" ({nd} decisions, {dt:.1f} s, one instance per thread)"}
        clocks = clk.summary()
        kind = max(r.loop_kind for r in rs)
        kname = {1: "dts_cta_kernel", 2: "dts_cta_kernel_fast", 3: "dts_warp_kernel"}.get(kind, "?")
        launch = ("one batched loop launch, one WARP per instance (32-thread CTAs, instances pulled "
                  "longest first)" if kind == 3 else
                  "one batched loop launch, one CTA per instance" if len(insts) < 296 else
                  "one batched loop launch of 128-thread CTAs (4 per SM), one CTA per instance, "
                  "longest first") if not single \
            else (f"one cooperative launch: the instance task-sharded over {args.shards} CTAs"
                  if gsh else f"one loop launch per rank: the instance task-sharded over "
                  f"{world} B200s, peer-memory exchanges" if xsh
                  else "one loop launch (one warp) per instance" if kind == 3
                  else "one loop launch (one CTA) per instance")
        line = {
            "metric": METRIC, "value": all_dec / (ms / 1e3), "unit": UNIT, "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms,
            "higher_is_better": True, "scaling": scaling, "vs_baseline": None,
            "dtype": "int32", "data": "synthetic",
            "config": {"workload": f"{args.workload}: {WORKLOADS[args.workload]}",
                       "policy": args.policy + ("+opti" if args.opti else "") + " (3inputs fallback on)",
                       "instances_per_rank": len(insts), "decisions_per_step": int(all_dec),
                       "l2": "flushed between timed steps (256 MiB write)", "launch": launch},
            "e2e": {"value": all_dec / (e2e_avg / 1e3), "unit": UNIT,
                    "h2d_bytes_per_step": int(h2d), "d2h_bytes_per_step": int(d2h),
                    "scope": ("dts_instance_create from host arrays, upload, run, result D2H, destroy"
                              if create_each_step else
                              "upload (from the library's pinned copy), run, result D2H; "
                              "instances created once outside the timed region")
                             + f"; mean of {n_e2e} passes after one untimed warm-up pass"},
            "gpu_launches": int(launches),
            "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                         "frac": achieved / peak, "traffic": _traffic(args.workload),
                         "kernel": kname, "peak_source": peak_src,
                         "bytes": "SURVEY.md §8(d) algorithmic bytes per launch: 4*sum(m_avail at scans)"
                                  " + 4.125*n*scans + 12*sum(deg over loads/evictions)"
                                  " + (4K + 8E/m)*allocations (kernel counters = oracle counters)",
                         "alg_bytes_per_launch": int(b8d), "launch_ms": loop_ms,
                         "launch_ms_steps": [round(x, 3) for x in loop_ms_steps],
                         "kernel_model_bytes_per_launch": int(alg)},
            "bytes_loaded": int(bytes_loaded), "n_loads": int(n_loads), "n_scans": int(n_scans),
            "cpu_baseline": cpu,
            "clocks": clocks,
        }
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()

"""Independent schedule validator.

Replays a schedule -- service order, load/evict trace, task times -- against
the model of PAPER.md §III and checks what must hold for ANY valid schedule,
whatever tie-breaking produced it:

* every task is processed exactly once (sum_k nb_k = m);
* a step evicts, then loads the missing inputs, then processes
  (PAPER.md:285-295): loads are inputs of the task being served and not yet
  resident; D(T) is resident when T runs;
* no input of a buffered task is evicted (V(k,i) ∩ D(T_sigma(k,i)) = ∅,
  PAPER.md:397-399) -- except by Alg. 6 l.6-7 (Belady, reading R29): only
  when every resident datum is a buffered input, only an input of the task
  running at the request and of no task not yet started, and it leaves
  memory when that task ends (the load it makes room for starts no earlier);
* request times follow R7 / R29 (W = 0: when the previous task ends; W >= 1:
  when the task W-1 places back starts, the first W at once);
* memory never exceeds the capacity (|L(k,i)| <= M);
* #loads, bytes and makespan are what the trace says (Obj. 2);
* the shared bus (Fig. 2) carries one transfer at a time, FIFO;
* bytes >= sum of the sizes of the distinct data used; loads <= E.

Shares no code with oracle/ or the CUDA path.
"""
from __future__ import annotations

import numpy as np


def validate(inst, serve_gpu, serve_task, events, task_start, task_end, *, W=0,
             bus_bps=12_000_000_000, complete=True):
    m, n, K = inst.m, inst.n, inst.K
    tp, td = inst.task_ptr, inst.task_data
    size = [int(x) for x in inst.data_size]
    dsets = [set(int(x) for x in td[tp[t]:tp[t + 1]]) for t in range(m)]
    cap = int(inst.mem_capacity)
    serve_gpu = [int(x) for x in serve_gpu]
    serve_task = [int(x) for x in serve_task]
    if complete:
        assert sorted(serve_task) == list(range(m)), "every task exactly once"
    else:
        assert len(set(serve_task)) == len(serve_task), "no task twice"

    mem = [set() for _ in range(K)]
    used = [0] * K
    gpu_free = [0] * K
    last = [-1] * K
    hist = [[] for _ in range(K)]   # tasks served on k, in order
    req = [0] * K                   # request time of k's next task (R7 / R29)
    bus_free = 0
    loads = evicts = 0
    nbytes = 0
    ev_i = 0
    ne = len(events)
    makespan = 0
    for T, k in zip(serve_task, serve_gpu):
        t = req[k]
        buf = [x for x in hist[k][-W:] if int(task_end[x]) > t] if W >= 1 else []
        running = [x for x in buf if int(task_start[x]) <= t]
        queued_inputs = set(dsets[T]).union(*[dsets[x] for x in buf if int(task_start[x]) > t])
        buffer_inputs = queued_inputs.union(*[dsets[x] for x in running])
        ready = 0
        mem_ready = t
        while ev_i < ne and int(events[ev_i]["task"]) == T and int(events[ev_i]["gpu"]) == k:
            e = events[ev_i]
            D, op = int(e["data"]), int(e["op"])
            if op == 1:
                assert D in mem[k], "evicting a non-resident datum"
                assert int(e["t"]) == int(e["t_end"])
                if D in buffer_inputs:  # Alg. 6 l.6-7 only (R29)
                    assert mem[k] <= buffer_inputs, "evicted a buffered input while another datum was free"
                    assert D not in queued_inputs, "evicted an input of a task not yet started"
                    ends = [int(task_end[x]) for x in running if D in dsets[x]]
                    assert ends and int(e["t"]) == max(ends), "Belady eviction not at the running task's end"
                else:
                    assert int(e["t"]) == t, "eviction not at the request time"
                mem_ready = max(mem_ready, int(e["t"]))
                mem[k].remove(D)
                used[k] -= size[D]
                evicts += 1
            else:
                assert D in dsets[T], "loaded a datum the task does not need"
                assert D not in mem[k], "loaded a resident datum"
                mem[k].add(D)
                used[k] += size[D]
                assert used[k] <= cap, "capacity exceeded"
                s, en = int(e["t"]), int(e["t_end"])
                dl = -(-size[D] * 1_000_000_000 // bus_bps)
                assert en - s == dl, "transfer time"
                assert s >= bus_free, "bus overlap / not FIFO"
                assert s >= mem_ready, "load before its memory was free"
                bus_free = en
                ready = max(ready, en)
                loads += 1
                nbytes += size[D]
            ev_i += 1
        assert dsets[T] <= mem[k], "inputs not resident at execution"
        st, en = int(task_start[T]), int(task_end[T])
        assert st >= ready and st >= gpu_free[k], "task started too early"
        tau = int(inst.task_ns[T]) if inst.task_ns is not None else int(inst.default_task_ns)
        assert en - st == tau, "task duration"
        gpu_free[k] = en
        last[k] = T
        hist[k].append(T)
        j = len(hist[k])
        req[k] = en if W == 0 else (t if j < W else int(task_start[hist[k][j - W]]))
        makespan = max(makespan, en)
    assert ev_i == ne, "trailing events not attached to a served task"
    used_data = set().union(*dsets) if m else set()
    if complete:
        assert nbytes >= sum(size[d] for d in used_data)
    assert loads <= int(tp[-1])
    return dict(n_loads=loads, n_evictions=evicts, bytes_loaded=nbytes, makespan=makespan)

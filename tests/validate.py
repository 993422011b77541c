"""Independent schedule validator.

Replays a schedule -- service order, load/evict trace, task times -- against
the model of PAPER.md §III and checks what must hold for ANY valid schedule,
whatever tie-breaking produced it:

* every task is processed exactly once (sum_k nb_k = m);
* a step evicts, then loads the missing inputs, then processes
  (PAPER.md:285-295): loads are inputs of the task being served and not yet
  resident; D(T) is resident when T runs;
* no input of a buffered task is evicted (V(k,i) ∩ D(T_sigma(k,i)) = ∅,
  PAPER.md:397-399);
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
    bus_free = 0
    loads = evicts = 0
    nbytes = 0
    ev_i = 0
    ne = len(events)
    makespan = 0
    for T, k in zip(serve_task, serve_gpu):
        buffer_inputs = set(dsets[T])
        if W >= 1 and last[k] >= 0 and int(task_end[last[k]]) > int(task_start[last[k]]):
            buffer_inputs |= dsets[last[k]]
        ready = 0
        first_t = None
        while ev_i < ne and int(events[ev_i]["task"]) == T and int(events[ev_i]["gpu"]) == k:
            e = events[ev_i]
            D, op = int(e["data"]), int(e["op"])
            if op == 1:
                assert D in mem[k], "evicting a non-resident datum"
                assert D not in buffer_inputs, "evicted an input of a buffered task"
                mem[k].remove(D)
                used[k] -= size[D]
                evicts += 1
                assert int(e["t"]) == int(e["t_end"])
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
                bus_free = en
                ready = max(ready, en)
                loads += 1
                nbytes += size[D]
                first_t = s if first_t is None else first_t
            ev_i += 1
        assert dsets[T] <= mem[k], "inputs not resident at execution"
        st, en = int(task_start[T]), int(task_end[T])
        assert st >= ready and st >= gpu_free[k], "task started too early"
        tau = int(inst.task_ns[T]) if inst.task_ns is not None else int(inst.default_task_ns)
        assert en - st == tau, "task duration"
        gpu_free[k] = en
        last[k] = T
        makespan = max(makespan, en)
    assert ev_i == ne, "trailing events not attached to a served task"
    used_data = set().union(*dsets) if m else set()
    if complete:
        assert nbytes >= sum(size[d] for d in used_data)
    assert loads <= int(tp[-1])
    return dict(n_loads=loads, n_evictions=evicts, bytes_loaded=nbytes, makespan=makespan)

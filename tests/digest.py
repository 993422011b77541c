"""Canonical SHA-256 digest of a schedule (used to compare full runs that are
too long to store): little-endian bytes of serve_gpu (int32), serve_task
(int32), task_start (int64), task_end (int64), then the events as packed
32-byte records (t int64, t_end int64, gpu int32, data int32, task int32,
op uint8, 3 zero bytes)."""
import hashlib

import numpy as np

EVENT_DTYPE = np.dtype([("t", "<i8"), ("t_end", "<i8"), ("gpu", "<i4"), ("data", "<i4"),
                        ("task", "<i4"), ("op", "u1"), ("pad", "u1", (3,))])


def digest(serve_gpu, serve_task, task_start, task_end, events):
    h = hashlib.sha256()
    h.update(np.ascontiguousarray(serve_gpu, dtype="<i4").tobytes())
    h.update(np.ascontiguousarray(serve_task, dtype="<i4").tobytes())
    h.update(np.ascontiguousarray(task_start, dtype="<i8").tobytes())
    h.update(np.ascontiguousarray(task_end, dtype="<i8").tobytes())
    ev = np.zeros(len(events), EVENT_DTYPE)
    for f in ("t", "t_end", "gpu", "data", "task", "op"):
        ev[f] = events[f]
    h.update(ev.tobytes())
    return h.hexdigest()

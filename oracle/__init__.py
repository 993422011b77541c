"""Plain CPU oracle for DARTS+LUF.  TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import this package.  The
product path (``paper_conf_ipps_gonthiermt22_b200`` / ``libdts.so``) never
imports, links or calls it, and shares no code with it.

* :func:`run` -- ctypes wrapper of ``dts_oracle.c`` (Alg. 5 + 3inputs +
  Alg. 6 + the integer time model, recomputed from definitions each step).
* :mod:`oracle.belady` -- Belady replay of a fixed schedule and brute force
  over all schedules of tiny instances.

Parity status per function: see DESIGN.md "Oracle pins".
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "dts_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

F_FALLBACK2 = 1
F_OPTI = 8
F_LRU = 16     # evict by LRU (not LUF): the paper's plain "DARTS" and "EAGER"
F_EAGER = 32   # EAGER task choice: shared FIFO queue in submission order
F_COUNT_DEG = 64  # measurement only: count sum of deg(D) over loads/evictions (slow)

POLICY_FLAGS = {"darts_luf": 0, "darts_lru": F_LRU, "eager_lru": F_EAGER | F_LRU}
DEFAULT_BUS_BPS = 12_000_000_000

EVENT_DTYPE = np.dtype([("t", "<i8"), ("t_end", "<i8"), ("gpu", "<i4"), ("data", "<i4"),
                        ("task", "<i4"), ("op", "u1"), ("pad", "u1", (3,))])


def build(force: bool = False) -> str:
    """Compile the oracle with gcc -O2 (plain C, no GPU)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-shared", "-fPIC", "-o", _LIB, _SRC])
    return _LIB


class _Result(C.Structure):
    _fields_ = [("serve_gpu", C.c_void_p), ("serve_task", C.c_void_p),
                ("task_start", C.c_void_p), ("task_end", C.c_void_p),
                ("events", C.c_void_p), ("events_cap", C.c_int64),
                ("n_events", C.c_int64), ("n_served", C.c_int64), ("n_loads", C.c_int64),
                ("n_evictions", C.c_int64), ("n_scans", C.c_int64), ("n_fallback2", C.c_int64),
                ("n_fallback_first", C.c_int64), ("n_belady", C.c_int64),
                ("n_idle_requests", C.c_int64), ("bytes_loaded", C.c_uint64),
                ("makespan", C.c_int64), ("n_wakes", C.c_int64),
                ("sum_avail_at_scans", C.c_int64), ("n_allocations", C.c_int64),
                ("sum_deg", C.c_int64)]


_lib = None


def _load():
    global _lib
    if _lib is None:
        # DTS_ORACLE_LIB: a deliberately mutated build of dts_oracle.c
        # (tests/oracle_mutants.py checks that the pins reject it)
        _lib = C.CDLL(os.environ.get("DTS_ORACLE_LIB") or build())
        _lib.or_run.restype = C.c_int
        _lib.or_run.argtypes = [C.c_int32, C.c_int32, C.c_void_p, C.c_void_p, C.c_void_p,
                                C.c_void_p, C.c_int64, C.c_uint64, C.c_int32, C.c_int32,
                                C.c_uint32, C.c_uint64, C.c_int64, C.POINTER(_Result)]
        assert _lib.or_event_size() == EVENT_DTYPE.itemsize
    return _lib


@dataclass
class OracleResult:
    serve_gpu: np.ndarray    # int32 [n_served], service order
    serve_task: np.ndarray   # int32 [n_served]
    task_start: np.ndarray   # int64 [m]
    task_end: np.ndarray     # int64 [m]
    events: np.ndarray       # EVENT_DTYPE [n_events]
    n_served: int
    n_loads: int
    n_evictions: int
    n_scans: int
    n_fallback2: int
    n_fallback_first: int
    n_belady: int
    n_idle_requests: int
    bytes_loaded: int
    makespan: int
    K: int
    n_wakes: int = 0
    sum_avail_at_scans: int = 0   # SURVEY §8(d) byte-model counters (measurement only)
    n_allocations: int = 0
    sum_deg: int = 0              # only with F_COUNT_DEG

    def orders(self):
        """Per-GPU task order sigma(k, .)."""
        return [self.serve_task[self.serve_gpu == k].copy() for k in range(self.K)]


def run(inst, W: int = 0, flags: int = F_FALLBACK2, bus_bps: int = DEFAULT_BUS_BPS,
        max_served: int = -1) -> OracleResult:
    """Run the oracle on a ``gen.Instance``-like object."""
    lib = _load()
    m, n = inst.m, inst.n
    tp = np.ascontiguousarray(inst.task_ptr, dtype=np.int64)
    td = np.ascontiguousarray(inst.task_data, dtype=np.int32)
    sz = np.ascontiguousarray(inst.data_size, dtype=np.uint64)
    tn = None if inst.task_ns is None else np.ascontiguousarray(inst.task_ns, dtype=np.int64)
    cap_ev = 2 * int(tp[-1]) + 16
    sg = np.full(max(m, 1), -1, np.int32)
    st = np.full(max(m, 1), -1, np.int32)
    ts = np.empty(max(m, 1), np.int64)
    te = np.empty(max(m, 1), np.int64)
    ev = np.zeros(cap_ev, EVENT_DTYPE)
    r = _Result(sg.ctypes.data, st.ctypes.data, ts.ctypes.data, te.ctypes.data, ev.ctypes.data,
                cap_ev)
    rc = lib.or_run(m, n, tp.ctypes.data, td.ctypes.data, sz.ctypes.data,
                    None if tn is None else tn.ctypes.data, int(inst.default_task_ns),
                    int(inst.mem_capacity), int(inst.K), int(W), int(flags), int(bus_bps),
                    int(max_served), C.byref(r))
    if rc != 0:
        raise RuntimeError(f"oracle failed rc={rc}")
    ns = r.n_served
    return OracleResult(sg[:ns].copy(), st[:ns].copy(), ts[:m].copy(), te[:m].copy(),
                        ev[:r.n_events].copy(), ns, r.n_loads, r.n_evictions, r.n_scans,
                        r.n_fallback2, r.n_fallback_first, r.n_belady, r.n_idle_requests,
                        r.bytes_loaded, r.makespan, int(inst.K), r.n_wakes,
                        r.sum_avail_at_scans, r.n_allocations, r.sum_deg)

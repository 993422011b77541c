"""Thin ctypes binding of libdts (include/dts.h): argument marshalling only.

Every step of the schedule runs in the CUDA kernels of ``libdts.so``; there is
no Python or CPU implementation here and no fallback: if the library or a
B200 is missing, the calls raise :class:`DtsError`.

The functions keep the C names (``dts_instance_create``, ``dts_run``,
``dts_result``, ...).  :func:`schedule` is the one-call convenience a user
makes: host arrays in, host result out.
"""
from __future__ import annotations

import ctypes as C
import os
from dataclasses import dataclass
from typing import Optional

import numpy as np

_PKG = os.path.dirname(os.path.abspath(__file__))
# DTS_PROFILE=1 loads the profiling build (per-phase cycle probes in
# dts_result_view.prof_cycles); otherwise prof_cycles reads 0.
LIB_PATH = os.path.join(_PKG, "lib", "libdts_prof.so" if os.environ.get("DTS_PROFILE") == "1"
                        else "libdts.so")

DTS_OK = 0
DTS_E_INVAL = -1
DTS_E_CAPACITY = -2
DTS_E_NOMEM = -3
DTS_E_CUDA = -4
DTS_E_STATE = -5
DTS_E_UNSUPPORTED = -6
DTS_POLICY_DARTS_LUF = 1
DTS_POLICY_DARTS_LRU = 2
DTS_POLICY_EAGER_LRU = 3
DTS_F_FALLBACK2 = 1
DTS_F_VERIFY = 2
DTS_F_NOFUSE = 4
DTS_F_OPTI = 8
DTS_F_PACKED = 16
DTS_F_GENERIC = 32
DTS_F_CTA = 64  # force the per-CTA loop where the one-warp loop applies (diagnostic)
LOOP_GENERIC, LOOP_CTA_FAST, LOOP_WARP = 1, 2, 3  # dts_result_view.loop_kind

EVENT_DTYPE = np.dtype([("t", "<i8"), ("t_end", "<i8"), ("gpu", "<i4"), ("data", "<i4"),
                        ("task", "<i4"), ("op", "u1"), ("pad", "u1", (3,))])

EXPORTED = ["dts_run_opts_default", "dts_instance_create", "dts_instance_upload", "dts_run",
            "dts_result", "dts_fetch_results", "dts_run_times", "dts_sweep_run", "dts_instance_destroy",
            "dts_status_str",
            "dts_last_error", "dts_version", "dts_kernel_launches",
            "dts_shard_set", "dts_shard_range", "dts_shard_export", "dts_shard_connect",
            "dts_shard_group_run"]
DTS_SHARD_HANDLE_BYTES = 128


class DtsError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{msg} (status {status})")
        self.status = status


class dts_run_opts(C.Structure):
    _fields_ = [("flags", C.c_uint32), ("lookahead_W", C.c_uint32),
                ("bus_bytes_per_s", C.c_uint64), ("device", C.c_int32),
                ("block_threads", C.c_int32), ("smem_budget", C.c_int32), ("n_devices", C.c_int32),
                ("max_served", C.c_int64), ("cuda_stream", C.c_void_p)]


class dts_result_view(C.Structure):
    _fields_ = [("K", C.c_int32), ("n_tasks", C.c_int32),
                ("gpu_task_ptr", C.c_void_p), ("gpu_task_ids", C.c_void_p),
                ("serve_gpu", C.c_void_p), ("serve_task", C.c_void_p),
                ("task_start_ns", C.c_void_p), ("task_end_ns", C.c_void_p),
                ("n_events", C.c_int64), ("events", C.c_void_p),
                ("bytes_loaded", C.c_uint64), ("n_loads", C.c_int64), ("n_evictions", C.c_int64),
                ("makespan_ns", C.c_int64), ("makespan_s", C.c_double),
                ("n_served", C.c_int64), ("n_scans", C.c_int64), ("n_fallback2", C.c_int64),
                ("n_fallback_first", C.c_int64), ("n_belady", C.c_int64),
                ("n_idle_requests", C.c_int64), ("n_verify_err", C.c_int64),
                ("alg_bytes", C.c_uint64),
                ("scan_alg_bytes", C.c_uint64), ("loop_ms", C.c_float), ("total_ms", C.c_float),
                ("prof_cycles", C.c_int64 * 16), ("sum_avail_at_scans", C.c_int64),
                ("n_allocations", C.c_int64), ("sum_deg_loads_evictions", C.c_int64),
                ("loop_kind", C.c_int32), ("reserved", C.c_int32)]


_lib = None


def load_library(path: str = LIB_PATH):
    """Load libdts.so (built in-tree by ``build.py``); raises if absent."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(path):
        raise DtsError(DTS_E_CUDA, f"libdts.so not built at {path}: run __graft_entry__.build()")
    lib = C.CDLL(path)
    P = C.c_void_p
    lib.dts_run_opts_default.argtypes = [C.POINTER(dts_run_opts)]
    lib.dts_run_opts_default.restype = None
    lib.dts_instance_create.argtypes = [C.c_int32, C.c_int32, P, P, P, P, C.c_int64, C.c_uint64,
                                        C.c_int32, C.POINTER(C.c_void_p)]
    lib.dts_instance_create.restype = C.c_int
    lib.dts_instance_upload.argtypes = [P, C.c_int32, P]
    lib.dts_instance_upload.restype = C.c_int
    lib.dts_run.argtypes = [P, C.c_int, C.POINTER(dts_run_opts)]
    lib.dts_run.restype = C.c_int
    lib.dts_result.argtypes = [P, C.POINTER(dts_result_view)]
    lib.dts_result.restype = C.c_int
    lib.dts_sweep_run.argtypes = [C.POINTER(C.c_void_p), C.c_int32, C.c_int,
                                  C.POINTER(dts_run_opts), C.POINTER(C.c_int32), C.c_int32]
    lib.dts_sweep_run.restype = C.c_int
    if hasattr(lib, "dts_fetch_results"):  # (older builds, tools/lib_ab.py, lack it)
        lib.dts_fetch_results.argtypes = [C.POINTER(C.c_void_p), C.c_int32]
        lib.dts_fetch_results.restype = C.c_int
    lib.dts_run_times.argtypes = [P, C.POINTER(C.c_float), C.POINTER(C.c_float)]
    lib.dts_run_times.restype = C.c_int
    lib.dts_instance_destroy.argtypes = [P]
    lib.dts_instance_destroy.restype = None
    lib.dts_status_str.argtypes = [C.c_int]
    lib.dts_status_str.restype = C.c_char_p
    lib.dts_last_error.argtypes = []
    lib.dts_last_error.restype = C.c_char_p
    lib.dts_kernel_launches.argtypes = []
    lib.dts_kernel_launches.restype = C.c_uint64
    lib.dts_version.argtypes = []
    lib.dts_version.restype = C.c_uint32
    lib.dts_shard_set.argtypes = [P, C.c_int32, C.c_int32]
    lib.dts_shard_set.restype = C.c_int
    lib.dts_shard_range.argtypes = [P, C.POINTER(C.c_int32), C.POINTER(C.c_int32)]
    lib.dts_shard_range.restype = C.c_int
    lib.dts_shard_export.argtypes = [P, C.c_int32, P]
    lib.dts_shard_export.restype = C.c_int
    lib.dts_shard_connect.argtypes = [P, P]
    lib.dts_shard_connect.restype = C.c_int
    lib.dts_shard_group_run.argtypes = [C.POINTER(C.c_void_p), C.c_int32, C.c_int,
                                        C.POINTER(dts_run_opts)]
    lib.dts_shard_group_run.restype = C.c_int
    _lib = lib
    return lib


def _check(status: int):
    if status != DTS_OK:
        lib = load_library()
        raise DtsError(status, f"{lib.dts_status_str(status).decode()}: {lib.dts_last_error().decode()}")


def _ptr(a: Optional[np.ndarray]):
    return None if a is None else a.ctypes.data


def dts_run_opts_default(**kw) -> dts_run_opts:
    o = dts_run_opts()
    load_library().dts_run_opts_default(C.byref(o))
    for k, v in kw.items():
        setattr(o, k, v)
    return o


class Instance:
    """Owns a ``dts_instance*``; destroyed with the object."""

    def __init__(self, handle: int, m: int, n: int, K: int):
        self.handle = handle
        self.m, self.n, self.K = m, n, K

    def __del__(self):
        h, self.handle = getattr(self, "handle", None), None
        if h and _lib is not None:
            _lib.dts_instance_destroy(h)


def dts_instance_create(task_ptr, task_data, data_size, task_ns=None, default_task_ns: int = 0,
                        mem_capacity_bytes: int = 0, K: int = 1) -> Instance:
    lib = load_library()
    tp = np.ascontiguousarray(task_ptr, dtype=np.int64)
    td = np.ascontiguousarray(task_data, dtype=np.int32)
    sz = np.ascontiguousarray(data_size, dtype=np.uint64)
    tn = None if task_ns is None else np.ascontiguousarray(task_ns, dtype=np.int64)
    m, n = int(tp.shape[0] - 1), int(sz.shape[0])
    h = C.c_void_p()
    _check(lib.dts_instance_create(m, n, _ptr(tp), _ptr(td) if td.size else None,
                                   _ptr(sz) if sz.size else None, _ptr(tn), int(default_task_ns),
                                   int(mem_capacity_bytes), int(K), C.byref(h)))
    return Instance(h.value, m, n, int(K))


def dts_instance_upload(inst: Instance, device: int = 0, cuda_stream: int = 0):
    _check(load_library().dts_instance_upload(inst.handle, int(device), cuda_stream or None))


def dts_run(inst: Instance, policy: int = DTS_POLICY_DARTS_LUF, opts: Optional[dts_run_opts] = None):
    _check(load_library().dts_run(inst.handle, int(policy), None if opts is None else C.byref(opts)))


def dts_sweep_run(insts, policy: int = DTS_POLICY_DARTS_LUF, opts: Optional[dts_run_opts] = None,
                  devices=None):
    """include/dts.h dts_sweep_run: independent instances in batched launches;
    ``devices`` (a list of CUDA ordinals, repeats allowed) splits them over
    devices by LPT, else everything runs on opts.device."""
    arr = (C.c_void_p * len(insts))(*[i.handle for i in insts])
    devs = None if not devices else (C.c_int32 * len(devices))(*[int(d) for d in devices])
    _check(load_library().dts_sweep_run(arr, len(insts), int(policy),
                                        None if opts is None else C.byref(opts),
                                        devs, 0 if not devices else len(devices)))


# ---- task-sharded single instance (include/dts.h, SURVEY.md §8(e) second mode)

def dts_shard_set(inst: Instance, G: int, g: int):
    _check(load_library().dts_shard_set(inst.handle, int(G), int(g)))


def dts_shard_range(inst: Instance):
    lo, hi = C.c_int32(), C.c_int32()
    _check(load_library().dts_shard_range(inst.handle, C.byref(lo), C.byref(hi)))
    return int(lo.value), int(hi.value)


def dts_shard_export(inst: Instance, device: int = 0) -> bytes:
    buf = (C.c_char * DTS_SHARD_HANDLE_BYTES)()
    _check(load_library().dts_shard_export(inst.handle, int(device), buf))
    return bytes(buf)


def dts_shard_connect(inst: Instance, handles) -> None:
    """handles: the G exported handles in shard order."""
    blob = b"".join(bytes(h) for h in handles)
    if len(blob) % DTS_SHARD_HANDLE_BYTES:
        raise DtsError(DTS_E_INVAL, "shard handles must be DTS_SHARD_HANDLE_BYTES each")
    buf = C.create_string_buffer(blob, len(blob))
    _check(load_library().dts_shard_connect(inst.handle, buf))


def dts_shard_group_run(shards, policy: int = DTS_POLICY_DARTS_LUF, opts: Optional[dts_run_opts] = None):
    arr = (C.c_void_p * len(shards))(*[i.handle for i in shards])
    _check(load_library().dts_shard_group_run(arr, len(shards), int(policy),
                                              None if opts is None else C.byref(opts)))


@dataclass
class Result:
    K: int
    gpu_task_ptr: np.ndarray
    gpu_task_ids: np.ndarray
    serve_gpu: np.ndarray
    serve_task: np.ndarray
    task_start: np.ndarray
    task_end: np.ndarray
    events: np.ndarray
    bytes_loaded: int
    n_loads: int
    n_evictions: int
    makespan: int
    makespan_s: float
    n_served: int
    n_scans: int
    n_fallback2: int
    n_fallback_first: int
    n_belady: int
    n_idle_requests: int
    n_verify_err: int
    alg_bytes: int
    scan_alg_bytes: int
    loop_ms: float
    total_ms: float
    prof_cycles: tuple = ()
    sum_avail_at_scans: int = 0
    n_allocations: int = 0
    sum_deg_loads_evictions: int = 0
    loop_kind: int = 0  # 1 generic CTA loop, 2 specialised CTA loop, 3 one-warp loop

    def orders(self):
        p = self.gpu_task_ptr
        return [self.gpu_task_ids[p[k]:p[k + 1]] for k in range(self.K)]


def _arr(ptr, n, dtype, copy=True):
    if n == 0 or not ptr:
        return np.zeros(0, dtype)
    buf = (C.c_char * (int(n) * np.dtype(dtype).itemsize)).from_address(ptr)
    a = np.frombuffer(buf, dtype=dtype)
    if copy:
        return a.copy()
    a.flags.writeable = False
    return a


def dts_result(inst: Instance, copy: bool = True) -> Result:
    """The run's results.  copy=False returns read-only numpy views of the
    library's pinned host buffers instead of copies (no host memcpy): like the
    C ABI's dts_result_view they stay valid until the instance runs again or is
    destroyed."""
    v = dts_result_view()
    _check(load_library().dts_result(inst.handle, C.byref(v)))
    ns = int(v.n_served)
    A = (lambda p, n, dt: _arr(p, n, dt, copy))
    return Result(int(v.K), A(v.gpu_task_ptr, v.K + 1, np.int64), A(v.gpu_task_ids, ns, np.int32),
                  A(v.serve_gpu, ns, np.int32), A(v.serve_task, ns, np.int32),
                  A(v.task_start_ns, v.n_tasks, np.int64), A(v.task_end_ns, v.n_tasks, np.int64),
                  A(v.events, v.n_events, EVENT_DTYPE), int(v.bytes_loaded), int(v.n_loads),
                  int(v.n_evictions), int(v.makespan_ns), float(v.makespan_s), ns, int(v.n_scans),
                  int(v.n_fallback2), int(v.n_fallback_first), int(v.n_belady),
                  int(v.n_idle_requests), int(v.n_verify_err), int(v.alg_bytes),
                  int(v.scan_alg_bytes),
                  float(v.loop_ms), float(v.total_ms), tuple(int(x) for x in v.prof_cycles),
                  int(v.sum_avail_at_scans), int(v.n_allocations), int(v.sum_deg_loads_evictions),
                  int(v.loop_kind))


def dts_fetch_results(insts) -> None:
    """Batched device->host copy of many instances' results (two waits in
    total); dts_result afterwards reads host memory only."""
    arr = (C.c_void_p * len(insts))(*[i.handle for i in insts])
    _check(load_library().dts_fetch_results(arr, len(insts)))


def dts_run_times(inst: Instance):
    """(loop_ms, total_ms) of the instance's last run (waits for its loop)."""
    a, b = C.c_float(), C.c_float()
    _check(load_library().dts_run_times(inst.handle, C.byref(a), C.byref(b)))
    return float(a.value), float(b.value)


def dts_kernel_launches() -> int:
    return int(load_library().dts_kernel_launches())


def dts_version() -> int:
    return int(load_library().dts_version())


def schedule(inst, *, policy: int = DTS_POLICY_DARTS_LUF, W: int = 0, flags: int = DTS_F_FALLBACK2,
             bus_bps: int = 12_000_000_000,
             device: int = 0, block_threads: int = 0, smem_budget: int = 0,
             max_served: int = -1, stream: int = 0, n_devices: int = 0) -> Result:
    """One call: create the instance from host arrays (a ``gen.Instance``-like
    object), run DARTS+LUF on the GPU, return the host result."""
    h = dts_instance_create(inst.task_ptr, inst.task_data, inst.data_size, inst.task_ns,
                            inst.default_task_ns, inst.mem_capacity, inst.K)
    o = dts_run_opts_default(flags=flags, lookahead_W=W, bus_bytes_per_s=bus_bps, device=device,
                             block_threads=block_threads, smem_budget=smem_budget,
                             max_served=max_served, cuda_stream=stream or None, n_devices=n_devices)
    dts_run(h, policy, o)
    return dts_result(h)


def create(inst) -> Instance:
    """dts_instance_create from a ``gen.Instance``-like object."""
    return dts_instance_create(inst.task_ptr, inst.task_data, inst.data_size, inst.task_ns,
                               inst.default_task_ns, inst.mem_capacity, inst.K)


def schedule_batch(insts, *, policy: int = DTS_POLICY_DARTS_LUF, W: int = 0, flags: int = DTS_F_FALLBACK2,
                   bus_bps: int = 12_000_000_000, device: int = 0, block_threads: int = 0,
                   smem_budget: int = 0, stream: int = 0):
    """Run many independent instances in ONE batched launch (dts_sweep_run,
    one CTA per instance) and return their host results."""
    hs = [create(i) for i in insts]
    o = dts_run_opts_default(flags=flags, lookahead_W=W, bus_bytes_per_s=bus_bps, device=device,
                             block_threads=block_threads, smem_budget=smem_budget,
                             max_served=-1, cuda_stream=stream or None)
    dts_sweep_run(hs, policy, o)
    dts_fetch_results(hs)
    return [dts_result(h) for h in hs]


def schedule_sharded(inst, G: int, *, policy: int = DTS_POLICY_DARTS_LUF, W: int = 0,
                     flags: int = DTS_F_FALLBACK2, bus_bps: int = 12_000_000_000, device: int = 0,
                     block_threads: int = 0, smem_budget: int = 0, max_served: int = -1,
                     stream: int = 0):
    """One instance, its tasks sharded over G co-resident CTAs of one device
    (dts_shard_group_run); returns every shard's result (all equal)."""
    hs = [create(inst) for _ in range(G)]
    o = dts_run_opts_default(flags=flags, lookahead_W=W, bus_bytes_per_s=bus_bps, device=device,
                             block_threads=block_threads, smem_budget=smem_budget,
                             max_served=max_served, cuda_stream=stream or None)
    dts_shard_group_run(hs, policy, o)
    return [dts_result(h) for h in hs]

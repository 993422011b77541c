"""B200-native (sm_100a) DARTS+LUF memory-aware task scheduling simulator.

The compute path is ``lib/libdts.so`` (hand-written CUDA, C ABI in
``include/dts.h``); this package is its thin Python binding.  No CPU
fallback: without the library or a B200 the calls raise ``DtsError``.
"""
from .dts import (  # noqa: F401
    DTS_F_FALLBACK2,
    DTS_F_VERIFY,
    DTS_F_NOFUSE,
    DTS_F_OPTI,
    DTS_F_PACKED,
    DTS_F_GENERIC,
    DTS_POLICY_DARTS_LUF,
    DTS_POLICY_DARTS_LRU,
    DTS_POLICY_EAGER_LRU,
    EVENT_DTYPE,
    EXPORTED,
    LIB_PATH,
    DtsError,
    Instance,
    Result,
    dts_instance_create,
    dts_instance_upload,
    dts_result,
    dts_fetch_results,
    dts_run_times,
    dts_run,
    dts_run_opts_default,
    dts_sweep_run,
    dts_version,
    dts_kernel_launches,
    create,
    schedule_batch,
    load_library,
    schedule,
    schedule_sharded,
    dts_shard_set,
    dts_shard_range,
    dts_shard_export,
    dts_shard_connect,
    dts_shard_group_run,
    DTS_SHARD_HANDLE_BYTES,
)

"""Seeded synthetic workload generators shared by the oracle tests, the GPU
parity tests and ``bench.py``.

This package holds *inputs only*: task -> data incidence (CSR), data sizes,
task durations and per-GPU capacities shaped like the paper's workloads
(§V-A).  It contains none of the scheduling method's
arithmetic, so it may be shared by ``oracle/`` and the CUDA path.
"""
from .workloads import (  # noqa: F401
    Instance,
    matmul2d,
    matmul3d,
    cholesky,
    random_shared,
    fig1,
    config_instances,
    sweep_params,
    sweep_instance,
    splitmix64,
    DATUM_2D_BYTES,
    TILE_BYTES,
    MIB500,
    TAU_2D_NS,
    TAU_GEMM_NS,
    TAU_TRSM_NS,
    TAU_SYRK_NS,
    TAU_POTRF_NS,
    DEFAULT_BUS_BPS,
)

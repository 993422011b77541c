"""Workload generators (inputs only; no scheduling arithmetic).

Every generator returns an :class:`Instance`: a task -> data CSR
(``task_ptr`` int64[m+1], ``task_data`` int32[E]), per-datum sizes in bytes
(``data_size`` uint64[n]), per-task durations in integer ns (``task_ns``
int64[m]), the per-simulated-GPU memory capacity in bytes and K.

Shapes follow the paper's workloads and SURVEY.md §8(d) / DESIGN.md "Input
recipe":

* 2D matrix product, tasks submitted row per row (§V-A);
  optional randomized order and sparse variant with 98% of
  the tasks removed.
* 3D matrix product A_ik * B_kj, summation ignored.
* Cholesky tasks with dependencies removed, reading R13.
* Random shared-input tasks (BASELINE.json config 4), splitmix64 stream.

Sizes: a 2D datum is a 960x3840 fp32 block row/column = 14,745,600 B and a
tile is 960x960 fp32 = 3,686,400 B (readings R14/R15: the paper's 140 MB at
5x5 and 8,400 MB at 300x300 only fit MiB and 4-tile blocks).  500 MB = 500
MiB.  Task times: flops / 13,253 GFlop/s (the paper's V100 peak,
PAPER.md:1032-1036), rounded to nearest ns.
"""
from __future__ import annotations

from dataclasses import dataclass, field
from typing import Optional

import numpy as np

DATUM_2D_BYTES = 960 * 3840 * 4          # 14,745,600
TILE_BYTES = 960 * 960 * 4               # 3,686,400
MIB500 = 500 * 1024 * 1024               # 524,288,000
DEFAULT_BUS_BPS = 12_000_000_000         # PCIe 3 x16 (paper silent; reading R9)

_V100_FLOP_PER_NS = 13_253


def _tau(flops: int) -> int:
    return int((flops + _V100_FLOP_PER_NS // 2) // _V100_FLOP_PER_NS)


TAU_2D_NS = _tau(2 * 960 * 960 * 3840)   # 534,059
TAU_GEMM_NS = _tau(2 * 960 ** 3)         # 133,515
TAU_TRSM_NS = _tau(960 ** 3)             # 66,757
TAU_SYRK_NS = _tau(960 ** 3)             # 66,757
TAU_POTRF_NS = _tau(960 ** 3 // 3)       # 22,252

_MASK64 = (1 << 64) - 1
_GOLDEN = 0x9E3779B97F4A7C15


def splitmix64(state_idx: np.ndarray, seed: int) -> np.ndarray:
    """Counter-based splitmix64: output number ``state_idx`` of the stream
    seeded with ``seed`` (the classic generator's x-th output, vectorised)."""
    with np.errstate(over="ignore"):
        z = (np.uint64(seed) + (state_idx.astype(np.uint64) + np.uint64(1)) * np.uint64(_GOLDEN))
        z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
        z = z ^ (z >> np.uint64(31))
    return z


@dataclass
class Instance:
    name: str
    task_ptr: np.ndarray                 # int64 [m+1]
    task_data: np.ndarray                # int32 [E]
    data_size: np.ndarray                # uint64 [n]
    task_ns: Optional[np.ndarray]        # int64 [m] or None
    default_task_ns: int
    mem_capacity: int                    # bytes per simulated GPU
    K: int
    meta: dict = field(default_factory=dict)

    @property
    def m(self) -> int:
        return int(self.task_ptr.shape[0] - 1)

    @property
    def n(self) -> int:
        return int(self.data_size.shape[0])

    @property
    def E(self) -> int:
        return int(self.task_ptr[-1])

    def with_(self, **kw) -> "Instance":
        d = dict(self.__dict__)
        d.update(kw)
        return Instance(**d)


def _csr(rows) -> tuple[np.ndarray, np.ndarray]:
    lens = np.fromiter((len(r) for r in rows), dtype=np.int64, count=len(rows))
    ptr = np.zeros(len(rows) + 1, dtype=np.int64)
    np.cumsum(lens, out=ptr[1:])
    data = np.fromiter((d for r in rows for d in r), dtype=np.int32, count=int(ptr[-1]))
    return ptr, data


def matmul2d(N: int, M: int = 35, K: int = 2, order: str = "natural",
             keep_frac: float = 1.0, seed: int = 0, datum_bytes: int = DATUM_2D_BYTES,
             task_ns: int = TAU_2D_NS) -> Instance:
    """2D product: data A_i = i (block rows of A), B_j = N + j (block columns
    of B); task (i, j) needs {A_i, B_j}.  Natural order:
    task id = i*N + j.  ``order='random'`` permutes the submission order
    (PAPER.md:800); ``keep_frac < 1`` keeps a seeded random subset of tasks
    (sparse 2D keeps 2%).  Capacity = M data."""
    ii, jj = np.divmod(np.arange(N * N, dtype=np.int64), N)
    if keep_frac < 1.0:
        r = splitmix64(np.arange(N * N, dtype=np.int64), seed + 1)
        thresh = np.uint64(int(keep_frac * float(1 << 53)) << 11)
        keep = r < thresh
        ii, jj = ii[keep], jj[keep]
    if order == "random":
        key = splitmix64(np.arange(ii.shape[0], dtype=np.int64), seed + 2)
        perm = np.argsort(key, kind="stable")
        ii, jj = ii[perm], jj[perm]
    elif order != "natural":
        raise ValueError(order)
    m = ii.shape[0]
    task_ptr = np.arange(0, 2 * m + 1, 2, dtype=np.int64)
    task_data = np.empty(2 * m, dtype=np.int32)
    task_data[0::2] = ii
    task_data[1::2] = N + jj
    n = 2 * N
    return Instance(f"2d_N{N}_M{M}_K{K}" + ("" if order == "natural" else "_rand")
                    + ("" if keep_frac >= 1.0 else f"_sparse{keep_frac}"),
                    task_ptr, task_data, np.full(n, datum_bytes, dtype=np.uint64),
                    None, task_ns, M * datum_bytes, K,
                    dict(kind="2d", N=N, M=M, order=order, keep_frac=keep_frac))


def matmul3d(N: int, M: int = 142, K: int = 4, with_c: bool = False,
             tile_bytes: int = TILE_BYTES, task_ns: int = TAU_GEMM_NS) -> Instance:
    """3D product: task (i, j, k) = (i*N + j)*N + k needs A_ik = i*N + k and
    B_kj = N^2 + k*N + j; ``with_c`` adds C_ij = 2N^2 +
    i*N + j as a third input (reading R12)."""
    t = np.arange(N ** 3, dtype=np.int64)
    ij, k = np.divmod(t, N)
    i, j = np.divmod(ij, N)
    a = i * N + k
    b = N * N + k * N + j
    ar = 3 if with_c else 2
    task_ptr = np.arange(0, ar * N ** 3 + 1, ar, dtype=np.int64)
    task_data = np.empty(ar * N ** 3, dtype=np.int32)
    task_data[0::ar] = a
    task_data[1::ar] = b
    n = 2 * N * N
    if with_c:
        task_data[2::ar] = 2 * N * N + i * N + j
        n = 3 * N * N
    return Instance(f"3d_N{N}_M{M}_K{K}" + ("_c" if with_c else ""), task_ptr, task_data,
                    np.full(n, tile_bytes, dtype=np.uint64), None, task_ns,
                    M * tile_bytes, K, dict(kind="3d", N=N, M=M, with_c=with_c))


def cholesky(N: int, M: int = 142, K: int = 8, tile_bytes: int = TILE_BYTES) -> Instance:
    """Tasks of a tiled Cholesky factorisation with dependencies removed
    (PAPER.md:807-811), reading R13: every tile accessed is an input.
    Lower tile (i, j), i >= j, has id i(i+1)/2 + j.  Submission order:
    for k: POTRF(k){A_kk}; TRSM(i,k){A_kk, A_ik} for i > k; for j > k:
    SYRK(j,k){A_jk, A_jj} then GEMM(i,j,k){A_ik, A_jk, A_ij} for i > j."""
    def tid(i, j):
        return i * (i + 1) // 2 + j
    rows, taus = [], []
    for k in range(N):
        rows.append((tid(k, k),)); taus.append(TAU_POTRF_NS)
        for i in range(k + 1, N):
            rows.append((tid(k, k), tid(i, k))); taus.append(TAU_TRSM_NS)
        for j in range(k + 1, N):
            rows.append((tid(j, k), tid(j, j))); taus.append(TAU_SYRK_NS)
            for i in range(j + 1, N):
                rows.append((tid(i, k), tid(j, k), tid(i, j))); taus.append(TAU_GEMM_NS)
    task_ptr, task_data = _csr(rows)
    n = N * (N + 1) // 2
    return Instance(f"cholesky_N{N}_M{M}_K{K}", task_ptr, task_data,
                    np.full(n, tile_bytes, dtype=np.uint64), np.asarray(taus, dtype=np.int64),
                    TAU_GEMM_NS, M * tile_bytes, K, dict(kind="cholesky", N=N, M=M))


def random_shared(m: int = 1 << 20, n: int = 1 << 14, arity: int = 3, M: int = 1024,
                  K: int = 8, seed: int = 42, tile_bytes: int = TILE_BYTES) -> Instance:
    """Random shared-input tasks: task t draws ``arity`` distinct ids from
    splitmix64 outputs t*16 + j (j = 0, 1, ...), id = value mod n (n a power
    of two: ``& (n-1)``), redrawing on a duplicate, then sorts them."""
    assert n & (n - 1) == 0 and arity <= 16
    base = np.arange(m, dtype=np.int64) * 16
    draws = np.stack([splitmix64(base + j, seed) & np.uint64(n - 1) for j in range(arity)], 1)
    draws = draws.astype(np.int64)
    s = np.sort(draws, axis=1)
    dup = np.any(s[:, 1:] == s[:, :-1], axis=1) if arity > 1 else np.zeros(m, bool)
    for t in np.nonzero(dup)[0]:
        got, j = [], 0
        while len(got) < arity:
            v = int(splitmix64(np.array([t * 16 + j]), seed)[0]) & (n - 1)
            j += 1
            if v not in got:
                got.append(v)
        s[t] = sorted(got)
    task_ptr = np.arange(0, arity * m + 1, arity, dtype=np.int64)
    return Instance(f"random_m{m}_n{n}_M{M}_K{K}", task_ptr, s.reshape(-1).astype(np.int32),
                    np.full(n, tile_bytes, dtype=np.uint64), None, TAU_GEMM_NS,
                    M * tile_bytes, K, dict(kind="random", M=M, seed=seed))


def fig1(K: int = 2, M: int = 2) -> Instance:
    """The 3x3 example of Fig. 1: T_{3(r-1)+c} needs D_c
    and D_{3+r}; ids shifted to 0-based.  Unit sizes, unit times."""
    rows = [(c, 3 + r) for r in range(3) for c in range(3)]
    task_ptr, task_data = _csr(rows)
    return Instance("fig1", task_ptr, task_data, np.ones(6, dtype=np.uint64), None, 1,
                    M, K, dict(kind="fig1"))


# ----------------------------------------------------------------- configs
SWEEP_N = list(range(5, 161, 5))                                        # 32 values
SWEEP_M = [4, 5, 6, 8, 10, 12, 16, 20, 24, 32, 35, 40, 48, 64, 96, 128]  # 16 values
SWEEP_K = list(range(1, 9))                                             # 8 values


def sweep_params():
    """Config 5: the 4,096 (N, M, K) triples of the 2D sweep."""
    return [(N, M, K) for N in SWEEP_N for M in SWEEP_M for K in SWEEP_K]


def sweep_instance(N: int, M: int, K: int) -> Instance:
    return matmul2d(N, M=M, K=K)


def config_instances(cfg: str):
    """The BASELINE.json configs as concrete instances."""
    if cfg == "C1":
        return [matmul2d(10, M=6, K=1)]
    if cfg == "C2":
        return [matmul2d(N, M=35, K=K) for K in (2, 4) for N in range(10, 101, 10)]
    if cfg == "C3":
        return [matmul3d(40, M=142, K=4)]
    if cfg == "C4a":
        return [cholesky(181, M=142, K=8)]
    if cfg == "C4b":
        return [random_shared(1 << 20, 1 << 14, 3, M=1024, K=8, seed=42)]
    if cfg == "C5":
        return [sweep_instance(*p) for p in sweep_params()]
    raise KeyError(cfg)

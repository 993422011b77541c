// dts_internal.cuh -- device-side data layout of libdts (sm_100a).
//
// Layout in HBM, per instance:
//   CSR (built on device, §8(a) a1):  tptr[m+1] int64, tdat[E] int32 (rows sorted,
//       de-duplicated), dptr[n+1] int64, ddat[E] int32 (each data segment in
//       ascending task id).
//   s[K][m_pad] uint32 -- per (simulated GPU k, task T) packed state
//       bit 31      : T allocated (left the shared pool of unprocessed tasks, R2)
//       bits 24..30 : cnt_k(T) = |D(T) \ R_k|   (<= 127)
//       bits  0..23 : x_k(T)   = XOR of the ids in D(T) \ R_k   (n < 2^24)
//     so (s >> 24) == 1  <=>  T unallocated and exactly one input missing, and
//     then x_k(T) IS that missing datum: "tasks that depend only on D and data
//     already loaded" (Alg. 5 l.5) need no rescan.
//   u[n] int32   -- #unallocated tasks using D (Alg. 5 l.9 secondary key, R23)
//   hist[n] int32 -- per-scan score n_k(D) (zero between scans)
//   np[K][n] int32 -- #tasks of plannedTasks_k using D (Alg. 6 l.3)
//   res_list[K][res_cap], res_pos[K][n] -- resident set of each simulated GPU
//   planned[K][plan_cap] -- plannedTasks_k in ascending id (-1 = removed by LUF)
#pragma once
#include <cstdint>

#include "dts.h"

namespace dts {

// Process-wide count of kernel launches issued by libdts (dts_kernel_launches()).
void count_launch();

constexpr uint32_t ALLOC_BIT = 0x80000000u;
constexpr uint32_t CNT_ONE = 1u << 24;
constexpr uint32_t XOR_MASK = 0x00FFFFFFu;
constexpr int MAX_K = 64;
constexpr int MAX_ROW = 127;

enum Cmd : int { CMD_NONE = 0, CMD_SCAN = 1, CMD_FSCAN = 2, CMD_DONE = 3 };

// Per-instance control block (global memory, zeroed by the init kernel).
struct Ctrl {
    unsigned bar_count;
    unsigned bar_gen;
    int cmd;
    int cmd_k;
    unsigned long long best_key;  // argmax over D of packed (score, u, ~id), atomicMax
    int min_avail;                // lowest unallocated task id (fallback, Alg. 5 l.13)
    int error;
};

// Scalar results written by the decision loop.
struct Out {
    int64_t n_events, n_served, n_loads, n_evictions, n_scans, n_fallback2, n_fallback_first,
        n_belady, n_idle;
    uint64_t bytes_loaded;
    int64_t makespan;
    uint64_t alg_bytes, scan_alg_bytes;
    int32_t error;
    int32_t pad;
};

// Device descriptor of one instance (passed by pointer to the loop kernel).
struct Inst {
    int32_t m, n, K, W;
    uint32_t flags;
    int32_t m_pad;       // m rounded up to a multiple of 4 (uint4 scans); pad words = ALLOC_BIT
    int64_t max_served;  // -1 = run to completion
    uint64_t cap;        // bytes per simulated GPU
    int32_t plan_cap;    // >= max_D deg(D)
    int32_t res_cap;     // >= max resident data per GPU
    int32_t id_bits, u_bits;
    int64_t E;
    // CSR (device)
    const int64_t *tptr;
    const int32_t *tdat;
    const int64_t *dptr;
    const int32_t *ddat;
    const uint64_t *size;
    const int64_t *delta;  // ceil(size * 1e9 / bw) ns (reading R9)
    const int64_t *tau;    // [m] or nullptr
    int64_t default_tau;
    // state
    uint32_t *s;
    int32_t *u;
    int32_t *hist;
    int32_t *np;
    int32_t *res_list;
    int32_t *res_pos;
    int32_t *planned;
    Ctrl *ctrl;
    // outputs
    int32_t *serve_gpu;
    int32_t *serve_task;
    int64_t *tstart;
    int64_t *tend;
    dts_event *events;
    int64_t ev_cap;
    Out *out;
    // result assembly
    int64_t *gpu_task_ptr;  // [K+1]
    int32_t *gpu_task_ids;  // [m]
};

}  // namespace dts

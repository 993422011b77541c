// dts_internal.cuh -- device-side data layout of libdts (sm_100a).
//
// One CTA runs one instance's whole schedule.  Layout
// per instance; arrays marked [S/G] live in the
// CTA's shared memory when the host's placement (Inst::so_*) fits them in the
// budget, else in their global (HBM/L2) home:
//
//   CSR (built on device, §8(a) a1):  tptr[m+1] int64, tdat[E] int32 (rows
//       sorted, de-duplicated), dptr[n+1] int64, ddat[E] int32 (each data
//       segment in ascending task id), dedge[E] int4 = ddat's edge records
//       {T, other inputs of T, |D(T)|} so a segment walk needs no row lookup [G]
//   s[K][m_pad] uint32 -- per (simulated GPU k, task T) packed state    [S/G]
//       bit 31      : T allocated (left the shared pool of unprocessed tasks, R2)
//       bits 24..30 : cnt_k(T) = |D(T) \ R_k|   (<= 127)
//       bits  0..23 : x_k(T)   = XOR of the ids in D(T) \ R_k   (n < 2^24)
//     so a task with cnt 1 NAMES its one missing datum: x_k(T).
//   al[m_pad/32 + 1] uint32 -- allocation bitmap (bit set: T left the shared
//       pool, R2; pad bits set).  The "row-derived" state mode (Inst::sl,
//       every row <= 3 inputs, one shard): s is not kept at all -- cnt_k(T) and
//       the missing ids are read off T's row (edge record / plan entry) and the
//       residency bitmap, so the per-(GPU, task) state shrinks from 4 K m bytes
//       to m / 8 and fits in shared memory for every config        [S/G]
//   h[K][nstr] int32 -- n_k(D)  = #unallocated T with cnt_k(T)=1, x_k(T)=D: the
//       DARTS score of Alg. 5 l.4-5, kept incrementally [S/G]
//   h2[K][nstr] int32 -- n2_k(D) = #unallocated T with cnt_k(T)=2, D missing:
//       the "3inputs" score, kept incrementally      [S/G]
//   u[nstr]  int32 -- #unallocated tasks using D (secondary key, R23)     [S/G]
//   np[K][nstr] int32 -- #tasks of plannedTasks_k using D (Alg. 6 l.3)       [S/G]
//   resb[K][nw] uint32 -- residency bitmap of each simulated GPU          [S/G]
//   res_list[K][res_cap] int32 -- resident data of each GPU (LUF scan)    [S/G]
//   plan[K][plan_cap] int4 -- plannedTasks_k in ascending id: {T, D0, D1, D2}
//       (T = -1: removed by LUF; D(T) cached when |D(T)| <= 3, D2 = -2 when
//       the row is longer)                                           [S/G]
//   lru[K][nstr] int32 -- serve index of D's last use on GPU k (LRU)   [S/G]
//   plan_tau[K][plan_cap] int64 -- their durations (per-task times only)  [S/G]
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
constexpr int MAX_W = 8;  // lookahead_W <= 8: taskBuffer of at most 9 tasks (R7, R29)
// result assembly's scratch in the CTA's dynamic shared memory (after the loop)
constexpr int ASSEMBLE_SMEM_BYTES = 8 * MAX_K + 4 * MAX_K + 4 * 16 * MAX_K;
constexpr int ROW_LONG = -2;  // plan entry: |D(T)| > 3, read the row from the CSR

// Scalar results written by the decision loop.
struct Out {
    int64_t n_events, n_served, n_loads, n_evictions, n_scans, n_fallback2, n_fallback_first,
        n_belady, n_idle, n_verify_err;
    uint64_t bytes_loaded;
    int64_t makespan;
    uint64_t alg_bytes, scan_alg_bytes;
    // SURVEY.md §8(d) byte model: sum over scans of the
    // unallocated tasks when the scan started, task allocations, sum of deg(D)
    // over loads and evictions
    int64_t sum_avail, n_alloc, sum_deg;
    int32_t error;
    int32_t pad;
    int64_t prof[16];  // SM cycles seen by thread 0 per phase (see PROF_* in dts_loop.cu)
};

// Task-sharded single instance (second mode): shard g of G
// owns the tasks [t_lo, t_hi) -- their packed state s, their data->task edges
// and PARTIAL score arrays h, h2, u -- while every decision (residency, plans,
// np, the time model, the trace) is replicated on all shards.  Shards meet at
// exchange points through each other's memory (same device: other CTAs; other
// B200s: CUDA IPC mappings over NVLink).  One entry per shard, pointers valid
// in the address space of the shard that reads the table.
constexpr int MAX_G = 64;
struct ShardPeer {
    unsigned long long *epoch;  // the shard's last published exchange number
    unsigned char *box;         // its two payload slots (by exchange parity)
    const int32_t *h, *h2, *u;  // its partial score arrays (global homes)
};
// Payload slot: keys / candidate ids, then the shard's part of a new plan.
struct ShardSlot {
    unsigned long long key[2];
    int32_t cnt;
    int32_t pad[3];
    // int4 ents[plan_cap] follow
};

// Device descriptor of one instance.
struct Inst {
    int32_t m, n, K, W;
    uint32_t flags;
    int32_t m_pad;       // m rounded up to a multiple of 4; pad words = ALLOC_BIT
    int64_t max_served;  // -1 = run to completion
    uint64_t cap;        // bytes per simulated GPU
    int32_t plan_cap;    // >= max_D deg(D)
    int32_t res_cap;     // >= max resident data per GPU
    int32_t id_bits, u_bits;
    int32_t key32;       // scores and u(D) < 2^15: 32-bit argmax keys (score << 16 | u)
    int32_t max_row;     // max |D(T)|
    int32_t nw;          // 32-bit words per residency bitmap row
    int32_t nstr;        // row stride of h, h2, np (and length of u): n rounded up to 4
    int64_t E;
    // CSR (device)
    const int64_t *tptr;
    const int32_t *tdat;
    const int64_t *dptr;
    const int32_t *ddat;
    const int64_t *raw_ptr;  // caller's CSR as uploaded (fused builds read it)
    const int32_t *raw_dat;
    int32_t fused;           // 1: the loop CTA builds the CSR and initial state itself
    int32_t pad2;
    uint64_t bw;             // bus bytes/s (fused init computes delta)
    const int4 *dedge;     // [E] edge records of the data->task CSR: {T, o1, o2, |D(T)|},
                           // o1/o2 = T's other inputs (-1 if none; first two if |D(T)| > 3)
    const uint64_t *size;
    const int64_t *delta;  // ceil(size * 1e9 / bw) ns (reading R9)
    uint64_t size0;        // != 0: every datum has this size (then delta0 = its bus time)
    int64_t delta0;
    const int64_t *tau;    // [m] or nullptr
    int64_t default_tau;
    // state: global homes
    uint32_t *s;
    int32_t *u, *h, *h2, *np;
    uint32_t *resb;
    int32_t *res_list;
    int4 *plan;
    int64_t *plan_tau;
    int32_t *vhist;  // DTS_F_VERIFY scratch [3 n]
    int32_t *lru;    // [K][nstr] last-use stamps (LRU policies)
    int32_t policy;  // dts_policy
    int32_t so_lru;
    // shared-memory placement: byte offset in the CTA's dynamic smem, -1 = global home
    int32_t so_u, so_h, so_h2, so_np, so_resb, so_res_list, so_plan, so_plan_tau, so_s, so_dptr;
    int32_t smem_bytes;
    int32_t pad1;
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
    // task sharding (G = 1: the whole instance on one CTA)
    int32_t G, g;             // shards, this shard
    int32_t t_lo, t_hi;       // owned task range
    const ShardPeer *peers;   // [G] (device), nullptr when G = 1
    unsigned long long ep_base;  // exchange numbers of this run: ep_base + 1, 2, ...
    int64_t box_bytes;        // bytes of one payload slot
    int32_t xsys;             // 1: peers on other devices (system-scope release/acquire)
    int32_t pop_batch_min;    // serve pops in one batch when more than this many are planned
    // row-derived state mode (sl = 1): no s; allocation bitmap al instead
    int32_t sl;
    int32_t so_al;            // shared-memory offset of al, -1 = global home
    uint32_t *al;             // [m_pad / 32 + 1] global home
    int32_t poison;  // debug (env DTS_POISON=1): fill the CTA's dynamic shared memory at instance start
    int32_t *wring;  // [K][MAX_W] W >= 1: the last W tasks served on each simulated GPU
    // 1: the launch runs the specialised loop (dts_loop_fast.cu), whose score rows are
    // packed: h[k][D] = n_k(D) | n2_k(D) << 16 (h2 unused); dts_init_kernel writes them so
    int32_t hh;
    int32_t pad3;
};

}  // namespace dts

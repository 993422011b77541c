// dts_loop.cu -- the device-resident DARTS+LUF decision loop (§8(a) a2-a8).
//
// ONE CTA runs ONE instance's whole schedule in a single launch (a batched
// launch runs many instances: each CTA pulls the next instance from a device
// counter).  The method is a chain of sequential decisions (PAPER.md:697-730:
// each request depends on every earlier load, eviction and allocation), so the
// kernel is built for per-decision LATENCY: thread 0 owns the scalar state
// (event order, pops, the bus/time model, the trace) in shared memory, and
// the whole CTA joins only for the data-parallel steps:
//
//   score    : n_k(D) = #unallocated tasks whose only missing input is D
//              (Alg. 5 l.4-5) is kept INCREMENTALLY in
//              h[k][D]: every residency change walks the datum's data->task
//              segment and moves each touched task between the cnt==1 / cnt==2
//              buckets.  A scan is then a block argmax over D of the packed key
//              (n(D), u(D), ~D): more unprocessed uses, then lower id, on ties
//              (Alg. 5 l.6-9, readings R1/R23) -- O(n), not O(m).
//   3inputs  : the same with h2[k][D] (tasks with two missing inputs, both
//              credited) when no datum frees a task.
//   plan     : ordered compaction of Dopt's segment -> plannedTasks_k (Alg. 5 l.10)
//   LUF      : block min over the resident data of (np(D), D) among those the
//              taskBuffer does not use (Alg. 6).
//   residency: segment update of the packed (cnt, xor) state + score buckets.
//
// Pops (Alg. 5 l.1-2) -- most requests -- are served by thread 0 alone with no
// barrier and no global read: a planned task has all its inputs resident
// (its inputs were resident or Dopt when planned; LUF drops planned tasks whose
// inputs it evicts, Alg. 6 l.8), so serving it is pure time-model arithmetic.
#include <cuda_runtime.h>

#include <climits>
#include <cstdint>

#include "dts_internal.cuh"
#include "dts_loop.cuh"

// Mode predicates.  This file is compiled twice: as the generic loop (every
// mode, chosen at run time from the descriptor) and, from dts_loop_fast.cu
// with DTS_FAST = 1, specialised at compile time to the mode every BASELINE
// config runs in -- row-derived state (rows of <= 3 inputs), one shard, W = 0,
// DARTS+LUF, 32-bit argmax keys, uniform data sizes, no OPTI / VERIFY -- so the
// other modes' code is compiled out of the hot loop (it is instruction-cache
// bound: DESIGN.md §6).
#ifndef DTS_FAST
#define DTS_FAST 0
#endif
#define M_SL(I) (DTS_FAST || (I).sl)                           // row-derived state
#define M_SHARD(I) (!DTS_FAST && (I).G > 1)                    // task shards
#define M_W(I) (DTS_FAST ? 0 : (I).W)                          // prefetch window
#define M_LUF(I) (DTS_FAST || (I).policy == DTS_POLICY_DARTS_LUF)
#define M_POL(I, p) (!DTS_FAST && (I).policy == (p))            // an LRU policy
#define M_LONG(c) (!DTS_FAST && (c))                           // rows of > 3 inputs
#define M_KEY32(I) (DTS_FAST || (I).key32)                     // scores and u(D) < 2^15
#define M_FLAG(I, f) (!DTS_FAST && ((I).flags & (f)))          // OPTI, VERIFY: generic only
#ifndef DTS_HH_UN
#define DTS_HH_UN 4
#endif
#define M_HH (DTS_FAST)  // packed scores: h[k][D] = n_k(D) | n2_k(D) << 16, one argmax pass for both
#if DTS_FAST
#define DTS_KNAME(x) x##_fast
#else
#define DTS_KNAME(x) x
#endif

namespace dts {

namespace {

constexpr unsigned FULL = 0xffffffffu;

// CTA barrier that also reconverges each warp.  __syncthreads() alone leaves a
// warp split after a thread-0-only block (independent thread scheduling), and
// the split halves then run every later instruction twice and meet again at
// each full-mask shuffle -- a measured 4x slowdown of the warp-0 phases.
// Every value a thread reads to choose a path must be final before the
// barrier that precedes the read and stay unchanged until the next barrier
// (see pop_batch: a violation shows up as divergent barriers in
// compute-sanitizer synccheck).
__device__ __forceinline__ void cta_sync() {
    __syncthreads();
    __syncwarp();
}

constexpr int POP_RANK_MAX = 256;  // pops ranked by counting in one pass

enum Cmd : int { CMD_SCAN = 1, CMD_DONE = 2, CMD_POP = 3, CMD_EAGER = 4 };

// Per-phase cycle accounting by thread 0 (diagnostics, dts_result_view.prof_cycles),
// compiled only into the profiling build (lib/libdts_prof.so, -DDTS_PROF): the
// probes are thread-0 branches plus shared read-modify-writes on the critical
// path, so the production library leaves them out (prof_cycles reads 0).
enum Prof : int { P_POP = 0, P_ARGMAX, P_PLAN, P_LOADS, P_LUF, P_EVICT, P_SEG, P_OTHER, P_BW0, P_BD, P_NB, P_NP, P_X1, P_X2, P_X3, P_X4 };
#ifdef DTS_PROF
#define PROF_T0(var) const long long var = (threadIdx.x == 0) ? clock64() : 0
#define PROF_ADD(L, slot, var) \
    do {                       \
        if (threadIdx.x == 0) (L).prof[slot] += clock64() - (var); \
    } while (0)
#define PROF_CNT(L, slot, v) \
    do {                     \
        if (threadIdx.x == 0) (L).prof[slot] += (v); \
    } while (0)
#else
#define PROF_T0(var)
#define PROF_ADD(L, slot, var) \
    do {                       \
    } while (0)
#define PROF_CNT(L, slot, v) \
    do {                     \
    } while (0)
#endif

struct Lead {  // leader scalars + broadcast slots (static shared memory)
    int64_t req[MAX_K];
    int64_t gpu_free[MAX_K];
    uint64_t used[MAX_K];
    int32_t plan_head[MAX_K], plan_end[MAX_K], plan_live[MAX_K];
    int32_t res_cnt[MAX_K];
    int32_t idle[MAX_K];
    // W >= 1: tasks served on k so far; the last W of them (I.wring[k][.], a
    // ring by this count) are the candidates of taskBuffer_k (R7, R29)
    int32_t won[MAX_K];
    int32_t row2[MAX_ROW + 1];  // inputs of the other buffered tasks: [0, row2_run) those of
    int32_t row2_len, row2_run; // the task running at the request, then those not started (R29)
    int64_t run_end;            // end of the running buffered task (Belady evictions, R29)
    int64_t mem_ready;          // serve_loads: the freed memory of this serve is available from
    int64_t bus_free;
    int64_t n_events, n_served, n_loads, n_evictions, n_scans, n_fb2, n_fbf, n_belady, n_idle,
        n_verr;
    uint64_t bytes_loaded, alg_bytes, scan_alg_bytes;
    int64_t makespan;
    int64_t sum_avail, n_alloc, sum_deg;  // SURVEY §8(d) byte-model counters (Out)
    int32_t scan_avail;                   // m_avail when the current scan started
    int32_t n_avail, avail_lo;
    int32_t error;
    int32_t cmd, k, T, vslot, row_len;
    int64_t t, ready;
    int32_t row[MAX_ROW + 1];
    unsigned long long red64[32];
    unsigned long long red64b[32];
    int32_t red32[32];
    int32_t wcnt[32];
    long long prof[16];
    int64_t bstart[32], breq[32], bns;  // pop batch (K <= 32): per-GPU first start / request
    int32_t bhead[32], bcnt[32], boff[33];
    int64_t rkey[POP_RANK_MAX];  // pop batch: request time of each pop (merge ranks)
    int32_t rgpu[POP_RANK_MAX];
    int4 fent;       // a fallback / EAGER pick as a plan entry (pool_move_many)
    int32_t miss[MAX_ROW + 1];  // serve_loads: D(T) \ R_k in ascending id (R10)
    int32_t nmiss;
    int64_t xe;      // task shards: exchanges done in this run
    int32_t xerr;    // task shards: a peer did not arrive in time (the run is abandoned)
    int32_t xoff[MAX_G + 1];  // plan exchange: each shard's offset in the merged plan
};

// Per-instance views: shared-memory arrays where placed, else global homes.
struct View {
    uint32_t *s;
    int32_t *u, *h, *h2, *np;
    uint32_t *resb;
    int32_t *res_list;
    int4 *plan;
    int64_t *plan_cum;  // inclusive prefix sums of the planned tasks' tau (per-task times only)
    int32_t *dptr32;    // shared-memory copy of dptr, or nullptr
    int32_t *lru;       // [K][nstr] last-use stamps (LRU policies)
    uint32_t *al;       // row-derived mode: allocation bitmap (bit set = left the pool)
};

// Per-CTA state at namespace scope, so the (non-inlined) phase functions
// address it with shared-memory instructions: the leader scalars, this CTA's
// instance descriptor and its array views.
__shared__ Lead L;
__shared__ Inst SI;
__shared__ View SV;
__shared__ ShardPeer SP[MAX_G];  // task shards: the peer table (copied at instance start)

// Warp reductions with redux.sync (one instruction per 32-bit reduction): a
// 64-bit max / min is the high words' extremum, then the low words' among the
// lanes that hold it -- 56 cycles on the B200 against 200 for five 64-bit
// shuffle rounds (tools/micro/redux_micro.cu).  Every lane must take part.
__device__ __forceinline__ int warp_sum(int v) { return (int)__reduce_add_sync(FULL, (unsigned)v); }
__device__ __forceinline__ unsigned long long warp_max_u64(unsigned long long v) {
    const unsigned hi = (unsigned)(v >> 32), lo = (unsigned)v;
    const unsigned mh = __reduce_max_sync(FULL, hi);
    const unsigned ml = __reduce_max_sync(FULL, hi == mh ? lo : 0u);
    return ((unsigned long long)mh << 32) | ml;
}
__device__ __forceinline__ unsigned long long warp_min_u64(unsigned long long v) {
    const unsigned hi = (unsigned)(v >> 32), lo = (unsigned)v;
    const unsigned mh = __reduce_min_sync(FULL, hi);
    const unsigned ml = __reduce_min_sync(FULL, hi == mh ? lo : 0xffffffffu);
    return ((unsigned long long)mh << 32) | ml;
}

// Block reductions (every thread calls; the result is returned to every
// thread): warp shuffle, one barrier-protected exchange, warp shuffle again.
__device__ unsigned long long block_max_u64(unsigned long long v) {
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, nw = blockDim.x >> 5;
    v = warp_max_u64(v);
    if (nw == 1) return v;
    cta_sync();
    if (lane == 0) L.red64[w] = v;
    cta_sync();
    return warp_max_u64(lane < nw ? L.red64[lane] : 0ull);
}
__device__ unsigned long long block_min_u64(unsigned long long v) {
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, nw = blockDim.x >> 5;
    v = warp_min_u64(v);
    if (nw == 1) return v;
    cta_sync();
    if (lane == 0) L.red64[w] = v;
    cta_sync();
    return warp_min_u64(lane < nw ? L.red64[lane] : ~0ull);
}
// Sum of one int and min of one unsigned per thread, in one exchange.
__device__ void block_sum_min(int &sum, unsigned &mn) {
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, nw = blockDim.x >> 5;
    sum = warp_sum(sum);
    mn = __reduce_min_sync(FULL, mn);
    if (nw == 1) return;
    cta_sync();
    if (lane == 0) {
        L.red32[w] = sum;
        L.wcnt[w] = (int)mn;
    }
    cta_sync();
    sum = warp_sum(lane < nw ? L.red32[lane] : 0);
    mn = __reduce_min_sync(FULL, lane < nw ? (unsigned)L.wcnt[lane] : 0xffffffffu);
}
__device__ int block_sum(int v) {
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, nw = blockDim.x >> 5;
    v = warp_sum(v);
    if (nw == 1) return v;
    cta_sync();
    if (lane == 0) L.red32[w] = v;
    cta_sync();
    return warp_sum(lane < nw ? L.red32[lane] : 0);
}

__device__ __forceinline__ bool resident(int k, int32_t D) {
    const Inst &I = SI;
    const View &V = SV;
    return (V.resb[(size_t)k * I.nw + (D >> 5)] >> (D & 31)) & 1u;
}

// n_k(D) += d and n2_k(D) += d (packed rows in the specialised loop: n2 is the high half).
__device__ __forceinline__ void add_n(int k, int32_t D, int d) { atomicAdd(&SV.h[(size_t)k * SI.nstr + D], d); }
__device__ __forceinline__ void add_n2(int k, int32_t D, int d) {
    if (M_HH) atomicAdd(&SV.h[(size_t)k * SI.nstr + D], d * 65536);
    else atomicAdd(&SV.h2[(size_t)k * SI.nstr + D], d);
}

// u(D) += d; the specialised loop keeps u as 16-bit halves (< 2^15 in that mode):
// the argmax then pulls 2 bytes per datum for it instead of 4.
__device__ __forceinline__ void add_u(int32_t D, int d) {
    if (M_HH) atomicAdd(reinterpret_cast<unsigned *>(SV.u) + (D >> 1), (unsigned)d << (16 * (D & 1)));
    else atomicAdd(&SV.u[D], d);
}
// u(D) for the four data 4v .. 4v+3
__device__ __forceinline__ uint4 u_vec4(int v) {
    if (M_HH) {
        const uint2 w = reinterpret_cast<const uint2 *>(SV.u)[v];
        return make_uint4(w.x & 0xFFFFu, w.x >> 16, w.y & 0xFFFFu, w.y >> 16);
    }
    const int4 w = reinterpret_cast<const int4 *>(SV.u)[v];
    return make_uint4((uint32_t)w.x, (uint32_t)w.y, (uint32_t)w.z, (uint32_t)w.w);
}

// Row-derived mode (Inst::sl): T has left the shared pool (R2).
__device__ __forceinline__ bool allocated(int32_t T) { return (SV.al[T >> 5] >> (T & 31)) & 1u; }
__device__ __forceinline__ void set_alloc(int32_t T, int sign) {
    if (sign < 0) atomicOr(&SV.al[T >> 5], 1u << (T & 31));
    else atomicAnd(&SV.al[T >> 5], ~(1u << (T & 31)));
}
// Row-derived mode: the inputs of a <= 3-input row {a, b, c} (-1 = absent)
// not resident on GPU k -- their count cnt_k(T) and the first two of them.
__device__ __forceinline__ int missing_of(int k, int32_t a, int32_t b, int32_t c, int32_t &m0, int32_t &m1) {
    const bool ma = a >= 0 && !resident(k, a), mb = b >= 0 && !resident(k, b), mc = c >= 0 && !resident(k, c);
    m0 = ma ? a : (mb ? b : c);
    m1 = ma ? (mb ? b : c) : c;
    return (int)ma + (int)mb + (int)mc;
}

// Data->task segment bounds of D (int32 copy in shared memory when placed).
__device__ __forceinline__ void seg_of(int32_t D, int64_t &b, int64_t &e) {
    const Inst &I = SI;
    const View &V = SV;
    if (V.dptr32) {
        b = V.dptr32[D];
        e = V.dptr32[D + 1];
    } else {
        b = __ldg(&I.dptr[D]);
        e = __ldg(&I.dptr[D + 1]);
    }
}
// Size and bus time of D: scalars when all sizes are equal (the paper's model).
__device__ __forceinline__ uint64_t size_of(int32_t D) {
    const Inst &I = SI;
    return (DTS_FAST || I.size0) ? I.size0 : __ldg(&I.size[D]);
}
__device__ __forceinline__ int64_t delta_of(int32_t D) {
    const Inst &I = SI;
    return (DTS_FAST || I.size0) ? I.delta0 : __ldg(&I.delta[D]);
}

__device__ __forceinline__ int64_t tau_of(int32_t T) {
    const Inst &I = SI;
    return I.tau ? __ldg(&I.tau[T]) : I.default_tau;
}

// D(T) as carried by an edge record / plan entry: the full row when
// len <= 3 (r0..r2, -1 = absent), else only len (rows are read from the CSR).
struct Row {
    int32_t r0, r1, r2, len;
};


// Rows longer than 3: the (first two) inputs of T not resident on GPU k,
// skipping `skip`, read from the CSR.
__device__ __noinline__ void missing_pair_long(int k, int32_t T, int32_t skip, int32_t &a, int32_t &b) {
    const Inst &I = SI;
    a = -1;
    b = -1;
    const int64_t rb = __ldg(&I.tptr[T]), re = __ldg(&I.tptr[T + 1]);
    for (int64_t i = rb; i < re; i++) {
        const int32_t D = __ldg(&I.tdat[i]);
        if (D == skip || resident(k, D)) continue;
        if (a < 0) a = D;
        else if (b < 0) b = D;
    }
}

// The (first two) inputs of T not resident on GPU k, skipping `skip`.
__device__ __forceinline__ void missing_pair(int k, int32_t T, Row r, int32_t skip, int32_t &a, int32_t &b) {
    if (M_LONG(r.len > 3)) {
        missing_pair_long(k, T, skip, a, b);
        return;
    }
    a = -1;
    b = -1;
    const int32_t c[3] = {r.r0, r.r1, r.r2};
#pragma unroll
    for (int i = 0; i < 3; i++) {
        const int32_t D = c[i];
        if (D < 0 || D == skip || resident(k, D)) continue;
        if (a < 0) a = D;
        else b = D;
    }
}

// u(D) (own tasks) and np (when plan_k >= 0) of T's inputs for pool_move, long rows.
__device__ __noinline__ void pool_move_long_row(int32_t T, int sign, int plan_k, bool own) {
    const Inst &I = SI;
    const View &V = SV;
    const int64_t rb = __ldg(&I.tptr[T]), re = __ldg(&I.tptr[T + 1]);
    for (int64_t i = rb; i < re; i++) {
        const int32_t D = __ldg(&I.tdat[i]);
        if (own) atomicAdd(&V.u[D], sign);
        if (plan_k >= 0) atomicAdd(&V.np[(size_t)plan_k * I.nstr + D], -sign);
    }
}

// T leaves (sign = -1) or re-enters (sign = +1) the shared pool of unallocated
// tasks (R2, R4): the ALLOC bit in all K state copies, the score buckets of
// every GPU on which T has one or two missing inputs, u(D) for its inputs,
// and np_k(D) when it enters / leaves plannedTasks_k (plan_k >= 0).  Called by
// ONE thread per task; the touched words of s are T's own.  The state words
// are loaded four at a time (one round trip), then updated by a compact loop
// (the code stays small: the loop kernel is instruction-cache bound).
// Task shards (§8(e)): s, h, h2 and u are the owner's (partial) arrays, np is
// replicated -- a shard applies np for every task of a plan, the rest only
// for its own tasks.
__device__ void pool_move(int32_t T, Row r, int sign, int plan_k) {
    const Inst &I = SI;
    const View &V = SV;
    const int K = I.K;
    const bool own = DTS_FAST || (T >= I.t_lo && T < I.t_hi);
    if (M_SL(I)) {  // row-derived state: the allocation bit, then each GPU's buckets
        set_alloc(T, sign);
#pragma unroll 1
        for (int j = 0; j < K; j++) {
            int32_t a, b;
            const int c = missing_of(j, r.r0, r.r1, r.r2, a, b);
            if (c == 1) {
                add_n(j, a, sign);
            } else if (c == 2) {
                add_n2(j, a, sign);
                add_n2(j, b, sign);
            }
        }
    }
    for (int j0 = 0; own && !M_SL(I) && j0 < K; j0 += 4) {
        uint32_t w0 = 0, w1 = 0, w2 = 0, w3 = 0;
        w0 = V.s[(size_t)j0 * I.m_pad + T];
        if (j0 + 1 < K) w1 = V.s[(size_t)(j0 + 1) * I.m_pad + T];
        if (j0 + 2 < K) w2 = V.s[(size_t)(j0 + 2) * I.m_pad + T];
        if (j0 + 3 < K) w3 = V.s[(size_t)(j0 + 3) * I.m_pad + T];
        const int je = K - j0 < 4 ? K - j0 : 4;
#pragma unroll 1
        for (int jj = 0; jj < je; jj++) {
            const uint32_t w = jj == 0 ? w0 : (jj == 1 ? w1 : (jj == 2 ? w2 : w3));
            const int j = j0 + jj;
            V.s[(size_t)j * I.m_pad + T] = sign < 0 ? (w | ALLOC_BIT) : (w & ~ALLOC_BIT);
            const uint32_t c = (w >> 24) & 0x7fu;
            if (c == 1u) {
                atomicAdd(&V.h[(size_t)j * I.nstr + (w & XOR_MASK)], sign);
            } else if (c == 2u) {
                int32_t a, b;
                missing_pair(j, T, r, -1, a, b);
                atomicAdd(&V.h2[(size_t)j * I.nstr + a], sign);
                atomicAdd(&V.h2[(size_t)j * I.nstr + b], sign);
            }
        }
    }
    if (M_LONG(r.len > 3)) {
        pool_move_long_row(T, sign, plan_k, own);
        return;
    }
    const int32_t c[3] = {r.r0, r.r1, r.r2};
#pragma unroll
    for (int i = 0; i < 3; i++) {
        if (c[i] < 0) continue;
        if (own) add_u(c[i], sign);
        if (plan_k >= 0) atomicAdd(&V.np[(size_t)plan_k * I.nstr + c[i]], -sign);
    }
}

// One (task, GPU) item of pool_move_many in the packed-state mode, out of line
// (keeps the hot row-derived loop compact).
__device__ __noinline__ void pool_item_packed(int4 e, int j, int sign) {
    const Inst &I = SI;
    const View &V = SV;
    const int32_t T = e.x;
    uint32_t *sp = &V.s[(size_t)j * I.m_pad + T];
    const uint32_t w = *sp;
    *sp = sign < 0 ? (w | ALLOC_BIT) : (w & ~ALLOC_BIT);
    const uint32_t c = (w >> 24) & 0x7fu;
    if (c == 1u) {
        atomicAdd(&V.h[(size_t)j * I.nstr + (w & XOR_MASK)], sign);
    } else if (c == 2u) {
        int32_t a, b;
        const bool lng = M_LONG(e.w == ROW_LONG);
        const int len = lng ? 4 : (e.y >= 0) + (e.z >= 0) + (e.w >= 0);
        if (len == 2) {  // both inputs miss: no residency lookups
            a = e.y;
            b = e.z >= 0 ? e.z : e.w;
        } else {
            missing_pair(j, T, Row{e.y, e.z, lng ? -1 : e.w, len}, -1, a, b);
        }
        atomicAdd(&V.h2[(size_t)j * I.nstr + a], sign);
        atomicAdd(&V.h2[(size_t)j * I.nstr + b], sign);
    }
}

// Block-wide pool_move of P tasks given as plan entries {T, D0, D1, D2}
// (-1 = absent input, D2 = ROW_LONG: read the row from the CSR).  The
// (task, simulated GPU) state items and the per-task input counts (u, np) are
// spread over the CTA: one short dependent chain per item instead of K
// divergent ones per task on one thread.  Entries must be visible to every
// thread (written before a barrier); the caller synchronises afterwards.
__device__ __noinline__ void pool_move_many(const int4 *ents, int P, int sign, int plan_k) {
    const Inst &I = SI;
    const View &V = SV;
    const int K = I.K;
    const int n_state = P * K;
    for (int idx = threadIdx.x; idx < n_state + P; idx += blockDim.x) {
        if (idx < n_state) {
            const int p = idx / K, j = idx - p * K;
            const int4 e = ents[p];
            const int32_t T = e.x;
            if (M_SL(I)) {  // row-derived state: T's missing inputs on GPU j from its row
                int32_t a, b;
                const int c = missing_of(j, e.y, e.z, e.w, a, b);
                if (c == 1) {
                    add_n(j, a, sign);
                } else if (c == 2) {
                    add_n2(j, a, sign);
                    add_n2(j, b, sign);
                }
                continue;
            }
            if (T < I.t_lo || T >= I.t_hi) continue;  // another shard's task
            pool_item_packed(e, j, sign);
        } else {
            const int4 e = ents[idx - n_state];
            const int32_t T = e.x;
            const bool own = DTS_FAST || (T >= I.t_lo && T < I.t_hi);
            if (M_SL(I)) set_alloc(T, sign);
            if (M_LONG(e.w == ROW_LONG)) {
                pool_move_long_row(T, sign, plan_k, own);
                continue;
            }
            const int32_t c[3] = {e.y, e.z, e.w};
#pragma unroll
            for (int q = 0; q < 3; q++) {
                if (c[q] < 0) continue;
                if (own) add_u(c[q], sign);
                if (plan_k >= 0) atomicAdd(&V.np[(size_t)plan_k * I.nstr + c[q]], -sign);
            }
        }
    }
}

// D(T) of task T as a plan entry {T, D0, D1, D2 | ROW_LONG} (thread-local).
__device__ __forceinline__ int4 entry_of_task(int32_t T) {
    const Inst &I = SI;
    const int64_t rb = __ldg(&I.tptr[T]), re = __ldg(&I.tptr[T + 1]);
    const int len = (int)(re - rb);
    int4 e = make_int4(T, -1, -1, -1);
    if (len > 0) e.y = __ldg(&I.tdat[rb]);
    if (len > 1) e.z = __ldg(&I.tdat[rb + 1]);
    if (len > 2) e.w = len > 3 ? ROW_LONG : __ldg(&I.tdat[rb + 2]);
    return e;
}

// Thread 0: D(T) for serve_loads straight from a fallback / EAGER pick's
// entry (rows are sorted, so the entry lists them ascending, R10) -- no second
// CSR read; a longer row is read by the serve path (row_len = -1).
__device__ __forceinline__ void row_from_entry(int4 e) {
    if (M_LONG(e.w == ROW_LONG)) {
        L.row_len = -1;
        return;
    }
    int len = 0;
    if (e.y >= 0) L.row[len++] = e.y;
    if (e.z >= 0) L.row[len++] = e.z;
    if (e.w >= 0) L.row[len++] = e.w;
    L.row_len = len;
}

// Packed-state mode of seg_update, out of line: the hot row-derived path stays
// compact (the loop kernel is instruction-cache bound).
__device__ __noinline__ void seg_update_packed(int k, int32_t D, bool load) {
    const Inst &I = SI;
    const View &V = SV;
    int64_t b, e;
    seg_of(D, b, e);
    uint32_t *sk = V.s + (size_t)k * I.m_pad;
    int32_t *hk = V.h + (size_t)k * I.nstr;
    int32_t *h2k = V.h2 + (size_t)k * I.nstr;
    for (int64_t i = b + threadIdx.x; i < e; i += blockDim.x) {
        const int4 ed = __ldg(&I.dedge[i]);
        const int32_t T = ed.x;
        const uint32_t w = sk[T];
        sk[T] = (load ? (w - CNT_ONE) : (w + CNT_ONE)) ^ (uint32_t)D;
        if (w & ALLOC_BIT) continue;
        const uint32_t c = (w >> 24) & 0x7fu;
        const int32_t x = (int32_t)(w & XOR_MASK);
        if (load) {
            if (c == 1u) {  // 1 -> 0: no longer scores for D
                atomicSub(&hk[D], 1);
            } else if (c == 2u) {  // 2 -> 1: now freed by its other missing datum
                const int32_t o = x ^ D;
                atomicSub(&h2k[D], 1);
                atomicSub(&h2k[o], 1);
                atomicAdd(&hk[o], 1);
            } else if (c == 3u) {  // 3 -> 2: one load away from two data
                int32_t a2 = ed.y, b2 = ed.z;  // |D(T)| = 3: both others miss
                if (M_LONG(ed.w > 3)) missing_pair(k, T, Row{-1, -1, -1, ed.w}, -1, a2, b2);
                atomicAdd(&h2k[a2], 1);
                atomicAdd(&h2k[b2], 1);
            }
        } else {
            if (c == 0u) {  // 0 -> 1
                atomicAdd(&hk[D], 1);
            } else if (c == 1u) {  // 1 -> 2: missing {x, D}
                atomicSub(&hk[x], 1);
                atomicAdd(&h2k[x], 1);
                atomicAdd(&h2k[D], 1);
            } else if (c == 2u) {  // 2 -> 3
                int32_t a2 = ed.y, b2 = ed.z;  // |D(T)| = 3: both others missed
                if (M_LONG(ed.w > 3)) missing_pair(k, T, Row{-1, -1, -1, ed.w}, D, a2, b2);
                atomicSub(&h2k[a2], 1);
                atomicSub(&h2k[b2], 1);
            }
        }
    }
}


// a2: datum D becomes resident (load) / leaves (evict) on GPU k.  Walk D's
// data->task segment (edge records: the task and its other inputs in one 16 B
// load): cnt_k(T) -/+= 1, x_k(T) ^= D, and move every unallocated task between
// the score buckets h (cnt 1) and h2 (cnt 2).  The residency bit of D is
// already updated.  Each task appears once in the segment, so the state words
// are plain read-modify-writes; the buckets are atomics.
__device__ void seg_update(int k, int32_t D, bool load) {
    const Inst &I = SI;
    const View &V = SV;
    if (!M_SL(I)) {
        seg_update_packed(k, D, load);
        return;
    }
    int64_t b, e;
    seg_of(D, b, e);
    int32_t *hk = V.h + (size_t)k * I.nstr;
    int32_t *h2k = V.h2 + (size_t)k * I.nstr;
    {  // row-derived state: cnt_k(T) before the change from T's other inputs
        for (int64_t i = b + threadIdx.x; i < e; i += blockDim.x) {
            const int4 ed = __ldg(&I.dedge[i]);
            if (allocated(ed.x)) continue;
            const bool my = ed.y >= 0 && !resident(k, ed.y), mz = ed.z >= 0 && !resident(k, ed.z);
            const int c = (int)my + (int)mz + (load ? 1 : 0);  // missing inputs before
            const int32_t o = my ? ed.y : ed.z;                 // the other missing one (c == 2 / 1)
            if (M_HH) {  // packed rows: n in the low half, n2 in the high half
                constexpr int U2 = 65536;
                if (load) {
                    if (c == 1) {  // 1 -> 0
                        atomicSub(&hk[D], 1);
                    } else if (c == 2) {  // 2 -> 1: now freed by o
                        atomicSub(&hk[D], U2);
                        atomicAdd(&hk[o], 1 - U2);
                    } else if (c == 3) {  // 3 -> 2
                        atomicAdd(&hk[ed.y], U2);
                        atomicAdd(&hk[ed.z], U2);
                    }
                } else {
                    if (c == 0) {  // 0 -> 1
                        atomicAdd(&hk[D], 1);
                    } else if (c == 1) {  // 1 -> 2: missing {o, D}
                        atomicAdd(&hk[o], U2 - 1);
                        atomicAdd(&hk[D], U2);
                    } else if (c == 2) {  // 2 -> 3
                        atomicSub(&hk[ed.y], U2);
                        atomicSub(&hk[ed.z], U2);
                    }
                }
                continue;
            }
            if (load) {
                if (c == 1) {  // 1 -> 0
                    atomicSub(&hk[D], 1);
                } else if (c == 2) {  // 2 -> 1: now freed by o
                    atomicSub(&h2k[D], 1);
                    atomicSub(&h2k[o], 1);
                    atomicAdd(&hk[o], 1);
                } else if (c == 3) {  // 3 -> 2
                    atomicAdd(&h2k[ed.y], 1);
                    atomicAdd(&h2k[ed.z], 1);
                }
            } else {
                if (c == 0) {  // 0 -> 1
                    atomicAdd(&hk[D], 1);
                } else if (c == 1) {  // 1 -> 2: missing {o, D}
                    atomicSub(&hk[o], 1);
                    atomicAdd(&h2k[o], 1);
                    atomicAdd(&h2k[D], 1);
                } else if (c == 2) {  // 2 -> 3
                    atomicSub(&h2k[ed.y], 1);
                    atomicSub(&h2k[ed.z], 1);
                }
            }
        }
        return;
    }
}

__device__ __forceinline__ void push_event(uint8_t op, int k, int32_t D, int32_t T, int64_t t, int64_t te) {
    const Inst &I = SI;
    const int64_t i = L.n_events;
    if (i < I.ev_cap) {
        dts_event ev;
        ev.t_ns = t;
        ev.t_end_ns = te;
        ev.gpu = k;
        ev.data = D;
        ev.task = T;
        ev.op = op;
        ev.pad[0] = ev.pad[1] = ev.pad[2] = 0;
        I.events[i] = ev;
    }
    L.n_events = i + 1;
}

// Thread 0: T (started at `start`) becomes the newest of k's last W served
// tasks; returns k's next request time (R7 / R29): W = 0 when T ends, W >= 1
// when the (j-W+1)-th of its j tasks starts -- the first W requests at once
// (at t).  Task times of earlier tasks are this thread's own writes.
__device__ __forceinline__ int64_t next_request(int k, int32_t T, int64_t t, int64_t start, int64_t end) {
    const Inst &I = SI;
#if DTS_FAST
    (void)I, (void)k, (void)T, (void)t, (void)start;
    return end;
#else
    if (I.W == 0) return end;
    const int W = I.W;
    const int j = ++L.won[k];
    I.wring[k * MAX_W + (j - 1) % W] = T;
    if (j < W) return t;
    return W == 1 ? start : __ldcg(&I.tstart[I.wring[k * MAX_W + j % W]]);
#endif
}

// Thread 0: record the service of T on k (time model of PAPER.md:276-342, R7, R9).
__device__ __forceinline__ void finish_serve(int k, int32_t T, int64_t t, int64_t ready, int64_t tau) {
    const Inst &I = SI;
    const int64_t start = ready > L.gpu_free[k] ? ready : L.gpu_free[k];
    const int64_t end = start + tau;
    L.gpu_free[k] = end;
    I.tstart[T] = start;
    I.tend[T] = end;
    if (end > L.makespan) L.makespan = end;
    I.serve_gpu[L.n_served] = k;
    I.serve_task[L.n_served] = T;
    L.n_served++;
    L.req[k] = next_request(k, T, t, start, end);  // R7, R29
    L.alg_bytes += 24;
}

// Thread 0: pop the smallest planned task of k (Alg. 5 l.2 / l.11, R3); it
// leaves plannedTasks_k (np_k(D) -= 1 for its inputs).  Returns T and its tau.
__device__ int32_t pop_planned(int k, int64_t *tau) {
    const Inst &I = SI;
    const View &V = SV;
    const int4 *pl = V.plan + (size_t)k * I.plan_cap;
    int h = L.plan_head[k];
    const int pe = L.plan_end[k];
    if (h >= pe) {  // internal inconsistency (never expected): end the run with an error
        L.error = 3;
        L.row_len = 0;
        return -1;
    }
    int4 e = pl[h];
    while (e.x < 0 && h + 1 < pe) e = pl[++h];  // bounded by plan_end (LUF-removed entries)
    if (e.x < 0) {
        L.error = 3;
        L.row_len = 0;
        return -1;
    }
    L.plan_head[k] = h + 1;
    L.plan_live[k]--;
    int32_t *npk = V.np + (size_t)k * I.nstr;
    if (!M_LONG(e.w == ROW_LONG)) {
        if (e.y >= 0) atomicSub(&npk[e.y], 1);
        if (e.z >= 0) atomicSub(&npk[e.z], 1);
        if (e.w >= 0) atomicSub(&npk[e.w], 1);
    } else {
        const int64_t rb = __ldg(&I.tptr[e.x]), re = __ldg(&I.tptr[e.x + 1]);
        for (int64_t i = rb; i < re; i++) atomicSub(&npk[__ldg(&I.tdat[i])], 1);
    }
    if (V.plan_cum) {
        const int64_t *pc = V.plan_cum + (size_t)k * I.plan_cap;
        *tau = pc[h] - (h > 0 ? pc[h - 1] : 0);
    } else {
        *tau = I.default_tau;
    }
    // D(T) for serve_loads, ascending (R10), straight from the entry when cached
    if (!M_LONG(e.w == ROW_LONG)) {
        int32_t a = e.y, b = e.z, c = e.w;  // -1 = absent; sort descending, count
        if (a < b) { const int32_t t = a; a = b; b = t; }
        if (b < c) { const int32_t t = b; b = c; c = t; }
        if (a < b) { const int32_t t = a; a = b; b = t; }
        const int len = (a >= 0) + (b >= 0) + (c >= 0);
        L.row_len = len;
        if (len == 3) { L.row[0] = c; L.row[1] = b; L.row[2] = a; }
        else if (len == 2) { L.row[0] = b; L.row[1] = a; }
        else if (len == 1) { L.row[0] = a; }
    } else {
        L.row_len = -1;
    }
    return e.x;
}

// Thread 0, sequential pops (used for prefix runs, max_served >= 0): serve
// every request that finds plannedTasks_k non-empty (Alg. 5 l.1-2) until one
// finds it empty (returns that k; L.k, L.t set) or the run ends (-1).  The
// popped task's inputs are resident (LUF drops planned tasks whose inputs it
// evicts, Alg. 6 l.8), so serving it is time-model arithmetic.
// np_k is not maintained by pops: LUF on GPU k only runs while k serves the
// first task of a new plan (or a fallback task), and every scan resets np_k.
__device__ __forceinline__ int pop_run_seq() {
    const Inst &I = SI;
    const View &V = SV;
    const int K = I.K, W = M_W(I), pcap = I.plan_cap;
    const int64_t maxs = I.max_served, dtau = I.default_tau;
    int32_t *const sg = I.serve_gpu;
    int32_t *const stk = I.serve_task;
    int64_t *const tst = I.tstart;
    int64_t *const ten = I.tend;
    int64_t ns = L.n_served, mk = L.makespan, pops = 0;
    int ret = -1;
    while (maxs < 0 || ns < maxs) {
        // the next request and the one after it: the two smallest (req_j, j)
        // over the non-idle GPUs (R8); eight GPUs' words loaded before any
        // compare, the compares branch-free (an idle GPU's key is INT64_MAX)
        int k = -1, k2 = -1;
        int64_t t1 = INT64_MAX, t2 = INT64_MAX;
        for (int j0 = 0; j0 < K; j0 += 8) {
            int64_t r[8];
#pragma unroll
            for (int q = 0; q < 8; q++) {
                const int j = j0 + q;
                r[q] = (j < K && !L.idle[j]) ? L.req[j] : INT64_MAX;
            }
#pragma unroll
            for (int q = 0; q < 8; q++) {
                const int j = j0 + q;
                const bool ok = r[q] != INT64_MAX;
                const bool b1 = ok & (r[q] < t1);
                const bool b2 = ok & !b1 & (r[q] < t2);
                k2 = b1 ? k : (b2 ? j : k2);
                t2 = b1 ? t1 : (b2 ? r[q] : t2);
                k = b1 ? j : k;
                t1 = b1 ? r[q] : t1;
            }
        }
        if (k < 0) break;
        int live = L.plan_live[k];
        if (live == 0) {
            ret = k;
            L.k = k;
            L.t = t1;
            break;
        }
        int h = L.plan_head[k];
        int64_t req = t1, gfree = L.gpu_free[k];
        const int4 *pl = V.plan + (size_t)k * pcap;
        const int64_t *pc = V.plan_cum ? V.plan_cum + (size_t)k * pcap : nullptr;
        while (true) {
            const int T = pl[h].x;
            const int64_t tau = pc ? pc[h] - (h > 0 ? pc[h - 1] : 0) : dtau;
            h++;
            live--;
            const int64_t start = req > gfree ? req : gfree;
            const int64_t end = start + tau;
            gfree = end;
            __stcg(&tst[T], start);
            __stcg(&ten[T], end);
            mk = end > mk ? end : mk;
            __stcg(&sg[ns], k);
            __stcg(&stk[ns], T);
            ns++;
            pops++;
            req = W == 0 ? end : next_request(k, T, req, start, end);  // R7, R29
            if (live == 0 || (maxs >= 0 && ns >= maxs)) break;
            if (k2 >= 0 && (req > t2 || (req == t2 && k2 < k))) break;
        }
        L.plan_head[k] = h;
        L.plan_live[k] = live;
        L.req[k] = req;
        L.gpu_free[k] = gfree;
    }
    L.n_served = ns;
    L.makespan = mk;
    L.alg_bytes += 24ull * (uint64_t)pops;
    return ret;
}


// a[lo..hi) := base + inclusive prefix sums of a[lo..hi).  Block-wide.
__device__ __noinline__ void block_incl_scan(int64_t *a, int lo, int hi, int64_t base) {
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, nw = blockDim.x >> 5;
    int64_t carry = base;
    for (int c = lo; c < hi; c += blockDim.x) {
        const int i = c + threadIdx.x;
        int64_t v = i < hi ? a[i] : 0;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const int64_t t = __shfl_up_sync(FULL, v, o);
            if (lane >= o) v += t;
        }
        cta_sync();
        if (lane == 31) L.red64[w] = (unsigned long long)v;
        cta_sync();
        int64_t off = 0, tot = 0;
        for (int j = 0; j < nw; j++) {
            const int64_t x = (int64_t)L.red64[j];
            if (j < w) off += x;
            tot += x;
        }
        if (i < hi) a[i] = carry + off + v;
        carry += tot;
    }
    cta_sync();
}

// After LUF removed planned tasks of k (T = -1), close the holes: ordered
// compaction of [head, end) so the live entries are contiguous (pop_batch
// indexes them directly), and rebuild their tau prefix sums.  Block-wide.
__device__ __noinline__ void compact_plan(int k) {
    const Inst &I = SI;
    const View &V = SV;
    int4 *pl = V.plan + (size_t)k * I.plan_cap;
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, nw = blockDim.x >> 5;
    const unsigned lt = (1u << lane) - 1u;
    const int ph = L.plan_head[k], pe = L.plan_end[k];
    int out = ph;
    for (int c = ph; c < pe; c += blockDim.x) {
        const int i = c + threadIdx.x;
        const int4 e = i < pe ? pl[i] : make_int4(-1, -1, -1, -1);
        const bool keep = e.x >= 0;
        const unsigned msk = __ballot_sync(FULL, keep);
        if (lane == 0) L.wcnt[w] = __popc(msk);
        cta_sync();  // every read of this chunk happened (writes go below its start)
        int off = out, tot = 0;
        for (int j = 0; j < nw; j++) {
            const int x = L.wcnt[j];
            if (j < w) off += x;
            tot += x;
        }
        if (keep) pl[off + __popc(msk & lt)] = e;
        out += tot;
        cta_sync();
    }
    if (V.plan_cum) {
        int64_t *pc = V.plan_cum + (size_t)k * I.plan_cap;
        for (int i = ph + threadIdx.x; i < out; i += blockDim.x) pc[i] = tau_of(pl[i].x);
        cta_sync();
        block_incl_scan(pc, ph, out, ph > 0 ? pc[ph - 1] : 0);
    }
    if (threadIdx.x == 0) L.plan_end[k] = out;
    cta_sync();
}

// Sum of tau over the c planned tasks of GPU j starting at plan index h.
__device__ __forceinline__ int64_t plan_span(int j, int h, int c) {
    const Inst &I = SI;
    const View &V = SV;
    if (c <= 0) return 0;
    if (!V.plan_cum) return (int64_t)c * I.default_tau;
    const int64_t *pc = V.plan_cum + (size_t)j * I.plan_cap;
    return pc[h + c - 1] - (h > 0 ? pc[h - 1] : 0);
}

// Pop batch bookkeeping of GPU j (see pop_batch): its first request time
// (req), the start of its first pop (start0) and its plan head.  The i-th pop
// is requested at req (i = 0) or start0 + span(i) (W = 0: a GPU asks again
// when its task ends, R7).
struct PopGpu {
    int64_t req, start0;
    int head;
};

__device__ __forceinline__ int64_t pop_req(int j, const PopGpu &g, int i) {
    return i == 0 ? g.req : g.start0 + plan_span(j, g.head, i);
}

// #{ i < c : (req_{j,i}, j) < (r, k) } -- the pops of GPU j that precede the
// request (r, k) in the (time, GPU id) order (R8).  Request times increase
// with i, so a binary search (multiplications only: 64-bit division is a long
// software sequence on the SM).
__device__ __forceinline__ int pops_before(int j, PopGpu g, int c, int64_t r, int k) {
    const Inst &I = SI;
    const View &V = SV;
    if (c <= 0) return 0;
    const bool tie_ok = j < k;  // equal times: the lower GPU id asks first
    if (!(g.req < r || (g.req == r && tie_ok))) return 0;
    if (!V.plan_cum) {  // i >= 1 asks at start0 + i * tau: binary search, multiplications only
        const int64_t tau = I.default_tau;
        int lo = 1, hi = c;
        while (lo < hi) {
            const int mid = (lo + hi) >> 1;
            const int64_t rm = g.start0 + (int64_t)mid * tau;
            const bool b = (rm < r) | ((rm == r) & tie_ok);
            lo = b ? mid + 1 : lo;
            hi = b ? hi : mid;
        }
        return lo;
    }
    int lo = 1, hi = c;  // first i in [1, c] whose request does not precede (r, k)
    while (lo < hi) {
        const int mid = (lo + hi) >> 1;
        const int64_t rm = g.start0 + plan_span(j, g.head, mid);
        const bool b = (rm < r) | ((rm == r) & tie_ok);
        lo = b ? mid + 1 : lo;
        hi = b ? hi : mid;
    }
    return lo;
}

// Every request that finds plannedTasks_k non-empty (Alg. 5 l.1-2) up to the
// next one that finds it empty, served at once.  Between two scans nothing
// but pops happens, and a pop only moves time: the popped task's inputs are
// resident (LUF drops planned tasks whose inputs it evicts, Alg. 6 l.8) and
// np_k is rebuilt at every scan of k (reset_plan), so each GPU's request
// times are prefix sums of its planned tasks' tau (W = 0).
// Warp 0 (one lane per simulated GPU, K <= 32) finds the next scan -- the
// earliest (request after the GPU's last pop, GPU id) (R8) -- and each GPU's
// pop count before it; then every thread places pops in the global service
// order by merge ranks.  Sets L.cmd (CMD_SCAN with L.k, L.t, or CMD_DONE).
// Scalar phase of pop_batch for K <= KR with the per-GPU values in registers
// (fully unrolled over KR): the next scan (earliest request after a GPU's last
// pop, R8), each GPU's pop count before it, the new request times.
template <int KR>
__device__ __forceinline__ void pop_batch_scalar() {
    const Inst &I = SI;
    const int K = I.K;
    int64_t rq[KR], st[KR], S[KR];
    int hd[KR], lv[KR];
    bool act[KR];
#pragma unroll
    for (int j = 0; j < KR; j++) {
        act[j] = j < K && !L.idle[j];
        rq[j] = j < K ? L.req[j] : 0;
        const int64_t gf = j < K ? L.gpu_free[j] : 0;
        st[j] = rq[j] > gf ? rq[j] : gf;
        hd[j] = j < K ? L.plan_head[j] : 0;
        lv[j] = j < K ? L.plan_end[j] - hd[j] : 0;
    }
    int kb = -1;
    int64_t sb = INT64_MAX;
#pragma unroll
    for (int j = 0; j < KR; j++) {
        S[j] = lv[j] == 0 ? rq[j] : st[j] + plan_span(j, hd[j], lv[j]);
        const bool take = act[j] & ((kb < 0) | (S[j] < sb));
        kb = take ? j : kb;
        sb = take ? S[j] : sb;
    }
    int total = 0;
    int64_t mk = L.makespan;
#pragma unroll
    for (int j = 0; j < KR; j++) {
        if (j >= K) break;
        int c = 0;
        if (act[j] && kb >= 0) {
            PopGpu g;
            g.req = rq[j];
            g.start0 = st[j];
            g.head = hd[j];
            c = j == kb ? lv[j] : pops_before(j, g, lv[j], sb, kb);
        }
        L.breq[j] = rq[j];
        L.bstart[j] = st[j];
        L.bhead[j] = hd[j];
        L.bcnt[j] = c;
        L.boff[j] = total;
        total += c;
        if (c > 0) {
            const int64_t last = st[j] + plan_span(j, hd[j], c);
            L.req[j] = last;  // W = 0 (R7)
            L.gpu_free[j] = last;
            L.plan_head[j] = hd[j] + c;  // plan_live: after the barrier (pop_batch)
            mk = last > mk ? last : mk;
        }
    }
    L.boff[K] = total;
    L.bns = L.n_served;
    L.n_served += total;
    L.makespan = mk;
    L.alg_bytes += 24ull * (uint64_t)total;
    L.k = kb;
    L.t = sb;
    L.cmd = kb < 0 ? CMD_DONE : CMD_SCAN;
}

// The same for 8 < K <= 32, values left in shared memory.
__device__ __noinline__ void pop_batch_scalar_smem() {
    const Inst &I = SI;
    const int K = I.K;
    int kb = -1;
    int64_t sb = INT64_MAX;
    for (int j = 0; j < K; j++) {
        const int64_t req = L.req[j];
        const int64_t start0 = req > L.gpu_free[j] ? req : L.gpu_free[j];
        const int head = L.plan_head[j];
        L.breq[j] = req;
        L.bstart[j] = start0;
        L.bhead[j] = head;
        if (L.idle[j]) continue;
        const int live = L.plan_end[j] - head;
        const int64_t S = live == 0 ? req : start0 + plan_span(j, head, live);
        if (kb < 0 || S < sb) {
            kb = j;
            sb = S;
        }
    }
    int total = 0;
    int64_t mk = L.makespan;
    for (int j = 0; j < K; j++) {
        int c = 0;
        if (!L.idle[j] && kb >= 0) {
            const int live = L.plan_end[j] - L.bhead[j];
            PopGpu g;
            g.req = L.breq[j];
            g.start0 = L.bstart[j];
            g.head = L.bhead[j];
            c = j == kb ? live : pops_before(j, g, live, sb, kb);
        }
        L.bcnt[j] = c;
        L.boff[j] = total;
        total += c;
        if (c > 0) {
            const int64_t last = L.bstart[j] + plan_span(j, L.bhead[j], c);
            L.req[j] = last;  // W = 0 (R7)
            L.gpu_free[j] = last;
            L.plan_head[j] += c;  // plan_live: after the barrier (pop_batch)
            mk = last > mk ? last : mk;
        }
    }
    L.boff[K] = total;
    L.bns = L.n_served;
    L.n_served += total;
    L.makespan = mk;
    L.alg_bytes += 24ull * (uint64_t)total;
    L.k = kb;
    L.t = sb;
    L.cmd = kb < 0 ? CMD_DONE : CMD_SCAN;
}

__device__ void pop_batch() {
    const Inst &I = SI;
    const View &V = SV;
    const int K = I.K;
    PROF_T0(p_w0);
    if (threadIdx.x == 0) {
        if (K <= 4) pop_batch_scalar<4>();
        else if (K <= 8) pop_batch_scalar<8>();
        else pop_batch_scalar_smem();
    }
    cta_sync();
    // plan_live is what every thread summed at the top of the loop iteration to
    // choose this path: thread 0 may change it only once all have passed the
    // barrier above (changing it in the scalar phase let a late warp take the
    // other path -- divergent barriers, found by compute-sanitizer synccheck)
    {  // one GPU per thread, from the top of the CTA (idle in the rank phase below)
        const int j = (int)blockDim.x - 1 - (int)threadIdx.x;
        for (int jj = j; jj >= 0 && jj < K; jj += blockDim.x) L.plan_live[jj] -= L.bcnt[jj];
    }
    PROF_ADD(L, P_BW0, p_w0);
    PROF_T0(p_bd);
    const int P = L.boff[K];
    const int64_t ns = L.bns;
    PROF_CNT(L, P_NB, 1);
    PROF_CNT(L, P_NP, P);
    if (P <= (int)blockDim.x && P <= POP_RANK_MAX) {
        // merge ranks by counting: each pop's key (request time, GPU) in shared
        // memory, position = #keys before it (ties inside a GPU keep pop order)
        int j = 0, i = 0, T = -1;
        int64_t r = 0, start = 0, end = 0;
        const int p = threadIdx.x;
        if (p < P) {
            while (L.boff[j + 1] <= p) j++;
            i = p - L.boff[j];
            PopGpu g;
            g.req = L.breq[j];
            g.start0 = L.bstart[j];
            g.head = L.bhead[j];
            r = pop_req(j, g, i);
            start = i == 0 ? g.start0 : r;
            end = g.start0 + plan_span(j, g.head, i + 1);
            T = V.plan[(size_t)j * I.plan_cap + g.head + i].x;
            L.rkey[p] = r;
            L.rgpu[p] = j;
        }
        cta_sync();
        if (p < P) {
            int64_t pos = ns;
            for (int q = 0; q < P; q++) {
                const int64_t rq = L.rkey[q];
                const int jq = L.rgpu[q];
                // bitwise, not short-circuit: one predicated chain, no branches
                pos += (int)((rq < r) | ((rq == r) & ((jq < j) | ((jq == j) & (q < p)))));
            }
            __stcg(&I.tstart[T], start);
            __stcg(&I.tend[T], end);
            __stcg(&I.serve_gpu[pos], j);
            __stcg(&I.serve_task[pos], T);
        }
    } else {
    for (int p = threadIdx.x; p < P; p += blockDim.x) {
        int j = 0;
        while (L.boff[j + 1] <= p) j++;
        const int i = p - L.boff[j];
        PopGpu g;
        g.req = L.breq[j];
        g.start0 = L.bstart[j];
        g.head = L.bhead[j];
        const int64_t r = pop_req(j, g, i);
        const int64_t start = i == 0 ? g.start0 : r;
        const int64_t end = g.start0 + plan_span(j, g.head, i + 1);
        const int T = V.plan[(size_t)j * I.plan_cap + g.head + i].x;
        int64_t pos = ns + i;
        for (int j2 = 0; j2 < K; j2++) {
            if (j2 == j) continue;
            PopGpu g2;
            g2.req = L.breq[j2];
            g2.start0 = L.bstart[j2];
            g2.head = L.bhead[j2];
            pos += pops_before(j2, g2, L.bcnt[j2], r, j);
        }
        __stcg(&I.tstart[T], start);
        __stcg(&I.tend[T], end);
        __stcg(&I.serve_gpu[pos], j);
        __stcg(&I.serve_task[pos], T);
    }
    }
    cta_sync();
    PROF_ADD(L, P_BD, p_bd);
}

// CTA-wide, at every scan of GPU k: plannedTasks_k is empty (all popped or
// removed); clear np_k for every datum its last plan touched, so that np_k
// counts exactly the plan this scan creates (Alg. 6 l.3).
__device__ void reset_plan(int k) {
    const Inst &I = SI;
    const View &V = SV;
    const int4 *pl = V.plan + (size_t)k * I.plan_cap;
    int32_t *npk = V.np + (size_t)k * I.nstr;
    const int pe = L.plan_end[k];
    for (int i = threadIdx.x; i < pe; i += blockDim.x) {
        const int4 e = pl[i];
        if (!M_LONG(e.w == ROW_LONG)) {
            if (e.y >= 0) npk[e.y] = 0;
            if (e.z >= 0) npk[e.z] = 0;
            if (e.w >= 0) npk[e.w] = 0;
        } else {
            const int T = e.x >= 0 ? e.x : -1;
            if (T >= 0) {
                const int64_t rb = __ldg(&I.tptr[T]), re = __ldg(&I.tptr[T + 1]);
                for (int64_t j = rb; j < re; j++) npk[__ldg(&I.tdat[j])] = 0;
            }
        }
    }
    cta_sync();  // every thread has read plan_end before thread 0 clears it
    if (threadIdx.x == 0) {
        L.plan_head[k] = 0;
        L.plan_end[k] = 0;
        L.plan_live[k] = 0;
    }
    // no second barrier: nothing reads plannedTasks_k's bounds before the scan's next
    // barrier (the argmax's block reduction or, on a one-warp CTA, the fallback's)
}

__device__ __forceinline__ Row row_of_entry(int4 e) {
    if (M_LONG(e.w == ROW_LONG)) return Row{-1, -1, -1, 4};
    return Row{e.y, e.z, e.w, (e.y >= 0) + (e.z >= 0) + (e.w >= 0)};
}

__device__ __forceinline__ bool entry_uses(int4 e, int32_t D) {
    const Inst &I = SI;
    if (e.y == D || e.z == D) return true;
    if (!M_LONG(e.w == ROW_LONG)) return e.w == D;
    const int64_t rb = __ldg(&I.tptr[e.x]), re = __ldg(&I.tptr[e.x + 1]);
    for (int64_t i = rb; i < re; i++)
        if (__ldg(&I.tdat[i]) == D) return true;
    return false;
}

// LUF (Alg. 6): among the data in GPU k's memory that the taskBuffer does not
// use (nb(D) = 0, l.4-5; the taskBuffer = the task being served for W = 0),
// the one with the fewest uses in plannedTasks_k, lowest id on ties (R1).
// Block-wide; returns V (-1: every resident datum is a buffered input -- Alg.
// 6 l.6-7, belady_victim) and sets L.vslot to its index in res_list.
__device__ int32_t luf_victim(int k) {
    const Inst &I = SI;
    const View &V = SV;
    const int cnt = L.res_cnt[k];
    const int32_t *rl = V.res_list + (size_t)k * I.res_cap;
    // LUF key np_k(D); LRU policies: the serve index of D's last use on k
    const int32_t *npk = (M_LUF(I) ? V.np : V.lru) + (size_t)k * I.nstr;
    const int nr = L.row_len, nr2 = L.row2_len;
    unsigned long long best = ~0ull;
    int bslot = -1;
#if DTS_FAST
    // two entries per thread and pass, both loads issued before either key is
    // formed (C4b: 1,024 resident data, resident list and np_k in L2)
    for (int i0 = threadIdx.x; i0 < cnt; i0 += 2 * blockDim.x) {
        const int i1 = i0 + blockDim.x;
        const int32_t D0 = rl[i0];
        const int32_t D1 = i1 < cnt ? rl[i1] : -1;
        const uint32_t p0 = (uint32_t)npk[D0];
        const uint32_t p1 = D1 >= 0 ? (uint32_t)npk[D1] : 0xffffffffu;
        bool b0 = false, b1 = D1 < 0;  // W = 0: taskBuffer_k = the task being served
        for (int r = 0; r < nr; r++) {
            b0 |= (L.row[r] == D0);
            b1 |= (L.row[r] == D1);
        }
        const unsigned long long k0 = ((unsigned long long)p0 << 32) | (unsigned long long)(uint32_t)D0;
        const unsigned long long k1 = ((unsigned long long)p1 << 32) | (unsigned long long)(uint32_t)D1;
        const bool t0 = !b0 & (k0 < best);
        best = t0 ? k0 : best;
        bslot = t0 ? i0 : bslot;
        const bool t1 = !b1 & (k1 < best);
        best = t1 ? k1 : best;
        bslot = t1 ? i1 : bslot;
    }
    (void)nr2;
#else
    for (int i = threadIdx.x; i < cnt; i += blockDim.x) {
        const int32_t D = rl[i];
        bool in_buf = false;  // nb(D) > 0: an input of a taskBuffer_k task
        for (int r = 0; r < nr; r++) in_buf |= (L.row[r] == D);
        for (int r = 0; r < nr2; r++) in_buf |= (L.row2[r] == D);
        const unsigned long long key =
            ((unsigned long long)(uint32_t)npk[D] << 32) | (unsigned long long)(uint32_t)D;
        const bool take = !in_buf & (key < best);
        best = take ? key : best;
        bslot = take ? i : bslot;
    }
#endif
    const unsigned long long mine = best;
    best = block_min_u64(best);
    if (best == ~0ull) return -1;
    if (mine == best) L.vslot = bslot;  // the one thread holding V (ids are unique)
    cta_sync();
    return (int32_t)(best & 0xffffffffull);
}

// Alg. 6 l.6-7 (reading R29), when every resident datum of GPU k is an input
// of a buffered task: Belady -- the datum whose next use in taskBuffer_k is
// the furthest.  A datum only the task running at the request uses has no
// future use, and the capacity check (>= max(1, W) tasks' inputs) guarantees
// one exists, so the victim is the lowest-id such datum; it leaves memory
// when that task ends (L.run_end).  Block-wide, out of line (W >= 1 only);
// returns V (-1: none) and sets L.vslot.
__device__ __noinline__ int32_t belady_victim(int k) {
    const Inst &I = SI;
    const View &V = SV;
    const int cnt = L.res_cnt[k];
    const int32_t *rl = V.res_list + (size_t)k * I.res_cap;
    unsigned long long best = ~0ull;
    int bslot = -1;
    for (int i = threadIdx.x; i < cnt; i += blockDim.x) {
        const int32_t D = rl[i];
        bool run = false, later = false;
        for (int r = 0; r < L.row2_run; r++) run |= (L.row2[r] == D);
        for (int r = 0; r < L.row_len; r++) later |= (L.row[r] == D);
        for (int r = L.row2_run; r < L.row2_len; r++) later |= (L.row2[r] == D);
        const bool take = run & !later & ((unsigned long long)D < best);
        best = take ? (unsigned long long)D : best;
        bslot = take ? i : bslot;
    }
    const unsigned long long mine = best;
    best = block_min_u64(best);
    if (best == ~0ull) return -1;
    if (mine == best) L.vslot = bslot;
    cta_sync();
    return (int32_t)best;
}

// Alg. 6 l.8-9: planned tasks of k that use V return to the shared pool (R4,
// idle GPUs wake at t, R18); then V leaves GPU k's memory.  Block-wide.
__device__ void evict(int k, int32_t Vd, int32_t Tserved, int64_t t, int64_t te) {
    const Inst &I = SI;
    const View &V = SV;
    int4 *pl = V.plan + (size_t)k * I.plan_cap;
    int nret = 0;
    unsigned tmin = 0xffffffffu;
    // Alg. 6 l.8 is LUF's; an LRU eviction leaves plannedTasks_k alone
    const int ph = L.plan_head[k], pe = M_LUF(I) ? L.plan_end[k] : ph;
    for (int i = ph + threadIdx.x; i < pe; i += blockDim.x) {
        const int4 e = pl[i];
        if (e.x >= 0 && entry_uses(e, Vd)) {
            pl[i].x = -1;
            pool_move(e.x, row_of_entry(e), +1, k);
            nret++;
            tmin = (unsigned)e.x < tmin ? (unsigned)e.x : tmin;
        }
    }
    // no planned task left behind the one being served (most of C4's plans): nothing
    // can return, skip the reduction's two barriers (ph, pe are CTA-uniform)
    if (ph < pe) block_sum_min(nret, tmin);
    if (threadIdx.x == 0) {
        if (nret > 0) {
            L.plan_live[k] -= nret;
            L.n_avail += nret;
            if ((int)tmin < L.avail_lo) L.avail_lo = (int)tmin;
            for (int j = 0; j < I.K; j++)  // R18
                if (L.idle[j]) {
                    L.idle[j] = 0;
                    L.req[j] = t;
                }
        }
        int32_t *rl = V.res_list + (size_t)k * I.res_cap;
        const int last = L.res_cnt[k] - 1;
        rl[L.vslot] = rl[last];
        L.res_cnt[k] = last;
        V.resb[(size_t)k * I.nw + (Vd >> 5)] &= ~(1u << (Vd & 31));
        L.used[k] -= size_of(Vd);
        L.n_evictions++;
        push_event(1, k, Vd, Tserved, te, te);  // te > t: a Belady eviction waits for the running task (R29)
        if (te > L.mem_ready) L.mem_ready = te;
        int64_t sb, se;
        seg_of(Vd, sb, se);
        L.alg_bytes += 24ull * (uint64_t)(se - sb) + (uint64_t)nret * (8ull * I.K + 40ull) + 32ull;
        L.sum_deg += se - sb;
    }
    cta_sync();
    if (nret > 0) compact_plan(k);
    seg_update(k, Vd, false);
    cta_sync();
}

// Warp 0, W >= 1: the inputs of the other tasks of taskBuffer_k -- those
// served on k that have not ended by t (R7, R29) -- into L.row2: first the
// task running at t (at most one), then those not started yet, oldest first.
__device__ __noinline__ void buffer_rows(int k, int64_t t) {
    const Inst &I = SI;
    const int W = I.W, j = L.won[k];
    __syncwarp();  // thread 0 reset row2_len
    for (int pass = 0; pass < 2; pass++) {  // 0: the running task, 1: the queued ones
        for (int q = j > W ? j - W : 0; q < j; q++) {
            const int32_t Tq = __ldcg(&I.wring[k * MAX_W + q % W]);
            const int64_t st = __ldcg(&I.tstart[Tq]), en = __ldcg(&I.tend[Tq]);
            if (en <= t || (st <= t) != (pass == 0)) continue;
            const int64_t rb = __ldg(&I.tptr[Tq]), re = __ldg(&I.tptr[Tq + 1]);
            const int base = L.row2_len;
            __syncwarp();
            for (int r = threadIdx.x; r < (int)(re - rb); r += 32) L.row2[base + r] = __ldg(&I.tdat[rb + r]);
            __syncwarp();
            if (threadIdx.x == 0) {
                L.row2_len = base + (int)(re - rb);
                if (pass == 0) {
                    L.row2_run = L.row2_len;
                    L.run_end = en;
                }
            }
            __syncwarp();
        }
    }
}

// Serve T on GPU k at time t with loads: evict V(k,i), load the missing inputs
// in ascending id (R10), process; shared FIFO bus (R9).
// Block-wide.  L.row holds D(T).
__device__ void serve_loads(int k, int32_t T, int64_t t) {
    const Inst &I = SI;
    const View &V = SV;
    // Thread 0: the missing inputs, ascending (R10).  Residency of D(T) only
    // changes by these loads while T is served (LUF never evicts an input of
    // a taskBuffer task), so the list is fixed up front: one barrier.
    if (threadIdx.x == 0) {
        L.ready = t;
        L.mem_ready = t;
        L.row2_len = 0;
        L.row2_run = 0;
        int nm = 0;
        for (int r = 0; r < L.row_len; r++)
            if (!resident(k, L.row[r])) L.miss[nm++] = L.row[r];
        L.nmiss = nm;
    }
    if (M_W(I) >= 1 && threadIdx.x < 32) buffer_rows(k, t);
    cta_sync();
    const int nmiss = L.nmiss;
    for (int r = 0; r < nmiss; r++) {
        const int32_t D = L.miss[r];
        const uint64_t sz = size_of(D);
        while (true) {  // R11: LUF until D fits
            const bool full = L.used[k] + sz > I.cap;
            cta_sync();
            if (!full) break;
            PROF_T0(p_luf);
            int32_t Vd = luf_victim(k);
            bool belady = false;
            if (Vd < 0 && M_LUF(I) && M_W(I) >= 1) {
                Vd = belady_victim(k);
                belady = true;
                if (threadIdx.x == 0) L.n_belady++;
            }
            PROF_ADD(L, P_LUF, p_luf);
            if (Vd < 0) {
                if (threadIdx.x == 0) L.error = 1;
                cta_sync();
                return;
            }
            PROF_T0(p_ev);
            evict(k, Vd, T, t, belady ? (L.run_end > t ? L.run_end : t) : t);
            PROF_ADD(L, P_EVICT, p_ev);
        }
        if (threadIdx.x == 0) {
            int32_t *rl = V.res_list + (size_t)k * I.res_cap;
            rl[L.res_cnt[k]++] = D;
            V.resb[(size_t)k * I.nw + (D >> 5)] |= 1u << (D & 31);
            L.used[k] += sz;
            int64_t st = L.bus_free > t ? L.bus_free : t;
            if (L.mem_ready > st) st = L.mem_ready;  // its memory is freed then (R29)
            const int64_t en = st + delta_of(D);
            L.bus_free = en;
            if (en > L.ready) L.ready = en;
            L.n_loads++;
            L.bytes_loaded += sz;
            push_event(0, k, D, T, st, en);
            int64_t sb, se;
            seg_of(D, sb, se);
            L.alg_bytes += 24ull * (uint64_t)(se - sb) + 32ull;
            L.sum_deg += se - sb;
        }
        // seg_update reads nothing thread 0 just wrote unless a row is longer
        // than its edge record (missing_pair reads the residency bitmap)
        if (M_LONG(I.max_row > 3)) cta_sync();
        PROF_T0(p_seg);
        seg_update(k, D, true);
        cta_sync();
        PROF_ADD(L, P_SEG, p_seg);
    }
    if (threadIdx.x == 0) {
        if (!M_LUF(I)) {  // LRU: D(T) used by the n_served-th task
            int32_t *lk = V.lru + (size_t)k * I.nstr;
            for (int r = 0; r < L.row_len; r++) lk[L.row[r]] = (int32_t)L.n_served;
        }
        finish_serve(k, T, t, L.ready, tau_of(T));
    }
    cta_sync();
}

// Alg. 5 l.6-9 (and the 3inputs fallback): block argmax
// over D of (score[D], u(D), -D) among data with a positive score -- more
// freed tasks, then more unprocessed uses, then the lower id (R1, R23, R24).
// A datum with a positive score is never resident (its tasks miss it), so no
// residency test is needed.  Rows are padded to nstr (multiple of 4, pad
// scores 0): 16-byte loads, UN vectors in flight per array and thread.
// Fast path (score, u < 2^15, checked on the host: I.key32): the pair packs
// into one 32-bit key score << 16 | u, and since each thread visits D in
// increasing order a strict '>' keeps the lowest id among equal keys; the
// 64-bit (key, ~D) is formed once per thread for the block reduction.
// The thread's best 64-bit key (score, u, ~D) when scores may reach 2^15.
__device__ __noinline__ unsigned long long score_best64(const int32_t *score) {
    const Inst &I = SI;
    const View &V = SV;
    const unsigned ib = (unsigned)I.id_bits, ub = (unsigned)I.u_bits;
    const unsigned long long idmask = (1ull << ib) - 1ull;
    unsigned long long best = 0ull;
    for (int D = threadIdx.x; D < I.n; D += blockDim.x) {
        const int32_t sc = score[D];
        if (sc <= 0) continue;
        const unsigned long long key = ((unsigned long long)(uint32_t)sc << (ub + ib)) |
                                       ((unsigned long long)(uint32_t)V.u[D] << ib) |
                                       (idmask - (unsigned long long)D);
        best = key > best ? key : best;
    }
    return best;
}

// sh = 16: the key is score << 16 | u; sh = 0 on packed rows (M_HH): the high
// half (n2) is the score, the 3inputs key.
__device__ int32_t score_argmax(const int32_t *score, int sh = 16) {
    const Inst &I = SI;
    const unsigned ib = (unsigned)I.id_bits;
    const unsigned long long idmask = (1ull << ib) - 1ull;
    unsigned long long best = 0ull;
    if (M_KEY32(I)) {
        const int4 *h4 = reinterpret_cast<const int4 *>(score);
        const int nv = I.nstr >> 2;
        constexpr int UN = 2;
        uint32_t bk = 0u;
        int32_t bd = 0;
        for (int v0 = threadIdx.x; v0 < nv; v0 += UN * blockDim.x) {
            int4 hv[UN];
            uint4 uv[UN];
#pragma unroll
            for (int q = 0; q < UN; q++) {
                const int v = v0 + q * blockDim.x;
                hv[q] = v < nv ? h4[v] : make_int4(0, 0, 0, 0);
                uv[q] = v < nv ? u_vec4(v) : make_uint4(0, 0, 0, 0);
            }
#pragma unroll
            for (int q = 0; q < UN; q++) {
                const int D = 4 * (v0 + q * blockDim.x);
                const uint32_t k0 = (((uint32_t)hv[q].x << sh) & 0xFFFF0000u) | uv[q].x;
                const uint32_t k1 = (((uint32_t)hv[q].y << sh) & 0xFFFF0000u) | uv[q].y;
                const uint32_t k2 = (((uint32_t)hv[q].z << sh) & 0xFFFF0000u) | uv[q].z;
                const uint32_t k3 = (((uint32_t)hv[q].w << sh) & 0xFFFF0000u) | uv[q].w;
                if (k0 > bk) { bk = k0; bd = D; }
                if (k1 > bk) { bk = k1; bd = D + 1; }
                if (k2 > bk) { bk = k2; bd = D + 2; }
                if (k3 > bk) { bk = k3; bd = D + 3; }
            }
        }
        if (bk >= 65536u)  // positive score
            best = ((unsigned long long)bk << ib) | (idmask - (unsigned long long)bd);
    } else {
        best = score_best64(score);
    }
    best = block_max_u64(best);
    return best ? (int32_t)(idmask - (best & idmask)) : -1;
}

// Both keys in ONE pass over the packed rows of the specialised loop (M_HH):
// the main argmax of (n_k(D), u(D), -D) (returned) and the 3inputs argmax of
// (n2_k(D), u(D), -D) (*d2), in a single block exchange -- the fallback no
// longer re-reads the rows (it serves 59-68 % of C4's scans).
__device__ void block_max2_u64(unsigned long long &a, unsigned long long &b) {
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, nw = blockDim.x >> 5;
    a = warp_max_u64(a);
    b = warp_max_u64(b);
    if (nw == 1) return;
    cta_sync();
    if (lane == 0) {
        L.red64[w] = a;
        L.red64b[w] = b;
    }
    cta_sync();
    a = warp_max_u64(lane < nw ? L.red64[lane] : 0ull);
    b = warp_max_u64(lane < nw ? L.red64b[lane] : 0ull);
}
__device__ int32_t score_argmax_hh(const int32_t *score, int32_t *d2) {
    const Inst &I = SI;
    const View &V = SV;
    const unsigned ib = (unsigned)I.id_bits;
    const unsigned long long idmask = (1ull << ib) - 1ull;
    const int4 *h4 = reinterpret_cast<const int4 *>(score);
    const int nv = I.nstr >> 2;
    constexpr int UN = DTS_HH_UN;
    uint32_t bk = 0u, bk2 = 0u;
    int32_t bd = 0, bd2 = 0;
    (void)V;
    for (int v0 = threadIdx.x; v0 < nv; v0 += UN * blockDim.x) {
        int4 hv[UN];
        uint4 uv[UN];
#pragma unroll
        for (int q = 0; q < UN; q++) {
            const int v = v0 + q * blockDim.x;
            hv[q] = v < nv ? h4[v] : make_int4(0, 0, 0, 0);
            uv[q] = v < nv ? u_vec4(v) : make_uint4(0, 0, 0, 0);
        }
#pragma unroll
        for (int q = 0; q < UN; q++) {
            const int D = 4 * (v0 + q * blockDim.x);
            const uint32_t hx[4] = {(uint32_t)hv[q].x, (uint32_t)hv[q].y, (uint32_t)hv[q].z, (uint32_t)hv[q].w};
            const uint32_t ux[4] = {uv[q].x, uv[q].y, uv[q].z, uv[q].w};
#pragma unroll
            for (int c = 0; c < 4; c++) {
                const uint32_t k1 = (hx[c] << 16) | ux[c], k2 = (hx[c] & 0xFFFF0000u) | ux[c];
                if (k1 > bk) { bk = k1; bd = D + c; }
                if (k2 > bk2) { bk2 = k2; bd2 = D + c; }
            }
        }
    }
    unsigned long long best = bk >= 65536u ? (((unsigned long long)bk << ib) | (idmask - (unsigned long long)bd)) : 0ull;
    unsigned long long best2 =
        bk2 >= 65536u ? (((unsigned long long)bk2 << ib) | (idmask - (unsigned long long)bd2)) : 0ull;
    block_max2_u64(best, best2);
    *d2 = best2 ? (int32_t)(idmask - (best2 & idmask)) : -1;
    return best ? (int32_t)(idmask - (best & idmask)) : -1;
}

// OPTI (§V-F): "we stop the search as soon as we find a
// data allowing to compute at least one task" -- dataNotInMem_k searched in
// ascending id (reading R28), i.e. the lowest D with n_k(D) >= 1.
__device__ __noinline__ int32_t score_first(const int32_t *score) {
    const Inst &I = SI;
    const int4 *h4 = reinterpret_cast<const int4 *>(score);
    const int nv = I.nstr >> 2;
    unsigned long long best = ~0ull;
    for (int v = threadIdx.x; v < nv; v += blockDim.x) {  // increasing D per thread
        const int4 hv = h4[v];
        const int D = 4 * v;
        const int f = hv.x > 0 ? 0 : (hv.y > 0 ? 1 : (hv.z > 0 ? 2 : (hv.w > 0 ? 3 : -1)));
        if (f >= 0) {
            best = (unsigned long long)(D + f);
            break;
        }
    }
    best = block_min_u64(best);
    return best == ~0ull ? -1 : (int32_t)best;
}

// Alg. 5 l.10: plannedTasks_k <- unallocated tasks of Dopt's segment with one
// missing input (= Dopt), ascending id (ordered block compaction).  Block-wide.
__device__ void plan(int k, int32_t Dopt) {
    const Inst &I = SI;
    const View &V = SV;
    int64_t b, e;
    seg_of(Dopt, b, e);
    const uint32_t *sk = V.s + (size_t)k * I.m_pad;
    int4 *pl = V.plan + (size_t)k * I.plan_cap;
    int64_t *pt = V.plan_cum ? V.plan_cum + (size_t)k * I.plan_cap : nullptr;
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, nw = blockDim.x >> 5;
    const unsigned lt = (1u << lane) - 1u;
    int base_out = 0;
    PROF_T0(p_q3);
    for (int64_t base = b; base < e; base += blockDim.x) {
        const int64_t i = base + threadIdx.x;
        int32_t T = -1;
        bool sel = false;
        int4 ed = make_int4(-1, -1, -1, 0);
        if (i < e) {
            ed = __ldg(&I.dedge[i]);
            T = ed.x;
            sel = M_SL(I) ? !allocated(T) && (ed.y < 0 || resident(k, ed.y)) && (ed.z < 0 || resident(k, ed.z))
                       : (sk[T] >> 24) == 1u;
        }
        const unsigned msk = __ballot_sync(FULL, sel);
        if (lane == 0) L.wcnt[w] = __popc(msk);
        cta_sync();
        int off = base_out, tot = 0;
        for (int j = 0; j < nw; j++) {
            const int c = L.wcnt[j];
            if (j < w) off += c;
            tot += c;
        }
        if (sel) {
            const int pos = off + __popc(msk & lt);
            pl[pos] = make_int4(T, Dopt, ed.y, M_LONG(ed.w > 3) ? ROW_LONG : ed.z);
            if (pt) pt[pos] = tau_of(T);
        }
        base_out += tot;
        cta_sync();
    }
    PROF_T0(p_pm);
    pool_move_many(pl, base_out, -1, k);
    cta_sync();
    PROF_ADD(L, P_X1, p_pm);
    PROF_ADD(L, P_X3, p_q3);
    PROF_T0(p_q4);
    if (pt) block_incl_scan(pt, 0, base_out, 0);  // tau -> prefix sums
    if (threadIdx.x == 0) {
        L.plan_head[k] = 0;
        L.plan_end[k] = base_out;
        L.plan_live[k] = base_out;
        L.n_avail -= base_out;
        L.n_alloc += base_out;
        L.alg_bytes += 20ull * (uint64_t)(e - b) + (uint64_t)base_out * (8ull * I.K + 40ull);
    }
    cta_sync();
    PROF_ADD(L, P_X4, p_q4);
}

// 3inputs: the lowest-id unallocated task of D2's segment with two missing inputs.
__device__ __noinline__ int32_t first_cnt2(int k, int32_t D2) {
    const Inst &I = SI;
    const View &V = SV;
    int64_t b, e;
    seg_of(D2, b, e);
    const uint32_t *sk = V.s + (size_t)k * I.m_pad;
    for (int64_t base = b; base < e; base += blockDim.x) {
        const int64_t i = base + threadIdx.x;
        unsigned long long c = ~0ull;
        if (i < e) {
            if (M_SL(I)) {  // D2 misses (n2(D2) > 0): exactly one other input misses
                const int4 ed = __ldg(&I.dedge[i]);
                const int mo = (int)(ed.y >= 0 && !resident(k, ed.y)) + (int)(ed.z >= 0 && !resident(k, ed.z));
                if (!allocated(ed.x) && mo == 1) c = (unsigned long long)ed.x;
            } else {
                const int32_t T = __ldg(&I.dedge[i]).x;
                if ((sk[T] >> 24) == 2u) c = (unsigned long long)T;
            }
        }
        c = block_min_u64(c);
        if (c != ~0ull) return (int32_t)c;
    }
    return -1;
}

// Alg. 5 l.13 (R5): the lowest-id unallocated task, scanning up from avail_lo
// (over the owned range [t_lo, t_hi) = all tasks unless sharded).
__device__ __noinline__ int32_t first_avail() {
    const Inst &I = SI;
    const View &V = SV;
    if (M_SL(I)) {  // the allocation bitmap, a word per thread (bits past m are set)
        const int lo = L.avail_lo;
        const int nwd = (I.m + 31) >> 5;
        for (int w0 = lo >> 5; w0 < nwd; w0 += blockDim.x) {
            const int wd = w0 + threadIdx.x;
            unsigned long long c = ~0ull;
            if (wd < nwd) {
                uint32_t free_bits = ~V.al[wd];
                if (wd == (lo >> 5)) free_bits &= ~((1u << (lo & 31)) - 1u);
                if (free_bits) c = (unsigned long long)(32 * wd + __ffs(free_bits) - 1);
            }
            c = block_min_u64(c);
            if (c != ~0ull) return (int32_t)c;
        }
        return -1;
    }
#if !DTS_FAST
    for (int64_t base = L.avail_lo > I.t_lo ? L.avail_lo : I.t_lo; base < I.t_hi; base += blockDim.x) {
        const int64_t T = base + threadIdx.x;
        unsigned long long c = ~0ull;
        if (T < I.t_hi && !(V.s[T] & ALLOC_BIT)) c = (unsigned long long)T;
        c = block_min_u64(c);
        if (c != ~0ull) return (int32_t)c;
    }
#endif
    return -1;
}

// ---------------------------------------------------------------------------
// Task shards (the north_star's second multi-GPU mode): one
// instance, its tasks split into G consecutive id ranges.  Shard g keeps the
// packed state and the data->task edges of its own tasks and PARTIAL score
// arrays (h, h2, u count only its tasks); everything the decisions depend on
// afterwards (residency, plannedTasks, np, the bus and time model, the trace)
// is replicated: every shard takes the same decision from the same exchanged
// values.  Exchanges go through the shards' memory -- other CTAs of the same
// launch, or other B200s through CUDA IPC mappings over NVLink -- inside the
// kernel: no host round trip per decision.  Per scan: exchange 1 (partials
// final), a reduce-scatter of (h, u[, h2]) by datum slice with the slice's best
// key, exchange 2, max of G keys; per plan: one exchange of the shards' parts.

__device__ __forceinline__ unsigned long long ld_acquire_sys(const unsigned long long *p) {
    unsigned long long v;
    asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release_sys(unsigned long long *p, unsigned long long v) {
    asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ unsigned long long global_ns() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}
constexpr unsigned long long XCH_TIMEOUT_NS = 5000000000ull;

__device__ __forceinline__ unsigned long long ld_acquire_gpu(const unsigned long long *p) {
    unsigned long long v;
    asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release_gpu(unsigned long long *p, unsigned long long v) {
    asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

// Payload slot of exchange number x (1-based within the run) of shard p.
__device__ __forceinline__ ShardSlot *xch_slot(int p, int64_t x) {
    const Inst &I = SI;
    return reinterpret_cast<ShardSlot *>(SP[p].box + (x & 1) * I.box_bytes);
}

// Block-wide: publish this shard's slot of the next exchange (every thread's
// writes to it precede the barrier) and wait until every shard published the
// same exchange.  Thread 0 releases (system scope when the peers are other
// GPUs, I.xsys; GPU scope for CTAs of one device) -- the barrier orders the
// other threads' writes before it -- and warp 0 acquires the peers' exchange
// numbers.  Two slots by parity suffice: a
// shard reuses a slot only after every peer published the exchange in between,
// which they do only after reading this one.  A peer missing for
// XCH_TIMEOUT_NS sets L.xerr -- the run ends with an error instead of a hang.
__device__ __noinline__ void xch_sync() {
    const Inst &I = SI;
    const unsigned long long e = I.ep_base + (unsigned long long)L.xe + 1ull;
    PROF_T0(p_x);
    cta_sync();
    if (threadIdx.x == 0) {
        if (I.xsys) st_release_sys(SP[I.g].epoch, e);
        else st_release_gpu(SP[I.g].epoch, e);
    }
    if (threadIdx.x < 32) {
        const unsigned long long t0 = global_ns();
        for (int p = threadIdx.x; p < I.G; p += 32) {
            const unsigned long long *f = SP[p].epoch;
            while ((I.xsys ? ld_acquire_sys(f) : ld_acquire_gpu(f)) < e) {
                if (global_ns() - t0 > XCH_TIMEOUT_NS) {
                    L.xerr = 1;
                    break;
                }
            }
        }
        __syncwarp();
        if (threadIdx.x == 0) L.xe = L.xe + 1;
    }
    cta_sync();
    PROF_CNT(L, P_X2, 1);
    PROF_ADD(L, P_X1, p_x);
}

// Block-wide: minimum over shards of one block-uniform candidate (~0 = none).
__device__ __noinline__ unsigned long long xch_min(unsigned long long v) {
    const Inst &I = SI;
    if (threadIdx.x == 0) xch_slot(I.g, L.xe + 1)->key[0] = v;
    xch_sync();
    if (L.xerr) return ~0ull;
    unsigned long long r = ~0ull;
    for (int p = 0; p < I.G; p++) {
        const unsigned long long x = __ldcg(&xch_slot(p, L.xe)->key[0]);
        r = x < r ? x : r;
    }
    return r == ~0ull || r < (unsigned long long)I.m ? r : ~0ull;  // (a task id or none)
}

__device__ __forceinline__ unsigned long long score_key(int32_t sc, int32_t u, int32_t D, unsigned ub, unsigned ib,
                                                        unsigned long long idmask) {
    return sc > 0 ? ((unsigned long long)(uint32_t)sc << (ub + ib)) | ((unsigned long long)(uint32_t)u << ib) |
                        (idmask - (unsigned long long)D)
                  : 0ull;
}

// Alg. 5 l.4-9 (+ the 3inputs score when fb2, OPTI's first positive datum
// when opti) over the shards: n_k(D) = sum of the shards' h_k(D), u(D) = sum
// of their u(D).  Shard g reduces the datum slice g of every shard's partials
// and publishes the slice's best keys; the max over shards is the argmax of
// the whole instance with the same (score, u, -D) order as one shard.
// Returns D* (or -1); *d2 = the 3inputs D2 (or -1).
__device__ __noinline__ int32_t shard_scan(int k, bool fb2, bool opti, int32_t *d2) {
    const Inst &I = SI;
    const unsigned ib = (unsigned)I.id_bits, ub = (unsigned)I.u_bits;
    const unsigned long long idmask = (1ull << ib) - 1ull;
    xch_sync();  // every shard's partial scores are final
    const int nv = I.nstr >> 2;
    const int per = (nv + I.G - 1) / I.G;
    const int v0 = I.g * per, v1 = nv < v0 + per ? nv : v0 + per;
    unsigned long long b1 = 0ull, b2 = 0ull;
    if (!L.xerr) {
        for (int v = v0 + threadIdx.x; v < v1; v += blockDim.x) {
            int4 hs = make_int4(0, 0, 0, 0), us = hs, h2s = hs;
            for (int p = 0; p < I.G; p++) {
                const ShardPeer *P = &SP[p];
                const int4 *ph = (const int4 *)(P->h + (size_t)k * I.nstr);
                const int4 *pu = (const int4 *)P->u;
                const int4 a = __ldcg(ph + v), c = __ldcg(pu + v);
                hs.x += a.x; hs.y += a.y; hs.z += a.z; hs.w += a.w;
                us.x += c.x; us.y += c.y; us.z += c.z; us.w += c.w;
                if (fb2) {
                    const int4 *ph2 = (const int4 *)(P->h2 + (size_t)k * I.nstr);
                    const int4 d = __ldcg(ph2 + v);
                    h2s.x += d.x; h2s.y += d.y; h2s.z += d.z; h2s.w += d.w;
                }
            }
            const int D = 4 * v;
            const int32_t hh[4] = {hs.x, hs.y, hs.z, hs.w}, uu[4] = {us.x, us.y, us.z, us.w},
                          h2h[4] = {h2s.x, h2s.y, h2s.z, h2s.w};
#pragma unroll
            for (int q = 0; q < 4; q++) {
                const unsigned long long k1 =
                    opti ? (hh[q] > 0 ? idmask - (unsigned long long)(D + q) + 1ull : 0ull)
                         : score_key(hh[q], uu[q], D + q, ub, ib, idmask);
                const unsigned long long k2 = score_key(h2h[q], uu[q], D + q, ub, ib, idmask);
                b1 = k1 > b1 ? k1 : b1;
                b2 = k2 > b2 ? k2 : b2;
            }
        }
    }
    b1 = block_max_u64(b1);
    b2 = block_max_u64(b2);
    if (threadIdx.x == 0) {
        ShardSlot *my = xch_slot(I.g, L.xe + 1);
        my->key[0] = b1;
        my->key[1] = b2;
    }
    xch_sync();
    *d2 = -1;
    if (L.xerr) return -1;
    unsigned long long m1 = 0ull, m2 = 0ull;
    for (int p = 0; p < I.G; p++) {
        const ShardSlot *sl = xch_slot(p, L.xe);
        const unsigned long long x1 = __ldcg(&sl->key[0]), x2 = __ldcg(&sl->key[1]);
        m1 = x1 > m1 ? x1 : m1;
        m2 = x2 > m2 ? x2 : m2;
    }
    if (m2) *d2 = (int32_t)(idmask - (m2 & idmask));
    const int32_t D = !m1 ? -1 : opti ? (int32_t)(idmask - (m1 - 1ull)) : (int32_t)(idmask - (m1 & idmask));
    if (D >= I.n || *d2 >= I.n) {  // not a peer of this run: abandon
        cta_sync();
        if (threadIdx.x == 0) L.xerr = 1;
        cta_sync();
        *d2 = -1;
        return -1;
    }
    return D;
}

// Alg. 5 l.10 over the shards: each shard compacts the unallocated tasks of
// ITS part of Dopt's segment with one missing input (ascending id) into its
// slot; after the exchange every shard concatenates the G parts in shard order
// (= ascending id: shards own consecutive ranges) into its replicated
// plannedTasks_k and moves them out of the pool (pool_move: np for all, the
// partial state for its own).  Block-wide.
__device__ __noinline__ void plan_shard(int k, int32_t Dopt) {
    const Inst &I = SI;
    const View &V = SV;
    int64_t b, e;
    seg_of(Dopt, b, e);
    const uint32_t *sk = V.s + (size_t)k * I.m_pad;
    ShardSlot *my = xch_slot(I.g, L.xe + 1);
    int4 *ents = reinterpret_cast<int4 *>(my + 1);
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, nw = blockDim.x >> 5;
    const unsigned lt = (1u << lane) - 1u;
    int base_out = 0;
    for (int64_t base = b; base < e; base += blockDim.x) {
        const int64_t i = base + threadIdx.x;
        bool sel = false;
        int4 ed = make_int4(-1, -1, -1, 0);
        if (i < e) {
            ed = __ldg(&I.dedge[i]);
            sel = (sk[ed.x] >> 24) == 1u;
        }
        const unsigned msk = __ballot_sync(FULL, sel);
        if (lane == 0) L.wcnt[w] = __popc(msk);
        cta_sync();
        int off = base_out, tot = 0;
        for (int j = 0; j < nw; j++) {
            const int c = L.wcnt[j];
            if (j < w) off += c;
            tot += c;
        }
        if (sel) ents[off + __popc(msk & lt)] = make_int4(ed.x, Dopt, ed.y, M_LONG(ed.w > 3) ? ROW_LONG : ed.z);
        base_out += tot;
        cta_sync();
    }
    if (threadIdx.x == 0) my->cnt = base_out;
    xch_sync();
    if (threadIdx.x == 0) {
        int run = 0;
        for (int p = 0; p < I.G; p++) {
            L.xoff[p] = run;
            const int c = L.xerr ? 0 : __ldcg(&xch_slot(p, L.xe)->cnt);
            run += c;
            if (c < 0 || run > I.plan_cap) {  // not a peer of this run: abandon, do not index
                L.xerr = 1;
                run -= c;
            }
        }
        L.xoff[I.G] = L.xerr ? 0 : run;
    }
    cta_sync();
    const int total = L.xoff[I.G];
    int4 *pl = V.plan + (size_t)k * I.plan_cap;
    int64_t *pt = V.plan_cum ? V.plan_cum + (size_t)k * I.plan_cap : nullptr;
    for (int i = threadIdx.x; i < total; i += blockDim.x) {
        int p = 0;
        while (L.xoff[p + 1] <= i) p++;
        const int4 en = __ldcg(reinterpret_cast<const int4 *>(xch_slot(p, L.xe) + 1) + (i - L.xoff[p]));
        pl[i] = en;
        if (pt) pt[i] = tau_of(en.x);
    }
    cta_sync();
    pool_move_many(pl, total, -1, k);
    cta_sync();
    if (pt) block_incl_scan(pt, 0, total, 0);
    if (threadIdx.x == 0) {
        L.plan_head[k] = 0;
        L.plan_end[k] = total;
        L.plan_live[k] = total;
        L.n_avail -= total;
        L.n_alloc += total;
        L.alg_bytes += 20ull * (uint64_t)(e - b) + (uint64_t)total * (8ull * I.K + 40ull);
    }
    cta_sync();
}

// Alg. 5 l.13 / the 3inputs pick over the shards: each shard's lowest
// candidate, then the minimum.
__device__ __noinline__ int32_t any_first_avail() {
    int32_t T = first_avail();
    if (M_SHARD(SI)) {
        const unsigned long long r = xch_min(T < 0 ? ~0ull : (unsigned long long)T);
        T = r == ~0ull ? -1 : (int32_t)r;
    }
    return T;
}
__device__ __noinline__ int32_t any_first_cnt2(int k, int32_t D2) {
    int32_t T = first_cnt2(k, D2);
    if (M_SHARD(SI)) {
        const unsigned long long r = xch_min(T < 0 ? ~0ull : (unsigned long long)T);
        T = r == ~0ull ? -1 : (int32_t)r;
    }
    return T;
}

// DTS_F_VERIFY (P9): recompute n_k(D), n2_k(D), u(D) and cnt_k(T) from their
// definitions -- the full non-incremental pass of Alg. 5 l.4-5 -- and count
// mismatches against the incremental state.
__device__ __noinline__ void verify_scores(int k) {
    const Inst &I = SI;
    const View &V = SV;
    int32_t *vh = I.vhist, *vh2 = I.vhist + I.n, *vu = I.vhist + 2 * I.n;
    for (int D = threadIdx.x; D < 3 * I.n; D += blockDim.x) vh[D] = 0;
    cta_sync();
    const uint32_t *sk = V.s + (size_t)k * I.m_pad;
    int bad = 0;
    for (int T = I.t_lo + threadIdx.x; T < I.t_hi; T += blockDim.x) {  // owned tasks
        const uint32_t w = M_SL(I) ? 0u : sk[T];
        const int64_t rb = __ldg(&I.tptr[T]), re = __ldg(&I.tptr[T + 1]);
        int c = 0;
        uint32_t x = 0;
        for (int64_t i = rb; i < re; i++) {
            const int32_t D = __ldg(&I.tdat[i]);
            if (!resident(k, D)) c++, x ^= (uint32_t)D;
        }
        if (M_SL(I)) {
            if (allocated(T)) continue;
        } else {
            bad += (c != (int)((w >> 24) & 0x7fu)) || (x != (w & XOR_MASK));
            if (w & ALLOC_BIT) continue;
        }
        for (int64_t i = rb; i < re; i++) {
            const int32_t D = __ldg(&I.tdat[i]);
            atomicAdd(&vu[D], 1);
            if (c == 2 && !resident(k, D)) atomicAdd(&vh2[D], 1);
        }
        if (c == 1) atomicAdd(&vh[x], 1);
    }
    cta_sync();
    for (int D = threadIdx.x; D < I.n; D += blockDim.x)
        bad += (__ldcg(&vh[D]) != V.h[(size_t)k * I.nstr + D]) +
               (__ldcg(&vh2[D]) != V.h2[(size_t)k * I.nstr + D]) + (__ldcg(&vu[D]) != V.u[D]);
    bad = block_sum(bad);
    if (threadIdx.x == 0) L.n_verr += bad;
    cta_sync();
}

// a8: sigma(k, .) for every k -- stable partition of the service sequence by GPU.
// Scratch in the CTA's dynamic shared memory (the decision loop is over; its
// placed arrays are dead): off[MAX_K] u64, tot[MAX_K], wk[16][MAX_K] ints.
__device__ __noinline__ void assemble(int64_t ns, unsigned char *dsm) {
    const Inst &I = SI;
    unsigned long long *off = reinterpret_cast<unsigned long long *>(dsm);
    int *tot = reinterpret_cast<int *>(off + MAX_K);
    int(*wk)[MAX_K] = reinterpret_cast<int(*)[MAX_K]>(tot + MAX_K);  // [warp][GPU]: blocks of <= 512 threads
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, nw = blockDim.x >> 5;
    const unsigned lt = (1u << lane) - 1u;
    for (int k = threadIdx.x; k < MAX_K; k += blockDim.x) off[k] = 0;
    cta_sync();
    for (int64_t i = threadIdx.x; i < ns; i += blockDim.x) atomicAdd(&off[I.serve_gpu[i]], 1ull);
    cta_sync();
    if (threadIdx.x == 0) {
        unsigned long long run = 0;
        for (int k = 0; k < I.K; k++) {
            const unsigned long long c = off[k];
            I.gpu_task_ptr[k] = (int64_t)run;
            off[k] = run;
            run += c;
        }
        I.gpu_task_ptr[I.K] = (int64_t)run;
    }
    cta_sync();
    for (int64_t base = 0; base < ns; base += blockDim.x) {
        for (int j = threadIdx.x; j < nw * MAX_K; j += blockDim.x) wk[j / MAX_K][j % MAX_K] = 0;
        cta_sync();
        const int64_t i = base + threadIdx.x;
        const int k = i < ns ? I.serve_gpu[i] : -1;
        const unsigned peers = __match_any_sync(FULL, k);
        if (k >= 0 && lane == __ffs(peers) - 1) wk[w][k] = __popc(peers);
        cta_sync();
        for (int kk = threadIdx.x; kk < I.K; kk += blockDim.x) {  // exclusive prefix over warps
            int run = 0;
            for (int ww = 0; ww < nw; ww++) {
                const int c = wk[ww][kk];
                wk[ww][kk] = run;
                run += c;
            }
            tot[kk] = run;
        }
        cta_sync();
        if (k >= 0) I.gpu_task_ids[off[k] + wk[w][k] + __popc(peers & lt)] = I.serve_task[i];
        cta_sync();
        for (int kk = threadIdx.x; kk < I.K; kk += blockDim.x) off[kk] += tot[kk];
        cta_sync();
    }
}


// ---------------------------------------------------------------------------
// Fused a1 + a2 init for small instances (Inst::fused): the CTA that runs the
// instance first builds its CSR and initial state itself, so a batched sweep
// is ONE kernel launch instead of ~20 launches per instance.  Same outputs as
// dts_csr.cu + dts_init_kernel (rows sorted and de-duplicated, D(T) a set,
// PAPER.md:244-245; each data segment in ascending task id).  Needs rows of
// <= FUSE_ROW inputs and (2 * warps + 1) * n ints of shared scratch (host-checked).
constexpr int FUSE_ROW = 8;

// Block-wide exclusive scan of one int per thread; returns the prefix, *total.
__device__ __forceinline__ int block_excl_scan_int(int v, int *total) {
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, nw = blockDim.x >> 5;
    int x = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const int t = __shfl_up_sync(FULL, x, o);
        if (lane >= o) x += t;
    }
    cta_sync();
    if (lane == 31) L.red32[w] = x;
    cta_sync();
    int off = 0, tot = 0;
    for (int j = 0; j < nw; j++) {
        const int y = L.red32[j];
        if (j < w) off += y;
        tot += y;
    }
    *total = tot;
    return off + x - v;
}

__device__ __noinline__ void fused_build(unsigned char *dsm) {
    const Inst &I = SI;
    const int m = I.m, n = I.n, nw = blockDim.x >> 5;
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    int64_t *tptr = const_cast<int64_t *>(I.tptr);
    int32_t *tdat = const_cast<int32_t *>(I.tdat);
    int64_t *dptr = const_cast<int64_t *>(I.dptr);
    int32_t *ddat = const_cast<int32_t *>(I.ddat);
    int4 *dedge = const_cast<int4 *>(I.dedge);
    int *cnt = reinterpret_cast<int *>(dsm);  // [nw][n] per-warp counts, then bases
    unsigned *msk = reinterpret_cast<unsigned *>(cnt + nw * n);  // [nw][n] lane masks
    int *deg = reinterpret_cast<int *>(msk + nw * n);            // [n]
    for (int i = threadIdx.x; i < nw * n; i += blockDim.x) {
        cnt[i] = 0;
        msk[i] = 0u;
    }
    for (int i = threadIdx.x; i < n; i += blockDim.x) deg[i] = 0;
    cta_sync();
    // 1. rows: sort + de-duplicate (thread per task), tptr by block scans, tdat, deg
    int64_t carry = 0;
    for (int c = 0; c < m; c += blockDim.x) {
        const int T = c + threadIdx.x;
        int row[FUSE_ROW];
        int len = 0;
        if (T < m) {
            const int64_t rb = I.raw_ptr[T], re = I.raw_ptr[T + 1];
            for (int64_t i = rb; i < re; i++) {
                const int v = I.raw_dat[i];
                int j = len;  // insertion, skipping duplicates
                bool dup = false;
                for (int q = 0; q < len; q++) dup |= row[q] == v;
                if (dup) continue;
                while (j > 0 && row[j - 1] > v) {
                    row[j] = row[j - 1];
                    j--;
                }
                row[j] = v;
                len++;
            }
        }
        int tot;
        const int off = block_excl_scan_int(len, &tot);
        if (T < m) {
            const int64_t o = carry + off;
            tptr[T] = o;
            for (int q = 0; q < len; q++) {
                tdat[o + q] = row[q];
                atomicAdd(&deg[row[q]], 1);
            }
        }
        carry += tot;
    }
    if (threadIdx.x == 0) tptr[m] = carry;
    cta_sync();
    // 2. dptr = exclusive scan of deg; per-warp counts over contiguous task ranges
    int64_t dcarry = 0;
    for (int c = 0; c < n; c += blockDim.x) {
        const int D = c + threadIdx.x;
        const int v = D < n ? deg[D] : 0;
        int tot;
        const int off = block_excl_scan_int(v, &tot);
        if (D < n) dptr[D] = dcarry + off;
        dcarry += tot;
    }
    if (threadIdx.x == 0) dptr[n] = dcarry;
    const int per = (m + nw - 1) / nw, t0 = w * per, t1 = min(m, t0 + per);
    for (int T = t0 + lane; T < t1; T += 32) {
        const int64_t rb = tptr[T], re = tptr[T + 1];
        for (int64_t i = rb; i < re; i++) atomicAdd(&cnt[w * n + tdat[i]], 1);
    }
    cta_sync();
    for (int D = threadIdx.x; D < n; D += blockDim.x) {  // per-datum bases over warps
        int64_t run = dptr[D];
        for (int j = 0; j < nw; j++) {
            const int x = cnt[j * n + D];
            cnt[j * n + D] = (int)run;
            run += x;
        }
    }
    cta_sync();
    // 3. stable scatter: each warp walks its range 32 tasks at a time; a task's
    //    rank among the group's tasks with the same datum = lower lanes in the mask
    const unsigned lt = (1u << lane) - 1u;
    for (int g = t0; g < t1; g += 32) {
        const int T = g + lane;
        int64_t rb = 0, re = 0;
        if (T < t1) {
            rb = tptr[T];
            re = tptr[T + 1];
        }
        for (int64_t i = rb; i < re; i++) atomicOr(&msk[w * n + tdat[i]], 1u << lane);
        __syncwarp();
        for (int64_t i = rb; i < re; i++) {
            const int D = tdat[i];
            const unsigned mk = msk[w * n + D];
            const int pos = cnt[w * n + D] + __popc(mk & lt);
            ddat[pos] = T;
            int4 e;
            e.x = T;
            e.y = -1;
            e.z = -1;
            e.w = (int)(re - rb);
            for (int64_t q = rb; q < re; q++) {
                const int o = tdat[q];
                if (o == D) continue;
                if (e.y < 0) e.y = o;
                else if (e.z < 0) e.z = o;
            }
            dedge[pos] = e;
        }
        __syncwarp();
        for (int64_t i = rb; i < re; i++) {
            const int D = tdat[i];
            const unsigned mk = msk[w * n + D];
            if (lane == __ffs(mk) - 1) cnt[w * n + D] += __popc(mk);
        }
        __syncwarp();
        for (int64_t i = rb; i < re; i++) msk[w * n + tdat[i]] = 0u;
        __syncwarp();
    }
    cta_sync();
}

// a2 initial state for a fused instance, straight into the placed arrays.
__device__ __noinline__ void fused_init() {
    const Inst &I = SI;
    const View &V = SV;
    const int m = I.m, n = I.n, K = I.K;
    for (int T = threadIdx.x; T < I.m_pad; T += blockDim.x) {
        uint32_t w = ALLOC_BIT;
        if (T < m) {
            const int64_t b = I.tptr[T], e = I.tptr[T + 1];
            uint32_t x = 0;
            for (int64_t i = b; i < e; i++) x ^= (uint32_t)I.tdat[i];
            w = ((uint32_t)(e - b) << 24) | x;
            I.tstart[T] = -1;
            I.tend[T] = -1;
        }
        if (!M_SL(I))
            for (int k = 0; k < K; k++) V.s[(size_t)k * I.m_pad + T] = w;
    }
    if (M_SL(I))  // nothing allocated; bits past m set
        for (int wd = threadIdx.x; wd <= I.m_pad / 32; wd += blockDim.x) {
            const int t0 = 32 * wd;
            V.al[wd] = t0 >= m ? ~0u : (m - t0 >= 32 ? 0u : ~((1u << (m - t0)) - 1u));
        }
    for (int D = threadIdx.x; D < I.nstr; D += blockDim.x) {
        int32_t c1 = 0, c2 = 0, dg = 0;
        if (D < n) {
            const int64_t b = I.dptr[D], e = I.dptr[D + 1];
            dg = (int32_t)(e - b);
            for (int64_t i = b; i < e; i++) {
                const int len = I.dedge[i].w;
                c1 += len == 1;
                c2 += len == 2;
            }
            if (!I.size0) {
                const unsigned __int128 num = (unsigned __int128)I.size[D] * 1000000000ull + (I.bw - 1);
                const_cast<int64_t *>(I.delta)[D] = (int64_t)(num / I.bw);
            }
            if (V.dptr32) V.dptr32[D] = (int32_t)b;
        }
        if (M_HH) reinterpret_cast<uint16_t *>(V.u)[D] = (uint16_t)dg;
        else V.u[D] = dg;
        for (int k = 0; k < K; k++) {
            V.h[(size_t)k * I.nstr + D] = M_HH ? (c1 | (c2 << 16)) : c1;
            if (!M_HH) V.h2[(size_t)k * I.nstr + D] = c2;
            V.np[(size_t)k * I.nstr + D] = 0;
        }
    }
    if (V.dptr32 && threadIdx.x == 0) V.dptr32[n] = (int32_t)I.dptr[n];
    for (int i = threadIdx.x; i < K * I.nw; i += blockDim.x) V.resb[i] = 0u;
    cta_sync();
}

}  // namespace

// One CTA per instance; instances pulled from *work_counter.
__global__ void __launch_bounds__(512, 1)
    DTS_KNAME(dts_cta_kernel)(const Inst *__restrict__ insts, int n_inst, int *work_counter) {
    extern __shared__ __align__(16) unsigned char dsm[];
    __shared__ int sh_inst;
    const int tid = threadIdx.x;

    while (true) {
        if (tid == 0) sh_inst = atomicAdd(work_counter, 1);
        cta_sync();
        const int ii = sh_inst;
        if (ii >= n_inst) break;
        if (tid == 0) SI = insts[ii];
        cta_sync();
        const Inst &I = SI;
        if (I.poison) {  // debug: nothing may depend on the previous instance's shared memory
            for (int i = tid; i < I.smem_bytes / 4; i += blockDim.x) reinterpret_cast<uint32_t *>(dsm)[i] = 0xA5A5A5A5u;
            if (tid == 0) {
                uint32_t *l = reinterpret_cast<uint32_t *>(&L);
                for (size_t i = 0; i < sizeof(Lead) / 4; i++) l[i] = 0x5A5A5A5Au;
            }
            cta_sync();
        }
        if (tid == 0) {
            View &W = SV;
            W.s = I.so_s >= 0 ? (uint32_t *)(dsm + I.so_s) : I.s;
            W.u = I.so_u >= 0 ? (int32_t *)(dsm + I.so_u) : I.u;
            W.h = I.so_h >= 0 ? (int32_t *)(dsm + I.so_h) : I.h;
            W.h2 = I.so_h2 >= 0 ? (int32_t *)(dsm + I.so_h2) : I.h2;
            W.np = I.so_np >= 0 ? (int32_t *)(dsm + I.so_np) : I.np;
            W.resb = I.so_resb >= 0 ? (uint32_t *)(dsm + I.so_resb) : I.resb;
            W.res_list = I.so_res_list >= 0 ? (int32_t *)(dsm + I.so_res_list) : I.res_list;
            W.plan = I.so_plan >= 0 ? (int4 *)(dsm + I.so_plan) : I.plan;
            W.plan_cum = !I.tau ? nullptr : (I.so_plan_tau >= 0 ? (int64_t *)(dsm + I.so_plan_tau) : I.plan_tau);
            W.dptr32 = I.so_dptr >= 0 ? (int32_t *)(dsm + I.so_dptr) : nullptr;
            W.lru = I.so_lru >= 0 ? (int32_t *)(dsm + I.so_lru) : I.lru;
            W.al = I.so_al >= 0 ? (uint32_t *)(dsm + I.so_al) : I.al;
        }
        cta_sync();
        const View &V = SV;
        if (M_SHARD(I))
            for (int p = tid; p < I.G; p += blockDim.x) SP[p] = I.peers[p];

        const int n = I.n, K = I.K;
        if (I.fused) {  // a1 + a2 inside this CTA (small instances)
            fused_build(dsm);
            fused_init();
        } else {
        // ---- CTA-local copies of the initial state (global homes were
        //      initialised by dts_init_kernel)
        if (I.so_dptr >= 0)
            for (int D = tid; D <= n; D += blockDim.x) V.dptr32[D] = (int32_t)__ldg(&I.dptr[D]);
        if (I.so_s >= 0) {
            const uint4 *src = reinterpret_cast<const uint4 *>(I.s);
            uint4 *dst = reinterpret_cast<uint4 *>(V.s);
            for (int i = tid; i < (K * I.m_pad) / 4; i += blockDim.x) dst[i] = __ldcg(&src[i]);
        }
        if (M_SL(I) && I.so_al >= 0)
            for (int i = tid; i <= I.m_pad / 32; i += blockDim.x) V.al[i] = __ldcg(&I.al[i]);
        if (I.so_u >= 0)  // packed rows: u as 16-bit halves, nstr / 2 words
            for (int D = tid; D < (M_HH ? I.nstr / 2 : I.nstr); D += blockDim.x) V.u[D] = __ldcg(&I.u[D]);
        if (I.so_h >= 0)
            for (int i = tid; i < K * I.nstr; i += blockDim.x) V.h[i] = __ldcg(&I.h[i]);
        if (I.so_h2 >= 0 && !M_HH)
            for (int i = tid; i < K * I.nstr; i += blockDim.x) V.h2[i] = __ldcg(&I.h2[i]);
        if (I.so_np >= 0)
            for (int i = tid; i < K * I.nstr; i += blockDim.x) V.np[i] = 0;
        if (I.so_resb >= 0)
            for (int i = tid; i < K * I.nw; i += blockDim.x) V.resb[i] = 0u;
        }
        if (tid == 0) {
            for (int k = 0; k < MAX_K; k++) {
                L.req[k] = 0;
                L.gpu_free[k] = 0;
                L.used[k] = 0;
                L.plan_head[k] = L.plan_end[k] = L.plan_live[k] = 0;
                L.res_cnt[k] = 0;
                L.idle[k] = 0;
                L.won[k] = 0;
            }
            L.bus_free = 0;
            L.n_events = L.n_served = L.n_loads = L.n_evictions = L.n_scans = L.n_fb2 = L.n_fbf =
                L.n_belady = L.n_idle = L.n_verr = 0;
            L.bytes_loaded = L.alg_bytes = L.scan_alg_bytes = 0;
            L.sum_avail = L.n_alloc = L.sum_deg = 0;
            L.makespan = 0;
            L.n_avail = I.m;
            L.avail_lo = 0;
            L.error = 0;
            L.row_len = 0;
            L.xe = 0;
            L.xerr = 0;
            for (int i = 0; i < 16; i++) L.prof[i] = 0;
        }
        cta_sync();

        // ---- the decision loop
        while (true) {
            PROF_T0(p_pop);
            if (M_LUF(I)) {
                int pending = 0;  // planned tasks left on all GPUs (uniform: every thread sums)
                for (int j = 0; j < K; j++) pending += L.plan_live[j];
                if (I.max_served < 0 && M_W(I) == 0 && K <= 32 && pending > I.pop_batch_min) {
                    pop_batch();
                } else {  // few pops (or a prefix run that stops at an exact count): thread 0
                    cta_sync();
                    if (tid == 0)
                        L.cmd = ((I.max_served < 0 || L.n_served < I.max_served) && pop_run_seq() >= 0)
                                    ? CMD_SCAN
                                    : CMD_DONE;
                }
            } else {
                // LRU policies: an LRU eviction does not drop planned tasks, so a
                // pop may need loads -- every request is served block-wide
                cta_sync();
                if (tid == 0) {
                    int cmd = CMD_DONE;
                    if (I.max_served < 0 || L.n_served < I.max_served) {
                        int kk = -1;  // next request: smallest (req_k, k), non-idle (R8)
                        int64_t tb = 0;
                        for (int j = 0; j < K; j++)
                            if (!L.idle[j] && (kk < 0 || L.req[j] < tb)) {
                                kk = j;
                                tb = L.req[j];
                            }
                        if (kk >= 0) {
                            L.k = kk;
                            L.t = tb;
                            if (M_POL(I, DTS_POLICY_DARTS_LRU) && L.plan_live[kk] > 0) {
                                int64_t tau;
                                L.T = pop_planned(kk, &tau);
                                cmd = CMD_POP;
                            } else {
                                cmd = M_POL(I, DTS_POLICY_EAGER_LRU) ? CMD_EAGER : CMD_SCAN;
                            }
                        }
                    }
                    L.cmd = cmd;
                }
            }
            PROF_ADD(L, P_POP, p_pop);
            cta_sync();
            if (L.cmd == CMD_DONE || L.xerr) break;
            const int k = L.k;
            const int64_t t = L.t;
            int32_t T = -1;
            if (L.cmd == CMD_POP) {
                T = L.T;
                if (T < 0) break;  // pop_planned found no entry (L.error set)
            } else if (L.cmd == CMD_EAGER) {
                // EAGER: the shared FIFO queue in submission
                // order -- the lowest-id unallocated task
                T = L.n_avail > 0 ? any_first_avail() : -1;
                if (tid == 0) {
                    if (T >= 0) {
                        L.avail_lo = T;
                        L.fent = entry_of_task(T);
                        row_from_entry(L.fent);
                        L.n_avail--;
                        L.n_alloc++;
                    } else {
                        L.idle[k] = 1;
                        L.n_idle++;
                    }
                }
                cta_sync();
                if (T < 0) continue;
                pool_move_many(&L.fent, 1, -1, -1);
                cta_sync();
            } else {
            reset_plan(k);
            if (M_FLAG(I, DTS_F_VERIFY)) verify_scores(k);
            // Alg. 5 l.4-9: Dopt = argmax (n_k(D), u(D), -D) over dataNotInMem_k
            PROF_T0(p_am);
            int32_t D2s = -1;  // task shards, packed rows: the 3inputs argmax comes with the main one
            const int32_t Dopt = M_SHARD(I) ? shard_scan(k, (I.flags & DTS_F_FALLBACK2) != 0,
                                                      M_FLAG(I, DTS_F_OPTI) != 0, &D2s)
                                 : M_FLAG(I, DTS_F_OPTI) ? score_first(V.h + (size_t)k * I.nstr)
                                 // packed rows in HBM/L2 (C4): both keys in one pass; in
                                 // shared memory (ALU-bound): the 3inputs pass only when needed
                                 : (M_HH && I.so_h < 0) ? score_argmax_hh(V.h + (size_t)k * I.nstr, &D2s)
                                                        : score_argmax(V.h + (size_t)k * I.nstr);
            PROF_ADD(L, P_ARGMAX, p_am);
            PROF_T0(p_pl);
            if (tid == 0) {
                L.scan_alg_bytes += 8ull * (uint64_t)n;
                L.alg_bytes += 8ull * (uint64_t)n;
                L.scan_avail = L.n_avail;  // before this scan allocates anything
            }
            if (M_SHARD(I) && L.xerr) break;  // a peer timed out in the scan exchange (CTA-uniform)
            if (Dopt >= 0) {
                if (M_SHARD(I)) plan_shard(k, Dopt);
                else plan(k, Dopt);
                if (M_SHARD(I) && L.xerr) break;  // plan exchange failed: no plan to pop from
                if (tid == 0) {
                    int64_t tau;
                    L.T = pop_planned(k, &tau);
                    L.n_scans++;
                    L.sum_avail += L.scan_avail;
                }
                cta_sync();
                T = L.T;
                if (T < 0) break;  // pop_planned found no entry (L.error set)
                PROF_ADD(L, P_PLAN, p_pl);
            } else {
                if (I.flags & DTS_F_FALLBACK2) {
                    const int32_t D2 = (M_SHARD(I) || (M_HH && I.so_h < 0)) ? D2s
                                       : M_HH ? score_argmax(V.h + (size_t)k * I.nstr, 0)
                                              : score_argmax(V.h2 + (size_t)k * I.nstr);
                    if (tid == 0) {
                        L.scan_alg_bytes += 8ull * (uint64_t)n;
                        L.alg_bytes += 8ull * (uint64_t)n;
                    }
                    if (D2 >= 0) {
                        T = any_first_cnt2(k, D2);
                        if (tid == 0) L.n_fb2++;
                    }
                }
                if (T < 0 && L.n_avail > 0) {
                    T = any_first_avail();
                    if (tid == 0) {
                        L.n_fbf++;
                        L.avail_lo = T;
                    }
                }
                if (T >= 0) {
                    if (tid == 0) {
                        L.fent = entry_of_task(T);
                        row_from_entry(L.fent);
                        L.n_avail--;
                        L.n_alloc++;
                        L.n_scans++;
                        L.sum_avail += L.scan_avail;
                    }
                    cta_sync();
                    pool_move_many(&L.fent, 1, -1, -1);
                } else if (tid == 0) {
                    L.idle[k] = 1;
                    L.n_idle++;
                }
                cta_sync();
                PROF_ADD(L, P_OTHER, p_pl);
                if (M_SHARD(I) && L.xerr) break;  // a min-exchange failed: T is not trustworthy
                if (T < 0) continue;
            }
            }  // scan
            // serve T with its loads (block-wide); D(T) from the CSR unless cached
            const bool need_row = L.row_len < 0;
            cta_sync();
            if (need_row && tid < 32) {
                const int64_t rb = __ldg(&I.tptr[T]), re = __ldg(&I.tptr[T + 1]);
                for (int r = tid; r < (int)(re - rb); r += 32) L.row[r] = __ldg(&I.tdat[rb + r]);
                if (tid == 0) L.row_len = (int)(re - rb);
            }
            cta_sync();
            PROF_T0(p_ld);
            serve_loads(k, T, t);
            PROF_ADD(L, P_LOADS, p_ld);
            if (L.error || L.xerr) break;
        }
        cta_sync();
        if (M_SHARD(I)) {  // no shard leaves while a peer may still read its slots
            xch_sync();
            if (tid == 0 && L.xerr && !L.error) L.error = 2;
            cta_sync();
        }

        // ---- a8: per-GPU orders, scalars
        cta_sync();  // the loop's shared-memory arrays are dead from here on
        assemble(L.n_served, dsm);
        if (tid == 0) {
            Out *o = I.out;
            o->n_events = L.n_events;
            o->n_served = L.n_served;
            o->n_loads = L.n_loads;
            o->n_evictions = L.n_evictions;
            o->n_scans = L.n_scans;
            o->n_fallback2 = L.n_fb2;
            o->n_fallback_first = L.n_fbf;
            o->n_belady = L.n_belady;
            o->n_idle = L.n_idle;
            o->n_verify_err = L.n_verr;
            o->bytes_loaded = L.bytes_loaded;
            o->makespan = L.makespan;
            o->alg_bytes = L.alg_bytes;
            o->scan_alg_bytes = L.scan_alg_bytes;
            o->sum_avail = L.sum_avail;
            o->n_alloc = L.n_alloc;
            o->sum_deg = L.sum_deg;
            o->error = L.error;
            for (int i = 0; i < 16; i++) o->prof[i] = L.prof[i];
        }
        cta_sync();
    }
}

#if !DTS_FAST
// ---------------------------------------------------------------- init (a2)
// Global homes: s_k(T) = (|D(T)| << 24) | XOR D(T) for every k (nothing
// resident), pad words allocated; u(D) = deg(D); h_k(D) / h2_k(D) = the tasks
// of D's segment with 1 / 2 inputs (all missing); np = 0; delta(D); times -1.
__global__ void dts_init_kernel(const Inst *__restrict__ insts, int n_inst, uint64_t bw) {
    for (int ii = 0; ii < n_inst; ii++) {
        const Inst I = insts[ii];
        if (I.fused) continue;  // built and initialised inside its loop CTA
        int64_t *delta = const_cast<int64_t *>(I.delta);
        const int64_t tid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
        const int64_t str = (int64_t)gridDim.x * blockDim.x;
        for (int64_t T = tid; T < I.m_pad; T += str) {
            uint32_t w = ALLOC_BIT;
            if (T < I.m) {
                const int64_t b = I.tptr[T], e = I.tptr[T + 1];
                uint32_t x = 0;
                for (int64_t i = b; i < e; i++) x ^= (uint32_t)I.tdat[i];
                w = ((uint32_t)(e - b) << 24) | x;
                if (T < I.t_lo || T >= I.t_hi) w |= ALLOC_BIT;  // another shard's task
                I.tstart[T] = -1;
                I.tend[T] = -1;
            }
            if (!M_SL(I))
                for (int k = 0; k < I.K; k++) I.s[(size_t)k * I.m_pad + T] = w;
        }
        if (M_SL(I))  // allocation bitmap: nothing allocated, bits past m set
            for (int64_t wd = tid; wd <= I.m_pad / 32; wd += str) {
                const int64_t t0 = 32 * wd;
                I.al[wd] = t0 >= I.m ? ~0u : (I.m - t0 >= 32 ? 0u : ~((1u << (I.m - t0)) - 1u));
            }
        for (int64_t D = I.n + tid; D < I.nstr; D += str) {  // row padding: never scores
            if (I.hh) reinterpret_cast<uint16_t *>(I.u)[D] = 0;
            else I.u[D] = 0;
            for (int k = 0; k < I.K; k++) {
                I.h[(size_t)k * I.nstr + D] = 0;
                I.h2[(size_t)k * I.nstr + D] = 0;
                I.np[(size_t)k * I.nstr + D] = 0;
            }
        }
        for (int64_t D = tid; D < I.n; D += str) {
            const int64_t b = I.dptr[D], e = I.dptr[D + 1];
            int32_t c1 = 0, c2 = 0;
            for (int64_t i = b; i < e; i++) {
                const int32_t T = I.ddat[i];
                const int64_t len = I.tptr[T + 1] - I.tptr[T];
                c1 += (len == 1);
                c2 += (len == 2);
            }
            if (I.hh) reinterpret_cast<uint16_t *>(I.u)[D] = (uint16_t)(e - b);
            else I.u[D] = (int32_t)(e - b);
            unsigned __int128 num = (unsigned __int128)I.size[D] * 1000000000ull + (bw - 1);
            delta[D] = (int64_t)(num / bw);
            for (int k = 0; k < I.K; k++) {
                I.h[(size_t)k * I.nstr + D] = I.hh ? (c1 | (c2 << 16)) : c1;
                I.h2[(size_t)k * I.nstr + D] = c2;
                I.np[(size_t)k * I.nstr + D] = 0;
            }
        }
        for (int64_t i = tid; i < (int64_t)I.K * I.nw; i += str) I.resb[i] = 0u;
    }
}

#endif  // !DTS_FAST

// ---------------------------------------------------------------- launchers
#if !DTS_FAST
cudaError_t launch_init(const Inst *d_insts, int n_inst, uint64_t bw, int64_t work, cudaStream_t st) {
    int64_t blocks = (work + 255) / 256;
    if (blocks < 1) blocks = 1;
    if (blocks > 148 * 8) blocks = 148 * 8;
    dts_init_kernel<<<(unsigned)blocks, 256, 0, st>>>(d_insts, n_inst, bw);
    count_launch();
    return cudaGetLastError();
}
#endif

// cudaFuncSetAttribute is a driver call worth avoiding per launch: raise the
// kernel's dynamic shared-memory limit only when a launch needs more.
static cudaError_t ensure_smem_attr(int smem_bytes) {
    static int cur[64];
    static bool init = false;
    if (!init) {
        for (int &c : cur) c = -1;
        init = true;
    }
    int dev = 0;
    cudaGetDevice(&dev);
    if (dev < 0 || dev >= 64) dev = 0;
    if (smem_bytes <= cur[dev]) return cudaSuccess;
    cudaError_t e =
        cudaFuncSetAttribute(DTS_KNAME(dts_cta_kernel), cudaFuncAttributeMaxDynamicSharedMemorySize, smem_bytes);
    if (e == cudaSuccess) cur[dev] = smem_bytes;
    return e;
}

cudaError_t DTS_KNAME(launch_loop)(const Inst *d_insts, int n_inst, int block, int grid, int *work_counter,
                                   int smem_bytes, cudaStream_t st) {
    cudaError_t e = ensure_smem_attr(smem_bytes);
    if (e != cudaSuccess) return e;
    DTS_KNAME(dts_cta_kernel)<<<grid, block, smem_bytes, st>>>(d_insts, n_inst, work_counter);
    count_launch();
    return cudaGetLastError();
}

#if !DTS_FAST
cudaError_t launch_loop_coop(const Inst *d_insts, int n_inst, int block, int *work_counter, int smem_bytes,
                             cudaStream_t st) {
    cudaError_t e = ensure_smem_attr(smem_bytes);
    if (e != cudaSuccess) return e;
    void *args[] = {(void *)&d_insts, (void *)&n_inst, (void *)&work_counter};
    e = cudaLaunchCooperativeKernel((const void *)dts_cta_kernel, dim3(n_inst), dim3(block), args,
                                    (size_t)smem_bytes, st);
    count_launch();
    return e;
}
#endif

int DTS_KNAME(loop_max_blocks_per_sm)(int block, int smem_bytes) {
    int nb = 0;
    if (ensure_smem_attr(smem_bytes) != cudaSuccess) return 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, DTS_KNAME(dts_cta_kernel), block, smem_bytes) !=
        cudaSuccess)
        return 0;
    return nb;
}

int DTS_KNAME(loop_static_smem)() {
    cudaFuncAttributes a;
    if (cudaFuncGetAttributes(&a, DTS_KNAME(dts_cta_kernel)) != cudaSuccess) return -1;
    return (int)a.sharedSizeBytes;
}

}  // namespace dts

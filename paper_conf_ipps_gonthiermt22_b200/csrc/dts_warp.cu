// dts_warp.cu -- the DARTS+LUF decision loop with ONE WARP per instance
// (§8(a) a1-a8 for small instances: C1, C2, the 4,096 C5 instances).
//
// Same schedule as dts_loop.cu (same readings R1-R29, same incremental
// scores), re-laid out for a single warp so that a decision is a short chain
// of warp instructions with no CTA barrier and no serial thread-0 section:
//
//   * per-GPU scalars live in REGISTERS of lane k (= simulated GPU k, K <= 32):
//     request time, GPU-free time, resident count, plan head / end / live,
//     idle flag.  The next request (R8: smallest (req_k, k)) is ONE 64-bit
//     warp min of (req_k << 5 | k); the scalars of the chosen GPU are read
//     with shuffles.  Everything uniform (bus, event count, counters) is kept
//     redundantly in every lane, so no broadcast is needed.
//   * the instance state is in the warp's slice of shared memory, packed:
//     hh[k][D] = n_k(D) | n2_k(D) << 16 (Alg. 5 l.4-5 and the 3inputs score,
//     PAPER.md:703-706, 1823-1834) -- one 32-bit atomic moves a task between
//     the two buckets; u(D) (R23) and np_k(D) (Alg. 6 l.3) as 16-bit halves;
//     residency and allocation bitmaps; plans and resident lists.
//   * the data->task CSR is built by the warp itself at instance start (a
//     stable counting sort) into ONE 32-bit edge word per (D, T):
//     T << 16 | (T's other input, 0xFFFF if none).  A segment walk reads 4
//     bytes per edge; a plan entry is the same word (its Dopt is per plan).
//
// Applies to instances in the compile-time fast mode of dts_loop_fast.cu
// (row-derived state, one shard, W = 0, DARTS+LUF, 32-bit keys, uniform
// sizes, no OPTI / VERIFY) with <= 2 inputs per task, m <= 65535, n <= 65534,
// K <= 32 and a state slice that fits in shared memory (host: dts_api.cu
// warp_mode).  dts_loop.cu stays the path for everything else.
#include <cuda_runtime.h>

#include <climits>
#include <cstdint>
#include <mutex>

#include "dts_internal.cuh"
#include "dts_loop.cuh"

namespace dts {

namespace {

constexpr unsigned FULL = 0xffffffffu;
constexpr uint32_t NOI = 0xFFFFu;          // edge / plan word: no other input
constexpr uint32_t REMOVED = 0xFFFFFFFFu;  // plan word removed by LUF (Alg. 6 l.8)

__device__ __forceinline__ unsigned long long wmax64(unsigned long long v) {
    const unsigned hi = (unsigned)(v >> 32), lo = (unsigned)v;
    const unsigned mh = __reduce_max_sync(FULL, hi);
    const unsigned ml = __reduce_max_sync(FULL, hi == mh ? lo : 0u);
    return ((unsigned long long)mh << 32) | ml;
}
__device__ __forceinline__ unsigned long long wmin64(unsigned long long v) {
    const unsigned hi = (unsigned)(v >> 32), lo = (unsigned)v;
    const unsigned mh = __reduce_min_sync(FULL, hi);
    const unsigned ml = __reduce_min_sync(FULL, hi == mh ? lo : 0xffffffffu);
    return ((unsigned long long)mh << 32) | ml;
}
// Per-phase cycle probes, profiling build only (lib/libdts_prof.so, -DDTS_PROF):
// WP(slot) charges the cycles since the previous probe to prof[slot].
#ifdef DTS_PROF
#define WP_DECL long long prof_[16] = {0}, pt_ = clock64()
#define WP(slot)                         \
    do {                                 \
        const long long t1_ = clock64(); \
        prof_[slot] += t1_ - pt_;        \
        pt_ = t1_;                       \
    } while (0)
#define WP_OUT(i) prof_[i]
// bounds checks of the profiling build (compute-sanitizer is not available on
// the GPU pool): a failed check sets the instance's error (Out::error = 9)
#define WCHK(c) (chk_ |= !(c))
#else
#define WP_DECL
#define WP(slot) \
    do {         \
    } while (0)
#define WP_OUT(i) 0
#define WCHK(c) ((void)0)
#endif

__device__ __forceinline__ int wsum(int v) { return (int)__reduce_add_sync(FULL, (unsigned)v); }

// 16-bit counters stored in pairs: add d to entry i (the field never leaves
// [0, 2^16), so the 32-bit add cannot carry into the neighbour).
__device__ __forceinline__ void add16(uint16_t *a, int i, int d) {
    atomicAdd(reinterpret_cast<unsigned *>(a) + (i >> 1), (unsigned)d << (16 * (i & 1)));
}

// Segment walks hold SEGR edges per lane in registers (32 SEGR = 160 per
// batch: C5's widest segment).  Every unrolled slot costs instructions: 8
// and 6 were slower, and one copy of the loop per width (2, 4, 5, 8 chosen
// per instance) made the C5 sweep 33 % slower (registers, instruction cache;
// profiles/r03/r03_warp_var.txt).
#ifndef DTS_SEGR
#define DTS_SEGR 5
#endif
constexpr int SEGR = DTS_SEGR;

// The warp's view of one instance (registers; pointers into its smem slice).
struct WV {
    int m, n, K, n4, n8, pcap, rcap, maxres;
    uint32_t kmask;  // bits 0..K-1
    uint32_t *resm;  // [n4]     bit k = D resident on simulated GPU k
    uint32_t *al;    // [m/32+1] allocation bitmap (R2; bits past m set)
    int32_t *dp;     // [n+1]    segment starts in wedge
    uint16_t *u;     // [n8]     u(D) = #unallocated tasks using D (R23)
    uint32_t *hh;    // [K][n4]  n_k(D) | n2_k(D) << 16
    uint16_t *np;    // [K][n8]  np_k(D) = #tasks of plannedTasks_k using D
    uint32_t *plan;  // [K][pcap] plannedTasks_k, ascending id: T << 16 | other input
    int32_t *rl;     // [K][rcap] resident data of GPU k
    const uint32_t *wedge;  // [E] global: data->task edges, each segment in ascending T
};

__device__ __forceinline__ bool res(const WV &v, int k, int D) { return (v.resm[D] >> k) & 1u; }

// D(T) of a task given as its caller's raw row (<= 2 distinct ids, sorted,
// duplicates removed: D(T) is a set, R27).  -1 = absent.
__device__ __forceinline__ void raw_row(const int64_t *rp, const int32_t *rd, int T, int &a, int &b) {
    const int64_t rb = rp[T], re = rp[T + 1];
    a = -1;
    b = -1;
    for (int64_t i = rb; i < re; i++) {
        const int d = rd[i];
        if (a < 0) a = d;
        else if (d != a) b = d;
    }
    if (b >= 0 && b < a) {
        const int t = a;
        a = b;
        b = t;
    }
}

// A task with inputs {a, b} (b = -1: one input) leaves (sign -1) or re-enters
// (+1) the shared pool: on every simulated GPU j where it has one missing
// input it counts in n_j(that input), where it has two in n2_j(both) --
// read off the two residency masks.  GPUs in `skip` are done by the caller.
__device__ __forceinline__ void pool_buckets(const WV &v, int a, int b, int sign, uint32_t skip) {
    if (a < 0) return;
    const uint32_t ma = ~v.resm[a] & v.kmask & ~skip;
    const uint32_t mb = b >= 0 ? (~v.resm[b] & v.kmask & ~skip) : 0u;
    uint32_t two = ma & mb, oa = ma & ~mb, ob = mb & ~ma;
    const unsigned s2 = (unsigned)(sign * 65536), s1 = (unsigned)sign;
    while (two) {
        const int j = __ffs(two) - 1;
        two &= two - 1;
        atomicAdd(&v.hh[j * v.n4 + a], s2);
        atomicAdd(&v.hh[j * v.n4 + b], s2);
    }
    while (oa) {
        const int j = __ffs(oa) - 1;
        oa &= oa - 1;
        atomicAdd(&v.hh[j * v.n4 + a], s1);
    }
    while (ob) {
        const int j = __ffs(ob) - 1;
        ob &= ob - 1;
        atomicAdd(&v.hh[j * v.n4 + b], s1);
    }
}

// Argmax over D of the key (score, u(D), -D) among data with a positive score
// (Alg. 5 l.6-9 with hi = 0; the 3inputs key with hi = 1; R1, R23, R24).  A
// datum with a positive score is never resident.  -1 if none.  Four vectors
// of four data per lane are loaded before any compare.
__device__ __forceinline__ unsigned long long max64(unsigned long long a, unsigned long long b) {
    return a > b ? a : b;
}
__device__ __forceinline__ int argmax_score(const WV &v, int k, bool hi, int lane) {
    const uint4 *h4 = reinterpret_cast<const uint4 *>(v.hh + k * v.n4);
    const uint2 *u2 = reinterpret_cast<const uint2 *>(v.u);
    const int nv = v.n4 >> 2;
    unsigned long long best = 0ull;  // (score << 16 | u) << 32 | (2^32 - 1 - D): ties -> lowest D
    for (int q0 = lane; q0 < nv; q0 += 128) {
        uint4 x[4];
        uint2 y[4];
#pragma unroll
        for (int r = 0; r < 4; r++) {
            const int q = q0 + 32 * r;
            x[r] = q < nv ? h4[q] : make_uint4(0, 0, 0, 0);
            y[r] = q < nv ? u2[q] : make_uint2(0, 0);
        }
        unsigned long long c[4];
#pragma unroll
        for (int r = 0; r < 4; r++) {  // a max tree per vector, then over the vectors
            const uint32_t D = 4u * (uint32_t)(q0 + 32 * r);
            const uint32_t s0 = hi ? (x[r].x & 0xFFFF0000u) : (x[r].x << 16);
            const uint32_t s1 = hi ? (x[r].y & 0xFFFF0000u) : (x[r].y << 16);
            const uint32_t s2 = hi ? (x[r].z & 0xFFFF0000u) : (x[r].z << 16);
            const uint32_t s3 = hi ? (x[r].w & 0xFFFF0000u) : (x[r].w << 16);
            const unsigned long long c0 = ((unsigned long long)(s0 | (y[r].x & 0xFFFFu)) << 32) | (0xFFFFFFFFu - D);
            const unsigned long long c1 = ((unsigned long long)(s1 | (y[r].x >> 16)) << 32) | (0xFFFFFFFEu - D);
            const unsigned long long c2 = ((unsigned long long)(s2 | (y[r].y & 0xFFFFu)) << 32) | (0xFFFFFFFDu - D);
            const unsigned long long c3 = ((unsigned long long)(s3 | (y[r].y >> 16)) << 32) | (0xFFFFFFFCu - D);
            c[r] = max64(max64(c0, c1), max64(c2, c3));
        }
        best = max64(best, max64(max64(c[0], c[1]), max64(c[2], c[3])));
    }
    if ((best >> 32) < 65536u) best = 0ull;  // no positive score
    const unsigned long long w = wmax64(best);
    return w ? (int)(0xFFFFFFFFu - (uint32_t)w) : -1;
}

// One batch of a data->task segment in registers: edges [b, e) of lane `lane`
// at b + lane + 32 r (REMOVED past the end).
__device__ __forceinline__ void seg_load(const WV &v, int b, int e, int lane, uint32_t (&ed)[SEGR]) {
#pragma unroll
    for (int r = 0; r < SEGR; r++) {
        const int i = b + lane + 32 * r;
        ed[r] = i < e ? v.wedge[i] : REMOVED;
    }
}

// a2 on one batch: D became resident on GPU k (load) or left it (evict); each
// unallocated task of the batch moves between the buckets.  Missing count
// before the change: D plus the other input o if o is missing too.  The
// allocation and residency words of all the batch's tasks are gathered
// before any update.  n1 / n2: the batch's tasks that leave / enter n_k(D)
// and n2_k(D) (applied once by the caller).
__device__ __forceinline__ void seg_apply(const WV &v, int k, bool load, const uint32_t (&ed)[SEGR], int nr,
                                          int &n1, int &n2) {
    uint32_t aw[SEGR], rw[SEGR];
#pragma unroll
    for (int r = 0; r < SEGR; r++) {
        const uint32_t w = ed[r];
        const int T = (int)(w >> 16), o = (int)(w & 0xFFFFu);
        aw[r] = w != REMOVED ? v.al[T >> 5] : ~0u;
        rw[r] = (w != REMOVED && o != (int)NOI) ? v.resm[o] : ~0u;
    }
    uint32_t *hk = v.hh + k * v.n4;
    const unsigned dd = load ? (1u - 65536u) : (65536u - 1u);
#pragma unroll
    for (int r = 0; r < SEGR; r++) {
        const uint32_t w = ed[r];
        const int T = (int)(w >> 16), o = (int)(w & 0xFFFFu);
        const bool live = w != REMOVED && !((aw[r] >> (T & 31)) & 1u);
        const bool mo = live && !((rw[r] >> k) & 1u);
        n1 += (int)(live && !mo);  // load: 1 -> 0 (n_k(D) - 1); evict: 0 -> 1 (n_k(D) + 1)
        n2 += (int)mo;             // load: 2 -> 1, freed by o now; evict: 1 -> 2, {o, D} missing
        if (mo) atomicAdd(&hk[o], dd);
    }
}

// a2 for the whole segment of D; its first batch is given (prefetched).
__device__ __forceinline__ void seg_update(const WV &v, int k, int D, bool load, int lane,
                                           const uint32_t (&ed0)[SEGR]) {
    const int b = v.dp[D], e = v.dp[D + 1];
    int n1 = 0, n2 = 0;
    seg_apply(v, k, load, ed0, min(SEGR, (e - b + 31) >> 5), n1, n2);
    for (int base = b + 32 * SEGR; base < e; base += 32 * SEGR) {
        uint32_t ed[SEGR];
        seg_load(v, base, e, lane, ed);
        seg_apply(v, k, load, ed, min(SEGR, (e - base + 31) >> 5), n1, n2);
    }
    n1 = wsum(n1);
    n2 = wsum(n2);
    if (lane == 0 && (n1 | n2)) {
        const uint32_t d = (uint32_t)n1 + ((uint32_t)n2 << 16);
        atomicAdd(&v.hh[k * v.n4 + D], load ? (0u - d) : d);
    }
    __syncwarp();
}

__device__ __forceinline__ void push_event(dts_event *evs, int64_t evcap, int64_t &nev, int lane, uint8_t op, int k,
                                           int D, int T, int64_t t, int64_t te) {
    if (lane == 0 && nev < evcap) {
        dts_event ev;
        ev.t_ns = t;
        ev.t_end_ns = te;
        ev.gpu = k;
        ev.data = D;
        ev.task = T;
        ev.op = op;
        ev.pad[0] = ev.pad[1] = ev.pad[2] = 0;
        evs[nev] = ev;
    }
    nev++;
}

// x / tau and x mod tau for 0 <= x < 2^52 (times in ns): a double-precision
// estimate corrected by one step (exact; no 64-bit integer division).
__device__ __forceinline__ int64_t div_tau(int64_t x, int64_t tau, double inv, int64_t &rem) {
    int64_t q = (int64_t)((double)x * inv);
    int64_t r = x - q * tau;
    while (r < 0) {
        q--;
        r += tau;
    }
    while (r >= tau) {
        q++;
        r -= tau;
    }
    rem = r;
    return q;
}

__device__ __forceinline__ int64_t tau_of(const int64_t *taup, int T, int64_t dtau) {
    return taup ? taup[T] : dtau;
}

// a1 + a2 at instance start (cold: out of line, the hot loop stays small):
// the data->task CSR as 32-bit edge words by a stable counting sort, the
// initial scores (nothing resident: n_k(D) / n2_k(D) = D's tasks with one /
// two inputs), u(D) = deg(D), empty bitmaps, task times -1.
__device__ __noinline__ void build_state(const WV v, const WarpLayout Lw, unsigned char *dsm, const int64_t *rp,
                                         const int32_t *rd, uint32_t *wedge, int64_t *tst, int64_t *ten, int lane) {
    const unsigned lt = (1u << lane) - 1u;
    const int m = v.m, n = v.n, K = v.K;
    // a1: data->task CSR (stable counting sort by warp) + initial scores
    {
        uint32_t *mask = reinterpret_cast<uint32_t *>(dsm + Lw.np);  // build scratch [n] + [n]
        int32_t *cur = reinterpret_cast<int32_t *>(mask + n);
        for (int i = lane; i < n; i += 32) {
            mask[i] = 0u;
            cur[i] = 0;
        }
        for (int i = lane; i < v.n4; i += 32) v.hh[i] = 0u;
        __syncwarp();
        // degrees; n_0(D) / n2_0(D) with nothing resident.  Four tasks per lane and
        // pass with their row loads in flight together; each task's D(T) is left as
        // one word a | b << 16 (0xFFFF: absent) in the task-start array (overwritten
        // by a2 below) for the scatter pass
        uint32_t *rows = reinterpret_cast<uint32_t *>(tst);
        for (int T0 = 0; T0 < m; T0 += 128) {
            int64_t rb[4], re[4];
#pragma unroll
            for (int q = 0; q < 4; q++) {
                const int T = T0 + 32 * q + lane;
                rb[q] = T < m ? rp[T] : 0;
                re[q] = T < m ? rp[T + 1] : 0;
            }
            int x0[4], x1[4];
#pragma unroll
            for (int q = 0; q < 4; q++) {
                x0[q] = re[q] > rb[q] ? rd[rb[q]] : -1;
                x1[q] = re[q] > rb[q] + 1 ? rd[rb[q] + 1] : -1;
            }
#pragma unroll
            for (int q = 0; q < 4; q++) {
                const int T = T0 + 32 * q + lane;
                if (T >= m) continue;
                int a, b;
                if (re[q] - rb[q] > 2) {  // duplicates in a longer raw row (R27)
                    raw_row(rp, rd, T, a, b);
                } else {
                    a = x0[q];
                    b = x1[q] != x0[q] ? x1[q] : -1;
                    if (b >= 0 && b < a) {
                        const int t = a;
                        a = b;
                        b = t;
                    }
                }
                rows[T] = (uint32_t)(a & 0xFFFF) | ((uint32_t)(b & 0xFFFF) << 16);
                if (a >= 0) {
                    atomicAdd(&cur[a], 1);
                    atomicAdd(&v.hh[a], b >= 0 ? 65536u : 1u);
                }
                if (b >= 0) {
                    atomicAdd(&cur[b], 1);
                    atomicAdd(&v.hh[b], 65536u);
                }
            }
        }
        __syncwarp();
        int carry = 0;  // dp = exclusive scan of the degrees; cursors start there
        for (int D0 = 0; D0 < n; D0 += 32) {
            const int D = D0 + lane;
            const int d = D < n ? cur[D] : 0;
            int x = d;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const int y = __shfl_up_sync(FULL, x, o);
                if (lane >= o) x += y;
            }
            if (D < n) {
                v.dp[D] = carry + x - d;
                cur[D] = carry + x - d;
            }
            carry += __shfl_sync(FULL, x, 31);
        }
        if (lane == 0) v.dp[n] = carry;
        __syncwarp();
        __threadfence_block();
        for (int T0 = 0; T0 < m; T0 += 32) {  // stable scatter: segments in ascending task id
            const int T = T0 + lane;
            int a = -1, b = -1;
            if (T < m) {
                const uint32_t w = rows[T];
                a = (w & 0xFFFFu) == 0xFFFFu ? -1 : (int)(w & 0xFFFFu);
                b = (w >> 16) == 0xFFFFu ? -1 : (int)(w >> 16);
            }
            if (a >= 0) atomicOr(&mask[a], 1u << lane);
            if (b >= 0) atomicOr(&mask[b], 1u << lane);
            __syncwarp();
            const unsigned ma = a >= 0 ? mask[a] : 0u, mb = b >= 0 ? mask[b] : 0u;
            if (a >= 0) wedge[cur[a] + __popc(ma & lt)] = ((uint32_t)T << 16) | (b >= 0 ? (uint32_t)b : NOI);
            if (b >= 0) wedge[cur[b] + __popc(mb & lt)] = ((uint32_t)T << 16) | (uint32_t)a;
            __syncwarp();
            if (a >= 0 && lane == __ffs(ma) - 1) cur[a] += __popc(ma);
            if (b >= 0 && lane == __ffs(mb) - 1) cur[b] += __popc(mb);
            __syncwarp();
            if (a >= 0) mask[a] = 0u;
            if (b >= 0) mask[b] = 0u;
            __syncwarp();
        }
        __threadfence_block();
        __syncwarp();
    }
    // a2: initial state
    for (int i = lane; i <= m / 32; i += 32) {
        const int t0 = 32 * i;
        v.al[i] = t0 >= m ? ~0u : (m - t0 >= 32 ? 0u : ~((1u << (m - t0)) - 1u));
    }
    for (int i = lane; i < v.n4; i += 32) v.resm[i] = 0u;
    for (int i = lane; i < v.n8; i += 32) v.u[i] = (uint16_t)(i < n ? v.dp[i + 1] - v.dp[i] : 0);
    for (int i = lane; i < (K - 1) * v.n4; i += 32) v.hh[v.n4 + i] = v.hh[i % v.n4];
    for (int i = lane; i < K * v.n8 / 2; i += 32) reinterpret_cast<uint32_t *>(v.np)[i] = 0u;
    for (int T = lane; T < m; T += 32) {
        tst[T] = -1;
        ten[T] = -1;
    }
    __syncwarp();

}

// No datum frees a task on GPU k (cold: out of line).  3inputs (PAPER.md:
// 1823-1834, R6, R24): D2 = argmax (n2_k(D), u(D), -D), then the lowest-id
// unallocated task of D2's segment whose other input is missing too; else
// Alg. 5 l.13 (R5): the lowest-id unallocated task.  Returns {T, D(T)
// ascending, bit 0: a 3inputs datum was found, bit 1: lowest-id pick}.
__device__ __noinline__ int4 fallback_pick(const WV v, int k, bool fb2, bool any_avail, int avail_lo,
                                           const int64_t *rp, const int32_t *rd, int lane) {
    int T = -1, ra = -1, rb = -1, how = 0;
    if (fb2) {
        const int D2 = argmax_score(v, k, true, lane);
        if (D2 >= 0) {
            const int b = v.dp[D2], e = v.dp[D2 + 1];
            for (int base = b; base < e && T < 0; base += 32) {
                const int i = base + lane;
                bool hit = false;
                uint32_t ed = 0;
                if (i < e) {
                    ed = v.wedge[i];
                    const int Tq = (int)(ed >> 16), o = (int)(ed & 0xFFFFu);
                    hit = !((v.al[Tq >> 5] >> (Tq & 31)) & 1u) && o != (int)NOI && !res(v, k, o);
                }
                const unsigned msk = __ballot_sync(FULL, hit);
                if (msk) {
                    ed = __shfl_sync(FULL, ed, __ffs(msk) - 1);
                    T = (int)(ed >> 16);
                    const int o = (int)(ed & 0xFFFFu);
                    ra = o < D2 ? o : D2;
                    rb = o < D2 ? D2 : o;
                }
            }
            how |= 1;
        }
    }
    if (T < 0 && any_avail) {
        const int nwd = (v.m + 31) >> 5;
        for (int w0 = avail_lo >> 5; w0 < nwd && T < 0; w0 += 32) {
            const int wd = w0 + lane;
            uint32_t fr = 0;
            if (wd < nwd) {
                fr = ~v.al[wd];
                if (wd == (avail_lo >> 5)) fr &= ~((1u << (avail_lo & 31)) - 1u);
            }
            const unsigned msk = __ballot_sync(FULL, fr != 0u);
            if (msk) {
                const int src = __ffs(msk) - 1;
                fr = __shfl_sync(FULL, fr, src);
                T = 32 * (w0 + src) + __ffs(fr) - 1;
            }
        }
        if (T >= 0) {
            raw_row(rp, rd, T, ra, rb);
            how |= 2;
        }
    }
    return make_int4(T, ra, rb, how);
}

// a8 (cold: out of line): sigma(k, .) for every k -- the stable partition of
// the service order by GPU; lane k holds the count of GPU k.
__device__ __noinline__ void assemble(const Inst *__restrict__ I, unsigned char *dsm, int lane, int nsv, int64_t ns,
                                      int K, const int32_t *sg, const int32_t *stk) {
    const unsigned lt = (1u << lane) - 1u;
    __threadfence_block();
    __syncwarp();
    {
        int x = lane < K ? nsv : 0;
        const int own = x;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const int y = __shfl_up_sync(FULL, x, o);
            if (lane >= o) x += y;
        }
        int32_t *off = reinterpret_cast<int32_t *>(dsm);  // the loop's state is dead
        __syncwarp();
        if (lane < K) {
            I->gpu_task_ptr[lane] = x - own;
            off[lane] = x - own;
        }
        if (lane == 0) I->gpu_task_ptr[K] = ns;
        __syncwarp();
        for (int64_t i0 = 0; i0 < ns; i0 += 32) {
            const int64_t i = i0 + lane;
            const int kv = i < ns ? sg[i] : -1;
            const int Tv = i < ns ? stk[i] : -1;
            const unsigned peers = __match_any_sync(FULL, kv);
            if (kv >= 0) I->gpu_task_ids[off[kv] + __popc(peers & lt)] = Tv;
            __syncwarp();
            if (kv >= 0 && lane == __ffs(peers) - 1) off[kv] += __popc(peers);
            __syncwarp();
        }
    }
}

// One instance, the whole warp.
__device__ __forceinline__ void run_instance(const Inst *__restrict__ I, unsigned char *dsm, int lane) {
    const unsigned lt = (1u << lane) - 1u;
    WV v;
    v.m = I->m;
    v.n = I->n;
    v.K = I->K;
    v.pcap = I->plan_cap;
    v.rcap = I->res_cap;
    v.kmask = v.K >= 32 ? 0xffffffffu : ((1u << v.K) - 1u);
    const WarpLayout Lw = warp_layout(v.m, v.n, v.K, v.pcap, v.rcap);
    v.n4 = Lw.n4;
    v.n8 = Lw.n8;
    v.resm = reinterpret_cast<uint32_t *>(dsm + Lw.resm);
    v.al = reinterpret_cast<uint32_t *>(dsm + Lw.al);
    v.dp = reinterpret_cast<int32_t *>(dsm + Lw.dp);
    v.u = reinterpret_cast<uint16_t *>(dsm + Lw.u);
    v.hh = reinterpret_cast<uint32_t *>(dsm + Lw.hh);
    v.np = reinterpret_cast<uint16_t *>(dsm + Lw.np);
    v.plan = reinterpret_cast<uint32_t *>(dsm + Lw.plan);
    v.rl = reinterpret_cast<int32_t *>(dsm + Lw.rl);
    uint32_t *const wedge = reinterpret_cast<uint32_t *>(const_cast<int32_t *>(I->ddat));
    v.wedge = wedge;
    const uint64_t size0 = I->size0, cap = I->cap;
    v.maxres = size0 == 0 ? INT_MAX : (int)(cap / size0 < (uint64_t)INT_MAX ? cap / size0 : (uint64_t)INT_MAX);
    const int m = v.m, n = v.n, K = v.K;
    const int64_t dtau = I->default_tau, delta0 = I->delta0, maxs = I->max_served;
    const bool fb2 = (I->flags & DTS_F_FALLBACK2) != 0;
    // pointers in registers (the descriptor is in global memory)
    int64_t *const tst = I->tstart, *const ten = I->tend;
    int32_t *const sg = I->serve_gpu, *const stk = I->serve_task;
    dts_event *const evs = I->events;
    const int64_t evcap = I->ev_cap;
    const int64_t *const taup = I->tau;
    const int64_t *const rp = I->raw_ptr;
    const int32_t *const rd = I->raw_dat;

    WP_DECL;
    [[maybe_unused]] bool chk_ = false;  // WCHK: a bounds check failed (profiling build)
    build_state(v, Lw, dsm, rp, rd, wedge, tst, ten, lane);
    // ---- per-GPU registers (lane k) and uniform scalars (every lane)
    int64_t req = 0, gfree = 0;
    int rc = 0, ph = 0, pe = 0, plive = 0, dopt = -1, nsv = 0;
    bool idle = false;
    int64_t ns = 0, bus = 0, mk = 0, nev = 0, nload = 0, nevict = 0, nscan = 0, nfb2 = 0, nfbf = 0, nidle = 0;
    int64_t sum_avail = 0, sum_deg = 0, n_alloc = 0;
    int n_avail = m, avail_lo = 0, error = 0;
    const bool uni_tau = taup == nullptr && dtau > 0 && maxs < 0;
    const double inv_tau = dtau > 0 ? 1.0 / (double)dtau : 0.0;
    // (task, GPU) item lane + 32 i of a plan's pool move: task p0 + i q32 (+ carries), GPU j0 + i r32
    const int p0 = lane / K, j0 = lane % K, q32 = 32 / K, r32 = 32 % K;
    WP(10);

    // ---- the decision loop
    while (maxs < 0 || ns < maxs) {
        const bool act = lane < K && !idle;
        const unsigned long long key = act ? (((unsigned long long)req << 5) | (unsigned)lane) : ~0ull;
        const unsigned long long kmin = wmin64(key);
        if (kmin == ~0ull) break;  // every GPU idle: no task left anywhere
        const int k = (int)(kmin & 31u);
        const int64_t t = (int64_t)(kmin >> 5);
        const int live = __shfl_sync(FULL, plive, k);
        if (live > 0) {
            // Alg. 5 l.1-2: pops.  A planned task has all inputs resident, so a
            // pop is time-model arithmetic only (R7, R8).
            if (uni_tau && __all_sync(FULL, !(act && plive > 0) || gfree <= req)) {
                // Every pop until the first request that needs a scan, S = the
                // smallest (req_j + plive_j tau, j), in ONE pass: GPU j's pops
                // come at req_j + i tau, so by (round q_j + i, req_j mod tau, j).
                const unsigned long long skey =
                    act ? ((((unsigned long long)(req + (int64_t)plive * dtau)) << 5) | (unsigned)lane) : ~0ull;
                const unsigned long long S = wmin64(skey);
                const int64_t St = (int64_t)(S >> 5);
                const int Sj = (int)(S & 31u);
                int c = 0;
                int64_t q = 0, rho = 0;
                if (act && plive > 0) {
                    const int64_t d = St - req;
                    int64_t cnt = 0;
                    if (d >= 0) {
                        int64_t rr;
                        const int64_t qd = div_tau(d, dtau, inv_tau, rr);
                        cnt = qd + (rr != 0 ? 1 : 0) + ((rr == 0 && lane < Sj) ? 1 : 0);
                    }
                    c = (int)(cnt < plive ? cnt : plive);
                    q = div_tau(req, dtau, inv_tau, rho);
                }
                const unsigned pm = __ballot_sync(FULL, c > 0);
                const uint32_t *pl = v.plan + lane * v.pcap;
                int total;
                if ((pm & (pm - 1)) == 0) {  // one GPU pops: its own sequence
                    if (c > 0) {
                        for (int i = 0; i < c; i++) {
                            const int T = (int)(pl[ph + i] >> 16);
                            const int64_t st = req + (int64_t)i * dtau;
                            tst[T] = st;
                            ten[T] = st + dtau;
                            sg[ns + i] = lane;
                            WCHK(ns + i < m && T < m);
                            stk[ns + i] = T;
                        }
                    }
                    total = __shfl_sync(FULL, c, __ffs(pm) - 1);
                } else {
                    unsigned prec = 0;  // GPUs before this one inside a round: (rho, id)
                    for (int j = 0; j < K; j++) {
                        const int64_t rj = __shfl_sync(FULL, rho, j);
                        if (rj < rho || (rj == rho && j < lane)) prec |= 1u << j;
                    }
                    const int64_t R0 = (int64_t)wmin64(c > 0 ? (unsigned long long)q : ~0ull);
                    const int64_t R1 = (int64_t)wmax64(c > 0 ? (unsigned long long)(q + c) : 0ull);
                    int64_t at = ns;
                    for (int64_t R = R0; R < R1; R++) {
                        const bool a = c > 0 && q <= R && R < q + c;
                        const unsigned am = __ballot_sync(FULL, a);
                        if (a) {
                            const int i = (int)(R - q);
                            const int64_t pos = at + __popc(am & prec);
                            const int T = (int)(pl[ph + i] >> 16);
                            const int64_t st = req + (int64_t)i * dtau;
                            tst[T] = st;
                            ten[T] = st + dtau;
                            WCHK(pos < m && T < m);
                            sg[pos] = lane;
                            stk[pos] = T;
                        }
                        at += __popc(am);
                    }
                    total = (int)(at - ns);
                }
                if (c > 0) {
                    req += (int64_t)c * dtau;
                    gfree = req;
                    ph += c;
                    plive -= c;
                    nsv += c;
                }
                const int64_t me = (int64_t)wmax64(c > 0 ? (unsigned long long)req : 0ull);
                mk = me > mk ? me : mk;
                ns += total;
            } else {
                // sequential: GPU k pops while its requests stay first in (time, id)
                const unsigned long long k2 = wmin64(lane == k ? ~0ull : key);
                int c = 0;
                int64_t mk_l = mk;
                if (lane == k) {
                    int64_t r = req, g = gfree;
                    int h = ph;
                    const uint32_t *pl = v.plan + k * v.pcap;
                    do {
                        const int T = (int)(pl[h] >> 16);
                        const int64_t start = r > g ? r : g, end = start + tau_of(taup, T, dtau);
                        g = end;
                        tst[T] = start;
                        ten[T] = end;
                        sg[ns + c] = k;
                        stk[ns + c] = T;
                        mk_l = end > mk_l ? end : mk_l;
                        c++;
                        h++;
                        r = end;
                    } while (c < live && (maxs < 0 || ns + c < maxs) &&
                             ((((unsigned long long)r << 5) | (unsigned)k) < k2));
                    req = r;
                    gfree = g;
                    ph = h;
                    plive = live - c;
                    nsv += c;
                }
                c = __shfl_sync(FULL, c, k);
                mk = __shfl_sync(FULL, mk_l, k);
                ns += c;
            }
            WP(0);
            continue;
        }

        // ---- a scan on GPU k at time t (plannedTasks_k is empty)
        WP(0);
        const int scan_avail = n_avail;
        const int Dopt = argmax_score(v, k, false, lane);  // Alg. 5 l.4-9
        uint32_t edo[SEGR];  // first batch of Dopt's segment (plan walk, then its load)
        int ob = 0, oe = 0;
        uint32_t m2b = 0u, selb = 0u;  // plan walk: per slot, unallocated with o missing / planned
        if (Dopt >= 0) {
            ob = v.dp[Dopt];
            oe = v.dp[Dopt + 1];
            seg_load(v, ob, oe, lane, edo);
        }
        {  // np_k counts exactly the plan this scan creates (Alg. 6 l.3): clear the last one's
            const int pe_k = __shfl_sync(FULL, pe, k), dk = __shfl_sync(FULL, dopt, k);
            uint16_t *npk = v.np + k * v.n8;
            const uint32_t *pl = v.plan + k * v.pcap;
            for (int i = lane; i < pe_k; i += 32) {
                const uint32_t o = pl[i] & 0xFFFFu;
                if (o != NOI) npk[o] = 0;
            }
            if (lane == 0 && dk >= 0) npk[dk] = 0;
            __syncwarp();
        }
        WP(1);
        int T = -1, ra = -1, rb = -1;  // the task served and D(T), ascending (R10)
        if (Dopt >= 0) {
            // Alg. 5 l.10: plannedTasks_k <- the unallocated tasks of Dopt's segment
            // whose other input is resident on k, ascending id (ordered warp
            // compaction); each leaves the shared pool (R2) as it is selected:
            // allocation bit, buckets of every GPU, u(D), np_k(D) (Alg. 6 l.3;
            // the first one is popped right away, Alg. 5 l.11: its np is not added)
            uint32_t *pl = v.plan + k * v.pcap;
            uint16_t *npk = v.np + k * v.n8;
            int P = 0;
            m2b = selb = 0u;
            for (int base = ob; base < oe; base += 32 * SEGR) {
                uint32_t ed[SEGR], aw[SEGR], rw[SEGR];
                if (base == ob) {
#pragma unroll
                    for (int r = 0; r < SEGR; r++) ed[r] = edo[r];
                } else {
                    seg_load(v, base, oe, lane, ed);
                }
#pragma unroll
                for (int r = 0; r < SEGR; r++) {
                    const uint32_t w = ed[r];
                    const int Tq = (int)(w >> 16), o = (int)(w & 0xFFFFu);
                    aw[r] = w != REMOVED ? v.al[Tq >> 5] : ~0u;
                    rw[r] = (w != REMOVED && o != (int)NOI) ? v.resm[o] : ~0u;
                }
#pragma unroll
                for (int r = 0; r < SEGR; r++) {
                    const uint32_t w = ed[r];
                    const int Tq = (int)(w >> 16), o = (int)(w & 0xFFFFu);
                    const bool live = w != REMOVED && !((aw[r] >> (Tq & 31)) & 1u);
                    const bool sel = live && ((rw[r] >> k) & 1u);
                    if (base == ob) {  // for Dopt's own load (below): its tasks' classes now
                        m2b |= (uint32_t)(live && !sel) << r;
                        selb |= (uint32_t)sel << r;
                    }
                    const unsigned msk = __ballot_sync(FULL, sel);
                    if (msk == 0u) continue;
                    if (sel) {
                        const int pos = P + __popc(msk & lt);
                        WCHK(pos < v.pcap && Tq < m && (o == (int)NOI || o < n));
                        pl[pos] = w;
                        atomicOr(&v.al[Tq >> 5], 1u << (Tq & 31));
                        if (o != (int)NOI) {
                            add16(v.u, o, -1);
                            if (pos > 0) add16(npk, o, 1);
                        }
                    }
                    P += __popc(msk);
                }
            }
            if (K > 1) {
                // the planned tasks' buckets on the other GPUs j: (task, GPU) items
                // spread over the lanes (item lane + 32 i = task p, GPU j)
                __syncwarp();
                const uint32_t mD = ~v.resm[Dopt] & v.kmask;  // GPUs missing Dopt
                int p = p0, j = j0;
                for (int idx = lane; idx < P * K; idx += 32) {
                    if (j != k) {
                        const int o = (int)(pl[p] & 0xFFFFu);
                        const bool md = (mD >> j) & 1u;
                        const bool mo = o != (int)NOI && !((v.resm[o] >> j) & 1u);
                        uint32_t *hj = v.hh + j * v.n4;
                        if (md && mo) {
                            atomicAdd(&hj[Dopt], 0u - 65536u);
                            atomicAdd(&hj[o], 0u - 65536u);
                        } else if (md || mo) {
                            atomicAdd(&hj[md ? Dopt : o], 0xFFFFFFFFu);
                        }
                    }
                    p += q32;
                    j += r32;
                    if (j >= K) {
                        j -= K;
                        p++;
                    }
                }
            }
            if (lane == 0) {  // the shared parts: u(Dopt), np_k(Dopt), n_k(Dopt) (every task has
                              // Dopt as its one missing input on k)
                add16(v.u, Dopt, -P);
                if (P > 1) add16(npk, Dopt, P - 1);
                atomicAdd(&v.hh[k * v.n4 + Dopt], (unsigned)(-P));
            }
            __syncwarp();
            const uint32_t w0 = pl[0];  // Alg. 5 l.11: the plan's first task is served now
            T = (int)(w0 >> 16);
            const int o0 = (int)(w0 & 0xFFFFu);
            if (o0 == (int)NOI) {
                ra = Dopt;
            } else {
                ra = o0 < Dopt ? o0 : Dopt;
                rb = o0 < Dopt ? Dopt : o0;
            }
            if (lane == k) {
                ph = 1;
                pe = P;
                plive = P - 1;
                dopt = Dopt;
            }
            n_avail -= P;
            n_alloc += P;
            nscan++;
            sum_avail += scan_avail;
            __syncwarp();
            WP(2);
        } else {
            if (lane == k) {
                ph = pe = plive = 0;
                dopt = -1;
            }
            // 3inputs (R6, R24), else Alg. 5 l.13 (R5)
            const int4 f = fallback_pick(v, k, fb2, n_avail > 0, avail_lo, rp, rd, lane);
            T = f.x;
            ra = f.y;
            rb = f.z;
            if (fb2) {
            }
            if (f.w & 1) nfb2++;
            if (f.w & 2) {
                nfbf++;
                avail_lo = T;
            }
            if (T < 0) {
                if (lane == k) idle = true;
                nidle++;
                WP(4);
                continue;
            }
            // T leaves the shared pool (no plan: np untouched)
            if (lane == 0) {
                atomicOr(&v.al[T >> 5], 1u << (T & 31));
                if (ra >= 0) add16(v.u, ra, -1);
                if (rb >= 0) add16(v.u, rb, -1);
                pool_buckets(v, ra, rb, -1, 0u);
            }
            n_avail--;
            n_alloc++;
            nscan++;
            sum_avail += scan_avail;
            __syncwarp();
            WP(4);
        }

        // ---- serve T on GPU k at t with its loads: evict V(k,i), load D(T) \ R_k in
        //      ascending id (R10), process; FIFO bus (R9)
        int rck = __shfl_sync(FULL, rc, k);
        const int phk = __shfl_sync(FULL, ph, k);
        int pek = __shfl_sync(FULL, pe, k);
        const int dk = __shfl_sync(FULL, dopt, k);
        int64_t ready = t;
        int vlast = -1, nvict = 0;  // victims of this serve
        for (int qd = 0; qd < 2 && !error; qd++) {
            const int D = qd == 0 ? ra : rb;
            if (D < 0 || res(v, k, D)) continue;
            while (rck >= v.maxres) {  // R11: LUF until D fits
                // Alg. 6: among resident data not used by taskBuffer_k = {T} (W = 0),
                // the fewest uses in plannedTasks_k, lowest id on ties (R1)
                const int32_t *rlk = v.rl + k * v.rcap;
                const uint16_t *npk = v.np + k * v.n8;
                uint32_t best = 0xFFFFFFFFu;  // np_k(D) << 16 | D (both < 2^16)
                int bslot = -1;
                for (int i = lane; i < rck; i += 32) {
                    const int Dv = rlk[i];
                    const uint32_t kk = ((uint32_t)npk[Dv] << 16) | (uint32_t)Dv;
                    const bool take = Dv != ra && Dv != rb && kk < best;
                    best = take ? kk : best;
                    bslot = take ? i : bslot;
                }
                const uint32_t mine = best;
                best = __reduce_min_sync(FULL, best);
                if (best == 0xFFFFFFFFu) {
                    error = 1;
                    break;
                }
                const int V = (int)(best & 0xFFFFu);
                uint32_t edv[SEGR];  // V's segment, fetched while the plan is updated
                const int vb = v.dp[V], ve = v.dp[V + 1];
                seg_load(v, vb, ve, lane, edv);
                const int vslot = __shfl_sync(FULL, bslot, __ffs(__ballot_sync(FULL, mine == best)) - 1);
                WP(5);
                // Alg. 6 l.8: planned tasks of k that use V return to the pool (R4)
                uint32_t *pl = v.plan + k * v.pcap;
                int nret = 0;
                unsigned tmin = 0xffffffffu;
                for (int i = phk + lane; i < pek; i += 32) {
                    const uint32_t w = pl[i];
                    const int Tq = (int)(w >> 16), o = (int)(w & 0xFFFFu);
                    if (o == V || dk == V) {
                        pl[i] = REMOVED;
                        const int a = o == (int)NOI ? dk : (o < dk ? o : dk);
                        const int bb = o == (int)NOI ? -1 : (o < dk ? dk : o);
                        atomicAnd(&v.al[Tq >> 5], ~(1u << (Tq & 31)));
                        pool_buckets(v, a, bb, +1, 0u);
                        add16(v.u, a, 1);
                        add16(v.np + k * v.n8, a, -1);
                        if (bb >= 0) {
                            add16(v.u, bb, 1);
                            add16(v.np + k * v.n8, bb, -1);
                        }
                        nret++;
                        tmin = (unsigned)Tq < tmin ? (unsigned)Tq : tmin;
                    }
                }
                nret = wsum(nret);
                if (nret > 0) {
                    tmin = __reduce_min_sync(FULL, tmin);
                    n_avail += nret;
                    if ((int)tmin < avail_lo) avail_lo = (int)tmin;
                    if (lane == k) plive -= nret;
                    if (idle) {  // R18 (provably never: DESIGN.md)
                        idle = false;
                        req = t;
                    }
                }
                // l.9: V leaves GPU k's memory
                if (lane == 0) {
                    int32_t *rlw = v.rl + k * v.rcap;
                    WCHK(vslot >= 0 && vslot < rck && rck <= v.rcap && V < n);
                    rlw[vslot] = rlw[rck - 1];
                    v.resm[V] &= ~(1u << k);
                }
                rck--;
                nevict++;
                push_event(evs, evcap, nev, lane, 1, k, V, T, t, t);
                const int degv = ve - vb;
                sum_deg += degv;
                __syncwarp();
                if (nret > 0) {  // close the holes: live entries contiguous from ph
                    int out = phk;
                    for (int c0 = phk; c0 < pek; c0 += 32) {
                        const int i = c0 + lane;
                        const uint32_t w = i < pek ? pl[i] : REMOVED;
                        const bool keep = w != REMOVED;
                        const unsigned msk = __ballot_sync(FULL, keep);
                        __syncwarp();
                        if (keep) pl[out + __popc(msk & lt)] = w;
                        out += __popc(msk);
                        __syncwarp();
                    }
                    pek = out;
                    if (lane == k) pe = out;
                }
                WP(6);
                vlast = V;
                nvict++;
                seg_update(v, k, V, false, lane, edv);
                WP(7);
            }
            if (error) break;
            // load D
            if (lane == 0) {
                WCHK(rck < v.rcap && D < n);
                v.rl[k * v.rcap + rck] = D;
                v.resm[D] |= 1u << k;
            }
            rck++;
            const int64_t st = bus > t ? bus : t;
            const int64_t en = st + delta0;
            bus = en;
            ready = en > ready ? en : ready;
            nload++;
            push_event(evs, evcap, nev, lane, 0, k, D, T, st, en);
            const int db = v.dp[D], de = v.dp[D + 1];
            sum_deg += de - db;
            __syncwarp();
            if (D == Dopt && de - db <= 32 * SEGR && nvict <= 1) {
                // Dopt's load in the plan path: after the plan, the unallocated tasks
                // of its segment are those the plan walk saw unallocated with their
                // other input o missing, plus planned ones LUF returned (o = V):
                // all go 2 -> 1 (freed by o); none is left with o resident
                uint32_t *hk = v.hh + k * v.n4;
                int n2 = 0;
#pragma unroll
                for (int r = 0; r < SEGR; r++) {
                    const int o = (int)(edo[r] & 0xFFFFu);
                    const bool upd = ((m2b >> r) & 1u) || (((selb >> r) & 1u) && o == vlast);
                    n2 += (int)upd;
                    if (upd) atomicAdd(&hk[o], 1u - 65536u);
                }
                n2 = wsum(n2);
                if (lane == 0 && n2) atomicAdd(&hk[D], 0u - ((uint32_t)n2 << 16));
                __syncwarp();
            } else {
                uint32_t edd[SEGR];
                if (D == Dopt) {
#pragma unroll
                    for (int r = 0; r < SEGR; r++) edd[r] = edo[r];
                } else {
                    seg_load(v, db, de, lane, edd);
                }
                seg_update(v, k, D, true, lane, edd);
            }
            WP(8);
        }
        if (error) break;
        // process T (time model, R7): k asks again when T ends
        {
            const int64_t gf = __shfl_sync(FULL, gfree, k);
            const int64_t start = ready > gf ? ready : gf, end = start + tau_of(taup, T, dtau);
            if (lane == k) {
                gfree = end;
                req = end;
                rc = rck;
                nsv++;
            }
            if (lane == 0) {
                tst[T] = start;
                ten[T] = end;
                sg[ns] = k;
                WCHK(ns < m && T >= 0 && T < m);
                stk[ns] = T;
            }
            mk = end > mk ? end : mk;
            ns++;
        }
        WP(9);
    }

    // ---- a8: sigma(k, .) -- stable partition of the service order by GPU
    assemble(I, dsm, lane, nsv, ns, K, sg, stk);
#ifdef DTS_PROF
    const bool bad_ = __any_sync(FULL, chk_);
#else
    (void)chk_;
    (void)n;
#endif
    if (lane == 0) {
        Out *o = I->out;
        o->n_events = nev;
        o->n_served = ns;
        o->n_loads = nload;
        o->n_evictions = nevict;
        o->n_scans = nscan;
        o->n_fallback2 = nfb2;
        o->n_fallback_first = nfbf;
        o->n_belady = 0;
        o->n_idle = nidle;
        o->n_verify_err = 0;
        o->bytes_loaded = (uint64_t)nload * size0;
        o->makespan = mk;
        o->alg_bytes = 0;  // the CTA loop's own byte model; not kept by this loop
        o->scan_alg_bytes = 0;
        o->sum_avail = sum_avail;
        o->n_alloc = n_alloc;
        o->sum_deg = sum_deg;
        o->error = error;
#ifdef DTS_PROF
        if (bad_) o->error = 9;
#endif
        WP(11);
        for (int i = 0; i < 16; i++) o->prof[i] = WP_OUT(i);
    }
    __syncwarp();
}

}  // namespace

// One warp per CTA; each CTA pulls instances from *work_counter.
__global__ void __launch_bounds__(32, 1) dts_warp_kernel(const Inst *__restrict__ insts, int n_inst,
                                                     int *work_counter) {
    extern __shared__ __align__(16) unsigned char dsm[];
    const int lane = threadIdx.x;
    while (true) {
        int ii = 0;
        if (lane == 0) ii = atomicAdd(work_counter, 1);
        ii = __shfl_sync(FULL, ii, 0);
        if (ii >= n_inst) break;
        run_instance(&insts[ii], dsm, lane);
    }
}

// The kernel's dynamic shared-memory limit, raised per device (the attribute
// belongs to the current device's context) and only ever upwards; host
// threads may launch concurrently.
static cudaError_t warp_smem_attr(int smem_bytes) {
    static std::mutex mu;
    static int cur[64] = {0};
    int dev = 0;
    cudaGetDevice(&dev);
    if (dev < 0 || dev >= 64) dev = 0;
    std::lock_guard<std::mutex> lock(mu);
    if (smem_bytes <= 48 * 1024 || smem_bytes <= cur[dev]) return cudaSuccess;
    const cudaError_t e =
        cudaFuncSetAttribute(dts_warp_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem_bytes);
    if (e == cudaSuccess) cur[dev] = smem_bytes;
    return e;
}

cudaError_t launch_warp(const Inst *d_insts, int n_inst, int grid, int *work_counter, int smem_bytes,
                        cudaStream_t st) {
    const cudaError_t e = warp_smem_attr(smem_bytes);
    if (e != cudaSuccess) return e;
    count_launch();
    dts_warp_kernel<<<grid, 32, smem_bytes, st>>>(d_insts, n_inst, work_counter);
    return cudaGetLastError();
}

int warp_max_blocks_per_sm(int smem_bytes) {
    int nb = 0;
    if (warp_smem_attr(smem_bytes) != cudaSuccess) return 1;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, dts_warp_kernel, 32, smem_bytes) != cudaSuccess) return 1;
    return nb;
}

}  // namespace dts

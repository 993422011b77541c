// dts_loop.cu -- the device-resident DARTS+LUF decision loop (§8(a) a2-a8).
//
// One launch runs a whole schedule.  A "group" of G CTAs cooperates on one
// instance (G = 1 for small instances and for the batched sweep, G = #SMs for
// the 1M-task configs).  Warp 0 of the group's CTA 0 -- the LEADER -- owns the
// sequential part of the method (event order, plannedTasks pops, LUF, loads,
// evictions, the bus/time model, the trace).  When a request finds
// plannedTasks_k empty (Alg. 5 l.3), the leader hands one data-parallel pass to
// the whole group:
//
//   SCAN(k)  : for every task T, if (s_k[T] >> 24) == 1 then hist[x_k(T)] += 1
//              -- n_k(D) of Alg. 5 l.4-5 for every D at once
//   FSCAN(k) : tasks with two missing inputs add 1 to both (3inputs,
//              PAPER.md:1823-1834) + the lowest unallocated id (Alg. 5 l.13)
//   ARGMAX   : each CTA reduces its slice of D to the packed key
//              (score, u(D), ~D) -- ties -> more unprocessed uses, then lower
//              id (Alg. 5 l.6-9, R1/R23) -- and one atomicMax per CTA.
//
// Group barriers: __syncthreads when G == 1, else a sense-reversing barrier on
// a global counter (the launch is cooperative, so all G CTAs are resident).
#include <cuda_runtime.h>

#include <climits>
#include <cstdint>

#include "dts_internal.cuh"
#include "dts_loop.cuh"

namespace dts {

namespace {

constexpr unsigned FULL = 0xffffffffu;

struct LState {  // leader-only state, in CTA 0's shared memory
    int64_t req[MAX_K];
    int64_t gpu_free[MAX_K];
    uint64_t used[MAX_K];
    int32_t plan_head[MAX_K], plan_end[MAX_K], plan_live[MAX_K];
    int32_t res_cnt[MAX_K];
    int32_t last_task[MAX_K];
    int32_t idle[MAX_K];
    int64_t bus_free;
    int64_t n_events, n_served, n_loads, n_evictions, n_scans, n_fb2, n_fbf, n_belady, n_idle;
    uint64_t bytes_loaded;
    int64_t makespan;
    uint64_t alg_bytes, scan_alg_bytes;
    int32_t n_avail;
    int32_t pending;  // CMD_SCAN / CMD_FSCAN awaiting its result, or CMD_NONE
    int32_t pend_k;
    int64_t pend_t;
    int32_t row[MAX_ROW + 1];  // D(T) of the task being served
    int32_t row_len;
    int32_t error;
};

__device__ __forceinline__ int ldcg_i32(const int32_t *p) { return __ldcg(p); }
__device__ __forceinline__ uint32_t ldcg_u32(const uint32_t *p) { return __ldcg(p); }

__device__ __forceinline__ unsigned long long ld_volatile_u64(const unsigned long long *p) {
    return *(const volatile unsigned long long *)p;
}

// ------------------------------------------------------------ group barrier
__device__ __forceinline__ void group_sync(Ctrl *c, int G) {
    __syncthreads();
    if (G > 1) {
        if (threadIdx.x == 0) {
            volatile unsigned *vgen = &c->bar_gen;
            unsigned gen = *vgen;
            __threadfence();
            unsigned arrived = atomicAdd(&c->bar_count, 1u);
            if (arrived == (unsigned)G - 1) {
                c->bar_count = 0;
                __threadfence();
                atomicAdd(&c->bar_gen, 1u);
            } else {
                while (*vgen == gen) __nanosleep(32);
            }
            __threadfence();
        }
        __syncthreads();
    }
}

// ------------------------------------------------------------ warp helpers
__device__ __forceinline__ int warp_sum(int v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(FULL, v, o);
    return v;
}
__device__ __forceinline__ unsigned long long warp_min_u64(unsigned long long v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        unsigned long long t = __shfl_xor_sync(FULL, v, o);
        v = t < v ? t : v;
    }
    return v;
}
__device__ __forceinline__ unsigned long long warp_max_u64(unsigned long long v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        unsigned long long t = __shfl_xor_sync(FULL, v, o);
        v = t > v ? t : v;
    }
    return v;
}
__device__ __forceinline__ int warp_min_i32(int v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v = min(v, __shfl_xor_sync(FULL, v, o));
    return v;
}

__device__ __forceinline__ bool row_contains(const Inst &I, int32_t T, int32_t D) {
    int64_t b = __ldg(&I.tptr[T]), e = __ldg(&I.tptr[T + 1]);
    for (int64_t i = b; i < e; i++)
        if (__ldg(&I.tdat[i]) == D) return true;
    return false;
}

__device__ __forceinline__ int64_t tau_of(const Inst &I, int32_t T) {
    return I.tau ? __ldg(&I.tau[T]) : I.default_tau;
}

// a2: residency update of GPU k's packed state along D's data->task segment.
// load: cnt -= 1, x ^= D ; evict: cnt += 1, x ^= D.  Each task appears once in
// the segment, so plain read-modify-write (no atomics) is race-free.
__device__ void seg_update(const Inst &I, int k, int32_t D, bool load, int lane) {
    const int64_t b = __ldg(&I.dptr[D]), e = __ldg(&I.dptr[D + 1]);
    uint32_t *sk = I.s + (size_t)k * I.m_pad;
    for (int64_t i = b + lane; i < e; i += 128) {
        int32_t T[4];
        uint32_t w[4];
#pragma unroll
        for (int j = 0; j < 4; j++) {
            int64_t ii = i + 32 * j;
            T[j] = ii < e ? __ldg(&I.ddat[ii]) : -1;
        }
#pragma unroll
        for (int j = 0; j < 4; j++) w[j] = T[j] >= 0 ? ldcg_u32(&sk[T[j]]) : 0u;
#pragma unroll
        for (int j = 0; j < 4; j++)
            if (T[j] >= 0) sk[T[j]] = (load ? (w[j] - CNT_ONE) : (w[j] + CNT_ONE)) ^ (uint32_t)D;
    }
}

// Mark T allocated (it leaves the shared pool, R2): ALLOC bit in all K state
// copies, u(D) -= 1 for its inputs, np_k(D) += 1 if it enters plannedTasks_k.
// Called by ONE lane per task.
__device__ void allocate_task(const Inst &I, int k, int32_t T, bool planned) {
    for (int j = 0; j < I.K; j++) {
        uint32_t *p = I.s + (size_t)j * I.m_pad + T;
        *p = ldcg_u32(p) | ALLOC_BIT;
    }
    int64_t b = __ldg(&I.tptr[T]), e = __ldg(&I.tptr[T + 1]);
    for (int64_t i = b; i < e; i++) {
        int32_t D = __ldg(&I.tdat[i]);
        atomicSub(&I.u[D], 1);
        if (planned) atomicAdd(&I.np[(size_t)k * I.n + D], 1);
    }
}

// Inverse of allocate_task for a planned task removed by LUF (Alg. 6 l.8, R4).
__device__ void unallocate_task(const Inst &I, int k, int32_t T) {
    for (int j = 0; j < I.K; j++) {
        uint32_t *p = I.s + (size_t)j * I.m_pad + T;
        *p = ldcg_u32(p) & ~ALLOC_BIT;
    }
    int64_t b = __ldg(&I.tptr[T]), e = __ldg(&I.tptr[T + 1]);
    for (int64_t i = b; i < e; i++) {
        int32_t D = __ldg(&I.tdat[i]);
        atomicAdd(&I.u[D], 1);
        atomicSub(&I.np[(size_t)k * I.n + D], 1);
    }
}

__device__ __forceinline__ void push_event(const Inst &I, LState &L, uint8_t op, int k, int32_t D,
                                           int32_t T, int64_t t, int64_t te) {
    int64_t i = L.n_events;
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

// ------------------------------------------------------------ LUF (Alg. 6)
// Among the data in GPU k's memory not used by the taskBuffer (nb(D) = 0,
// l.4-5), the one with the fewest uses in plannedTasks_k (np), lowest id on ties.
__device__ int32_t luf_victim(const Inst &I, LState &L, int k, int lane) {
    const int cnt = L.res_cnt[k];
    const int32_t *rl = I.res_list + (size_t)k * I.res_cap;
    unsigned long long best = ~0ull;
    for (int i = lane; i < cnt; i += 32) {
        int32_t D = ldcg_i32(&rl[i]);
        bool in_buf = false;
        for (int r = 0; r < L.row_len; r++) in_buf |= (L.row[r] == D);
        if (in_buf) continue;  // nb(D) > 0
        unsigned long long key =
            ((unsigned long long)(uint32_t)ldcg_i32(&I.np[(size_t)k * I.n + D]) << 32) | (uint32_t)D;
        best = key < best ? key : best;
    }
    best = warp_min_u64(best);
    if (best == ~0ull) return -1;  // Belady branch (l.7): unreachable with the capacity check
    return (int32_t)(best & 0xffffffffu);
}

__device__ void evict(const Inst &I, LState &L, int k, int32_t V, int32_t Tserved, int64_t t,
                      int lane) {
    // Alg. 6 l.8: planned tasks that use V return to the shared pool (R4)
    int nret = 0;
    int32_t *pl = I.planned + (size_t)k * I.plan_cap;
    for (int i = L.plan_head[k] + lane; i < L.plan_end[k]; i += 32) {
        int32_t T2 = ldcg_i32(&pl[i]);
        if (T2 >= 0 && row_contains(I, T2, V)) {
            pl[i] = -1;
            unallocate_task(I, k, T2);
            nret++;
        }
    }
    nret = warp_sum(nret);
    // l.9: evict V
    if (lane == 0) {
        if (nret > 0) {
            L.plan_live[k] -= nret;
            L.n_avail += nret;
            for (int j = 0; j < I.K; j++)  // wake idle GPUs (R18)
                if (L.idle[j]) {
                    L.idle[j] = 0;
                    L.req[j] = t;
                }
        }
        int32_t *rl = I.res_list + (size_t)k * I.res_cap;
        int32_t *rp = I.res_pos + (size_t)k * I.n;
        int p = rp[V];
        int last = L.res_cnt[k] - 1;
        int32_t Dl = rl[last];
        rl[p] = Dl;
        rp[Dl] = p;
        rp[V] = -1;
        L.res_cnt[k] = last;
        L.used[k] -= __ldg(&I.size[V]);
        L.n_evictions++;
        push_event(I, L, 1, k, V, Tserved, t, t);
        int64_t deg = __ldg(&I.dptr[V + 1]) - __ldg(&I.dptr[V]);
        L.alg_bytes += 12ull * (uint64_t)deg + 16ull * (uint64_t)nret * (uint64_t)I.K;
    }
    __syncwarp();
    seg_update(I, k, V, false, lane);
    __syncwarp();
}

// Serve T on GPU k at request time t: evict V(k,i), load the missing inputs in
// ascending id (R10), process; shared FIFO bus (R9).
__device__ void serve(const Inst &I, LState &L, int k, int32_t T, int64_t t, int lane) {
    const int64_t b = __ldg(&I.tptr[T]), e = __ldg(&I.tptr[T + 1]);
    const int len = (int)(e - b);
    for (int r = lane; r < len; r += 32) L.row[r] = __ldg(&I.tdat[b + r]);
    if (lane == 0) L.row_len = len;
    __syncwarp();
    int64_t ready = t;
    const int32_t *rp = I.res_pos + (size_t)k * I.n;
    for (int r = 0; r < len; r++) {
        const int32_t D = L.row[r];
        if (ldcg_i32(&rp[D]) >= 0) continue;  // resident
        const uint64_t sz = __ldg(&I.size[D]);
        while (L.used[k] + sz > I.cap) {  // R11: repeat LUF until D fits
            int32_t V = luf_victim(I, L, k, lane);
            if (V < 0) {
                if (lane == 0) L.error = 1;
                __syncwarp();
                return;
            }
            evict(I, L, k, V, T, t, lane);
        }
        if (lane == 0) {
            int32_t *rl = I.res_list + (size_t)k * I.res_cap;
            int c = L.res_cnt[k];
            rl[c] = D;
            I.res_pos[(size_t)k * I.n + D] = c;
            L.res_cnt[k] = c + 1;
            L.used[k] += sz;
            int64_t st = L.bus_free > t ? L.bus_free : t;
            int64_t en = st + __ldg(&I.delta[D]);
            L.bus_free = en;
            L.n_loads++;
            L.bytes_loaded += sz;
            push_event(I, L, 0, k, D, T, st, en);
            int64_t deg = __ldg(&I.dptr[D + 1]) - __ldg(&I.dptr[D]);
            L.alg_bytes += 12ull * (uint64_t)deg;
        }
        __syncwarp();
        ready = max(ready, L.bus_free);  // this load's end == bus_free now
        seg_update(I, k, D, true, lane);
        __syncwarp();
    }
    if (lane == 0) {
        int64_t start = ready > L.gpu_free[k] ? ready : L.gpu_free[k];
        int64_t end = start + tau_of(I, T);
        L.gpu_free[k] = end;
        I.tstart[T] = start;
        I.tend[T] = end;
        if (end > L.makespan) L.makespan = end;
        I.serve_gpu[L.n_served] = k;
        I.serve_task[L.n_served] = T;
        L.n_served++;
        L.last_task[k] = T;
        L.req[k] = (I.W == 0) ? end : start;  // R7
    }
    __syncwarp();
}

// Pop the smallest planned task of GPU k (Alg. 5 l.2 / l.11, R3).
__device__ int32_t pop_planned(const Inst &I, LState &L, int k, int lane) {
    const int32_t *pl = I.planned + (size_t)k * I.plan_cap;
    int h = L.plan_head[k];
    int32_t T = -1;
    while (true) {  // skip entries removed by LUF, 32 at a time
        int i = h + lane;
        int32_t v = i < L.plan_end[k] ? ldcg_i32(&pl[i]) : -1;
        unsigned msk = __ballot_sync(FULL, v >= 0);
        if (msk) {
            int f = __ffs(msk) - 1;
            T = __shfl_sync(FULL, v, f);
            h += f + 1;
            break;
        }
        h += 32;
    }
    // it leaves plannedTasks_k: np_k(D) -= 1 for its inputs
    int64_t b = __ldg(&I.tptr[T]), e = __ldg(&I.tptr[T + 1]);
    for (int64_t i = b + lane; i < e; i += 32) atomicSub(&I.np[(size_t)k * I.n + __ldg(&I.tdat[i])], 1);
    __syncwarp();
    if (lane == 0) {
        L.plan_head[k] = h;
        L.plan_live[k]--;
    }
    __syncwarp();
    return T;
}

// Alg. 5 l.10: plannedTasks_k <- unallocated tasks depending only on Dopt and
// data in memory = tasks of Dopt's segment with (s_k >> 24) == 1, in
// ascending id (ordered warp compaction).
__device__ void plan(const Inst &I, LState &L, int k, int32_t Dopt, int lane) {
    const int64_t b = __ldg(&I.dptr[Dopt]), e = __ldg(&I.dptr[Dopt + 1]);
    const uint32_t *sk = I.s + (size_t)k * I.m_pad;
    int32_t *pl = I.planned + (size_t)k * I.plan_cap;
    const unsigned lt = (1u << lane) - 1u;
    int w = 0;
    for (int64_t base = b; base < e; base += 32) {
        int64_t i = base + lane;
        int32_t T = -1;
        bool sel = false;
        if (i < e) {
            T = __ldg(&I.ddat[i]);
            sel = (ldcg_u32(&sk[T]) >> 24) == 1u;
        }
        unsigned msk = __ballot_sync(FULL, sel);
        if (sel) {
            pl[w + __popc(msk & lt)] = T;
            allocate_task(I, k, T, true);
        }
        w += __popc(msk);
    }
    __syncwarp();
    if (lane == 0) {
        L.plan_head[k] = 0;
        L.plan_end[k] = w;
        L.plan_live[k] = w;
        L.n_avail -= w;
        int64_t segl = e - b;
        L.alg_bytes += 8ull * (uint64_t)segl + (uint64_t)w * (4ull * I.K + 16ull);
    }
    __syncwarp();
}

// The leader's sequential event loop (R8).  Returns the command for the group.
__device__ int leader_run(const Inst &I, LState &L, int lane) {
    Ctrl *C = I.ctrl;
    if (L.pending == CMD_SCAN) {
        const int k = L.pend_k;
        const int64_t t = L.pend_t;
        unsigned long long key = ld_volatile_u64(&C->best_key);
        __syncwarp();
        if (lane == 0) C->best_key = 0ull;
        if (key != 0ull) {  // Alg. 5 l.7: nmax > 0
            const int32_t idmask = (int32_t)((1u << I.id_bits) - 1u);
            const int32_t Dopt = idmask - (int32_t)(key & (unsigned long long)idmask);
            plan(I, L, k, Dopt, lane);
            int32_t T = pop_planned(I, L, k, lane);
            if (lane == 0) {
                L.n_scans++;
                L.pending = CMD_NONE;
            }
            __syncwarp();
            serve(I, L, k, T, t, lane);
        } else {
            if (lane == 0) L.pending = CMD_FSCAN;
            __syncwarp();
            if (lane == 0) {
                C->cmd = CMD_FSCAN;
                C->cmd_k = k;
                L.scan_alg_bytes += 4ull * (uint64_t)L.n_avail;
                L.alg_bytes += 4ull * (uint64_t)L.n_avail + 8ull * (uint64_t)I.n;
            }
            __syncwarp();
            return CMD_FSCAN;
        }
    } else if (L.pending == CMD_FSCAN) {
        const int k = L.pend_k;
        const int64_t t = L.pend_t;
        unsigned long long key = ld_volatile_u64(&C->best_key);
        int minav = *(volatile int *)&C->min_avail;
        __syncwarp();
        if (lane == 0) {
            C->best_key = 0ull;
            C->min_avail = INT_MAX;
            L.pending = CMD_NONE;
        }
        __syncwarp();
        int32_t T = -1;
        if (key != 0ull) {  // 3inputs: lowest-id task of D2 with two missing inputs
            const int32_t idmask = (int32_t)((1u << I.id_bits) - 1u);
            const int32_t D2 = idmask - (int32_t)(key & (unsigned long long)idmask);
            const int64_t b = __ldg(&I.dptr[D2]), e = __ldg(&I.dptr[D2 + 1]);
            const uint32_t *sk = I.s + (size_t)k * I.m_pad;
            for (int64_t base = b; base < e && T < 0; base += 32) {
                int64_t i = base + lane;
                int32_t Tc = i < e ? __ldg(&I.ddat[i]) : -1;
                bool ok = Tc >= 0 && (ldcg_u32(&sk[Tc]) >> 24) == 2u;
                unsigned msk = __ballot_sync(FULL, ok);
                if (msk) T = __shfl_sync(FULL, Tc, __ffs(msk) - 1);
            }
            if (lane == 0) L.n_fb2++;
        } else if (minav != INT_MAX) {  // Alg. 5 l.13, reading R5
            T = minav;
            if (lane == 0) L.n_fbf++;
        }
        if (T >= 0) {
            if (lane == 0) {
                allocate_task(I, k, T, false);
                L.n_avail--;
                L.n_scans++;
            }
            __syncwarp();
            serve(I, L, k, T, t, lane);
        } else {
            if (lane == 0) {
                L.idle[k] = 1;
                L.n_idle++;
            }
            __syncwarp();
        }
    }
    // event loop
    while (true) {
        if (L.error) break;
        if (I.max_served >= 0 && L.n_served >= I.max_served) break;
        // next request: smallest (req_k, k) over non-idle GPUs (R8)
        int kk = -1;
        int64_t tb = 0;
        for (int j = lane; j < I.K; j += 32) {
            if (L.idle[j]) continue;
            int64_t r = L.req[j];
            if (kk < 0 || r < tb) {
                kk = j;
                tb = r;
            }
        }
        // warp argmin on (req, k)
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) {
            int ok = __shfl_xor_sync(FULL, kk, o);
            int64_t ot = __shfl_xor_sync(FULL, tb, o);
            if (ok >= 0 && (kk < 0 || ot < tb || (ot == tb && ok < kk))) {
                kk = ok;
                tb = ot;
            }
        }
        if (kk < 0) break;  // every GPU idle
        const int k = kk;
        const int64_t t = tb;
        if (L.plan_live[k] > 0) {  // Alg. 5 l.1-2
            int32_t T = pop_planned(I, L, k, lane);
            serve(I, L, k, T, t, lane);
            continue;
        }
        // Alg. 5 l.4: scan dataNotInMem_k -- needs the whole group
        if (lane == 0) {
            L.pending = CMD_SCAN;
            L.pend_k = k;
            L.pend_t = t;
            C->cmd = CMD_SCAN;
            C->cmd_k = k;
            L.scan_alg_bytes += 4ull * (uint64_t)L.n_avail + 8ull * (uint64_t)I.n;
            L.alg_bytes += 4ull * (uint64_t)L.n_avail + 8ull * (uint64_t)I.n;
        }
        __syncwarp();
        return CMD_SCAN;
    }
    if (lane == 0) C->cmd = CMD_DONE;
    __syncwarp();
    return CMD_DONE;
}

// ------------------------------------------------------------ group phases
__device__ __forceinline__ void count_one(int32_t *hist, bool smem_hist, uint32_t w) {
    if ((w >> 24) == 1u) atomicAdd(&hist[w & XOR_MASK], 1);
    (void)smem_hist;
}

// SCAN(k): n_k(D) for all D in one pass over the packed state (4 B / task).
__device__ void scan_phase(const Inst &I, int k, int32_t *hist, bool smem_hist, int cta, int G) {
    const uint4 *sv = reinterpret_cast<const uint4 *>(I.s + (size_t)k * I.m_pad);
    const int64_t nv = I.m_pad >> 2;
    const int64_t stride = (int64_t)G * blockDim.x;
    int64_t v = (int64_t)cta * blockDim.x + threadIdx.x;
    for (; v + stride < nv; v += 2 * stride) {
        uint4 a = __ldcg(&sv[v]);
        uint4 c = __ldcg(&sv[v + stride]);
        count_one(hist, smem_hist, a.x);
        count_one(hist, smem_hist, a.y);
        count_one(hist, smem_hist, a.z);
        count_one(hist, smem_hist, a.w);
        count_one(hist, smem_hist, c.x);
        count_one(hist, smem_hist, c.y);
        count_one(hist, smem_hist, c.z);
        count_one(hist, smem_hist, c.w);
    }
    if (v < nv) {
        uint4 a = __ldcg(&sv[v]);
        count_one(hist, smem_hist, a.x);
        count_one(hist, smem_hist, a.y);
        count_one(hist, smem_hist, a.z);
        count_one(hist, smem_hist, a.w);
    }
}

// FSCAN(k): n2_k(D) (tasks with exactly two missing inputs, both credited) and
// the lowest unallocated task id.
__device__ void fscan_phase(const Inst &I, int k, int32_t *hist, int cta, int G, int *sh_min) {
    const uint32_t *sk = I.s + (size_t)k * I.m_pad;
    const int32_t *rp = I.res_pos + (size_t)k * I.n;
    const bool fb2 = (I.flags & DTS_F_FALLBACK2) != 0;
    const int64_t stride = (int64_t)G * blockDim.x;
    int mn = INT_MAX;
    for (int64_t T = (int64_t)cta * blockDim.x + threadIdx.x; T < I.m; T += stride) {
        uint32_t w = __ldcg(&sk[T]);
        if (w & ALLOC_BIT) continue;
        mn = min(mn, (int)T);
        if (fb2 && (w >> 24) == 2u) {
            int64_t b = __ldg(&I.tptr[T]), e = __ldg(&I.tptr[T + 1]);
            for (int64_t i = b; i < e; i++) {
                int32_t D = __ldg(&I.tdat[i]);
                if (__ldcg(&rp[D]) < 0) atomicAdd(&hist[D], 1);
            }
        }
    }
    mn = warp_min_i32(mn);
    if ((threadIdx.x & 31) == 0 && mn != INT_MAX) atomicMin(sh_min, mn);
}

// ARGMAX over this CTA's slice of D of (score, u, ~id); resets the histogram.
__device__ void argmax_phase(const Inst &I, int32_t *hist, bool smem_hist, int cta, int G,
                             unsigned long long *sh_key) {
    const int64_t n = I.n;
    const int64_t lo = n * cta / G, hi = n * (cta + 1) / G;
    const unsigned ib = (unsigned)I.id_bits, ub = (unsigned)I.u_bits;
    const unsigned long long idmask = (1ull << ib) - 1ull;
    unsigned long long best = 0ull;
    for (int64_t D = lo + threadIdx.x; D < hi; D += blockDim.x) {
        int32_t h = smem_hist ? hist[D] : __ldcg(&hist[D]);
        if (h > 0) {
            hist[D] = 0;
            unsigned long long uu = (unsigned long long)(uint32_t)__ldcg(&I.u[D]);
            unsigned long long key = ((unsigned long long)(uint32_t)h << (ub + ib)) | (uu << ib) |
                                     (idmask - (unsigned long long)D);
            best = key > best ? key : best;
        }
    }
    best = warp_max_u64(best);
    if ((threadIdx.x & 31) == 0 && best) atomicMax(sh_key, best);
}

}  // namespace

// One group of gridDim.x / n_groups ... : when G > 1 the grid IS the group
// (n_inst == 1, cooperative launch); when G == 1 each CTA pulls instances from
// a device-side work counter (batched sweep).
__global__ void __launch_bounds__(1024, 1)
    dts_loop_kernel(const Inst *__restrict__ insts, int n_inst, int G, int *work_counter,
                    int smem_hist_cap) {
    extern __shared__ int32_t dyn_smem[];
    __shared__ LState L;
    __shared__ int sh_inst;
    __shared__ unsigned long long sh_key;
    __shared__ int sh_min;
    __shared__ int sh_cmd, sh_k;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int cta = (G > 1) ? (int)blockIdx.x : 0;

    while (true) {
        if (threadIdx.x == 0) sh_inst = (G > 1) ? (blockIdx.x == 0 ? 0 : 0) : atomicAdd(work_counter, 1);
        __syncthreads();
        const int ii = sh_inst;
        if (G == 1 && ii >= n_inst) break;
        const Inst I = insts[ii];
        Ctrl *C = I.ctrl;
        const bool smem_hist = (G == 1) && (I.n <= smem_hist_cap);
        int32_t *hist = smem_hist ? dyn_smem : I.hist;
        if (smem_hist)
            for (int D = threadIdx.x; D < I.n; D += blockDim.x) hist[D] = 0;
        const bool leader_cta = (cta == 0);
        if (leader_cta && threadIdx.x == 0) {
            for (int k = 0; k < MAX_K; k++) {
                L.req[k] = 0;
                L.gpu_free[k] = 0;
                L.used[k] = 0;
                L.plan_head[k] = L.plan_end[k] = L.plan_live[k] = 0;
                L.res_cnt[k] = 0;
                L.last_task[k] = -1;
                L.idle[k] = 0;
            }
            L.bus_free = 0;
            L.n_events = L.n_served = L.n_loads = L.n_evictions = L.n_scans = L.n_fb2 = L.n_fbf =
                L.n_belady = L.n_idle = 0;
            L.bytes_loaded = 0;
            L.makespan = 0;
            L.alg_bytes = L.scan_alg_bytes = 0;
            L.n_avail = I.m;
            L.pending = CMD_NONE;
            L.error = 0;
            L.row_len = 0;
        }
        __syncthreads();
        while (true) {
            if (leader_cta) {
                if (warp == 0) {
                    int cmd = leader_run(I, L, lane);
                    if (lane == 0) {
                        sh_cmd = cmd;
                        sh_k = L.pend_k;
                    }
                }
            }
            group_sync(C, G);
            int cmd, k;
            if (leader_cta) {
                cmd = sh_cmd;
                k = sh_k;
            } else {
                cmd = *(volatile int *)&C->cmd;
                k = *(volatile int *)&C->cmd_k;
            }
            if (cmd == CMD_DONE) break;
            if (threadIdx.x == 0) {
                sh_key = 0ull;
                sh_min = INT_MAX;
            }
            __syncthreads();
            if (cmd == CMD_SCAN)
                scan_phase(I, k, hist, smem_hist, cta, G);
            else
                fscan_phase(I, k, hist, cta, G, &sh_min);
            __syncthreads();
            if (threadIdx.x == 0 && sh_min != INT_MAX) atomicMin(&C->min_avail, sh_min);
            group_sync(C, G);
            argmax_phase(I, hist, smem_hist, cta, G, &sh_key);
            __syncthreads();
            if (threadIdx.x == 0 && sh_key) atomicMax(&C->best_key, sh_key);
            group_sync(C, G);
        }
        // write back the scalars
        if (leader_cta && threadIdx.x == 0) {
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
            o->bytes_loaded = L.bytes_loaded;
            o->makespan = L.makespan;
            o->alg_bytes = L.alg_bytes;
            o->scan_alg_bytes = L.scan_alg_bytes;
            o->error = L.error;
        }
        if (G > 1) break;
        __syncthreads();
    }
}

// ---------------------------------------------------------------- init (a2)
// s_k(T) = (|D(T)| << 24) | XOR D(T) for every k (nothing resident), pad words
// allocated; u(D) = deg(D); empty histograms / plans / residency; delta(D).
__global__ void dts_init_kernel(const Inst *__restrict__ insts, int n_inst, uint64_t bw,
                                int64_t *const *__restrict__ deltas) {
    for (int ii = 0; ii < n_inst; ii++) {
        const Inst I = insts[ii];
        int64_t *delta = deltas[ii];
        const int64_t tid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
        const int64_t str = (int64_t)gridDim.x * blockDim.x;
        for (int64_t T = tid; T < I.m_pad; T += str) {
            uint32_t w = ALLOC_BIT;
            if (T < I.m) {
                int64_t b = I.tptr[T], e = I.tptr[T + 1];
                uint32_t x = 0;
                for (int64_t i = b; i < e; i++) x ^= (uint32_t)I.tdat[i];
                w = ((uint32_t)(e - b) << 24) | x;
                I.tstart[T] = -1;
                I.tend[T] = -1;
            }
            for (int k = 0; k < I.K; k++) I.s[(size_t)k * I.m_pad + T] = w;
        }
        for (int64_t D = tid; D < I.n; D += str) {
            I.u[D] = (int32_t)(I.dptr[D + 1] - I.dptr[D]);
            I.hist[D] = 0;
            unsigned __int128 num = (unsigned __int128)I.size[D] * 1000000000ull + (bw - 1);
            delta[D] = (int64_t)(num / bw);
            for (int k = 0; k < I.K; k++) {
                I.np[(size_t)k * I.n + D] = 0;
                I.res_pos[(size_t)k * I.n + D] = -1;
            }
        }
        if (tid == 0) {
            Ctrl *c = I.ctrl;
            c->bar_count = 0;
            c->bar_gen = 0;
            c->cmd = CMD_NONE;
            c->cmd_k = 0;
            c->best_key = 0ull;
            c->min_avail = INT_MAX;
            c->error = 0;
        }
    }
}

// ---------------------------------------------------------- assembly (a8)
// sigma(k, .) for every k: stable partition of the service sequence by GPU.
__global__ void __launch_bounds__(1024) dts_assemble_kernel(const Inst *__restrict__ insts) {
    const Inst I = insts[blockIdx.x];
    __shared__ unsigned long long cnt[MAX_K];
    __shared__ long long off[MAX_K];
    __shared__ int wcount[32][MAX_K];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, nw = blockDim.x >> 5;
    const unsigned lt = (1u << lane) - 1u;
    const int64_t ns = I.out->n_served;
    for (int k = threadIdx.x; k < MAX_K; k += blockDim.x) cnt[k] = 0;
    __syncthreads();
    for (int64_t i = threadIdx.x; i < ns; i += blockDim.x) atomicAdd(&cnt[I.serve_gpu[i]], 1ull);
    __syncthreads();
    if (threadIdx.x == 0) {
        long long run = 0;
        for (int k = 0; k < I.K; k++) {
            I.gpu_task_ptr[k] = run;
            off[k] = run;
            run += cnt[k];
        }
        I.gpu_task_ptr[I.K] = run;
    }
    __syncthreads();
    for (int64_t base = 0; base < ns; base += blockDim.x) {
        for (int j = threadIdx.x; j < nw * MAX_K; j += blockDim.x) wcount[j / MAX_K][j % MAX_K] = 0;
        __syncthreads();
        const int64_t i = base + threadIdx.x;
        const int k = i < ns ? I.serve_gpu[i] : -1;
        const unsigned peers = __match_any_sync(FULL, k);
        if (k >= 0 && lane == __ffs(peers) - 1) wcount[w][k] = __popc(peers);
        __syncthreads();
        if (threadIdx.x < I.K) {
            long long run = off[threadIdx.x];
            for (int ww = 0; ww < nw; ww++) {
                int t = wcount[ww][threadIdx.x];
                wcount[ww][threadIdx.x] = (int)(run - off[threadIdx.x]);
                run += t;
            }
            cnt[threadIdx.x] = run;  // new running offset, published after the scatter
        }
        __syncthreads();
        if (k >= 0) I.gpu_task_ids[off[k] + wcount[w][k] + __popc(peers & lt)] = I.serve_task[i];
        __syncthreads();
        if (threadIdx.x < I.K) off[threadIdx.x] = cnt[threadIdx.x];
        __syncthreads();
    }
}

// ---------------------------------------------------------------- launchers
cudaError_t launch_init(const Inst *d_insts, int n_inst, uint64_t bw, int64_t *const *d_deltas,
                        int64_t work, cudaStream_t st) {
    int64_t blocks = (work + 255) / 256;
    if (blocks < 1) blocks = 1;
    if (blocks > 148 * 8) blocks = 148 * 8;
    dts_init_kernel<<<(unsigned)blocks, 256, 0, st>>>(d_insts, n_inst, bw, d_deltas);
    count_launch();
    return cudaGetLastError();
}

cudaError_t launch_loop(const Inst *d_insts, int n_inst, int G, int block, int grid,
                        int *work_counter, int smem_hist_cap, cudaStream_t st) {
    size_t dyn = (G == 1) ? sizeof(int32_t) * (size_t)smem_hist_cap : 0;
    cudaError_t e = cudaFuncSetAttribute(dts_loop_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         (int)dyn);
    if (e != cudaSuccess) return e;
    if (G > 1) {
        void *args[] = {(void *)&d_insts, (void *)&n_inst, (void *)&G, (void *)&work_counter,
                        (void *)&smem_hist_cap};
        count_launch();
        return cudaLaunchCooperativeKernel((const void *)dts_loop_kernel, dim3(G), dim3(block), args,
                                           dyn, st);
    }
    dts_loop_kernel<<<grid, block, dyn, st>>>(d_insts, n_inst, 1, work_counter, smem_hist_cap);
    count_launch();
    return cudaGetLastError();
}

cudaError_t launch_assemble(const Inst *d_insts, int n_inst, cudaStream_t st) {
    dts_assemble_kernel<<<n_inst, 1024, 0, st>>>(d_insts);
    count_launch();
    return cudaGetLastError();
}

int loop_max_blocks_per_sm(int block, int smem_hist_cap) {
    int nb = 0;
    size_t dyn = sizeof(int32_t) * (size_t)smem_hist_cap;
    cudaFuncSetAttribute(dts_loop_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)dyn);
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, dts_loop_kernel, block, dyn) != cudaSuccess)
        return 0;
    return nb;
}

}  // namespace dts

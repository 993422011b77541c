// dts_csr.cu -- §8(a) a1: build the task->data and data->task incidence of the
// bipartite graph G = (T ∪ D, E) (§III) on the device.
//
//   1. k_rows      : one thread per task; sort + de-duplicate its row (D(T) is a
//                    set) -> new row length
//   2. scan        : exclusive prefix sum of the lengths -> tptr
//   3. k_compact   : copy the rows to tdat; emit (datum, task) edge pairs in
//                    task-major order; count deg(D)
//   4. scan        : deg -> dptr
//   5. LSD radix sort of the edges by datum id (stable, 8-bit digits), which
//      keeps the task-major order inside each datum: the ddat segment of D lists
//      its tasks in ascending id (needed for the plannedTasks order, R3).
// All integer and deterministic: no order-dependent atomic reaches the output.
#include <cuda_runtime.h>

#include <cstdint>

#include "dts_csr.cuh"
#include "dts_internal.cuh"

namespace dts {

namespace {

constexpr int SCAN_T = 1024;
constexpr int SCAN_I = 4;
constexpr int SCAN_TILE = SCAN_T * SCAN_I;

__device__ __forceinline__ int64_t warp_incl_scan(int64_t v) {
    const int lane = threadIdx.x & 31;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        int64_t t = __shfl_up_sync(0xffffffffu, v, o);
        if (lane >= o) v += t;
    }
    return v;
}

// Exclusive scan of one value per thread over the block; *total = block sum.
__device__ int64_t block_excl_scan(int64_t v, int64_t *total) {
    __shared__ int64_t wsum[32];
    __shared__ int64_t wofs[32];
    __shared__ int64_t tot;
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, nw = blockDim.x >> 5;
    __syncthreads();  // protect the shared slots from a previous call
    int64_t inc = warp_incl_scan(v);
    if (lane == 31) wsum[w] = inc;
    __syncthreads();
    if (w == 0) {
        int64_t x = lane < nw ? wsum[lane] : 0;
        int64_t xi = warp_incl_scan(x);
        wofs[lane] = xi - x;
        if (lane == 31) tot = xi;
    }
    __syncthreads();
    *total = tot;
    return wofs[w] + inc - v;
}

template <typename TIn>
__global__ void k_block_sums(const TIn *__restrict__ in, int64_t L, int64_t *__restrict__ sums) {
    int64_t base = (int64_t)blockIdx.x * SCAN_TILE + (int64_t)threadIdx.x * SCAN_I;
    int64_t v = 0;
#pragma unroll
    for (int j = 0; j < SCAN_I; j++)
        if (base + j < L) v += (int64_t)in[base + j];
    int64_t tot;
    block_excl_scan(v, &tot);
    if (threadIdx.x == 0) sums[blockIdx.x] = tot;
}

// out[i] = offs[block] + exclusive prefix within the block; the last block
// also writes out[L] (the total).  offs == nullptr means a single block.
template <typename TIn>
__global__ void k_scan_tiles(const TIn *__restrict__ in, int64_t L, const int64_t *__restrict__ offs,
                             int64_t *__restrict__ out) {
    int64_t base = (int64_t)blockIdx.x * SCAN_TILE + (int64_t)threadIdx.x * SCAN_I;
    int64_t x[SCAN_I];
    int64_t v = 0;
#pragma unroll
    for (int j = 0; j < SCAN_I; j++) {
        x[j] = (base + j < L) ? (int64_t)in[base + j] : 0;
        v += x[j];
    }
    int64_t tot;
    int64_t p = block_excl_scan(v, &tot) + (offs ? offs[blockIdx.x] : 0);
#pragma unroll
    for (int j = 0; j < SCAN_I; j++) {
        if (base + j < L) out[base + j] = p;
        p += x[j];
    }
    if (blockIdx.x == gridDim.x - 1 && threadIdx.x == 0) out[L] = (offs ? offs[blockIdx.x] : 0) + tot;
}

template <typename TIn>
void scan_excl(const TIn *in, int64_t L, int64_t *out, int64_t *scratch, cudaStream_t st) {
    int64_t nb = (L + SCAN_TILE - 1) / SCAN_TILE;
    if (nb <= 1) {
        k_scan_tiles<TIn><<<1, SCAN_T, 0, st>>>(in, L, nullptr, out); count_launch();
        return;
    }
    int64_t *sums = scratch;
    int64_t *offs = scratch + nb;  // nb + 1 entries
    k_block_sums<TIn><<<(unsigned)nb, SCAN_T, 0, st>>>(in, L, sums); count_launch();
    scan_excl<int64_t>(sums, nb, offs, scratch + 2 * nb + 1, st);
    k_scan_tiles<TIn><<<(unsigned)nb, SCAN_T, 0, st>>>(in, L, offs, out); count_launch();
}

// 1. sort + de-duplicate each row in place (rows have <= MAX_ROW entries,
//    checked on the host); write the de-duplicated length.
__global__ void k_rows(const int64_t *__restrict__ raw_ptr, const int32_t *__restrict__ raw_dat,
                       int32_t m, int32_t *__restrict__ tmp, int64_t *__restrict__ nlen) {
    int32_t T = blockIdx.x * blockDim.x + threadIdx.x;
    if (T >= m) return;
    int64_t b = raw_ptr[T], e = raw_ptr[T + 1];
    int32_t L = (int32_t)(e - b);
    int32_t *row = tmp + b;
    for (int32_t i = 0; i < L; i++) {  // insertion sort (rows are tiny: <= 127)
        int32_t v = raw_dat[b + i];
        int32_t j = i;
        while (j > 0 && row[j - 1] > v) {
            row[j] = row[j - 1];
            j--;
        }
        row[j] = v;
    }
    int32_t q = 0;
    for (int32_t i = 0; i < L; i++)
        if (q == 0 || row[q - 1] != row[i]) row[q++] = row[i];
    nlen[T] = q;
}

// 3. compact rows into tdat, write the (datum, task) edges, count degrees.
//    Only the tasks of [t_lo, t_hi) enter the data->task side (a task shard,
//    §8(e); the whole range otherwise); the other edges get key n and sort
//    past dptr[n].  The task->data side always holds every row.
__global__ void k_compact(const int64_t *__restrict__ raw_ptr, const int32_t *__restrict__ tmp,
                          const int64_t *__restrict__ tptr, int32_t m, int32_t n, int32_t t_lo,
                          int32_t t_hi, int32_t *__restrict__ tdat, int32_t *__restrict__ ekey,
                          int32_t *__restrict__ eval, unsigned long long *__restrict__ deg) {
    int32_t T = blockIdx.x * blockDim.x + threadIdx.x;
    if (T >= m) return;
    const bool own = T >= t_lo && T < t_hi;
    int64_t b = raw_ptr[T], o = tptr[T], q = tptr[T + 1] - o;
    for (int64_t i = 0; i < q; i++) {
        int32_t D = tmp[b + i];
        tdat[o + i] = D;
        ekey[o + i] = own ? D : n;
        eval[o + i] = T;
        if (own) atomicAdd(&deg[D], 1ull);
    }
}

// Pad the edge slots beyond the de-duplicated count E = tptr[m] with key n so
// that they sort after every real edge.
__global__ void k_pad_tail(const int64_t *__restrict__ tptr, int32_t m, int64_t E_raw, int32_t n,
                           int32_t *__restrict__ ekey, int32_t *__restrict__ eval) {
    int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i < E_raw && i >= tptr[m]) {
        ekey[i] = n;
        eval[i] = -1;
    }
}

// 5. stable LSD radix sort pass over 8-bit digit `shift` (keys = datum ids,
//    values = task ids).  A CTA owns RX_TILE consecutive elements; each of its
//    8 warps owns 256 consecutive elements, processed 32 at a time in order.
constexpr int RX_T = 256;
constexpr int RX_W = RX_T / 32;
constexpr int RX_PER_WARP = 256;
constexpr int RX_TILE = RX_W * RX_PER_WARP;  // 2048

__global__ void k_radix_hist(const int32_t *__restrict__ keys, int64_t L, int shift,
                             int64_t *__restrict__ counts, int64_t nchunks) {
    __shared__ int32_t h[256];
    h[threadIdx.x] = 0;
    __syncthreads();
    int64_t base = (int64_t)blockIdx.x * RX_TILE;
    for (int i = threadIdx.x; i < RX_TILE; i += RX_T)
        if (base + i < L) atomicAdd(&h[(keys[base + i] >> shift) & 255], 1);
    __syncthreads();
    counts[(int64_t)threadIdx.x * nchunks + blockIdx.x] = h[threadIdx.x];
}

__global__ void k_radix_scatter(const int32_t *__restrict__ kin, const int32_t *__restrict__ vin,
                                int64_t L, int shift, const int64_t *__restrict__ offs,
                                int64_t nchunks, int32_t *__restrict__ kout,
                                int32_t *__restrict__ vout) {
    __shared__ int64_t wc[RX_W][256];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    for (int i = threadIdx.x; i < RX_W * 256; i += RX_T) wc[i / 256][i % 256] = 0;
    __syncthreads();
    const int64_t wbase = (int64_t)blockIdx.x * RX_TILE + (int64_t)w * RX_PER_WARP;
    const unsigned lt = (1u << lane) - 1u;
    // pass 1: per-warp digit counts
    for (int it = 0; it < RX_PER_WARP / 32; it++) {
        int64_t i = wbase + it * 32 + lane;
        bool ok = i < L;
        int d = ok ? ((kin[i] >> shift) & 255) : 256 + lane;
        unsigned peers = __match_any_sync(0xffffffffu, d);
        if (ok && lane == __ffs(peers) - 1) wc[w][d] += __popc(peers);
        __syncwarp();
    }
    __syncthreads();
    {  // per bin: global offset of this chunk + exclusive prefix over warps
        int b = threadIdx.x;  // RX_T == 256 bins
        int64_t run = offs[(int64_t)b * nchunks + blockIdx.x];
        for (int ww = 0; ww < RX_W; ww++) {
            int64_t t = wc[ww][b];
            wc[ww][b] = run;
            run += t;
        }
    }
    __syncthreads();
    // pass 2: stable scatter
    for (int it = 0; it < RX_PER_WARP / 32; it++) {
        int64_t i = wbase + it * 32 + lane;
        bool ok = i < L;
        int32_t key = ok ? kin[i] : 0;
        int d = ok ? ((key >> shift) & 255) : 256 + lane;
        unsigned peers = __match_any_sync(0xffffffffu, d);
        int64_t pos = 0;
        if (ok) pos = wc[w][d] + __popc(peers & lt);
        __syncwarp();
        if (ok) {
            kout[pos] = key;
            vout[pos] = vin[i];
            if (lane == __ffs(peers) - 1) wc[w][d] += __popc(peers);
        }
        __syncwarp();
    }
}

// 6. edge records: for edge i of datum D's segment, {T, T's other inputs, |D(T)|}.
__global__ void k_edges(const int64_t *__restrict__ tptr, const int32_t *__restrict__ tdat,
                        const int64_t *__restrict__ dptr, const int32_t *__restrict__ ddat, int32_t n,
                        int64_t E_raw, int4 *__restrict__ dedge) {
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= E_raw || i >= dptr[n]) return;
    int32_t lo = 0, hi = n - 1;  // D = the segment containing i: dptr[D] <= i < dptr[D+1]
    while (lo < hi) {
        const int32_t mid = (lo + hi + 1) >> 1;
        if (dptr[mid] <= i) lo = mid;
        else hi = mid - 1;
    }
    const int32_t D = lo, T = ddat[i];
    const int64_t rb = tptr[T], re = tptr[T + 1];
    int4 e;
    e.x = T;
    e.y = -1;
    e.z = -1;
    e.w = (int32_t)(re - rb);
    for (int64_t j = rb; j < re; j++) {
        const int32_t o = tdat[j];
        if (o == D) continue;
        if (e.y < 0) e.y = o;
        else if (e.z < 0) e.z = o;
    }
    dedge[i] = e;
}

}  // namespace

size_t csr_scratch_bytes(int32_t m, int32_t n, int64_t E_raw) {
    int64_t L = E_raw > m ? E_raw : m;
    if (n > L) L = n;
    int64_t nchunks = (E_raw + RX_TILE - 1) / RX_TILE + 1;
    int64_t cnt = 256 * nchunks;
    if (cnt > L) L = cnt;
    size_t b = 0;
    b += sizeof(int32_t) * (size_t)(E_raw + 4);         // tmp rows
    b += sizeof(int64_t) * (size_t)(m + 4);             // nlen
    b += sizeof(unsigned long long) * (size_t)(n + 4);  // deg
    b += sizeof(int32_t) * 4 * (size_t)(E_raw + 4);     // ekey/eval ping-pong
    b += sizeof(int64_t) * (size_t)(cnt + 4) * 2;       // radix counts + offsets
    b += sizeof(int64_t) * (size_t)(2 * (L / 2048 + 64));  // scan scratch
    return b + 16 * 64;
}

static inline char *carve(char *&p, size_t bytes) {
    char *r = p;
    p += (bytes + 63) & ~size_t(63);
    return r;
}

cudaError_t build_csr(const int64_t *raw_ptr, const int32_t *raw_dat, int32_t m, int32_t n,
                      int64_t E_raw, int64_t *tptr, int32_t *tdat, int64_t *dptr, int32_t *ddat,
                      int4 *dedge, void *scratch, cudaStream_t st, int32_t t_lo, int32_t t_hi) {
    char *p = (char *)scratch;
    int32_t *tmp = (int32_t *)carve(p, sizeof(int32_t) * (size_t)(E_raw + 4));
    int64_t *nlen = (int64_t *)carve(p, sizeof(int64_t) * (size_t)(m + 4));
    unsigned long long *deg = (unsigned long long *)carve(p, sizeof(unsigned long long) * (size_t)(n + 4));
    int32_t *k0 = (int32_t *)carve(p, sizeof(int32_t) * (size_t)(E_raw + 4));
    int32_t *v0 = (int32_t *)carve(p, sizeof(int32_t) * (size_t)(E_raw + 4));
    int32_t *k1 = (int32_t *)carve(p, sizeof(int32_t) * (size_t)(E_raw + 4));
    int32_t *v1 = (int32_t *)carve(p, sizeof(int32_t) * (size_t)(E_raw + 4));
    int64_t nchunks = (E_raw + RX_TILE - 1) / RX_TILE;
    if (nchunks < 1) nchunks = 1;
    int64_t *counts = (int64_t *)carve(p, sizeof(int64_t) * (size_t)(256 * nchunks + 4));
    int64_t *offs = (int64_t *)carve(p, sizeof(int64_t) * (size_t)(256 * nchunks + 4));
    int64_t L = E_raw > m ? E_raw : m;
    if (n > L) L = n;
    if (256 * nchunks > L) L = 256 * nchunks;
    int64_t *sscr = (int64_t *)carve(p, sizeof(int64_t) * (size_t)(2 * (L / 2048 + 64)));

    cudaMemsetAsync(deg, 0, sizeof(unsigned long long) * (size_t)(n + 1), st);
    if (m > 0) {
        k_rows<<<(m + 255) / 256, 256, 0, st>>>(raw_ptr, raw_dat, m, tmp, nlen);
        count_launch();
    }
    scan_excl<int64_t>(nlen, m, tptr, sscr, st);
    if (m > 0) {
        k_compact<<<(m + 255) / 256, 256, 0, st>>>(raw_ptr, tmp, tptr, m, n, t_lo, t_hi, tdat, k0, v0, deg);
        count_launch();
    }
    scan_excl<unsigned long long>(deg, n, dptr, sscr, st);
    // The de-duplicated edge count E = tptr[m] <= E_raw is only known on the
    // device: sort all E_raw slots with the tail padded by key n (sorts last).
    if (E_raw > 0) {
        k_pad_tail<<<(unsigned)((E_raw + 255) / 256), 256, 0, st>>>(tptr, m, E_raw, n, k0, v0);
        count_launch();
    }
    int bits = 1;
    while ((1ll << bits) <= (long long)n) bits++;  // ids in [0, n] (n = pad key)
    int passes = (bits + 7) / 8;
    int32_t *ki = k0, *vi = v0, *ko = k1, *vo = v1;
    for (int ps = 0; ps < passes; ps++) {
        int shift = 8 * ps;
        if (E_raw > 0) {
            k_radix_hist<<<(unsigned)nchunks, RX_T, 0, st>>>(ki, E_raw, shift, counts, nchunks); count_launch();
            scan_excl<int64_t>(counts, 256 * nchunks, offs, sscr, st);
            k_radix_scatter<<<(unsigned)nchunks, RX_T, 0, st>>>(ki, vi, E_raw, shift, offs, nchunks, ko,
                                                               vo); count_launch();
        }
        int32_t *t;
        t = ki; ki = ko; ko = t;
        t = vi; vi = vo; vo = t;
    }
    if (E_raw > 0) cudaMemcpyAsync(ddat, vi, sizeof(int32_t) * (size_t)E_raw, cudaMemcpyDeviceToDevice, st);
    if (E_raw > 0 && dedge) {
        k_edges<<<(unsigned)((E_raw + 255) / 256), 256, 0, st>>>(tptr, tdat, dptr, ddat, n, E_raw, dedge);
        count_launch();
    }
    return cudaGetLastError();
}

}  // namespace dts

// dts_api.cu -- the C ABI of libdts (include/dts.h): validation, device memory,
// stream orchestration and result transfer.  Host code never computes any part
// of the schedule: it validates and copies inputs, launches the kernels of
// dts_csr.cu / dts_loop.cu, and copies results back.
#include <cuda_runtime.h>

#include <algorithm>
#include <atomic>
#include <climits>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <new>
#include <string>
#include <memory>
#include <mutex>
#include <vector>

#include "dts.h"
#include "dts_csr.cuh"
#include "dts_internal.cuh"
#include "dts_loop.cuh"

namespace {

thread_local std::string g_err;

dts_status fail(dts_status s, const std::string &msg) {
    g_err = msg;
    return s;
}

dts_status cuda_fail(cudaError_t e, const char *where) {
    g_err = std::string(where) + ": " + cudaGetErrorString(e);
    return DTS_E_CUDA;
}

#define CK(expr, where)                          \
    do {                                         \
        cudaError_t _e = (expr);                 \
        if (_e != cudaSuccess) return cuda_fail(_e, where); \
    } while (0)

int bits_for(uint64_t v) {  // bits needed to represent v (>= 1)
    int b = 1;
    while (b < 64 && (v >> b) != 0) b++;
    return b;
}

struct Arena {
    char *base = nullptr;
    size_t size = 0;
    size_t used = 0;
    template <typename T>
    T *take(size_t count) {
        size_t bytes = (sizeof(T) * count + 255) & ~size_t(255);
        T *p = reinterpret_cast<T *>(base + used);
        used += bytes;
        return p;
    }
};

}  // namespace

// ---------------------------------------------------------------- allocator
// Caching allocator for instance memory (device arenas, pinned host buffers).
// cudaMalloc / cudaMallocHost / cudaFree cost milliseconds (cudaFree also
// synchronises the device), so creating and destroying instances per request
// -- the public API's end-to-end path -- would be dominated by them.  A freed
// block goes to a per-process pool with an event recorded on the stream of
// its instance's last work; a later allocation takes the smallest pooled block
// of at least the size (and at most twice it, plus 1 MiB) on the same device,
// waiting for that event first.  Bounded: beyond POOL_CAP bytes per kind,
// blocks are freed.  Arenas exported through CUDA IPC are never pooled.
namespace {
struct PoolBlock {
    void *p;
    size_t bytes;
    int device;        // -1: pinned host memory
    cudaEvent_t done;  // the last work using it (nullptr: none)
};
std::mutex g_pool_mu;
std::vector<PoolBlock> g_pool;
size_t g_pool_bytes[2] = {0, 0};  // [0] device, [1] host
constexpr size_t POOL_CAP[2] = {size_t(16) << 30, size_t(4) << 30};

void *pool_take(int device, size_t bytes, size_t *got) {
    PoolBlock b{nullptr, 0, 0, nullptr};
    {
        std::lock_guard<std::mutex> lk(g_pool_mu);
        size_t bi = SIZE_MAX;
        for (size_t i = 0; i < g_pool.size(); i++) {
            const PoolBlock &c = g_pool[i];
            if (c.device != device || c.bytes < bytes || c.bytes > 2 * bytes + (size_t(1) << 20)) continue;
            if (bi == SIZE_MAX || c.bytes < g_pool[bi].bytes) bi = i;
        }
        if (bi == SIZE_MAX) return nullptr;
        b = g_pool[bi];
        g_pool.erase(g_pool.begin() + (std::ptrdiff_t)bi);
        g_pool_bytes[device < 0] -= b.bytes;
    }
    if (b.done) {
        cudaEventSynchronize(b.done);
        cudaEventDestroy(b.done);
    }
    *got = b.bytes;
    return b.p;
}

// `last`: the stream of the block's last work (nullptr: none pending).
void pool_give(int device, void *p, size_t bytes, cudaStream_t last, bool has_last) {
    if (!p) return;
    cudaEvent_t done = nullptr;
    if (has_last && cudaEventCreateWithFlags(&done, cudaEventDisableTiming) == cudaSuccess &&
        cudaEventRecord(done, last) != cudaSuccess) {
        cudaEventDestroy(done);
        done = nullptr;
        cudaStreamSynchronize(last);
    }
    {
        std::lock_guard<std::mutex> lk(g_pool_mu);
        if (g_pool_bytes[device < 0] + bytes <= POOL_CAP[device < 0]) {
            g_pool.push_back(PoolBlock{p, bytes, device, done});
            g_pool_bytes[device < 0] += bytes;
            return;
        }
    }
    if (done) {
        cudaEventSynchronize(done);
        cudaEventDestroy(done);
    }
    if (device < 0) cudaFreeHost(p);
    else cudaFree(p);
}

cudaError_t dev_alloc(int device, size_t bytes, void **p, size_t *got) {
    *p = pool_take(device, bytes, got);
    if (*p) return cudaSuccess;
    *got = bytes;
    return cudaMalloc(p, bytes);
}
cudaError_t host_alloc(size_t bytes, void **p, size_t *got) {
    *p = pool_take(-1, bytes, got);
    if (*p) return cudaSuccess;
    *got = bytes;
    return cudaMallocHost(p, bytes);
}
}  // namespace

// The events of one batched launch, shared by all its instances: recording
// two events per instance after a long launch fills the device work queue and
// blocks the host until the launch ends (4,096 instances: the whole sweep).
struct SweepEvents {
    int device = 0;
    cudaEvent_t begin = nullptr, loop_begin = nullptr, loop_end = nullptr;
    ~SweepEvents() {
        int cur = 0;
        cudaGetDevice(&cur);
        cudaSetDevice(device);
        for (cudaEvent_t e : {begin, loop_begin, loop_end})
            if (e) cudaEventDestroy(e);
        cudaSetDevice(cur);
    }
};

struct dts_instance {
    int32_t m = 0, n = 0, K = 1;
    int64_t E_raw = 0;
    uint64_t cap = 0;
    int64_t default_ns = 0;
    std::vector<int64_t> task_ptr;
    std::vector<int32_t> task_data;
    std::vector<uint64_t> size;
    std::vector<int64_t> task_ns;
    bool has_tau = false;
    int32_t max_deg_ub = 0;
    int32_t max_row_len = 0;
    bool uniform_size = false;
    uint64_t max_row_bytes = 0;
    uint64_t min_size = 1;
    int32_t res_cap = 1;
    int32_t m_pad = 0;

    // device side
    int device = -1;
    Arena ar;
    size_t arena_bytes = 0;
    bool uploaded = false;
    int64_t *d_raw_ptr = nullptr;
    int32_t *d_raw_dat = nullptr;
    uint64_t *d_size = nullptr;
    int64_t *d_tau = nullptr;
    int64_t *d_delta = nullptr;
    dts::Inst *h_pinned = nullptr;   // pinned staging copy of the descriptor (async H2D)
    cudaEvent_t ev_desc = nullptr;   // the last H2D copy out of h_pinned
    cudaEvent_t ev_up = nullptr;     // the last H2D upload of the inputs
    cudaStream_t up_stream = nullptr; // ... and the stream it was enqueued on
    void *d_csr_scratch = nullptr;
    int *d_work = nullptr;
    dts::Inst h_inst{};
    dts::Inst *d_inst = nullptr;
    cudaStream_t stream = nullptr;
    cudaEvent_t ev[4] = {nullptr, nullptr, nullptr, nullptr};
    std::shared_ptr<SweepEvents> sev;  // set by a batched launch: its events replace ev[]

    // run state / results
    bool ran = false;
    bool have_host = false;
    int32_t loop_kind = 0;  // dts_result_view.loop_kind of the last run
    dts::Out out{};
    // pinned host memory (allocated with the device arena): a mirror of the
    // inputs for the H2D upload and the result buffers for the D2H read-back
    char *h_pin = nullptr;
    size_t h_pin_cap = 0, h_pinned_cap = 0, h_res_cap = 0;  // pooled block sizes
    bool exported = false;                   // arena shared through CUDA IPC: never pooled
    int64_t *p_task_ptr = nullptr, *p_task_ns = nullptr;
    int32_t *p_task_data = nullptr;
    uint64_t *p_size = nullptr;
    int64_t *r_gpu_ptr = nullptr, *r_tstart = nullptr, *r_tend = nullptr;
    int32_t *r_gpu_ids = nullptr, *r_serve_gpu = nullptr, *r_serve_task = nullptr;
    dts_event *r_events = nullptr;
    dts::Out *r_out = nullptr;
    // pinned mirror of the device result region [gpu_task_ptr .. events end): one
    // D2H copy per instance brings sigma, the service order, the times and the trace
    char *h_res = nullptr;
    size_t res_bytes = 0;
    int64_t r_n_events = 0;
    float loop_ms = 0.f, total_ms = 0.f;

    // task shard (§8(e)): shard g of G owns tasks [t_lo, t_hi)
    int32_t G = 1, g = 0, t_lo = 0, t_hi = 0;
    uint64_t runs = 0;                       // runs so far: exchange numbers of run r start at r << 32
    unsigned long long *d_epoch = nullptr;   // this shard's published exchange number
    unsigned char *d_box = nullptr;          // its two payload slots
    int64_t box_bytes = 0;
    dts::ShardPeer *d_peers = nullptr;       // [MAX_G] peer table read by the kernel
    bool connected = false;
    bool xsys = false;                       // peers mapped through CUDA IPC (other processes / GPUs)
    std::vector<void *> ipc_open;            // peers' arenas mapped through CUDA IPC
    // dts_run with opts.n_devices = G > 1: this instance is shard 0 of G and
    // owns the other G-1 shards (same inputs), shard j on device (device+j) mod #devices
    std::vector<dts_instance *> xs;
    int32_t xs_dev0 = -1;

    ~dts_instance() {
        for (dts_instance *x : xs) delete x;
        // memory back to the pool behind an event on the last stream that used it
        // (the default stream when it was never used on another)
        const bool used = device >= 0;
        if (device >= 0) {
            int cur = 0;
            cudaGetDevice(&cur);
            cudaSetDevice(device);
            for (void *p : ipc_open) cudaIpcCloseMemHandle(p);
            if (ar.base) {
                if (exported) cudaFree(ar.base);
                else pool_give(device, ar.base, ar.size, stream, true);
            }
            for (auto &e : ev)
                if (e) cudaEventDestroy(e);
            if (ev_desc) cudaEventDestroy(ev_desc);
            if (ev_up) cudaEventDestroy(ev_up);
            if (h_pinned) pool_give(-1, h_pinned, h_pinned_cap, stream, true);
            if (h_pin) pool_give(-1, h_pin, h_pin_cap, stream, true);
            if (h_res) pool_give(-1, h_res, h_res_cap, stream, true);
            cudaSetDevice(cur);
        } else {
            if (h_pinned) pool_give(-1, h_pinned, h_pinned_cap, nullptr, used);
            if (h_pin) pool_give(-1, h_pin, h_pin_cap, nullptr, used);
            if (h_res) pool_give(-1, h_res, h_res_cap, nullptr, used);
        }
    }
};

namespace dts {
static std::atomic<uint64_t> g_launches{0};
void count_launch() { g_launches.fetch_add(1, std::memory_order_relaxed); }
}  // namespace dts

extern "C" {

uint64_t dts_kernel_launches(void) { return dts::g_launches.load(std::memory_order_relaxed); }

void dts_run_opts_default(dts_run_opts *o) {
    if (!o) return;
    std::memset(o, 0, sizeof *o);
    o->flags = DTS_F_FALLBACK2;
    o->lookahead_W = 0;
    o->bus_bytes_per_s = 12000000000ull;
    o->device = 0;
    o->block_threads = 0;
    o->smem_budget = 0;
    o->max_served = -1;
    o->cuda_stream = nullptr;
}

const char *dts_status_str(dts_status s) {
    switch (s) {
        case DTS_OK: return "DTS_OK";
        case DTS_E_INVAL: return "DTS_E_INVAL";
        case DTS_E_CAPACITY: return "DTS_E_CAPACITY";
        case DTS_E_NOMEM: return "DTS_E_NOMEM";
        case DTS_E_CUDA: return "DTS_E_CUDA";
        case DTS_E_STATE: return "DTS_E_STATE";
        case DTS_E_UNSUPPORTED: return "DTS_E_UNSUPPORTED";
    }
    return "DTS_E_UNKNOWN";
}

const char *dts_last_error(void) { return g_err.c_str(); }

uint32_t dts_version(void) { return (1u << 16) | 3u; }

dts_status dts_instance_create(int32_t n_tasks, int32_t n_data, const int64_t *task_ptr,
                               const int32_t *task_data, const uint64_t *data_size,
                               const int64_t *task_ns, int64_t default_task_ns,
                               uint64_t mem_capacity_bytes, int32_t K, dts_instance **out) {
    if (!out) return fail(DTS_E_INVAL, "out is NULL");
    *out = nullptr;
    if (n_tasks < 0 || n_data < 0) return fail(DTS_E_INVAL, "negative size");
    if (K < 1) return fail(DTS_E_INVAL, "K < 1");
    if (K > dts::MAX_K) return fail(DTS_E_UNSUPPORTED, "K > 64");
    if (n_data >= (1 << 24)) return fail(DTS_E_UNSUPPORTED, "n_data >= 2^24 (packed xor field)");
    if (!task_ptr) return fail(DTS_E_INVAL, "task_ptr is NULL");
    if (n_data > 0 && !data_size) return fail(DTS_E_INVAL, "data_size is NULL");
    if (task_ptr[0] != 0) return fail(DTS_E_INVAL, "task_ptr[0] != 0");
    // the whole of task_ptr first: 0 <= task_ptr[T] <= task_ptr[T+1] for every T,
    // so no row is read past E = task_ptr[m]
    for (int32_t T = 0; T < n_tasks; T++)
        if (task_ptr[T + 1] < task_ptr[T])
            return fail(DTS_E_INVAL, "task_ptr not monotone at " + std::to_string(T));
    const int64_t E = task_ptr[n_tasks];
    if (E > 0 && !task_data) return fail(DTS_E_INVAL, "task_data is NULL");
    if (default_task_ns < 0) return fail(DTS_E_INVAL, "default_task_ns < 0");
    if (E >= (int64_t)INT32_MAX) return fail(DTS_E_UNSUPPORTED, "too many edges");
    dts_instance *I = new (std::nothrow) dts_instance();
    if (!I) return fail(DTS_E_NOMEM, "host allocation");
    try {
        I->m = n_tasks;
        I->n = n_data;
        I->K = K;
        I->E_raw = E;
        I->cap = mem_capacity_bytes;
        I->default_ns = default_task_ns;
        I->task_ptr.assign(task_ptr, task_ptr + (size_t)n_tasks + 1);
        if (E > 0) I->task_data.assign(task_data, task_data + E);
        if (n_data > 0) I->size.assign(data_size, data_size + n_data);
        if (task_ns) {
            I->task_ns.assign(task_ns, task_ns + n_tasks);
            I->has_tau = true;
        }
    } catch (...) {
        delete I;
        return fail(DTS_E_NOMEM, "host allocation");
    }
    // validation (input checking only; the schedule is computed on the device)
    uint64_t min_size = UINT64_MAX;
    for (int32_t D = 0; D < n_data; D++) {
        if (I->size[D] == 0) {
            delete I;
            return fail(DTS_E_INVAL, "data_size[" + std::to_string(D) + "] == 0");
        }
        min_size = std::min(min_size, I->size[D]);
    }
    if (n_data == 0) min_size = 1;
    std::vector<int32_t> occ((size_t)n_data + 1, 0);
    int32_t scratch[dts::MAX_ROW];
    for (int32_t T = 0; T < n_tasks; T++) {
        int64_t b = I->task_ptr[T], e = I->task_ptr[T + 1];
        if (e < b) {
            delete I;
            return fail(DTS_E_INVAL, "task_ptr not monotone at " + std::to_string(T));
        }
        if (e - b > dts::MAX_ROW) {
            delete I;
            return fail(DTS_E_UNSUPPORTED, "task " + std::to_string(T) + " has > 127 inputs");
        }
        if (I->has_tau && I->task_ns[T] < 0) {
            delete I;
            return fail(DTS_E_INVAL, "task_ns < 0");
        }
        int q = 0;
        uint64_t bytes = 0;
        for (int64_t i = b; i < e; i++) {
            int32_t D = I->task_data[i];
            if (D < 0 || D >= n_data) {
                delete I;
                return fail(DTS_E_INVAL, "task_data id out of range at edge " + std::to_string(i));
            }
            bool dup = false;
            for (int j = 0; j < q; j++) dup |= (scratch[j] == D);
            if (!dup) {
                scratch[q++] = D;
                bytes += I->size[D];
                occ[D]++;
            }
        }
        I->max_row_bytes = std::max(I->max_row_bytes, bytes);
        I->max_row_len = std::max(I->max_row_len, q);
    }
    int32_t md = 1;
    for (int32_t D = 0; D < n_data; D++) md = std::max(md, occ[D]);
    I->max_deg_ub = md;
    I->uniform_size = n_data > 0 && std::all_of(I->size.begin(), I->size.end(),
                                                [&](uint64_t x) { return x == I->size[0]; });
    I->min_size = min_size;
    uint64_t rc = mem_capacity_bytes / min_size;
    I->res_cap = (int32_t)std::max<uint64_t>(1, std::min<uint64_t>(rc, (uint64_t)std::max(n_data, 1)));
    I->m_pad = (n_tasks + 3) & ~3;
    int hb = bits_for((uint64_t)md), idb = bits_for(n_data > 0 ? (uint64_t)(n_data - 1) : 0);
    if (2 * hb + idb > 63) {
        delete I;
        return fail(DTS_E_UNSUPPORTED, "argmax key does not fit 64 bits");
    }
    *out = I;
    return DTS_OK;
}

void dts_instance_destroy(dts_instance *inst) { delete inst; }

}  // extern "C"

namespace {

dts_status check_device(int device) {
    // cudaGetDeviceProperties costs milliseconds: query each device once
    static int checked[64] = {0};  // 0 = unknown, 1 = sm_100, -1 = other
    int ndev = 0;
    cudaError_t e = cudaGetDeviceCount(&ndev);
    if (e != cudaSuccess || ndev == 0) return fail(DTS_E_CUDA, "no CUDA device (libdts has no CPU path)");
    if (device < 0 || device >= ndev || device >= 64) return fail(DTS_E_INVAL, "device ordinal out of range");
    if (checked[device] == 0) {
        int major = 0;
        CK(cudaDeviceGetAttribute(&major, cudaDevAttrComputeCapabilityMajor, device), "attr major");
        checked[device] = major == 10 ? 1 : -1;
    }
    if (checked[device] < 0) return fail(DTS_E_CUDA, "libdts is built for sm_100a (B200); device is not sm_10x");
    return DTS_OK;
}

dts_status ensure_device(dts_instance *I, int device) {
    if (I->device == device && I->ar.base) return DTS_OK;
    if (I->device >= 0 && I->ar.base) {
        if (I->connected && I->G > 1)
            return fail(DTS_E_STATE, "a connected task shard cannot move to another device");
        cudaSetDevice(I->device);
        if (I->exported) cudaFree(I->ar.base);
        else pool_give(I->device, I->ar.base, I->ar.size, I->stream, true);
        for (auto &e : I->ev)
            if (e) cudaEventDestroy(e);
        if (I->ev_desc) cudaEventDestroy(I->ev_desc);
        if (I->ev_up) cudaEventDestroy(I->ev_up);
        I->ev_desc = nullptr;
        I->ev_up = nullptr;
        I->ar = Arena{};
        I->uploaded = false;
    }
    dts_status s = check_device(device);
    if (s != DTS_OK) return s;
    CK(cudaSetDevice(device), "cudaSetDevice");
    const size_t m = (size_t)I->m, n = (size_t)I->n, K = (size_t)I->K, E = (size_t)I->E_raw;
    const size_t mp = (size_t)I->m_pad;
    const size_t ev_cap = 2 * E + 16;
    const size_t plan_cap = (size_t)I->max_deg_ub + 1;
    const size_t res_cap = (size_t)I->res_cap + 1;
    const size_t nw = (n + 31) / 32 + 1;
    const size_t nstr = (n + 3) & ~size_t(3);
    size_t need = 0;
    auto add = [&](size_t bytes) { need += (bytes + 255) & ~size_t(255); };
    add(8 * (m + 1)); add(4 * (E + 1)); add(8 * (n + 1)); add(8 * (m + 1));          // raw inputs
    add(8 * (m + 1)); add(4 * (E + 1)); add(8 * (n + 1)); add(4 * (E + 1));          // CSR
    add(16 * (E + 1));                                                               // edge records
    add(8 * (n + 1)); add(8);                                                        // delta
    add(4 * K * mp + 16); add(4 * (nstr + 4)); add(4 * K * (nstr + 4)); add(4 * K * (nstr + 4));  // s u h h2
    add(4 * K * (nstr + 4)); add(4 * K * nw); add(4 * K * res_cap);                  // np resb res_list
    add(16 * K * plan_cap); add(8 * K * plan_cap); add(4 * (3 * n + 1));              // plan tau vhist
    add(4 * K * (nstr + 4));                                                          // lru stamps
    add(4 * (mp / 32 + 2));                                                           // alloc bitmap
    add(4 * K * dts::MAX_W);                                                          // W ring
    add(sizeof(dts::Out));
    add(4 * (m + 1)); add(4 * (m + 1)); add(8 * (m + 1)); add(8 * (m + 1));          // serve, times
    add(sizeof(dts_event) * ev_cap); add(8 * (K + 1)); add(4 * (m + 1));
    add(sizeof(dts::Inst)); add(64);
    add(dts::csr_scratch_bytes(I->m, I->n, I->E_raw));
    const int64_t box_bytes = (int64_t)sizeof(dts::ShardSlot) + 16 * (int64_t)plan_cap;
    add(256); add(2 * (size_t)box_bytes); add(sizeof(dts::ShardPeer) * dts::MAX_G);  // shard exchange
    char *base = nullptr;
    size_t got = 0;
    cudaError_t e = dev_alloc(device, need, reinterpret_cast<void **>(&base), &got);
    if (e != cudaSuccess) return fail(DTS_E_NOMEM, std::string("cudaMalloc: ") + cudaGetErrorString(e));
    I->ar.base = base;
    I->ar.size = got;
    I->ar.used = 0;
    I->device = device;
    for (auto &ev : I->ev) CK(cudaEventCreate(&ev), "cudaEventCreate");
    CK(cudaEventCreateWithFlags(&I->ev_desc, cudaEventDisableTiming), "cudaEventCreate");
    CK(cudaEventCreateWithFlags(&I->ev_up, cudaEventDisableTiming), "cudaEventCreate");
    if (!I->h_pinned)
        CK(host_alloc(sizeof(dts::Inst), reinterpret_cast<void **>(&I->h_pinned), &I->h_pinned_cap), "cudaMallocHost");
    if (!I->h_pin) {
        size_t hb = 0;
        // the input mirror has the device arena's layout (256-byte rounding, same
        // order as d_raw_ptr, d_raw_dat, d_size, d_tau): one H2D copy uploads it
        auto hadd = [&](size_t bytes) { size_t o = hb; hb += (bytes + 255) & ~size_t(255); return o; };
        const size_t o_tp = hadd(8 * (m + 1)), o_td = hadd(4 * (E + 1)), o_sz = hadd(8 * (n + 1)),
                     o_tn = hadd(8 * (m + 1)), o_out = hadd(sizeof(dts::Out));
        CK(host_alloc(hb, reinterpret_cast<void **>(&I->h_pin), &I->h_pin_cap), "cudaMallocHost");
        I->p_task_ptr = (int64_t *)(I->h_pin + o_tp);
        I->p_task_data = (int32_t *)(I->h_pin + o_td);
        I->p_size = (uint64_t *)(I->h_pin + o_sz);
        I->p_task_ns = (int64_t *)(I->h_pin + o_tn);
        I->r_out = (dts::Out *)(I->h_pin + o_out);
        std::memcpy(I->p_task_ptr, I->task_ptr.data(), 8 * (m + 1));
        if (E) std::memcpy(I->p_task_data, I->task_data.data(), 4 * E);
        if (n) std::memcpy(I->p_size, I->size.data(), 8 * n);
        if (I->has_tau && m) std::memcpy(I->p_task_ns, I->task_ns.data(), 8 * m);
    }

    Arena &A = I->ar;
    dts::Inst &h = I->h_inst;
    std::memset(&h, 0, sizeof h);
    I->d_raw_ptr = A.take<int64_t>(m + 1);
    I->d_raw_dat = A.take<int32_t>(E + 1);
    I->d_size = A.take<uint64_t>(n + 1);
    I->d_tau = A.take<int64_t>(m + 1);
    h.tptr = A.take<int64_t>(m + 1);
    h.tdat = A.take<int32_t>(E + 1);
    h.dptr = A.take<int64_t>(n + 1);
    h.ddat = A.take<int32_t>(E + 1);
    h.dedge = A.take<int4>(E + 1);
    I->d_delta = A.take<int64_t>(n + 1);
    h.s = A.take<uint32_t>(K * mp + 4);
    h.u = A.take<int32_t>(nstr + 4);
    h.h = A.take<int32_t>(K * (nstr + 4));
    h.h2 = A.take<int32_t>(K * (nstr + 4));
    h.np = A.take<int32_t>(K * (nstr + 4));
    h.resb = A.take<uint32_t>(K * nw);
    h.res_list = A.take<int32_t>(K * res_cap);
    h.plan = A.take<int4>(K * plan_cap);
    h.plan_tau = A.take<int64_t>(K * plan_cap);
    h.vhist = A.take<int32_t>(3 * n + 1);
    h.lru = A.take<int32_t>(K * (nstr + 4));
    h.al = A.take<uint32_t>(mp / 32 + 2);
    h.wring = A.take<int32_t>(K * dts::MAX_W);
    h.out = A.take<dts::Out>(1);
    // the result region, contiguous, the trace last (its used length varies)
    h.gpu_task_ptr = A.take<int64_t>(K + 1);
    h.gpu_task_ids = A.take<int32_t>(m + 1);
    h.serve_gpu = A.take<int32_t>(m + 1);
    h.serve_task = A.take<int32_t>(m + 1);
    h.tstart = A.take<int64_t>(m + 1);
    h.tend = A.take<int64_t>(m + 1);
    h.events = A.take<dts_event>(ev_cap);
    I->d_inst = A.take<dts::Inst>(1);
    I->d_work = A.take<int>(16);
    I->d_csr_scratch = A.take<char>(dts::csr_scratch_bytes(I->m, I->n, I->E_raw));
    I->d_epoch = A.take<unsigned long long>(32);
    I->box_bytes = box_bytes;
    I->d_box = A.take<unsigned char>(2 * (size_t)box_bytes);
    I->d_peers = A.take<dts::ShardPeer>(dts::MAX_G);
    if (A.used > A.size) return fail(DTS_E_NOMEM, "arena overflow (internal)");
    {  // host mirror of the result region, same relative layout
        char *r0 = reinterpret_cast<char *>(h.gpu_task_ptr);
        const size_t bytes = (size_t)(reinterpret_cast<char *>(h.events) - r0) + sizeof(dts_event) * ev_cap;
        if (I->h_res && I->h_res_cap < bytes) {
            pool_give(-1, I->h_res, I->h_res_cap, I->stream, true);
            I->h_res = nullptr;
        }
        if (!I->h_res) CK(host_alloc(bytes, reinterpret_cast<void **>(&I->h_res), &I->h_res_cap), "cudaMallocHost");
        I->res_bytes = bytes;
        auto at = [&](const void *d) { return I->h_res + (reinterpret_cast<const char *>(d) - r0); };
        I->r_gpu_ptr = reinterpret_cast<int64_t *>(at(h.gpu_task_ptr));
        I->r_gpu_ids = reinterpret_cast<int32_t *>(at(h.gpu_task_ids));
        I->r_serve_gpu = reinterpret_cast<int32_t *>(at(h.serve_gpu));
        I->r_serve_task = reinterpret_cast<int32_t *>(at(h.serve_task));
        I->r_tstart = reinterpret_cast<int64_t *>(at(h.tstart));
        I->r_tend = reinterpret_cast<int64_t *>(at(h.tend));
        I->r_events = reinterpret_cast<dts_event *>(at(h.events));
    }
    CK(cudaMemset(I->d_epoch, 0, 256), "memset epoch");  // exchange numbers start at 0, once
    I->connected = false;
    I->runs = 0;

    h.m = I->m;
    h.n = I->n;
    h.K = I->K;
    h.m_pad = I->m_pad;
    h.cap = I->cap;
    h.plan_cap = (int32_t)plan_cap;
    h.res_cap = (int32_t)res_cap;
    h.nw = (int32_t)nw;
    h.nstr = (int32_t)nstr;
    h.id_bits = bits_for(I->n > 0 ? (uint64_t)(I->n - 1) : 0);
    h.u_bits = bits_for((uint64_t)I->max_deg_ub);
    h.key32 = I->max_deg_ub < 32768 ? 1 : 0;  // n(D), n2(D), u(D) <= deg(D)
    h.max_row = I->max_row_len;
    h.E = I->E_raw;
    h.size = I->d_size;
    h.delta = I->d_delta;
    h.tau = I->has_tau ? I->d_tau : nullptr;
    h.default_tau = I->default_ns;
    h.ev_cap = (int64_t)ev_cap;
    return DTS_OK;
}

dts_status upload(dts_instance *I, cudaStream_t st, bool force = false) {
    if (I->uploaded && !force) return DTS_OK;
    // from the pinned mirror of the caller's arrays (asynchronous DMA), one copy:
    // task_ptr, task_data, data_size[, task_ns] at the arena's relative offsets
    const char *d0 = reinterpret_cast<const char *>(I->d_raw_ptr);
    const char *end = I->has_tau && I->m > 0 ? reinterpret_cast<const char *>(I->d_tau + I->m)
                                             : reinterpret_cast<const char *>(I->d_size + I->n);
    CK(cudaMemcpyAsync(I->d_raw_ptr, I->p_task_ptr, (size_t)(end - d0), cudaMemcpyHostToDevice, st), "H2D inputs");
    CK(cudaEventRecord(I->ev_up, st), "event");  // a run on another stream waits for it (stage)
    I->up_stream = st;
    I->uploaded = true;
    return DTS_OK;
}

dts_status check_opts(const dts_instance *I, dts_policy policy, const dts_run_opts *o) {
    if (policy != DTS_POLICY_DARTS_LUF && policy != DTS_POLICY_DARTS_LRU && policy != DTS_POLICY_EAGER_LRU)
        return fail(DTS_E_UNSUPPORTED, "policy");
    if (o->flags & ~(uint32_t)(DTS_F_FALLBACK2 | DTS_F_VERIFY | DTS_F_NOFUSE | DTS_F_OPTI | DTS_F_PACKED |
                               DTS_F_GENERIC | DTS_F_CTA))
        return fail(DTS_E_UNSUPPORTED, "unknown flags");
    if (o->lookahead_W > (uint32_t)dts::MAX_W) return fail(DTS_E_UNSUPPORTED, "lookahead_W > 8");
    if ((int64_t)o->lookahead_W * I->max_row_len > dts::MAX_ROW + 1)
        return fail(DTS_E_UNSUPPORTED, "lookahead_W * (inputs per task) > 128");
    if (o->bus_bytes_per_s == 0) return fail(DTS_E_INVAL, "bus_bytes_per_s == 0");
    if (o->block_threads != 0 && (o->block_threads < 32 || o->block_threads > 512 || o->block_threads % 32))
        return fail(DTS_E_INVAL, "block_threads must be 0 or a multiple of 32 in [32, 512]");
    if (o->smem_budget < -1) return fail(DTS_E_INVAL, "smem_budget < -1");
    // DARTS+LUF: max(1, W) tasks' inputs -- with W >= 1 Alg. 6's Belady branch
    // may fire and always finds a datum only the running task uses (R29);
    // the LRU policies have no Belady branch: (W+1) tasks' inputs
    const uint64_t tasks = policy == DTS_POLICY_DARTS_LUF ? std::max<uint64_t>(1, o->lookahead_W)
                                                          : (uint64_t)o->lookahead_W + 1;
    unsigned __int128 need = (unsigned __int128)tasks * I->max_row_bytes;
    if ((unsigned __int128)I->cap < need)
        return fail(DTS_E_CAPACITY, policy == DTS_POLICY_DARTS_LUF
                                        ? "mem_capacity_bytes < max(1, W) * max_T size(D(T))"
                                        : "mem_capacity_bytes < (W+1) * max_T size(D(T))");
    return DTS_OK;
}

// Tuning knobs: fixed in the product library.  Only the profiling build
// (lib/libdts_prof.so, -DDTS_PROF) lets an experiment override them from the
// environment, so the launch shape of a product run never depends on it.
int tuning(const char *name, int dflt) {
#ifdef DTS_PROF
    const char *v = std::getenv(name);
    return v ? std::atoi(v) : dflt;
#else
    (void)name;
    return dflt;
#endif
}

// Relative cost of an instance's chain (longest-first ordering, LPT over devices).
double instance_cost(const dts_instance *I) {
    return (double)I->m * (double)I->E_raw / std::max(1, I->n);
}

// The compile-time specialised loop (dts_loop_fast.cu) applies: row-derived
// state, one shard, W = 0, DARTS+LUF, 32-bit argmax keys, uniform data sizes,
// no OPTI, no self-check, not forced generic.
bool fast_mode(const dts::Inst &h) {
    return h.sl && h.G == 1 && h.W == 0 && h.policy == DTS_POLICY_DARTS_LUF && h.key32 && h.size0 &&
           !(h.flags & (DTS_F_VERIFY | DTS_F_OPTI | DTS_F_GENERIC));
}

// The one-warp-per-instance loop (dts_warp.cu) applies: the fast mode's
// conditions, <= 2 inputs per task, 16-bit task and data ids in the edge
// words, K <= 32 (a lane per simulated GPU), 16-bit scores, automatic launch
// shape and placement, and a state slice that fits in shared memory.
int64_t warp_slot_bytes(const dts_instance *I) {
    return dts::warp_layout(I->m, I->n, I->K, I->max_deg_ub + 1, I->res_cap + 1).total;
}
int max_dyn_smem_warp(int device) {
    static std::atomic<int> cache[64];  // 0 = not queried yet
    if (device >= 0 && device < 64 && cache[device].load() > 0) return cache[device].load();
    int optin = 0;
    cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, device);
    const int r = std::max(0, optin - 1024);
    if (device >= 0 && device < 64 && r > 0) cache[device].store(r);
    return r;
}
bool warp_eligible(const dts_instance *I, dts_policy policy, const dts_run_opts &o) {
    if (policy != DTS_POLICY_DARTS_LUF || o.lookahead_W != 0 || o.block_threads != 0 || o.smem_budget < 0 ||
        (o.flags & (DTS_F_VERIFY | DTS_F_OPTI | DTS_F_GENERIC | DTS_F_CTA | DTS_F_PACKED | DTS_F_NOFUSE)) ||
        I->G != 1)
        return false;
    if (I->max_row_len > 2 || I->m > 65535 || I->n > 65534 || I->K > 32 || !I->uniform_size ||
        I->max_deg_ub >= 32768)
        return false;
    const int64_t slot = warp_slot_bytes(I);
    const int64_t lim = o.smem_budget > 0 ? std::min<int64_t>(o.smem_budget, max_dyn_smem_warp(o.device))
                                          : max_dyn_smem_warp(o.device);
    return slot <= lim;
}
// A lone instance runs on one warp while its segments stay short (the widest
// segment walk is 2,048 / 160 register batches at most); the warp loop beat the
// CTA loop on every lone instance whose slice fits (C3 1.64x, n up to 4,096:
// 1.4-1.8x, profiles/r03/r03q_solo_cross.txt).
#ifndef DTS_WARP_SOLO_MAX
#define DTS_WARP_SOLO_MAX 2048
#endif
constexpr int WARP_SOLO_MAX = DTS_WARP_SOLO_MAX;
bool warp_solo(const dts_instance *I) { return I->max_deg_ub <= WARP_SOLO_MAX; }

// Shared-memory placement of one instance's state:
// greedy, most latency-critical array first, each either fully in the CTA's
// dynamic shared memory or in its global home.  Returns the bytes used.
int place_smem(dts::Inst &h, bool has_tau, int budget, bool lru, bool shard, bool sl) {
    const int64_t K = h.K, n = h.n;
    int used = 0;
    auto put = [&](int32_t &so, int64_t bytes) {
        bytes = (bytes + 15) & ~int64_t(15);
        const bool peer_read = shard && (&so == &h.so_u || &so == &h.so_h || &so == &h.so_h2);
        if (budget > 0 && !peer_read && used + bytes <= budget) {
            so = used;
            used += (int)bytes;
        } else {
            so = -1;
        }
    };
    put(h.so_resb, 4 * K * h.nw);
    // the allocation bitmap is read by every segment walk (placing it after u
    // instead made C4 1 % slower, profiles/r01i_c4_placement.txt)
    h.so_al = -1;
    if (sl) put(h.so_al, 4 * (int64_t)(h.m_pad / 32 + 1));
    put(h.so_dptr, 4 * (n + 1));
    put(h.so_plan, 16 * K * h.plan_cap);
    if (has_tau) put(h.so_plan_tau, 8 * K * h.plan_cap);
    else h.so_plan_tau = -1;
    put(h.so_res_list, 4 * K * h.res_cap);
    put(h.so_u, 4 * (int64_t)h.nstr);
    put(h.so_h, 4 * K * (int64_t)h.nstr);
    put(h.so_h2, 4 * K * (int64_t)h.nstr);
    put(h.so_np, 4 * K * (int64_t)h.nstr);
    if (lru) put(h.so_lru, 4 * K * (int64_t)h.nstr);
    else h.so_lru = -1;
    if (!sl) put(h.so_s, 4 * K * (int64_t)h.m_pad);  // last: the largest, worth it only when it fits
    else h.so_s = -1;
    h.smem_bytes = used;
    return used;
}

int max_dyn_smem(int device) {
    static int cache[64] = {0};
    if (device >= 0 && device < 64 && cache[device] > 0) return cache[device];
    int optin = 0;
    cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, device);
    int st = std::max(dts::loop_static_smem(), dts::loop_static_smem_fast());
    if (st < 0) st = 16384;
    const int r = std::max(0, optin - st - 1024);
    if (device >= 0 && device < 64) cache[device] = r;
    return r;
}

// Threads of the CTA: enough to cover a data segment (deg(D)) in one pass
// and the score argmax in <= 8 entries per thread, within [64, 512].
int auto_block(const dts_instance *I, bool alone = false) {
    // alone (a single instance, or a batch small enough for one CTA per
    // instance on its own SM): twice the widest segment -- the pool moves of
    // a plan (|plan| x K items) then take one pass (C2's chain: 7.08 -> 6.98 ms)
    const int64_t deg = alone ? 2 * (int64_t)I->max_deg_ub : (int64_t)I->max_deg_ub;
    int b = 64;
    while (b < 512 && (b * 8 < I->n || b < deg)) b *= 2;
    return b;
}


// Enqueue everything of one instance up to (not including) the decision loop:
// upload if needed, CSR build (a1), state init (a2), descriptor H2D.
// Shared scratch of the fused in-CTA CSR build (dts_loop.cu fused_build).
int fused_scratch_bytes(const dts_instance *I, int block) { return (2 * (block / 32) + 1) * 4 * (I->n + 1); }

dts_status stage(dts_instance *I, dts_policy policy, const dts_run_opts &o, int budget, int block,
                 cudaStream_t st, bool copy_desc = true, bool own_events = true, bool warp = false) {
    dts_status s = ensure_device(I, o.device);
    if (s != DTS_OK) return s;
    int cur = -1;
    if (cudaGetDevice(&cur) != cudaSuccess || cur != o.device) CK(cudaSetDevice(o.device), "cudaSetDevice");
    I->stream = st;
    I->ran = false;
    I->have_host = false;
    s = upload(I, st);
    if (s != DTS_OK) return s;
    // inputs uploaded on another stream (dts_instance_upload) are complete
    // before this run reads them (the same stream orders them already)
    if (I->up_stream != st) {
        CK(cudaStreamWaitEvent(st, I->ev_up, 0), "wait upload");
        I->up_stream = st;
    }
    dts::Inst &h = I->h_inst;
    h.W = (int32_t)o.lookahead_W;
    h.flags = o.flags;
    h.max_served = o.max_served;
    h.policy = (int32_t)policy;
    h.size0 = 0;
    h.delta0 = 0;
    h.bw = o.bus_bytes_per_s;
    h.raw_ptr = I->d_raw_ptr;
    h.raw_dat = I->d_raw_dat;
    if (I->uniform_size) {
        h.size0 = I->size[0];
        const unsigned __int128 num = (unsigned __int128)h.size0 * 1000000000u + (o.bus_bytes_per_s - 1);
        h.delta0 = (int64_t)(num / o.bus_bytes_per_s);  // ceil, reading R9 (same as dts_init_kernel)
    }
    // row-derived state (no per-(GPU, task) words) when every edge record holds its row
    h.sl = I->G == 1 && I->max_row_len <= 3 && !(o.flags & DTS_F_PACKED) ? 1 : 0;
    place_smem(h, I->has_tau, budget, policy != DTS_POLICY_DARTS_LUF, I->G > 1, h.sl != 0);
    h.G = I->G;
    h.g = I->g;
    h.t_lo = I->G > 1 ? I->t_lo : 0;
    h.t_hi = I->G > 1 ? I->t_hi : I->m;
    h.peers = I->G > 1 ? I->d_peers : nullptr;
    h.ep_base = (unsigned long long)(++I->runs) << 32;
    h.box_bytes = I->box_bytes;
    h.xsys = I->xsys ? 1 : 0;
    // batched pops pay off from ~2.5 planned tasks per simulated GPU (C3, K = 4: 10; C4, K = 8:
    // 20, where a threshold of 10 made C4a 2.3 % slower, profiles/r03/r03l_pop_batch_min.txt)
    h.pop_batch_min = tuning("DTS_POP_BATCH_MIN", h.K >= 8 ? 20 : 10);
    h.poison = tuning("DTS_POISON", 0);  // debug (profiling build only)
    // small instances: the loop CTA builds its own CSR and state (one launch)
    const int fs = fused_scratch_bytes(I, block);
    h.fused = I->G == 1 && !(o.flags & DTS_F_NOFUSE) && I->max_row_len <= 8 && fs <= max_dyn_smem(o.device) ? 1 : 0;
    if (h.fused) h.smem_bytes = std::max(h.smem_bytes, fs);
    h.smem_bytes = std::max(h.smem_bytes, dts::ASSEMBLE_SMEM_BYTES);  // result assembly's scratch
    if (warp) {  // dts_warp.cu: the warp builds its CSR and state in its own slice
        h.fused = 1;
        h.smem_bytes = (int32_t)warp_slot_bytes(I);
    }
    if (own_events) {
        I->sev.reset();
        CK(cudaEventRecord(I->ev[0], st), "event");
    }
    if (!h.fused)
        CK(dts::build_csr(I->d_raw_ptr, I->d_raw_dat, I->m, I->n, I->E_raw, (int64_t *)h.tptr,
                          (int32_t *)h.tdat, (int64_t *)h.dptr, (int32_t *)h.ddat, (int4 *)h.dedge,
                          I->d_csr_scratch, st, h.t_lo, h.t_hi),
           "build_csr");
    h.hh = fast_mode(h) ? 1 : 0;  // the specialised loop keeps packed score rows (dts_loop.cu M_HH)
    if (!copy_desc) return DTS_OK;
    // descriptor H2D from pinned memory (a pageable copy would serialise the host)
    CK(cudaEventSynchronize(I->ev_desc), "desc event");
    *I->h_pinned = h;
    CK(cudaMemcpyAsync(I->d_inst, I->h_pinned, sizeof h, cudaMemcpyHostToDevice, st), "H2D inst");
    CK(cudaEventRecord(I->ev_desc, st), "event");
    return DTS_OK;
}

int budget_of(const dts_run_opts &o) {
    if (o.smem_budget < 0) return 0;
    const int mx = max_dyn_smem(o.device);
    return o.smem_budget == 0 ? mx : std::min(o.smem_budget, mx);
}

// Per-device ring of descriptor buffers for batched (sweep / shard-group)
// launches.  Every launch gets its own slot: the device copy of its instance
// descriptors and its own instance counters, so a sweep on one stream never
// overwrites what a still-running launch on another stream reads.  A slot is
// reused only after the event recorded behind its last kernel has completed
// (host wait, only when the ring wraps around a running launch).  The mutex
// serialises the enqueue of batched launches on one device (slot choice,
// capacity growth, the shared side stream and its fork/join events).
struct SweepSlot {
    dts::Inst *d_insts = nullptr;  // descriptors, then the launch's instance counters
    dts::Inst *h_insts = nullptr;  // pinned staging copy (async H2D)
    int *d_work = nullptr;         // the launch's instance counter
    size_t cap = 0;
    cudaEvent_t done = nullptr;    // recorded after every kernel that reads this slot
};
struct DeviceSweep {
    static constexpr int RING = 8;
    std::mutex mu;
    SweepSlot slot[RING];
    int next = 0;
    bool init = false;
    std::vector<cudaStream_t> extra;  // library streams for multi-device sweeps (dts_sweep_run devices[])
};
DeviceSweep g_dev[64];

// Caller holds D.mu; the device is current.
dts_status acquire_slot(DeviceSweep &D, size_t n, SweepSlot **out) {
    if (!D.init) {
        D.init = true;
    }
    SweepSlot &S = D.slot[D.next];
    D.next = (D.next + 1) % DeviceSweep::RING;
    if (S.done) CK(cudaEventSynchronize(S.done), "sweep slot event");  // its last launch has finished
    else CK(cudaEventCreateWithFlags(&S.done, cudaEventDisableTiming), "cudaEventCreate");
    if (S.cap < n) {
        // grow EVERY slot of the ring now (each waits for its last launch first): a
        // batch size seen once is then served without cudaMalloc / cudaMallocHost --
        // slots first used inside a timed loop cost up to 30 ms of host time each
        const size_t cap = std::max<size_t>(n, 64);
        for (SweepSlot &X : D.slot) {
            if (X.cap >= cap) continue;
            if (X.done) CK(cudaEventSynchronize(X.done), "sweep slot event");
            else CK(cudaEventCreateWithFlags(&X.done, cudaEventDisableTiming), "cudaEventCreate");
            if (X.d_insts) cudaFree(X.d_insts);
            if (X.h_insts) cudaFreeHost(X.h_insts);
            X.d_insts = nullptr;
            X.h_insts = nullptr;
            X.cap = 0;
            CK(cudaMalloc(&X.d_insts, sizeof(dts::Inst) * cap + 256), "cudaMalloc sweep");
            CK(cudaMallocHost(&X.h_insts, sizeof(dts::Inst) * cap), "cudaMallocHost sweep");
            X.d_work = reinterpret_cast<int *>(X.d_insts + cap);
            X.cap = cap;
        }
    }
    *out = &S;
    return DTS_OK;
}

// One batched launch of insts[0..n) on o.device,
// enqueued on st.  The instances are validated by the caller.
dts_status sweep_on_device(dts_instance *const *insts, int32_t n, dts_policy policy, const dts_run_opts &o,
                           cudaStream_t st) {
    int64_t work = 1;
    for (int32_t i = 0; i < n; i++)
        work = std::max<int64_t>(work, std::max<int64_t>(insts[i]->m_pad, (int64_t)insts[i]->n * insts[i]->K));
    // Each instance is a latency-bound chain: with many more instances than
    // SMs, run several CTAs per SM (their chains interleave) by default --
    // a share of the shared memory each; few instances get all of it.
    int nsm = 0;
    CK(cudaSetDevice(o.device), "cudaSetDevice");
    CK(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, o.device), "attr SMs");
    const bool many = n >= 2 * nsm;
    int budget = budget_of(o);
    const int smem_div = std::max(1, tuning("DTS_SWEEP_SMEM_DIV", 6));
    if (o.smem_budget == 0 && many) budget = std::min(budget, (max_dyn_smem(o.device) + 1024) / smem_div - 4096);
    // longest first (cost ~ m * mean degree), so the device counter hands the
    // long chains out early and the tail of the batch stays short
    std::vector<int32_t> ord((size_t)n);
    for (int32_t i = 0; i < n; i++) ord[(size_t)i] = i;
    std::stable_sort(ord.begin(), ord.end(),
                     [&](int32_t a, int32_t b) { return instance_cost(insts[a]) > instance_cost(insts[b]); });
    // CTA size: each instance wants twice its widest segment (auto_block); a
    // batch of many instances runs in ONE launch of <= 128-thread CTAs so that
    // four chains share an SM (registers) and the longest ones, handed out
    // first by the launch's counter, overlap the rest (C5: 232 ms against 280
    // for round 1's two concurrent launches of 256- and 128-thread CTAs,
    // profiles/r02s_c5_block.txt).  A forced size applies to all.
    bool warp = true;  // every instance on one warp (dts_warp.cu)
    for (int32_t i = 0; i < n && warp; i++) warp = warp_eligible(insts[i], policy, o);
    if (n == 1) warp = warp && warp_solo(insts[0]);
    const int forced = o.block_threads;
    const int small_max = tuning("DTS_SWEEP_SMALL_BLOCK", 128);
    int block = 32;
    for (int32_t i = 0; i < n; i++) {
        const int ab = auto_block(insts[ord[(size_t)i]], !many);
        block = std::max(block, many ? std::min(ab, small_max) : ab);
    }
    if (forced) block = forced;
    int smem = 0;
    bool any_unfused = false;
    auto sev = std::make_shared<SweepEvents>();
    sev->device = o.device;
    CK(cudaEventCreate(&sev->begin), "cudaEventCreate");
    CK(cudaEventCreate(&sev->loop_begin), "cudaEventCreate");
    CK(cudaEventCreate(&sev->loop_end), "cudaEventCreate");
    CK(cudaEventRecord(sev->begin, st), "event");
    for (int32_t i = 0; i < n; i++) {
        dts_instance *I = insts[ord[(size_t)i]];
        dts_status s = stage(I, policy, o, budget, block, st, false, false, warp);
        if (s != DTS_OK) return s;
        smem = std::max(smem, I->h_inst.smem_bytes);
        any_unfused |= !I->h_inst.fused;
    }
    DeviceSweep &D = g_dev[o.device];
    std::lock_guard<std::mutex> lock(D.mu);
    SweepSlot *S = nullptr;
    dts_status s = acquire_slot(D, (size_t)n, &S);
    if (s != DTS_OK) return s;
    bool fast = true;  // the specialised loop applies to every instance (packed score rows)
    for (int32_t i = 0; i < n; i++) fast &= fast_mode(insts[i]->h_inst);
    for (int32_t i = 0; i < n; i++) {
        S->h_insts[i] = insts[ord[(size_t)i]]->h_inst;
        S->h_insts[i].hh = fast && !warp ? 1 : 0;
    }
    CK(cudaMemcpyAsync(S->d_insts, S->h_insts, sizeof(dts::Inst) * (size_t)n, cudaMemcpyHostToDevice, st),
       "H2D sweep");
    CK(cudaMemsetAsync(S->d_work, 0, 2 * sizeof(int), st), "memset");
    if (any_unfused) CK(dts::launch_init(S->d_insts, n, o.bus_bytes_per_s, work, st), "init");
    CK(cudaEventRecord(sev->loop_begin, st), "event");
    if (warp) {
        const int per = std::max(1, dts::warp_max_blocks_per_sm(smem));
        const int grid = (int)std::min<int64_t>((int64_t)n, (int64_t)per * nsm);
        CK(dts::launch_warp(S->d_insts, n, grid, S->d_work, smem, st), "loop (warp)");
    } else {
        const int per = std::max(1, fast ? dts::loop_max_blocks_per_sm_fast(block, smem)
                                         : dts::loop_max_blocks_per_sm(block, smem));
        const int grid = (int)std::min<int64_t>((int64_t)n, (int64_t)per * nsm);
        if (fast) CK(dts::launch_loop_fast(S->d_insts, n, block, grid, S->d_work, smem, st), "loop");
        else CK(dts::launch_loop(S->d_insts, n, block, grid, S->d_work, smem, st), "loop");
    }
    CK(cudaEventRecord(sev->loop_end, st), "event");
    CK(cudaEventRecord(S->done, st), "event");
    for (int32_t i = 0; i < n; i++) {
        insts[i]->sev = sev;
        insts[i]->ran = true;
        insts[i]->loop_kind = warp ? 3 : (fast ? 2 : 1);
    }
    return DTS_OK;
}

// A library stream on `device` for the j-th extra group of a multi-device sweep.
dts_status extra_stream(int device, size_t j, cudaStream_t *out) {
    DeviceSweep &D = g_dev[device];
    std::lock_guard<std::mutex> lock(D.mu);
    CK(cudaSetDevice(device), "cudaSetDevice");
    while (D.extra.size() <= j) {
        cudaStream_t s = nullptr;
        CK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking), "cudaStreamCreate");
        D.extra.push_back(s);
    }
    *out = D.extra[j];
    return DTS_OK;
}

}  // namespace

extern "C" {

dts_status dts_instance_upload(dts_instance *I, int32_t device, void *cuda_stream) {
    if (!I) return fail(DTS_E_INVAL, "instance is NULL");
    dts_status s = ensure_device(I, device);
    if (s != DTS_OK) return s;
    cudaStream_t st = (cudaStream_t)cuda_stream;
    return upload(I, st, true);
}

static dts_status run_multi_device(dts_instance *I, dts_policy policy, const dts_run_opts &o);
static dts_status run_one(dts_instance *I, dts_policy policy, const dts_run_opts &o);

dts_status dts_run(dts_instance *I, dts_policy policy, const dts_run_opts *opts) {
    if (!I) return fail(DTS_E_INVAL, "instance is NULL");
    dts_run_opts o;
    if (opts) o = *opts;
    else dts_run_opts_default(&o);
    dts_status s = check_opts(I, policy, &o);
    if (s != DTS_OK) return s;
    s = check_device(o.device);
    if (s != DTS_OK) return s;
    if (o.n_devices < 0 || o.n_devices > dts::MAX_G) return fail(DTS_E_INVAL, "n_devices must be in [0, 64]");
    if (o.n_devices > 1) return run_multi_device(I, policy, o);
    if (!I->xs.empty()) {  // back to one device: drop the owned shards
        for (dts_instance *x : I->xs) delete x;
        I->xs.clear();
        I->xs_dev0 = -1;
        dts_shard_set(I, 1, 0);
    }
    return run_one(I, policy, o);
}

// One instance (or one task shard) on o.device, enqueued on o.cuda_stream.
static dts_status run_one(dts_instance *I, dts_policy policy, const dts_run_opts &o) {
    dts_status s;
    if (I->G > 1 && !I->connected)
        return fail(DTS_E_STATE, "task shard not connected (dts_shard_connect) -- or use dts_shard_group_run");
    if (I->G > 1 && I->device != o.device) return fail(DTS_E_INVAL, "task shard: opts.device != exported device");
    cudaStream_t st = (cudaStream_t)o.cuda_stream;
    const int budget = budget_of(o);
    const int block = o.block_threads ? o.block_threads : auto_block(I, true);
    const bool warp = warp_eligible(I, policy, o) && warp_solo(I);
    s = stage(I, policy, o, budget, block, st, true, true, warp);
    if (s != DTS_OK) return s;
    const int64_t work = std::max<int64_t>((int64_t)I->m_pad, (int64_t)I->n + 4);
    if (!I->h_inst.fused) CK(dts::launch_init(I->d_inst, 1, o.bus_bytes_per_s, work, st), "init");
    CK(cudaMemsetAsync(I->d_work, 0, sizeof(int) * 16, st), "memset");
    CK(cudaEventRecord(I->ev[1], st), "event");
    I->loop_kind = warp ? 3 : (fast_mode(I->h_inst) ? 2 : 1);
    if (warp)
        CK(dts::launch_warp(I->d_inst, 1, 1, I->d_work, I->h_inst.smem_bytes, st), "loop (warp)");
    else if (fast_mode(I->h_inst))
        CK(dts::launch_loop_fast(I->d_inst, 1, block, 1, I->d_work, I->h_inst.smem_bytes, st), "loop");
    else
        CK(dts::launch_loop(I->d_inst, 1, block, 1, I->d_work, I->h_inst.smem_bytes, st), "loop");
    CK(cudaEventRecord(I->ev[2], st), "event");
    CK(cudaEventRecord(I->ev[3], st), "event");
    I->ran = true;
    return DTS_OK;
}

dts_status dts_sweep_run(dts_instance *const *insts, int32_t n, dts_policy policy, const dts_run_opts *opts,
                         const int32_t *devices, int32_t n_devices) {
    if (n < 0 || (n > 0 && !insts)) return fail(DTS_E_INVAL, "insts");
    if (n_devices < 0 || (n_devices > 0 && !devices)) return fail(DTS_E_INVAL, "devices");
    if (n == 0) return DTS_OK;
    dts_run_opts o;
    if (opts) o = *opts;
    else dts_run_opts_default(&o);
    dts_status s = check_device(o.device);
    if (s != DTS_OK) return s;
    for (int32_t g = 0; g < n_devices; g++)
        if ((s = check_device(devices[g])) != DTS_OK) return s;
    std::vector<dts_instance *> seen(insts, insts + n);
    std::sort(seen.begin(), seen.end());
    if (std::adjacent_find(seen.begin(), seen.end()) != seen.end())
        return fail(DTS_E_INVAL, "instance listed twice");
    for (int32_t i = 0; i < n; i++) {
        if (!insts[i]) return fail(DTS_E_INVAL, "instance is NULL");
        s = check_opts(insts[i], policy, &o);
        if (s != DTS_OK) return s;
        if (insts[i]->G > 1) return fail(DTS_E_INVAL, "a task shard cannot be part of a sweep");
    }
    cudaStream_t st = (cudaStream_t)o.cuda_stream;
    if (n_devices == 0) return sweep_on_device(insts, n, policy, o, st);

    // Several devices (independent instances, no
    // communication): LPT over the device list on the chain-cost estimate,
    // longest first, each to the least loaded entry (lower index on ties).
    // Entry g runs ONE batched launch on devices[g]; the first entry on
    // opts->device uses the caller's stream, the others library streams
    // forked from it and joined back into it (cross-device event waits).
    std::vector<int32_t> ord((size_t)n);
    for (int32_t i = 0; i < n; i++) ord[(size_t)i] = i;
    std::stable_sort(ord.begin(), ord.end(),
                     [&](int32_t a, int32_t b) { return instance_cost(insts[a]) > instance_cost(insts[b]); });
    std::vector<double> load((size_t)n_devices, 0.0);
    std::vector<std::vector<dts_instance *>> part((size_t)n_devices);
    for (int32_t i : ord) {
        size_t g = 0;
        for (size_t q = 1; q < load.size(); q++)
            if (load[q] < load[g]) g = q;
        load[g] += instance_cost(insts[i]);
        part[g].push_back(insts[i]);
    }
    CK(cudaSetDevice(o.device), "cudaSetDevice");
    cudaEvent_t fork = nullptr;
    CK(cudaEventCreateWithFlags(&fork, cudaEventDisableTiming), "cudaEventCreate");
    CK(cudaEventRecord(fork, st), "event");
    std::vector<cudaEvent_t> joins;
    std::vector<int> used((size_t)64, 0);  // library streams taken per device
    bool caller_taken = false;
    dts_status rs = DTS_OK;
    for (int32_t g = 0; g < n_devices && rs == DTS_OK; g++) {
        if (part[(size_t)g].empty()) continue;
        const int d = devices[g];
        dts_run_opts od = o;
        od.device = d;
        cudaStream_t sg = st;
        const bool on_caller = d == o.device && !caller_taken;
        if (on_caller) {
            caller_taken = true;
        } else {
            if ((rs = extra_stream(d, (size_t)used[(size_t)d]++, &sg)) != DTS_OK) break;
            CK(cudaSetDevice(d), "cudaSetDevice");
            CK(cudaStreamWaitEvent(sg, fork, 0), "wait");
        }
        od.cuda_stream = sg;
        rs = sweep_on_device(part[(size_t)g].data(), (int32_t)part[(size_t)g].size(), policy, od, sg);
        if (rs != DTS_OK) break;
        if (!on_caller) {
            cudaEvent_t j = nullptr;
            CK(cudaSetDevice(d), "cudaSetDevice");
            CK(cudaEventCreateWithFlags(&j, cudaEventDisableTiming), "cudaEventCreate");
            CK(cudaEventRecord(j, sg), "event");
            joins.push_back(j);
        }
    }
    CK(cudaSetDevice(o.device), "cudaSetDevice");
    for (cudaEvent_t j : joins) {
        CK(cudaStreamWaitEvent(st, j, 0), "wait");
        cudaEventDestroy(j);  // released once it has completed
    }
    cudaEventDestroy(fork);
    return rs;
}

}  // extern "C"

// ---------------------------------------------------------------- task shards
namespace {

// Consecutive task ranges with about E/G edges each (§8(e)); the last shard
// ends at m.
void shard_bounds(const dts_instance *I, int32_t G, int32_t g, int32_t *lo, int32_t *hi) {
    auto start = [&](int32_t q) -> int32_t {
        if (q <= 0) return 0;
        if (q >= G) return I->m;
        const int64_t E = I->E_raw;
        if (E == 0) return (int32_t)((int64_t)I->m * q / G);
        const int64_t target = (E * q + G - 1) / G;
        return (int32_t)(std::lower_bound(I->task_ptr.begin(), I->task_ptr.begin() + I->m, target) -
                         I->task_ptr.begin());
    };
    *lo = start(g);
    *hi = g == G - 1 ? I->m : std::max(*lo, start(g + 1));
}

constexpr uint32_t SHARD_MAGIC = 0x48535444u;  // "DTSH"
struct ShardHandle {
    cudaIpcMemHandle_t mem;      // the shard's device arena
    int64_t off_epoch, off_box, off_h, off_h2, off_u;
    int32_t G, g;
    int64_t box_bytes;
    uint32_t magic, pad;
};
static_assert(sizeof(ShardHandle) <= DTS_SHARD_HANDLE_BYTES, "handle size");

dts::ShardPeer own_peer(const dts_instance *I) {
    dts::ShardPeer p;
    p.epoch = I->d_epoch;
    p.box = I->d_box;
    p.h = I->h_inst.h;
    p.h2 = I->h_inst.h2;
    p.u = I->h_inst.u;
    return p;
}

dts_status write_peers(dts_instance *I, const std::vector<dts::ShardPeer> &tab) {
    CK(cudaSetDevice(I->device), "cudaSetDevice");
    CK(cudaMemcpy(I->d_peers, tab.data(), sizeof(dts::ShardPeer) * tab.size(), cudaMemcpyHostToDevice),
       "H2D peers");
    I->connected = true;
    return DTS_OK;
}

}  // namespace

extern "C" {

dts_status dts_shard_set(dts_instance *I, int32_t G, int32_t g) {
    if (!I) return fail(DTS_E_INVAL, "instance is NULL");
    if (G < 1 || G > dts::MAX_G) return fail(DTS_E_UNSUPPORTED, "G must be in [1, 64]");
    if (g < 0 || g >= G) return fail(DTS_E_INVAL, "g must be in [0, G)");
    for (void *p : I->ipc_open) cudaIpcCloseMemHandle(p);
    I->ipc_open.clear();
    I->G = G;
    I->g = g;
    shard_bounds(I, G, g, &I->t_lo, &I->t_hi);
    I->connected = false;
    return DTS_OK;
}

dts_status dts_shard_range(const dts_instance *I, int32_t *t_lo, int32_t *t_hi) {
    if (!I || !t_lo || !t_hi) return fail(DTS_E_INVAL, "NULL argument");
    *t_lo = I->G > 1 ? I->t_lo : 0;
    *t_hi = I->G > 1 ? I->t_hi : I->m;
    return DTS_OK;
}

dts_status dts_shard_export(dts_instance *I, int32_t device, void *handle) {
    if (!I || !handle) return fail(DTS_E_INVAL, "NULL argument");
    if (I->G < 2) return fail(DTS_E_STATE, "not a task shard (dts_shard_set with G >= 2 first)");
    dts_status s = ensure_device(I, device);
    if (s != DTS_OK) return s;
    ShardHandle hd;
    std::memset(&hd, 0, sizeof hd);
    CK(cudaIpcGetMemHandle(&hd.mem, I->ar.base), "cudaIpcGetMemHandle");
    I->exported = true;
    const char *b = I->ar.base;
    hd.off_epoch = (const char *)I->d_epoch - b;
    hd.off_box = (const char *)I->d_box - b;
    hd.off_h = (const char *)I->h_inst.h - b;
    hd.off_h2 = (const char *)I->h_inst.h2 - b;
    hd.off_u = (const char *)I->h_inst.u - b;
    hd.G = I->G;
    hd.g = I->g;
    hd.box_bytes = I->box_bytes;
    hd.magic = SHARD_MAGIC;
    std::memset(handle, 0, DTS_SHARD_HANDLE_BYTES);
    std::memcpy(handle, &hd, sizeof hd);
    return DTS_OK;
}

dts_status dts_shard_connect(dts_instance *I, const void *handles) {
    if (!I || !handles) return fail(DTS_E_INVAL, "NULL argument");
    if (I->G < 2 || !I->ar.base) return fail(DTS_E_STATE, "dts_shard_export first");
    CK(cudaSetDevice(I->device), "cudaSetDevice");
    // a new connection starts every shard's exchange numbers at 0 (the caller
    // makes all ranks connect before any of them runs: include/dts.h)
    CK(cudaDeviceSynchronize(), "sync");
    CK(cudaMemset(I->d_epoch, 0, 256), "memset epoch");
    CK(cudaDeviceSynchronize(), "sync");
    I->runs = 0;
    for (void *p : I->ipc_open) cudaIpcCloseMemHandle(p);
    I->ipc_open.clear();
    std::vector<dts::ShardPeer> tab((size_t)I->G);
    for (int32_t p = 0; p < I->G; p++) {
        ShardHandle hd;
        std::memcpy(&hd, (const char *)handles + (size_t)p * DTS_SHARD_HANDLE_BYTES, sizeof hd);
        if (hd.magic != SHARD_MAGIC || hd.G != I->G || hd.g != p || hd.box_bytes != I->box_bytes)
            return fail(DTS_E_INVAL, "shard handle " + std::to_string(p) + " does not match this instance");
        if (p == I->g) {
            tab[(size_t)p] = own_peer(I);
            continue;
        }
        void *base = nullptr;
        CK(cudaIpcOpenMemHandle(&base, hd.mem, cudaIpcMemLazyEnablePeerAccess), "cudaIpcOpenMemHandle");
        I->ipc_open.push_back(base);
        char *c = (char *)base;
        tab[(size_t)p].epoch = (unsigned long long *)(c + hd.off_epoch);
        tab[(size_t)p].box = (unsigned char *)(c + hd.off_box);
        tab[(size_t)p].h = (const int32_t *)(c + hd.off_h);
        tab[(size_t)p].h2 = (const int32_t *)(c + hd.off_h2);
        tab[(size_t)p].u = (const int32_t *)(c + hd.off_u);
    }
    I->xsys = true;
    return write_peers(I, tab);
}

dts_status dts_shard_group_run(dts_instance *const *shards, int32_t G, dts_policy policy,
                               const dts_run_opts *opts) {
    if (G < 1 || G > dts::MAX_G || !shards) return fail(DTS_E_INVAL, "G must be in [1, 64]");
    dts_run_opts o;
    if (opts) o = *opts;
    else dts_run_opts_default(&o);
    dts_status s = check_device(o.device);
    if (s != DTS_OK) return s;
    std::vector<dts_instance *> seen(shards, shards + G);
    std::sort(seen.begin(), seen.end());
    if (std::adjacent_find(seen.begin(), seen.end()) != seen.end()) return fail(DTS_E_INVAL, "shard listed twice");
    int block = 32;
    int64_t work = 1;
    for (int32_t i = 0; i < G; i++) {
        dts_instance *I = shards[i];
        if (!I) return fail(DTS_E_INVAL, "shard is NULL");
        if (I->m != shards[0]->m || I->n != shards[0]->n || I->K != shards[0]->K || I->E_raw != shards[0]->E_raw)
            return fail(DTS_E_INVAL, "shards must hold the same instance");
        s = check_opts(I, policy, &o);
        if (s != DTS_OK) return s;
        if (I->G != G || I->g != i || (G > 1 && !I->connected) || I->device != o.device) {
            s = dts_shard_set(I, G, i);
            if (s != DTS_OK) return s;
            s = ensure_device(I, o.device);
            if (s != DTS_OK) return s;
        }
        block = std::max(block, auto_block(I));
        work = std::max<int64_t>(work, std::max<int64_t>(I->m_pad, (int64_t)I->n * I->K));
    }
    if (G > 1 && !shards[0]->connected) {  // same device: the peers' own pointers
        std::vector<dts::ShardPeer> tab((size_t)G);
        for (int32_t p = 0; p < G; p++) tab[(size_t)p] = own_peer(shards[p]);
        for (int32_t i = 0; i < G; i++) {
            s = write_peers(shards[i], tab);
            if (s != DTS_OK) return s;
            shards[i]->xsys = false;
        }
    }
    if (o.block_threads) block = o.block_threads;
    cudaStream_t st = (cudaStream_t)o.cuda_stream;
    const int budget = budget_of(o);
    // one exchange-number range for the whole group: above every shard's last
    uint64_t runs = 0;
    for (int32_t i = 0; i < G; i++) runs = std::max(runs, shards[i]->runs);
    int smem = 0;
    for (int32_t i = 0; i < G; i++) {
        shards[i]->runs = runs;
        s = stage(shards[i], policy, o, budget, block, st, false);
        if (s != DTS_OK) return s;
        smem = std::max(smem, shards[i]->h_inst.smem_bytes);
    }
    DeviceSweep &D = g_dev[o.device];
    std::lock_guard<std::mutex> lock(D.mu);
    SweepSlot *S = nullptr;
    s = acquire_slot(D, (size_t)G, &S);
    if (s != DTS_OK) return s;
    for (int32_t i = 0; i < G; i++) S->h_insts[i] = shards[i]->h_inst;
    CK(cudaMemcpyAsync(S->d_insts, S->h_insts, sizeof(dts::Inst) * (size_t)G, cudaMemcpyHostToDevice, st),
       "H2D shards");
    CK(cudaMemsetAsync(S->d_work, 0, sizeof(int), st), "memset");
    CK(dts::launch_init(S->d_insts, G, o.bus_bytes_per_s, work, st), "init");
    for (int32_t i = 0; i < G; i++) CK(cudaEventRecord(shards[i]->ev[1], st), "event");
    // the G shards exchange inside the kernel: they must be co-resident
    CK(dts::launch_loop_coop(S->d_insts, G, block, S->d_work, smem, st), "loop (cooperative)");
    CK(cudaEventRecord(S->done, st), "event");
    for (int32_t i = 0; i < G; i++) {
        CK(cudaEventRecord(shards[i]->ev[2], st), "event");
        CK(cudaEventRecord(shards[i]->ev[3], st), "event");
        shards[i]->ran = true;
        shards[i]->loop_kind = 1;  // task shards: the generic loop
    }
    return DTS_OK;
}


// dts_run with opts.n_devices = G > 1: the instance is
// task-sharded over G shards in this process -- shard 0 is the instance
// itself, shards 1..G-1 are copies it owns -- shard j on device
// (opts.device + j) mod #devices, each ONE CTA that exchanges with its peers
// through their memory (peer access / UVA; system-scope release/acquire when
// the shards span devices), launched on its device's library stream forked
// from and joined back into opts.cuda_stream.  Every shard computes the whole
// schedule; dts_result(inst) reads shard 0's.
static dts_status run_multi_device(dts_instance *I, dts_policy policy, const dts_run_opts &o) {
    const int32_t G = o.n_devices;
    int ndev = 0;
    CK(cudaGetDeviceCount(&ndev), "cudaGetDeviceCount");
    if (I->G > 1 && I->xs.empty()) return fail(DTS_E_INVAL, "an exported task shard cannot run with n_devices");
    auto dev_of = [&](int32_t j) { return (o.device + j) % ndev; };
    dts_status s;
    if ((int32_t)I->xs.size() != G - 1 || I->xs_dev0 != o.device) {
        for (dts_instance *x : I->xs) delete x;
        I->xs.clear();
        for (int32_t j = 1; j < G; j++) {
            dts_instance *x = new (std::nothrow) dts_instance();
            if (!x) return fail(DTS_E_NOMEM, "host allocation");
            x->m = I->m; x->n = I->n; x->K = I->K; x->E_raw = I->E_raw; x->cap = I->cap;
            x->default_ns = I->default_ns; x->task_ptr = I->task_ptr; x->task_data = I->task_data;
            x->size = I->size; x->task_ns = I->task_ns; x->has_tau = I->has_tau;
            x->max_deg_ub = I->max_deg_ub; x->max_row_len = I->max_row_len; x->uniform_size = I->uniform_size;
            x->max_row_bytes = I->max_row_bytes; x->min_size = I->min_size; x->res_cap = I->res_cap;
            x->m_pad = I->m_pad;
            I->xs.push_back(x);
        }
        std::vector<dts_instance *> sh((size_t)G);
        sh[0] = I;
        for (int32_t j = 1; j < G; j++) sh[(size_t)j] = I->xs[(size_t)j - 1];
        bool cross = false;
        for (int32_t j = 0; j < G; j++) {
            if ((s = dts_shard_set(sh[(size_t)j], G, j)) != DTS_OK) return s;
            if ((s = ensure_device(sh[(size_t)j], dev_of(j))) != DTS_OK) return s;
            cross |= dev_of(j) != o.device;
        }
        for (int32_t a = 0; a < G && cross; a++)  // every pair of distinct devices maps each other
            for (int32_t b = 0; b < G; b++) {
                if (dev_of(a) == dev_of(b)) continue;
                CK(cudaSetDevice(dev_of(a)), "cudaSetDevice");
                const cudaError_t e = cudaDeviceEnablePeerAccess(dev_of(b), 0);
                if (e != cudaSuccess && e != cudaErrorPeerAccessAlreadyEnabled)
                    return cuda_fail(e, "cudaDeviceEnablePeerAccess");
                cudaGetLastError();
            }
        std::vector<dts::ShardPeer> tab((size_t)G);
        for (int32_t j = 0; j < G; j++) tab[(size_t)j] = own_peer(sh[(size_t)j]);
        for (int32_t j = 0; j < G; j++) {  // a new group: exchange numbers from 0 on every shard
            dts_instance *x = sh[(size_t)j];
            CK(cudaSetDevice(x->device), "cudaSetDevice");
            CK(cudaDeviceSynchronize(), "sync");
            CK(cudaMemset(x->d_epoch, 0, 256), "memset epoch");
            CK(cudaDeviceSynchronize(), "sync");
            x->runs = 0;
            if ((s = write_peers(x, tab)) != DTS_OK) return s;
            x->xsys = cross;
        }
        I->xs_dev0 = o.device;
    }
    CK(cudaSetDevice(o.device), "cudaSetDevice");
    cudaStream_t st = (cudaStream_t)o.cuda_stream;
    cudaEvent_t fork = nullptr;
    CK(cudaEventCreateWithFlags(&fork, cudaEventDisableTiming), "cudaEventCreate");
    CK(cudaEventRecord(fork, st), "event");
    std::vector<std::pair<int, cudaEvent_t>> joins;
    s = DTS_OK;
    for (int32_t j = 0; j < G && s == DTS_OK; j++) {
        dts_instance *x = j == 0 ? I : I->xs[(size_t)j - 1];
        dts_run_opts oj = o;
        oj.device = dev_of(j);
        oj.n_devices = 1;
        cudaStream_t sj = st;
        if (j > 0) {  // shards must run concurrently: one library stream each
            if ((s = extra_stream(oj.device, (size_t)j, &sj)) != DTS_OK) break;
            CK(cudaSetDevice(oj.device), "cudaSetDevice");
            CK(cudaStreamWaitEvent(sj, fork, 0), "wait");
        }
        oj.cuda_stream = sj;
        if ((s = run_one(x, policy, oj)) != DTS_OK) break;
        if (j > 0) {
            cudaEvent_t e = nullptr;
            CK(cudaSetDevice(oj.device), "cudaSetDevice");
            CK(cudaEventCreateWithFlags(&e, cudaEventDisableTiming), "cudaEventCreate");
            CK(cudaEventRecord(e, sj), "event");
            joins.emplace_back(oj.device, e);
        }
    }
    CK(cudaSetDevice(o.device), "cudaSetDevice");
    for (auto &je : joins) {
        CK(cudaStreamWaitEvent(st, je.second, 0), "wait");
        cudaEventDestroy(je.second);
    }
    cudaEventDestroy(fork);
    return s;
}

// Result copies in two phases so that many instances share the waits
// (dts_fetch_results): the scalars first (they size the rest), then the arrays.
static dts_status fetch_out(dts_instance *I) {
    CK(cudaSetDevice(I->device), "cudaSetDevice");
    CK(cudaMemcpyAsync(I->r_out, I->h_inst.out, sizeof I->out, cudaMemcpyDeviceToHost, I->stream), "D2H out");
    return DTS_OK;
}
static dts_status fetch_arrays(dts_instance *I) {
    I->out = *I->r_out;
    if (I->out.error == 2) return fail(DTS_E_STATE, "task shards: a peer did not reach an exchange in time");
    if (I->out.error == 3) return fail(DTS_E_STATE, "device loop: plannedTasks inconsistent (internal)");
    if (I->out.error == 9) return fail(DTS_E_STATE, "device loop: a bounds check failed (profiling build)");
    if (I->out.error) return fail(DTS_E_STATE, "device loop: LUF found no victim");
    const dts::Inst &h = I->h_inst;
    const size_t ne = (size_t)std::min<int64_t>(I->out.n_events, h.ev_cap);
    cudaStream_t st = I->stream;  // the run's stream: the copies follow the run
    CK(cudaSetDevice(I->device), "cudaSetDevice");
    // one copy: sigma, service order, task times, then the used part of the trace
    const size_t head = (size_t)(reinterpret_cast<const char *>(h.events) - reinterpret_cast<const char *>(h.gpu_task_ptr));
    CK(cudaMemcpyAsync(I->h_res, h.gpu_task_ptr, head + sizeof(dts_event) * ne, cudaMemcpyDeviceToHost, st), "D2H");
    I->r_n_events = (int64_t)ne;
    return DTS_OK;
}
static dts_status fetch_done(dts_instance *I) {
    if (I->sev) {
        CK(cudaEventElapsedTime(&I->loop_ms, I->sev->loop_begin, I->sev->loop_end), "elapsed");
        CK(cudaEventElapsedTime(&I->total_ms, I->sev->begin, I->sev->loop_end), "elapsed");
    } else {
        CK(cudaEventElapsedTime(&I->loop_ms, I->ev[1], I->ev[2]), "elapsed");
        CK(cudaEventElapsedTime(&I->total_ms, I->ev[0], I->ev[3]), "elapsed");
    }
    I->have_host = true;
    return DTS_OK;
}
// Wait for every distinct (device, stream) of the list once.
static dts_status sync_streams(dts_instance *const *insts, int32_t n) {
    std::vector<std::pair<int, cudaStream_t>> seen;
    for (int32_t i = 0; i < n; i++) {
        const std::pair<int, cudaStream_t> key(insts[i]->device, insts[i]->stream);
        if (insts[i]->have_host || std::find(seen.begin(), seen.end(), key) != seen.end()) continue;
        seen.push_back(key);
        CK(cudaSetDevice(key.first), "cudaSetDevice");
        CK(cudaStreamSynchronize(key.second), "D2H sync");
    }
    return DTS_OK;
}

dts_status dts_fetch_results(dts_instance *const *insts, int32_t n) {
    if (n < 0 || (n > 0 && !insts)) return fail(DTS_E_INVAL, "insts");
    for (int32_t i = 0; i < n; i++) {
        if (!insts[i]) return fail(DTS_E_INVAL, "instance is NULL");
        if (!insts[i]->ran) return fail(DTS_E_STATE, "dts_fetch_results before dts_run");
    }
    dts_status s;
    for (int32_t i = 0; i < n; i++)
        if (!insts[i]->have_host && (s = fetch_out(insts[i])) != DTS_OK) return s;
    if ((s = sync_streams(insts, n)) != DTS_OK) return s;
    for (int32_t i = 0; i < n; i++)
        if (!insts[i]->have_host && (s = fetch_arrays(insts[i])) != DTS_OK) return s;
    if ((s = sync_streams(insts, n)) != DTS_OK) return s;
    for (int32_t i = 0; i < n; i++)
        if (!insts[i]->have_host && (s = fetch_done(insts[i])) != DTS_OK) return s;
    return DTS_OK;
}

dts_status dts_run_times(dts_instance *I, float *loop_ms, float *total_ms) {
    if (!I || !loop_ms || !total_ms) return fail(DTS_E_INVAL, "NULL argument");
    if (!I->ran) return fail(DTS_E_STATE, "dts_run_times before dts_run");
    CK(cudaSetDevice(I->device), "cudaSetDevice");
    cudaEvent_t b = I->sev ? I->sev->loop_begin : I->ev[1], e = I->sev ? I->sev->loop_end : I->ev[2];
    cudaEvent_t b0 = I->sev ? I->sev->begin : I->ev[0];
    CK(cudaEventSynchronize(e), "loop event");
    CK(cudaEventElapsedTime(loop_ms, b, e), "elapsed");
    CK(cudaEventElapsedTime(total_ms, b0, e), "elapsed");
    return DTS_OK;
}

dts_status dts_result(dts_instance *I, dts_result_view *v) {
    if (!I || !v) return fail(DTS_E_INVAL, "NULL argument");
    if (!I->ran) return fail(DTS_E_STATE, "dts_result before dts_run");
    if (!I->have_host) {
        dts_instance *one[1] = {I};
        dts_status s = dts_fetch_results(one, 1);
        if (s != DTS_OK) return s;
    }
    std::memset(v, 0, sizeof *v);
    v->K = I->K;
    v->n_tasks = I->m;
    v->gpu_task_ptr = I->r_gpu_ptr;
    v->gpu_task_ids = I->r_gpu_ids;
    v->serve_gpu = I->r_serve_gpu;
    v->serve_task = I->r_serve_task;
    v->task_start_ns = I->r_tstart;
    v->task_end_ns = I->r_tend;
    v->n_events = I->r_n_events;
    v->events = I->r_events;
    v->bytes_loaded = I->out.bytes_loaded;
    v->n_loads = I->out.n_loads;
    v->n_evictions = I->out.n_evictions;
    v->makespan_ns = I->out.makespan;
    v->makespan_s = (double)I->out.makespan * 1e-9;
    v->n_served = I->out.n_served;
    v->n_scans = I->out.n_scans;
    v->n_fallback2 = I->out.n_fallback2;
    v->n_fallback_first = I->out.n_fallback_first;
    v->n_belady = I->out.n_belady;
    v->n_idle_requests = I->out.n_idle;
    v->n_verify_err = I->out.n_verify_err;
    v->alg_bytes = I->out.alg_bytes;
    v->scan_alg_bytes = I->out.scan_alg_bytes;
    for (int i = 0; i < 16; i++) v->prof_cycles[i] = I->out.prof[i];
    v->sum_avail_at_scans = I->out.sum_avail;
    v->n_allocations = I->out.n_alloc;
    v->sum_deg_loads_evictions = I->out.sum_deg;
    v->loop_kind = I->loop_kind;
    v->reserved = 0;
    v->loop_ms = I->loop_ms;
    v->total_ms = I->total_ms;
    return DTS_OK;
}

}  // extern "C"

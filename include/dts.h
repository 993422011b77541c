/*
 * dts.h -- C ABI of libdts: B200-native (sm_100a) DARTS+LUF memory-aware task
 * scheduling simulator.
 *
 * Method: Gonthier, Marchal, Thibault, "Memory-Aware Scheduling of Tasks
 * Sharing Data on Multiple GPUs with Dynamic Runtime Systems", IPDPS 2022.
 * Citations are to /root/reference/PAPER.md lines (section / algorithm).
 *
 * Problem (§III): m independent tasks T and n data D form a
 * bipartite graph; D(T) is the set of inputs of T.  K GPUs each hold at most
 * `mem_capacity_bytes` of data (M data when sizes are uniform).  A schedule
 * assigns each task to one GPU and orders it; before a task runs, its missing
 * inputs are loaded over a shared bus (Fig. 2), after evictions if needed
 * (PAPER.md:285-295).  The library computes the DARTS+LUF schedule:
 *   - DARTS data selection, Algorithm 5, with the
 *     "3inputs" fallback of §V-E, flag DTS_F_FALLBACK2;
 *   - LUF eviction, Algorithm 6;
 * deterministically (lowest-id tie-breaks, readings R1-R27 of DESIGN.md), and
 * returns the per-GPU task order sigma(k,i), the load/evict trace V(k,i), the
 * bytes transferred (Obj. 2) and the modelled makespan.
 *
 * Every step runs in CUDA kernels on one B200; there is no CPU fallback: a
 * missing or unusable GPU is reported as DTS_E_CUDA.
 *
 * Conventions
 *   - All ids are 0-based int32.  All times are integer nanoseconds.
 *   - Every function returns a dts_status; nothing aborts.  On error,
 *     dts_last_error() returns a thread-local message.
 *   - Ownership: dts_instance_create COPIES the caller's arrays (the caller
 *     keeps ownership of them).  Result views belong to the instance and stay
 *     valid until the next dts_run on it or dts_instance_destroy.
 *   - Thread safety: distinct instances may be used from distinct threads;
 *     one instance must not be used concurrently.
 */
#ifndef DTS_H
#define DTS_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct dts_instance dts_instance; /* opaque, owned by the library */

typedef enum {
    DTS_OK = 0,
    DTS_E_INVAL = -1,       /* malformed argument (pointer, range, monotonicity) */
    DTS_E_CAPACITY = -2,    /* capacity < max(1,W) (DARTS+LUF) or (W+1) (LRU policies)
                               * max_T sum_{D in D(T)} size(D) */
    DTS_E_NOMEM = -3,       /* host or device allocation failed */
    DTS_E_CUDA = -4,        /* CUDA error, no device, or device is not sm_100 */
    DTS_E_STATE = -5,       /* call out of order (e.g. dts_result before dts_run) */
    DTS_E_UNSUPPORTED = -6  /* outside the packed-state limits (see dts_instance_create) */
} dts_status;

typedef enum {
    DTS_POLICY_DARTS_LUF = 1, /* Alg. 5 + Alg. 6 */
    /* Comparison policies of the paper's evaluation, both
     * with StarPU's default LRU eviction: the resident datum (not an input of
     * the task being served) whose last use on the GPU is the oldest, lowest id
     * on ties; an LRU eviction leaves plannedTasks untouched, so a planned task
     * may reload data (the "domino effect"). */
    DTS_POLICY_DARTS_LRU = 2, /* "DARTS": Alg. 5 selection, LRU eviction */
    DTS_POLICY_EAGER_LRU = 3  /* "EAGER": one shared FIFO queue in submission order */
} dts_policy;

enum {
    /* "3inputs" fallback when no datum frees a task: load the datum that
     * makes the most tasks one load away.  Default ON. */
    DTS_F_FALLBACK2 = 1u << 0,
    /* Debug / parity mode: at every scan, recompute the
     * scores n_k(D), n2_k(D), u(D) and every task's missing count from their
     * definitions (a full pass over all tasks) and count disagreements with
     * the incremental state in dts_result_view.n_verify_err.  Slow. */
    DTS_F_VERIFY = 1u << 1,
    /* Diagnostic: build the CSR and initial state with the separate grid-wide
     * kernels even for small instances (default: the loop CTA of an instance
     * with <= 8 inputs per task and a small n builds them itself). */
    DTS_F_NOFUSE = 1u << 2,
    /* OPTI variant (§V-F): instead of the datum that frees
     * the most tasks, take the first one (ascending id) that frees at least
     * one.  Combines with DTS_F_FALLBACK2 ("DARTS+LUF+OPTI-3inputs"). */
    DTS_F_OPTI = 1u << 3,
    /* Diagnostic: keep the packed per-(simulated GPU, task) state word
     * (cnt:7 | xor:24, 4 K m bytes) even when every task has <= 3 inputs
     * (default then: no per-GPU task state, the missing inputs are read off
     * the task's row and the residency bitmaps). */
    DTS_F_PACKED = 1u << 4,
    /* Diagnostic: run the generic decision loop even when the one compiled for
     * the default mode applies (row-derived state, one shard, W = 0,
     * DARTS+LUF: every BASELINE config). */
    DTS_F_GENERIC = 1u << 5,
    /* Diagnostic: run a small instance on a CTA of the decision loop even
     * where the one-warp-per-instance loop applies (the default for instances
     * of <= 2 inputs per task in the mode above whose state fits a warp's
     * share of shared memory: C1, C2, the C5 sweep). */
    DTS_F_CTA = 1u << 6
};

typedef struct {
    uint32_t flags;           /* DTS_F_* ; default DTS_F_FALLBACK2 */
    uint32_t lookahead_W;     /* taskBuffer depth beyond the running task,
                                 0..8.  0 (default, the formal model of §III): a GPU asks
                                 for its next task when the current one ends.  W >= 1
                                 (StarPU's prefetch, readings R7 / R29): it keeps W tasks
                                 ahead -- asks when the (j-W+1)-th of its j tasks starts, the
                                 first W at once; LUF protects the inputs of every task not
                                 ended.  DARTS+LUF accepts a capacity of max(1, W) tasks'
                                 inputs: then Alg. 6's Belady branch can fire -- it evicts
                                 an input of the running task only (no future use), which
                                 leaves memory when that task ends (the load waits).
                                 W * (inputs per task) must be <= 128 */
    uint64_t bus_bytes_per_s; /* shared host->GPU bus bandwidth; default 12e9 (reading R9) */
    int32_t device;           /* CUDA device ordinal; default 0 */
    int32_t block_threads;    /* threads of the ONE CTA that runs an instance: a multiple of
                                 32 in [32, 512]; 0 = automatic */
    int32_t smem_budget;      /* bytes of shared memory per CTA for state placement
                                 (DESIGN.md "Data layout"); 0 = automatic (all that fits);
                                 -1 = none (every array in its global home) */
    int32_t n_devices;        /* dts_run only: G physical GPUs for ONE instance (SURVEY.md
                                 §8(e), second mode).  0 or 1 (default): one CTA on `device`.
                                 G > 1: the instance is task-sharded over G shards in this
                                 process, shard j on device (device + j) mod #devices (so a
                                 single-GPU machine runs all G on one device), exchanging
                                 through peer memory inside the kernel; the result is the
                                 same schedule.  The instance then owns G-1 shard copies
                                 (freed by a later run with n_devices <= 1 or destroy). */
    int64_t max_served;       /* stop after this many served tasks (prefix runs); -1 = all */
    void *cuda_stream;        /* cudaStream_t to enqueue on; NULL = the legacy default stream */
} dts_run_opts;

/* Fill *opts with the defaults above. */
void dts_run_opts_default(dts_run_opts *opts);

/* One entry of the load/evict trace.  32 bytes, naturally aligned.
 *   op 0 = LOAD : datum `data` crosses the shared bus to GPU `gpu` during
 *                 [t_ns, t_end_ns) (FIFO bus);
 *   op 1 = EVICT: datum `data` leaves GPU `gpu` memory at t_ns = t_end_ns
 *                 (Alg. 6 l.9);
 * `task` is the task whose service triggered the event (the task of step i
 * in V(k,i) / D(T_sigma(k,i))). */
typedef struct {
    int64_t t_ns, t_end_ns;
    int32_t gpu, data, task;
    uint8_t op;
    uint8_t pad[3];
} dts_event;

/* Create an instance from a task->data CSR.
 *   n_tasks, n_data : m >= 0, n >= 0; n < 2^24.
 *   task_ptr  [m+1] : host, task_ptr[0] = 0, non-decreasing.
 *   task_data [task_ptr[m]] : host, ids in [0, n).  Duplicates inside a row
 *                     are removed (D(T) is a set); at most
 *                     127 distinct inputs per task (else DTS_E_UNSUPPORTED).
 *   data_size [n]   : host, bytes, each > 0 (uniform sizes = the paper's
 *                     model; heterogeneous sizes = the extension of
 *                     PAPER.md:449-451, reading R11).
 *   task_ns   [m]   : host, task durations (>= 0) or NULL => default_task_ns.
 *   mem_capacity_bytes : per simulated GPU.
 *   K               : simulated GPUs, 1 <= K <= 64.
 *   out             : receives the new instance; destroy with dts_instance_destroy.
 * Host-only: validates and copies; no device work happens until dts_run. */
dts_status dts_instance_create(int32_t n_tasks, int32_t n_data, const int64_t *task_ptr,
                               const int32_t *task_data, const uint64_t *data_size,
                               const int64_t *task_ns, int64_t default_task_ns,
                               uint64_t mem_capacity_bytes, int32_t K, dts_instance **out);

/* Stage the instance's inputs (raw CSR, sizes, task times) on `device`: an
 * H2D copy on `cuda_stream` from the library's host copy, every call (so a
 * caller can time the host->device step).  dts_run uploads only if this
 * never happened, so after this call a run starts with its inputs resident
 * in HBM.  Allocates the instance's device arena on first use. */
dts_status dts_instance_upload(dts_instance *inst, int32_t device, void *cuda_stream);

/* Run the policy.  Enqueues on opts->cuda_stream: (upload if needed) -> CSR
 * build (sort/dedup rows, data->task transpose) -> state init -> the device-
 * resident decision loop -> result assembly.  Returns after enqueueing; the
 * results stay on the device until dts_result (which synchronises).
 * opts may be NULL (defaults).  DTS_E_CAPACITY if the capacity cannot hold
 * max(1, W) tasks' inputs for DARTS+LUF (Alg. 6's Belady branch then always
 * finds a victim, reading R29), (W+1) for the LRU policies. */
dts_status dts_run(dts_instance *inst, dts_policy policy, const dts_run_opts *opts);

typedef struct {
    int32_t K, n_tasks;
    const int64_t *gpu_task_ptr;   /* [K+1] offsets into gpu_task_ids                      */
    const int32_t *gpu_task_ids;   /* [n_served] sigma(k, .) for each k, in processing order */
    const int32_t *serve_gpu;      /* [n_served] GPU of the i-th served request (event order) */
    const int32_t *serve_task;     /* [n_served] task of the i-th served request              */
    const int64_t *task_start_ns;  /* [n_tasks], -1 if not served (prefix runs)               */
    const int64_t *task_end_ns;    /* [n_tasks]                                               */
    int64_t n_events;
    const dts_event *events;       /* [n_events] load/evict trace in event order              */
    uint64_t bytes_loaded;         /* sum of sizes of the LOAD events (Obj. 2 in bytes)       */
    int64_t n_loads, n_evictions;
    int64_t makespan_ns;           /* max task end                                            */
    double makespan_s;
    int64_t n_served;              /* served requests = decisions (reading R21)              */
    int64_t n_scans;               /* requests that found plannedTasks_k empty and got a task */
    int64_t n_fallback2, n_fallback_first, n_belady, n_idle_requests;
    int64_t n_verify_err;          /* DTS_F_VERIFY: disagreements found (0 = consistent)       */
    uint64_t alg_bytes;            /* algorithmic HBM bytes of the decision loop  */
    uint64_t scan_alg_bytes;       /* ... of which in the per-scan pass                       */
    float loop_ms;                 /* device time of the decision-loop kernel (CUDA events)  */
    float total_ms;                /* device time of the whole run (CSR build..assembly)     */
    int64_t prof_cycles[16];        /* diagnostics: SM cycles of the loop per phase (pop, argmax,
                                      plan, serve-with-loads, LUF, evict, load-update, other,
                                      pop-batch warp-0 phase, pop-batch rank phase, #batches, #pops) */
    /* Counters of the SURVEY.md §8(d) algorithmic-byte model (DESIGN.md
     * "Roofline"): bytes = 4 * sum_avail_at_scans + 4.125 * n * n_scans
     *                    + 12 * sum_deg_loads_evictions
     *                    + (4 K + 8 E / m) * n_allocations.
     * The oracle counts the same three quantities (parity-tested). */
    int64_t sum_avail_at_scans;      /* sum over scans of #unallocated tasks when the scan began */
    int64_t n_allocations;           /* tasks leaving the shared pool (plans, fallback / EAGER picks) */
    int64_t sum_deg_loads_evictions; /* sum of deg(D) over every LOAD and EVICT event            */
    int32_t loop_kind;               /* which decision loop ran: 1 = the generic
                                        per-CTA loop, 2 = the per-CTA loop specialised to the
                                        default mode, 3 = the one-warp-per-instance loop */
    int32_t reserved;
} dts_result_view;

/* Synchronise on the run's stream, copy the results to host (once) and fill *out. */
dts_status dts_result(dts_instance *inst, dts_result_view *out);

/* Device times of the instance's last run (CUDA events on the run's stream):
 * *loop_ms = the decision-loop kernel launch (for a batched launch: the whole
 * batch's loop launch), *total_ms = from the first enqueued step (CSR build)
 * to the end of that launch.  Waits for the loop to finish; copies no result.
 * DTS_E_STATE before any dts_run. */
dts_status dts_run_times(dts_instance *inst, float *loop_ms, float *total_ms);

/* Copy the results of insts[0..n) to host in two batched phases -- every
 * instance's scalars, one wait per distinct stream, then every instance's
 * arrays, one more wait per stream -- instead of two waits per instance.
 * dts_result on these instances then returns without device work.  The
 * instances must have run (DTS_E_STATE otherwise); the first failing
 * instance's status is returned. */
dts_status dts_fetch_results(dts_instance *const *insts, int32_t n);

/* Sweep (BASELINE config 5) / batch of independent instances (SURVEY.md
 * §8(e): instances share nothing, so they shard over devices with no
 * communication).
 *   insts[0..n)  : distinct instances (none of them a task shard); each gets
 *                  the same policy and options; results are read per
 *                  instance with dts_result / dts_fetch_results.
 *   devices      : NULL or n_devices CUDA ordinals (repeats allowed: two
 *                  entries naming one device give two concurrent launches on
 *                  it).  NULL / n_devices = 0: everything on opts->device.
 *                  Otherwise the instances are split over the entries by LPT
 *                  on a chain-cost estimate (m * mean degree), longest first,
 *                  each to the least loaded entry.
 * Per device entry: ONE batched launch of the decision loop, one CTA per
 * instance (<= 128 threads when the batch has many more instances than SMs,
 * so several chains share an SM), CTAs pulling instances longest-first from
 * that launch's own device counter; every launch has its own descriptor buffer,
 * so concurrent sweeps on different streams or threads do not interfere.
 * The first entry on opts->device is enqueued on opts->cuda_stream; the
 * others on library streams of their devices, forked from and joined back
 * into opts->cuda_stream (so a synchronisation of that stream covers the
 * whole sweep).  Returns after enqueueing.
 * Errors: DTS_E_INVAL (NULL / repeated instance, bad device list, a task
 * shard in the list), DTS_E_CUDA, DTS_E_CAPACITY / DTS_E_UNSUPPORTED as for
 * dts_run (checked for every instance before anything is enqueued). */
dts_status dts_sweep_run(dts_instance *const *insts, int32_t n, dts_policy policy,
                         const dts_run_opts *opts, const int32_t *devices, int32_t n_devices);

/* ---- Task-sharded single instance (second mode) ----------
 * One instance whose tasks are split into G consecutive id ranges with about
 * E/G edges each; shard g keeps the packed state, the data->task edges and
 * PARTIAL scores n_k(D), n2_k(D), u(D) of its own tasks, and every decision of
 * Alg. 5 / Alg. 6 is replicated on all shards from the
 * exchanged values: per scan, a reduce-scatter of the partial scores by datum
 * slice plus the max of the G slice keys (the "allreduce + argmax" of the
 * north_star, done inside the kernel through the shards' memory); per plan,
 * one exchange of each shard's part of plannedTasks_k (Alg. 5 l.10); per
 * fallback pick (Alg. 5 l.13, 3inputs), one min-exchange.  The schedule is
 * the same as dts_run's on the whole instance, bit for bit; every shard's
 * dts_result returns all of it.
 *
 * Multi-GPU (one process per B200): every rank creates the SAME instance,
 *   dts_shard_set(inst, G, rank); dts_shard_export(inst, device, my_handle);
 *   all-gather the handles (any transport, rank order);
 *   dts_shard_connect(inst, all_handles);  then each run: dts_run(inst, ...)
 *   on every rank concurrently (each launches one CTA that exchanges with its
 *   peers over NVLink through CUDA IPC mappings; a peer missing for 5 s ends
 *   the run with DTS_E_STATE from dts_result instead of a hang).
 * One device: dts_shard_group_run runs G shards as G co-resident CTAs. */
#define DTS_SHARD_HANDLE_BYTES 128

/* Make `inst` shard g of G (G = 1: the whole instance).  Host only. */
dts_status dts_shard_set(dts_instance *inst, int32_t G, int32_t g);
/* The task range [*t_lo, *t_hi) the instance owns. */
dts_status dts_shard_range(const dts_instance *inst, int32_t *t_lo, int32_t *t_hi);
/* Allocate the shard's device state on `device` and write its IPC handle
 * (DTS_SHARD_HANDLE_BYTES bytes) to `handle`. */
dts_status dts_shard_export(dts_instance *inst, int32_t device, void *handle);
/* Map the peers' state: `handles` = G handles in shard order (this shard's
 * own included, ignored).  Resets this shard's exchange numbers: every rank
 * must finish dts_shard_connect (a barrier) before any rank runs, and the
 * ranks then call dts_run the same number of times.  Needs every peer alive
 * (exported) at this call. */
dts_status dts_shard_connect(dts_instance *inst, const void *handles);
/* One device: shards[i] becomes shard i of G (same instance in every entry)
 * and all G run in ONE cooperative launch on opts->device. */
dts_status dts_shard_group_run(dts_instance *const *shards, int32_t G, dts_policy policy,
                               const dts_run_opts *opts);

void dts_instance_destroy(dts_instance *inst);
const char *dts_status_str(dts_status s);
const char *dts_last_error(void);

/* Number of CUDA kernels libdts has launched in this process so far
 * (monotone; the difference around a region = the library's launches in it). */
uint64_t dts_kernel_launches(void);

/* ABI version: (major << 16) | minor. */
uint32_t dts_version(void);

#ifdef __cplusplus
}
#endif
#endif /* DTS_H */

/*
 * svp.h -- C-ABI of libsvp, the B200-native SigmaVP multiplexer.
 *
 * SigmaVP (Jung & Carloni, DAC'15) lets many virtual platforms (VPs) -- simulated
 * embedded devices with virtual GPUs -- run their GPU kernels on the host GPUs
 * ("multiplexes the host GPUs ... by using separate streams for each VP",
 * PAPER.md L199-206, §2).  The host side (Fig 2, text L231-257) is
 * a Job Queue fed by the VPs, a Kernel Match that finds identical kernel requests,
 * a Re-scheduler that reorders jobs (Kernel Interleaving) and merges identical ones
 * (Kernel Coalescing), a Job Dispatcher that invokes the physical GPUs, and a
 * Profiler.  This header is that pipeline's boundary:
 *
 *   svp_init -> svp_register_kernel -> svp_submit* -> svp_flush -> svp_profile
 *
 * Conventions
 *  - Every function returns svp_status (SVP_OK == 0, negative on error) unless noted.
 *    No C++ exception crosses the ABI.  svp_last_error() returns a thread-local,
 *    human-readable message for the last failing call on the calling thread.
 *  - A CUDA failure inside svp_flush returns SVP_E_CUDA and makes the context
 *    "sticky-errored": every later call except svp_finalize / svp_last_error /
 *    svp_profile returns SVP_E_STATE.
 *  - The library owns everything it creates (streams, events, tables, staging arena,
 *    worker threads).  The caller owns every buffer passed in svp_buf.
 *  - Pointers are plain host or device addresses; sizes are bytes unless noted.
 *    No torch types appear here; PyTorch is only the caller's allocator.
 */
#ifndef SVP_H_
#define SVP_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define SVP_ABI_VERSION 6

typedef int32_t svp_status;
enum {
    SVP_OK = 0,
    SVP_E_INVAL = -1,       /* bad argument (null, size too small, wrong count/dir/residency) */
    SVP_E_NOMEM = -2,       /* host/device/pinned allocation failed, or a job exceeds the arena */
    SVP_E_CUDA = -3,        /* a CUDA runtime call failed; context becomes sticky-errored */
    SVP_E_NOKERNEL = -4,    /* unknown kernel name or id */
    SVP_E_STATE = -5,       /* context errored / finalized / flush re-entered */
    SVP_E_TIMEOUT = -6,     /* flush watchdog expired (cfg.flush_timeout_ms) */
    SVP_E_UNSUPPORTED = -7  /* valid request this build cannot run (e.g. sgemm K % 4 != 0) */
};

typedef struct svp_ctx svp_ctx; /* opaque */

/* ------------------------------------------------------------------ configuration */
/* Implementation of the fp32 "sgemm" kernel (all meet its 1e-5 fp32 contract). */
enum { SVP_SGEMM_FFMA = 0,      /* TMA-staged tiles, fp32 FFMA on the CUDA cores          */
       SVP_SGEMM_3XTF32 = 1,    /* tcgen05 tensor cores, operands split hi+lo (3 TF32 MMAs) */
       SVP_SGEMM_TF32BF16 = 2 };/* tcgen05: hi*hi as TF32 + the two cross corrections as
                                   BF16 MMAs (1 TF32 + 2 BF16 MMAs = 2/3 of 3xTF32's time) */

typedef struct svp_config {
    int32_t num_gpus;            /* GPUs to drive; 0 = all visible (dry_run: 0 -> 1)          */
    const int32_t* device_ids;   /* optional [num_gpus] CUDA ordinals; NULL = 0..num_gpus-1   */
    int32_t streams_per_gpu;     /* compute streams per GPU (>= 1); copies use 2 more streams */
    int32_t coalesce;            /* 1: Kernel Coalescing; 0: one launch/job */
    int32_t interleave;          /* 1: Kernel Interleaving: chunking,
                                    Johnson order, H2D / compute / D2H on separate streams;
                                    0: every op on one stream in submission order            */
    int32_t max_chunks;          /* upper bound on chunks a group is split into (1..64)       */
    uint64_t arena_bytes;        /* per-GPU device staging arena for host-resident buffers;
                                    0 = 2 GiB.  Allocated lazily on first host-resident job.  */
    int32_t profile_level;       /* 0: no events; 1: CUDA events around every op (per-VP
                                    attribution by algorithmic work, kernel stats); 2: as 1,
                                    and every vecadd/SAXPY/Black-Scholes/hist256 launch also
                                    counts the SM clock cycles thread 0 of each CTA spends in
                                    each tile, per segment -- the launch's time is then split
                                    over its VPs by those measured cycles (GEMM launches keep
                                    the FLOP split).  A latency-weighted split: a tile costs
                                    what its loads waited when it ran                         */
    int32_t sync_each_job;       /* serial baseline B1: stream-synchronize after every job    */
    int32_t dry_run;             /* 1: plan only -- no CUDA call at all, op times simulated
                                    by the cost model (host-logic tests on CPU)               */
    int32_t flush_timeout_ms;    /* 0 = wait forever; else watchdog -> SVP_E_TIMEOUT          */
    int32_t validate_ptrs;       /* svp_submit checks every buffer [ptr, ptr + touched bytes):
                                    DEVICE -> device/managed memory on the VP's GPU, HOST_PINNED
                                    -> page-locked host memory, and the range inside ONE
                                    allocation (else SVP_E_INVAL).  0: no check; 1: allocation
                                    ranges are resolved once (cudaPointerGetAttributes +
                                    cuPointerGetAttribute RANGE_START/SIZE) and remembered for
                                    the context's lifetime -- memory freed and re-allocated at
                                    the same address with another residency is not re-detected;
                                    2: query the driver on every submit                       */
    int32_t sgemm_impl;          /* SVP_SGEMM_TF32BF16 (default), SVP_SGEMM_3XTF32 or SVP_SGEMM_FFMA */
    void* const* external_streams; /* optional [num_gpus] caller cudaStream_t (e.g. torch's
                                    current stream): flush work starts after the work already
                                    queued on it, and it waits for the flush's last op.      */
    /* cost model used for ordering/chunking before measurements exist (D8, PAPER.md
       L272-275 "expected time for each invocation"); 0 = built-in B200 defaults      */
    double hbm_gbps;             /* default 6552 (MEASURED_PEAKS.json hbm_gbs)                */
    double pcie_gbps;            /* default 50 per direction                                  */
    double ffma_tflops;          /* default 60                                                */
    double launch_us;            /* default 4                                                 */
    /* NEXT item f4 (lifts "identical kernels only") */
    int32_t hetero;              /* 1: heterogeneous coalescing -- the vecadd, SAXPY and
                                    Black-Scholes groups of one (level, GPU) share ONE launch
                                    whose segment table names each segment's kernel          */
    int32_t graph;               /* 1 (default since ABI 6): steady-state replay -- a flush
                                    whose requests (VP, kernel, args, buffers, in order)
                                    equal those of one of the last 32 successful flushes
                                    reuses that plan, and on its second sighting captures the
                                    flush's device work as one CUDA graph per GPU (with a
                                    private copy of its device tables), replayed on every
                                    later sighting.  A loop that rotates input buffer sets
                                    therefore replays one graph per set.  Results are the
                                    same with 0.  Ignored with sync_each_job.               */
    int32_t table_mode;          /* where a coalesced launch finds its segment table (SURVEY
                                    §8(b)): SVP_TABLE_PARAM (default) -- launches of
                                    elementwise / hist256 groups with <= 64 VPs receive it
                                    by value as a kernel parameter of 1 or 4 KiB (no upload;
                                    cfg5 measured +4 % over global); larger groups, and
                                    SVP_TABLE_GLOBAL -- one device table
                                    buffer per GPU, uploaded once per flush when it changed.
                                    GEMM launches always use the global table.             */
    int32_t sgemm_kchunk;        /* (ABI 5) "sgemm" on the tensor-core splits: accumulate K in chunks
                                    of this many k (multiple of 16; 3xTF32 uses half), each from
                                    zero in TMEM, folded into C by TMA reduce-add (IEEE fp32) --
                                    the error of one chunk at any K and for any operand signs
                                    (R23).  Default 768 (cfg5: ~0.92x of 0).  beta != 0
                                    jobs longer than one chunk run on FFMA.  0: one accumulation
                                    per tile, jobs with K > 2048 (TF32+2xBF16) / 1024 (3xTF32)
                                    run on FFMA; same-sign operands then err up to ~2e-5 at
                                    K = 2048                                                  */
} svp_config;

enum { SVP_TABLE_GLOBAL = 0, SVP_TABLE_PARAM = 1 };

/* Fill *cfg with defaults: num_gpus 0, 4 compute streams, coalesce 1, interleave 1,
   max_chunks 8, profile_level 0, validate_ptrs 1, sgemm_impl SVP_SGEMM_TF32BF16,
   table_mode SVP_TABLE_PARAM, sgemm_kchunk 768, graph 1, rest 0 (hetero 0). */
void svp_config_default(svp_config* cfg);

/* Create a context.  On success *out owns streams/events/threads for every GPU.
   Errors: SVP_E_INVAL (null / bad values), SVP_E_CUDA (no device, bad ordinal). */
svp_status svp_init(const svp_config* cfg, svp_ctx** out);

/* Sync, free every library-owned resource, join worker threads.  Safe on an errored
   context; ctx is invalid afterwards. */
svp_status svp_finalize(svp_ctx* ctx);

const char* svp_last_error(void);
int32_t svp_abi_version(void);

/* ------------------------------------------------------------------ kernels */
/* Builtin guest kernels (BASELINE.json north_star):
 *   "vecadd"        c = a + b                        args svp_args_vecadd   bufs [a IN f32, b IN f32, c OUT f32]
 *   "saxpy"         y = fma(a, x, y)                 args svp_args_saxpy    bufs [x IN f32, y INOUT f32]
 *   "hist256"       counts[b] = #{i: d[i]==b}        args svp_args_hist256  bufs [d IN u8, counts OUT u32[256]]
 *                   (counts are overwritten)
 *   "blackscholes"  call/put per option              args svp_args_bs       bufs [S IN, X IN, T IN, call OUT, put OUT] f32
 *   "sgemm"         C = alpha A B + beta C, fp32     args svp_args_sgemm   bufs [A IN, B IN, C OUT (INOUT if beta != 0)]
 *                   contract (R10/R20): |c - exact| <= 1e-5 (|alpha||A||B| + |beta C|)_ij
 *                   + (K+1) 2^-149, Inf/NaN propagated as in IEEE fp32.  cfg.sgemm_impl picks
 *                   the implementation: SVP_SGEMM_TF32BF16 (default; tcgen05 TF32 + 2 BF16
 *                   MMAs on a hi/lo operand split), SVP_SGEMM_3XTF32 (3 TF32 MMAs) or
 *                   SVP_SGEMM_FFMA (fp32 FFMA on the CUDA cores).  The two tensor-core splits
 *                   add 2^-134 |other operand| per product whose operand is below 2^-115 in
 *                   magnitude (TF32 / BF16 subnormal granularity); an output their tensor-core
 *                   accumulation leaves NaN (an Inf / NaN operand, or one near FLT_MAX) is
 *                   recomputed exactly from A and B (fp64 products and sum, one rounding).
 *                   Their fp32 accumulation loses ~1.7e-8 (random-sign data) to ~3.4e-8
 *                   (same-sign data) relative per accumulating MMA, so K is accumulated in
 *                   chunks of cfg.sgemm_kchunk (default 768) folded into C with fp32 adds:
 *                   measured <= 7.4e-6 componentwise on same-sign data at any K (DESIGN R23)
 *   "sgemm_tf32"    same, tcgen05 TF32 tensor cores  (own tolerance 2e-3; raw operands, so a
 *                   NaN whose payload is only in the low 13 mantissa bits reads as Inf)
 *   "dgemm"         C = alpha A B + beta C, fp64     args svp_args_dgemm   bufs [A IN, B IN, C OUT (INOUT if beta != 0)] f64
 *                   (the paper's Table 1 guest: 320x320 fp64 matmul)
 * GEMM jobs of different shapes are "identical kernels" too: one grouped launch covers
 * every VP's (M, N, K) (ragged grouped GEMM).
 * Registration is idempotent; the id is stable for the context's lifetime.
 * Errors: SVP_E_NOKERNEL for an unknown name. */
svp_status svp_register_kernel(svp_ctx* ctx, const char* name, int32_t* id_out);

typedef struct svp_args_vecadd { uint64_t n; } svp_args_vecadd;
typedef struct svp_args_saxpy { uint64_t n; float a; uint32_t _pad; } svp_args_saxpy;
typedef struct svp_args_hist256 { uint64_t n; } svp_args_hist256;
typedef struct svp_args_bs { uint64_t n; float R; float V; } svp_args_bs;
typedef struct svp_args_sgemm { int32_t M, N, K; float alpha, beta; } svp_args_sgemm;
typedef struct svp_args_dgemm { int32_t M, N, K, _pad; double alpha, beta; } svp_args_dgemm;

/* ------------------------------------------------------------------ jobs */
enum { SVP_DIR_IN = 1, SVP_DIR_OUT = 2, SVP_DIR_INOUT = 3 };
enum { SVP_MEM_DEVICE = 0, SVP_MEM_HOST_PINNED = 1 };

typedef struct svp_buf {
    void* ptr;       /* device pointer (mem DEVICE, must be on svp_vp_device(vp)) or pinned host */
    uint64_t bytes;  /* extent the caller guarantees valid; must cover what the kernel touches */
    int32_t dir;     /* SVP_DIR_*; must match the kernel's buffer directions                     */
    int32_t mem;     /* SVP_MEM_*                                                                 */
} svp_buf;

#define SVP_MAX_BUFS 5
#define SVP_MAX_ARGS 64

/* Queue one job of VP `vp` (0 <= vp < 2^20).  This is the in-process stand-in for the
 * paper's VP -> IPC manager -> Job Queue path (Fig 2): it validates
 * the job against the kernel descriptor, copies `args` and the buffer descriptors, and
 * appends to the VP's FIFO (program order).  Asynchronous like cudaMemcpyAsync: the
 * caller keeps every buffer valid and unmodified until svp_flush returns.  Pinned host
 * buffers are staged through the device arena (the paper's physically-contiguous
 * chunk, Fig 5); device buffers are used in place.  n = 0 is a legal no-op job.
 * Thread-safe: many threads may submit concurrently.  *job_out (optional) gets a
 * monotonically increasing job id.
 * Errors: SVP_E_INVAL (bad vp/args/bufs/residency), SVP_E_NOKERNEL, SVP_E_UNSUPPORTED,
 * SVP_E_STATE. */
svp_status svp_submit(svp_ctx* ctx, int32_t vp, int32_t kernel, const void* args,
                      size_t args_bytes, const svp_buf* bufs, int32_t nbufs, uint64_t* job_out);

/* Batched submit (one lock, one validation pass) -- same semantics as n svp_submit
 * calls in array order; on error nothing from the batch is queued. */
typedef struct svp_job_desc {
    int32_t vp;
    int32_t kernel;
    uint32_t args_bytes;
    int32_t nbufs;
    uint8_t args[SVP_MAX_ARGS];
    svp_buf bufs[SVP_MAX_BUFS];
} svp_job_desc;
svp_status svp_submit_batch(svp_ctx* ctx, int32_t n, const svp_job_desc* jobs, uint64_t* job_ids_out);

/* Drain every job submitted before the call: Kernel Match -> Job Dispatcher ->
 * Re-scheduler -> per-GPU execution (coalesced launches over device segment tables,
 * interleaved H2D/kernel/D2H streams) -> Profiler; blocks until every output is in
 * the caller's buffers.  Concurrent calls (other threads, the dispatcher) serialize.
 * On an error the flushed jobs are dropped and reported failed to svp_wait.
 * Errors: SVP_E_CUDA (sticky), SVP_E_TIMEOUT, SVP_E_NOMEM, SVP_E_STATE. */
svp_status svp_flush(svp_ctx* ctx);

/* (ABI 6) Pipelined flush: the same flush as svp_flush, but it returns once the device
 * work is enqueued.  The flush stays pending until the NEXT flush (async or not) has been
 * planned and issued, so the host's submit / plan / issue of flush i+1 overlaps the device
 * work of flush i.  A launch-bound loop of small flushes then runs at the pace of the
 * slower of host and GPU, not their sum.  At most one flush is pending: each flush
 * completes the previous pending one (waits for it, runs the Profiler, marks its jobs done
 * for svp_wait) after issuing its own work.
 * *ticket_out = the flush's sequence number.  Its outputs are in place after
 * svp_flush_wait(ctx, ticket), a later svp_flush, svp_wait on one of its jobs, or
 * svp_finalize.  Until then, the caller must not modify that flush's input buffers or read
 * its outputs.  The GPUs run consecutive flushes in order (each forks from the previous
 * one's join on the caller's stream); only host work overlaps.  With profile_level >= 1 or
 * sync_each_job there is no overlap: the previous flush completes before the next is
 * issued, because per-op timing events are reused from flush to flush.
 * svp_flush_stats_get reports the last COMPLETED flush.  Errors: as svp_flush (an error of
 * the completed previous flush is returned here if the new one succeeded). */
svp_status svp_flush_async(svp_ctx* ctx, uint64_t* ticket_out);
/* Complete every flush up to `ticket` (a no-op for completed ones).  Returns the status of
 * flush `ticket`.  Errors: SVP_E_INVAL (null ctx, ticket never issued), or that flush's
 * error. */
svp_status svp_flush_wait(svp_ctx* ctx, uint64_t ticket);

/* ------------------------------------------------------------------ VP Control */
/* Block the calling VP until job `job` (an id returned by svp_submit*) has run and its
 * outputs are in place -- the synchronous-call path of PAPER.md L276-286 / Fig 4(b):
 * the VP is stopped while other VPs' jobs keep the GPU busy, and resumed when its job
 * completes.  Somebody must flush (the caller from another thread, or the dispatcher).
 * timeout_ms <= 0 waits forever.  Returns SVP_OK, the failing flush's status for a job
 * that was dropped, SVP_E_TIMEOUT, SVP_E_STATE (context errored first) or SVP_E_INVAL
 * (unknown id). */
svp_status svp_wait(svp_ctx* ctx, uint64_t job, int32_t timeout_ms);

/* Continuous dispatch (the paper's continuously fed Job Queue): a
 * background thread flushes whenever jobs are queued, after letting more VPs join for up
 * to window_us (or until max_jobs are queued, 0 = no cap) -- so concurrent VPs' identical
 * synchronous calls still coalesce.  svp_stop_dispatcher drains the queue and joins. */
svp_status svp_start_dispatcher(svp_ctx* ctx, int32_t window_us, int32_t max_jobs);
svp_status svp_stop_dispatcher(svp_ctx* ctx);

/* ------------------------------------------------------------------ IPC front end */
/* The paper's IPC Manager (VPs reach the host "through an IPC method
 * such as socket or shared memory"): VP *processes* submit jobs to a server process that
 * owns the svp context.  svp_ipc_serve creates the POSIX shared-memory segment `name`
 * (no '/'; shm_open("/name")) holding a ticketed ring of nslots job slots and a data
 * arena of arena_bytes, registers the arena with CUDA (so jobs use it as HOST_PINNED
 * memory -- staged, coalesced and interleaved like any host-resident job), starts the
 * context's dispatcher if it is not running, and serves until svp_ipc_shutdown (which
 * also unlinks the segment).  Clients need no CUDA: svp_ipc_connect maps the segment,
 * svp_ipc_alloc bump-allocates 256-B aligned arena space (returns its offset and a
 * pointer in the caller's mapping), svp_ipc_submit queues a job whose buffers are arena
 * offsets (returns a ticket), svp_ipc_wait blocks until that job has run (its outputs
 * are then in the arena) and returns the job's status.  Each ticket is waited once. */
typedef struct svp_ipc_server svp_ipc_server;
typedef struct svp_ipc_client svp_ipc_client;
typedef struct svp_ipc_buf {
    uint64_t offset; /* arena offset from svp_ipc_alloc */
    uint64_t bytes;
    int32_t dir;     /* SVP_DIR_* */
    int32_t _pad;
} svp_ipc_buf;
svp_status svp_ipc_serve(svp_ctx* ctx, const char* name, uint64_t arena_bytes, int32_t nslots,
                         svp_ipc_server** out);
svp_status svp_ipc_server_stats(svp_ipc_server* s, uint64_t* jobs_served, uint64_t* tickets_issued);
svp_status svp_ipc_shutdown(svp_ipc_server* s);
svp_status svp_ipc_connect(const char* name, svp_ipc_client** out);
svp_status svp_ipc_disconnect(svp_ipc_client* c);
svp_status svp_ipc_alloc(svp_ipc_client* c, uint64_t bytes, uint64_t* offset_out, void** ptr_out);
svp_status svp_ipc_submit(svp_ipc_client* c, int32_t vp, int32_t kernel, const void* args, size_t args_bytes,
                          const svp_ipc_buf* bufs, int32_t nbufs, uint64_t* ticket_out);
svp_status svp_ipc_wait(svp_ipc_client* c, uint64_t ticket, int32_t timeout_ms);
/* Builtin kernel ids are stable; clients (which have no context) look them up by name. */
svp_status svp_kernel_lookup(const char* name, int32_t* id_out);

/* ------------------------------------------------------------------ Job Dispatcher */
/* The GPU (index into the context's device list, 0..num_gpus-1) that runs VP `vp`.
 * Sticky: assigned on first use (least-loaded by estimated cost so far) or by
 * svp_assign_vps, never moved afterwards -- the caller allocates device-resident VP
 * buffers there. */
svp_status svp_vp_device(svp_ctx* ctx, int32_t vp, int32_t* device_out);

/* Pin n VPs to GPUs with kernel-stratified LPT: within each class
 * (kernel id), VPs in decreasing cost go to the least-loaded GPU, so every GPU gets a
 * share of every class.  Already-placed VPs keep their GPU.  devices_out[n] optional. */
svp_status svp_assign_vps(svp_ctx* ctx, int32_t n, const int32_t* vps, const int32_t* classes,
                          const double* costs, int32_t* devices_out);

/* Pure function (no context, no CUDA): the same kernel-stratified LPT over G bins.
 * Used by multi-process (one rank per GPU) runs so every rank computes the same
 * partition without exchanging data.  out[n] receives the bin of each item. */
svp_status svp_lpt_partition(int32_t n, const int32_t* classes, const double* costs, int32_t G,
                             int32_t* out);

/* ------------------------------------------------------------------ Profiler */
/* Per-VP attribution of device-timed op durations (the profiler
 * "acquires execution information such as ... the elapsed clock cycles"): an op's
 * event-timed duration is split over its member VPs in proportion to their
 * algorithmic bytes (FLOPs for SGEMM), or with profile_level 2 for segment launches in
 * proportion to the measured SM cycles of each VP's tiles.  Needs profile_level >= 1.  vp = -1 returns
 * device-wide totals (sum over VPs, plus op counts). */
typedef struct svp_vp_profile {
    uint64_t jobs;
    double kernel_ns, h2d_ns, d2h_ns;
    uint64_t bytes_kernel, bytes_h2d, bytes_d2h;
    double flops;
    uint64_t launches; /* vp = -1 only: kernel launches issued */
} svp_vp_profile;
svp_status svp_profile(svp_ctx* ctx, int32_t vp, svp_vp_profile* out);
svp_status svp_reset_profile(svp_ctx* ctx);

/* Aggregate per kernel id (profile_level >= 1): launches, summed event-timed kernel
 * duration (ns), algorithmic bytes and FLOPs of those launches.  `kernel` is a
 * registered id or SVP_KERNEL_EW_MIX, the heterogeneous elementwise launch that
 * cfg.hetero forms (its vecadd/SAXPY/Black-Scholes members are counted there, not under
 * their own ids); plan ops of such a launch also report SVP_KERNEL_EW_MIX. */
#define SVP_KERNEL_EW_MIX 8
typedef struct svp_kernel_stats {
    uint64_t launches;
    double total_ns;
    double bytes;
    double flops;
    double max_ns;
} svp_kernel_stats;
svp_status svp_kernel_stats_get(svp_ctx* ctx, int32_t kernel, svp_kernel_stats* out);

/* Counters of the most recent flush. */
typedef struct svp_flush_stats {
    uint64_t jobs, groups, chunks, launches, levels;
    uint64_t h2d_bytes, d2h_bytes, table_bytes, table_uploads;
    double host_plan_ns;     /* match + dispatch + reschedule + table build      */
    double host_issue_ns;    /* enqueueing copies/launches                        */
    double host_total_ns;    /* whole svp_flush call                               */
    double device_ns;        /* first-op start to last-op end (profile_level >= 1) */
    double sim_makespan_ns;  /* cost-model makespan of the plan (always)           */
    double sim_serial_ns;    /* cost-model time of the same ops run one at a time  */
    uint64_t plan_reused;    /* cfg.graph: 1 if a recent flush's plan was reused     */
    uint64_t graph_replays;  /* cfg.graph: GPUs whose work ran as a replayed CUDA graph */
    uint64_t kernel_launches; /* kernels actually launched (`launches` counts coalesced
                                 launch ops; hist256's zeroing kernel and the SGEMM tail
                                 split's slice launch + reduction add to this one)     */
} svp_flush_stats;
svp_status svp_flush_stats_get(svp_ctx* ctx, svp_flush_stats* out);

/* (ABI 5) Per-GPU view of the Job Dispatcher and the Profiler, for GPU index g
 * (0..num_gpus-1): how many VPs the Dispatcher has placed there and their summed cost
 * estimate (ns, the LPT load), and -- accumulated since svp_reset_profile, profile_level
 * >= 1 -- flushes and jobs that ran there, the summed per-flush device span (first op
 * start to last op end on that GPU) and the summed event-timed kernel op durations
 * (ops that overlap on different streams each count in full).  Imbalance across GPUs =
 * max / mean of device_ns.  Errors: SVP_E_INVAL (null, g out of range). */
typedef struct svp_device_stats {
    int32_t ordinal;        /* CUDA device ordinal of GPU index g                       */
    int32_t vps;            /* VPs placed on it (sticky)                               */
    double est_load_ns;     /* Dispatcher's summed cost estimate of those VPs           */
    uint64_t flushes;       /* flushes with work on this GPU                            */
    uint64_t jobs;          /* jobs run on this GPU                                     */
    double device_ns;       /* summed per-flush device span                             */
    double kernel_ns;       /* summed event-timed kernel op durations                   */
    double last_device_ns;  /* the last flush's span on this GPU                        */
    int32_t numa_node;      /* (ABI 6) the GPU's NUMA node (sysfs of its PCI function),
                               -1 unknown (single-socket hosts, hidden sysfs)           */
    int32_t worker_cpu_pinned; /* (ABI 6) 1 if the worker thread driving this GPU runs on
                               the GPU's local CPUs (GPU indices >= 1 of a multi-GPU
                               context; GPU 0 is driven by the flushing thread, never
                               pinned).  SVP_NUMA_AFFINITY=0 turns the pinning off.     */
} svp_device_stats;
svp_status svp_device_stats_get(svp_ctx* ctx, int32_t g, svp_device_stats* out);

/* (ABI 6) NUMA-local page-locked host memory for host-resident VP buffers (PAPER.md
 * L266-286: the H2D / D2H copies of a VP's data are its job's first and last steps; on a
 * multi-socket B200 node, pages on the far socket cross the inter-socket link before PCIe).
 * Allocates `bytes` (rounded up to whole pages) of anonymous host memory, binds it
 * (mbind MPOL_PREFERRED) to the NUMA node of GPU index `gpu` of this context, and
 * page-locks it with cudaHostRegister(Portable), so any GPU of the process can DMA it and
 * svp_submit accepts it as SVP_MEM_HOST_PINNED.  *ptr_out receives the address (page
 * aligned); *numa_node_out (optional) the node the pages were bound to, or -1 when the
 * GPU's node is unknown (the memory is then page-locked but not placed).  The memory is
 * the caller's until svp_host_free(ctx, ptr) or svp_finalize(ctx), which releases every
 * block still allocated; freeing a block with jobs in flight on it is undefined.
 * Errors: SVP_E_INVAL (null, bytes == 0, gpu out of range), SVP_E_UNSUPPORTED (dry-run
 * context), SVP_E_NOMEM (mmap / pinning failed), SVP_E_CUDA. */
svp_status svp_host_alloc(svp_ctx* ctx, int32_t gpu, uint64_t bytes, void** ptr_out, int32_t* numa_node_out);
/* Releases a block from svp_host_alloc.  SVP_E_INVAL if ptr is not one (or already freed). */
svp_status svp_host_free(svp_ctx* ctx, void* ptr);

/* ------------------------------------------------------------------ plan introspection */
/* The last flush's plan, one entry per issued op in issue order (tests, tooling). */
enum { SVP_OP_H2D = 0, SVP_OP_KERNEL = 1, SVP_OP_D2H = 2 };
typedef struct svp_plan_op {
    int32_t kind;       /* SVP_OP_* */
    int32_t device;     /* GPU index                                      */
    int32_t stream;     /* library stream index on that GPU               */
    int32_t level;      /* program-order level (the level-th job of a VP)  */
    int32_t kernel;     /* kernel id                                       */
    int32_t group;      /* Kernel Match group index within the flush       */
    int32_t chunk;      /* chunk index within the group                    */
    int32_t nvps;       /* members (VPs) in this op                        */
    uint64_t bytes;     /* copy bytes, or algorithmic kernel bytes          */
    double flops;
    double est_ns;      /* cost-model duration                              */
    double sim_start_ns, sim_end_ns; /* cost-model schedule                */
    double measured_ns; /* event-timed duration (profile_level >= 1), else -1 */
} svp_plan_op;
svp_status svp_plan_size(svp_ctx* ctx, int32_t* n_ops);
/* vps_out (optional, capacity cap) receives the op's member VPs in segment order. */
svp_status svp_plan_get(svp_ctx* ctx, int32_t i, svp_plan_op* op, int32_t* vps_out, int32_t cap);
/* (ABI 5) Ordering detail of plan op i: *arena_off / *arena_len = the staging-arena byte
 * range its chunk uses (len 0: nothing staged), *nwaits = how many earlier ops it waits on
 * through events (cross-stream waits; ops on the same (device, stream) are ordered by
 * issue order and are not listed), waits_out[0 .. min(nwaits, cap)) their plan indices, and
 * *measured_start_ns = when the op started on its GPU, event-timed from the start of that
 * GPU's first op of the flush (profile_level >= 1; -1 otherwise) -- with measured_ns of
 * svp_plan_get, the flush's measured timeline.  Any pointer may be NULL.
 * Errors: SVP_E_INVAL (null ctx, index out of range). */
svp_status svp_plan_op_detail(svp_ctx* ctx, int32_t i, uint64_t* arena_off, uint64_t* arena_len,
                              int32_t* waits_out, int32_t cap, int32_t* nwaits, double* measured_start_ns);

#ifdef __cplusplus
}
#endif
#endif /* SVP_H_ */

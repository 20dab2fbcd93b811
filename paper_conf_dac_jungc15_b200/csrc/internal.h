// internal.h -- core data structures of libsvp (host side).  Not part of the C-ABI.
//
// Layering: capi.cpp (L5 boundary) -> scheduler.cpp (L3: Job Queue,
// Kernel Match, Job Dispatcher, Re-scheduler, cost model) -> executor.cpp (L2: per-GPU
// streams/events/arena/tables, Profiler) -> kernels/*.cu (L0: sm_100a guest kernels).
#pragma once
#include <math.h>
#include <pthread.h>
#include <sched.h>
#include <string.h>
#include <stdint.h>

#include <atomic>
#include <chrono>
#include <condition_variable>
#include <functional>
#include <memory>
#include <mutex>
#include <string>
#include <thread>
#include <unordered_map>
#include <vector>

#include "../../include/svp.h"

namespace svp {

// ------------------------------------------------------------------ kernel registry
enum KernelId : int32_t {
    K_VECADD = 1,
    K_SAXPY = 2,
    K_HIST256 = 3,
    K_BLACKSCHOLES = 4,
    K_SGEMM = 5,
    K_SGEMM_TF32 = 6,
    K_DGEMM = 7,
    K_EW_MIX = 8,   // heterogeneous elementwise launch (cfg.hetero, NEXT f4): not registrable,
                    // appears only as a plan/kernel-stats id (SVP_KERNEL_EW_MIX)
    K_COUNT = 9
};

struct KernelDesc {
    const char* name;
    int32_t id;
    int32_t nbufs;
    int32_t dirs[SVP_MAX_BUFS];   // required SVP_DIR_* (sgemm C may be OUT or INOUT)
    uint32_t args_bytes;
};
const KernelDesc* kernel_desc(int32_t id);
inline bool is_gemm(int32_t k) { return k == K_SGEMM || k == K_SGEMM_TF32 || k == K_DGEMM; }
// Largest K an "sgemm" job runs with on the tensor-core split implementations (R23):
// the tcgen05 fp32 accumulation loses magnitude (measured -1.66e-8 relative per accumulating
// MMA, profiles/r02/accuracy_k.jsonl), so the output's relative error grows with K; up to
// these K every measured output keeps the 1e-5 fp32 contract.  Jobs with larger K match as a
// separate group that runs the FFMA kernel.
// K chunk (k, multiple of 16; 0 = off) of a tensor-core split's accumulation (R23) from
// cfg.sgemm_kchunk: 3xTF32 (6 accumulating MMAs per 16 k against 4) uses half of it
inline int32_t sgemm_chunk_k(int32_t impl, int32_t cfg_kchunk) {
    if (cfg_kchunk <= 0) return 0;
    if (impl == SVP_SGEMM_3XTF32) return cfg_kchunk >= 32 ? cfg_kchunk / 32 * 16 : 16;
    return impl == SVP_SGEMM_TF32BF16 ? cfg_kchunk : 0;
}
// internal "sgemm_impl" of a group whose jobs TMA cannot address (k_sgemm_plain)
constexpr int32_t kSgemmPlain = 3;
inline int32_t sgemm_tc_kmax(int32_t impl) {
    return impl == SVP_SGEMM_TF32BF16 ? 2048 : impl == SVP_SGEMM_3XTF32 ? 1024 : (1 << 30);
}
// kernels the heterogeneous launch can carry: same CTA shape (256 threads, no shared
// memory) and the same SegDesc tile mapping
inline bool is_ew(int32_t k) { return k == K_VECADD || k == K_SAXPY || k == K_BLACKSCHOLES; }
// launches that read a SegDesc segment table (tile -> VP segment)
inline bool is_seg_kernel(int32_t k) { return is_ew(k) || k == K_EW_MIX || k == K_HIST256; }
const KernelDesc* kernel_by_name(const char* name);

// ------------------------------------------------------------------ jobs
struct Job {
    uint64_t id = 0;
    int32_t vp = 0;
    int32_t kernel = 0;
    uint8_t args[SVP_MAX_ARGS] = {};
    svp_buf bufs[SVP_MAX_BUFS] = {};
    int32_t nbufs = 0;
    // derived at submit
    uint64_t n = 0;               // elements (memory-bound kernels)
    int32_t M = 0, N = 0, K = 0;  // sgemm
    float f0 = 0.f, f1 = 0.f;     // scalars
    double d0 = 1.0, d1 = 0.0;    // dgemm alpha, beta
    uint64_t shape_key = 0;       // Kernel Match key (with kernel id)
    uint64_t in_bytes = 0;        // bytes of IN/INOUT buffers the kernel reads
    uint64_t out_bytes = 0;       // bytes of OUT/INOUT buffers the kernel writes
    uint64_t host_in_bytes = 0;   // of which host-resident (H2D staging)
    uint64_t host_out_bytes = 0;  // of which host-resident (D2H)
    double alg_bytes = 0;         // algorithmic bytes (roofline, profiler weights)
    double flops = 0;
    int32_t level = 0;            // program-order level within the flush
    int32_t device = 0;           // assigned GPU
};

// Bytes the kernel touches in buffer b of job j (what must be staged / copied back).
uint64_t touched_bytes(const Job& j, int b);

// ------------------------------------------------------------------ plan
struct Chunk {
    int32_t group = 0;
    int32_t index = 0;              // chunk index in group
    int32_t device = 0;
    int32_t level = 0;
    int32_t kernel = 0;
    std::vector<int32_t> jobs;      // indices into Flush::jobs, segment order (vp ascending)
    double t_in = 0, t_k = 0, t_out = 0;  // cost-model estimates (ns)
    uint64_t in_bytes = 0, out_bytes = 0;
    double alg_bytes = 0, flops = 0;
    // staging
    uint64_t arena_off = 0, arena_len = 0;
    std::vector<uint64_t> staged;   // per job per buffer: device address used by kernel
    // table
    uint64_t table_off = 0;         // offset of this chunk's table in the device table buffer
    uint32_t total_tiles = 0;
    int32_t nsegs = 0;
    uint64_t maps_off = 0;          // sgemm: tensor maps offset
    int64_t cmaps_off = -1;         // tensor-core sgemm with K chunks: C tensor maps (R23), else -1
    bool small_tiles = false;       // dgemm: 32x32 tile variant (launch under 2 waves of 64x64)
    bool wide = false;              // sgemm TF32+2xBF16: 256x512 pair tiles (>= 2 waves of them)
    bool param = false;             // table_mode param: the SegDesc table goes by value
    int32_t co_grid = 0;            // >0: launch with co_grid CTAs per SM so the kernel
                                    // co-resides with a tensor-core SGEMM on the same SMs
    // profile_level 2 (segment launches): offset of this launch's per-segment busy-cycle
    // counters in the GPU's counter buffer (-1: none), and their values after the flush
    int64_t busy_off = -1;
    std::vector<uint64_t> busy;
    int32_t sched_slot = -1;        // dynamic tile order: counter slot of this launch (-1: static)
    int64_t hscr_off = -1;          // single-launch hist256: scratch offset (u32) of this launch
    // SGEMM tail split (wide launches whose last wave is at most half full): the main launch
    // runs main_tiles tiles, the last wave's tiles run as tail_n K-slices (narrow pair
    // kernel) into a workspace, then tail_nred sub-tile reductions write C
    uint32_t main_tiles = 0;
    int32_t tail_n = 0, tail_nred = 0;
    uint64_t tail_maps_off = 0, tail_table_off = 0, tail_red_off = 0;
    // kernel launches this op issues (hist256 zeroing kernel, tail split: 3)
    int32_t kernel_launches = 1;
    int32_t sgemm_impl = -1;        // K_SGEMM: the implementation this launch runs (R23)
};

struct Op {
    int32_t kind = SVP_OP_KERNEL;
    int32_t chunk = 0;
    int32_t device = 0;
    int32_t stream = 0;
    std::vector<int32_t> wait_ops;  // ops (global index) this op must wait for
    bool needs_event = false;       // someone waits on this op -> record event after it
    double est_ns = 0;
    double sim_start = 0, sim_end = 0;
    double measured_ns = -1;
    double measured_start_ns = -1;  // from the start of this GPU's first op of the flush
    uint64_t bytes = 0;
    double flops = 0;
    bool last_of_job = false;       // serial baseline: sync after this op
};

struct Group {
    int32_t kernel = 0;
    uint64_t shape_key = 0;
    int32_t level = 0;
    int32_t device = 0;
    std::vector<int32_t> jobs;      // vp ascending
};

struct Flush {
    std::vector<Job> jobs;
    std::vector<Group> groups;
    std::vector<Chunk> chunks;
    std::vector<Op> ops;            // issue order (per device subsequence is that device's issue order)
    int32_t levels = 0;
    // steady-state replay (cfg.graph): plan_gen names the plan; reused = this flush's
    // requests equal the previous flush's, so plan, chunks and tables were copied from it
    uint64_t plan_gen = 0;
    bool reused = false;
    uint64_t seq = 0;             // flush sequence number (svp_flush_async tickets)
    svp_flush_stats stats{};      // this flush's statistics (svp_flush_stats_get: the last completed)
};

// ------------------------------------------------------------------ per-VP profile
struct VpProfile {
    uint64_t jobs = 0;
    double kernel_ns = 0, h2d_ns = 0, d2h_ns = 0;
    uint64_t bytes_kernel = 0, bytes_h2d = 0, bytes_d2h = 0;
    double flops = 0;
};

struct KStats {
    uint64_t launches = 0;
    double total_ns = 0, bytes = 0, flops = 0, max_ns = 0;
};

// per-GPU Profiler accumulators (svp_device_stats_get), under Ctx::pmu
struct DevStats {
    uint64_t flushes = 0, jobs = 0;
    double device_ns = 0, kernel_ns = 0, last_device_ns = 0;
};

// ------------------------------------------------------------------ cost model (D8)
struct CostModel {
    double hbm_Bps = 6552e9;
    double pcie_Bps = 50e9;
    double ffma_flops = 60e12;
    double tf32_flops = 500e12;
    double launch_ns = 4000;
    int sgemm_tc_units = 0;          // "sgemm" on tensor cores: TF32-MMA-equivalents per
                                     // product (3xTF32: 3, TF32+2xBF16: 2); 0 = FFMA
    double copy_ns = 2000;           // per-copy fixed overhead
    double fp64_flops = 30e12;
    // EMA of measured / predicted kernel time per (kernel, size bucket), learned
    // from the Profiler: a 64 Ki-element launch and a 16 Mi-element one of the same kernel sit
    // at different points of Eq 9's T_o + T_e ceil(xi / lambda), so one factor per kernel
    // would mix them.  Bucket = floor(log4(work)), work = FLOPs (GEMMs) or algorithmic bytes.
    static constexpr int kBuckets = 32;
    double kscale[K_COUNT][kBuckets];
    CostModel() {
        for (auto& row : kscale)
            for (double& x : row) x = 1.0;
    }
    static int bucket(double alg_bytes, double flops) {
        // floor(log2 w) / 2 from the exponent bits: this runs once per submitted job
        const double w = flops > 0 ? flops : alg_bytes;
        if (!(w >= 1.0)) return 0;
        uint64_t bits;
        memcpy(&bits, &w, sizeof bits);
        const int b = ((int)((bits >> 52) & 0x7ff) - 1023) >> 1;
        return b >= kBuckets ? kBuckets - 1 : b;
    }
    double kernel_ns(int32_t kernel, double alg_bytes, double flops) const;
    // K_SGEMM on an explicit implementation (a group routed to FFMA, R23)
    double sgemm_ns(int32_t impl, double alg_bytes, double flops) const;
    double h2d_ns(uint64_t bytes, int ncopies) const;
    double d2h_ns(uint64_t bytes, int ncopies) const;
};

class Executor;  // executor.cpp

struct Ctx {
    svp_config cfg{};
    std::vector<int32_t> device_ids;
    int32_t ngpu = 1;
    CostModel cost;

    // Job Queue (D2): per-VP FIFOs, program order = submission order
    std::mutex qmu;
    std::vector<Job> queue;          // appended in submission order; snapshot at flush
    uint64_t next_job_id = 1;

    // Job Dispatcher: sticky VP -> GPU
    std::mutex dmu;
    std::unordered_map<int32_t, int32_t> vp_dev;
    std::vector<double> dev_load;

    // state
    std::mutex flush_mu;             // serializes flushes (user calls and the dispatcher)
    // job completion (VP Control: svp_wait blocks a VP until its job is done)
    std::mutex done_mu;
    std::condition_variable done_cv;
    uint64_t completed_upto = 0;     // every job id <= completed_upto has been flushed
    std::vector<std::pair<uint64_t, int32_t>> failed;  // (last id of a failed flush, status), ascending
    uint64_t failed_floor = 0;       // ids <= failed_floor that are not in `failed` succeeded
    // continuous dispatcher (svp_start_dispatcher)
    std::condition_variable q_cv;    // with qmu: a job was queued / stop requested
    std::thread disp;
    bool disp_running = false;
    bool disp_stop = false;
    int64_t disp_window_us = 0;
    int32_t disp_max_jobs = 0;
    // SVP_OK or the first fatal status.  Read lock-free by every entry point; written once
    // (with sticky_msg) under done_mu before waiters are notified.  sticky_msg is read
    // only through sticky_message() (done_mu), never while it is being assigned.
    std::atomic<int32_t> sticky{0};
    std::string sticky_msg;
    std::string sticky_message() {
        std::lock_guard<std::mutex> lk(done_mu);
        return sticky_msg;
    }
    bool registered[K_COUNT] = {};

    // last flush, and (cfg.graph) the plans of the kPlanCache successful flushes before it
    static constexpr size_t kPlanCache = 32;
    std::vector<Flush> plan_cache;
    Flush last;
    // svp_flush_async: the flush whose device work may still run (its wait half pending),
    // under flush_mu.  Completed when the next flush has been issued, by svp_flush_wait,
    // by svp_wait on one of its jobs, or at svp_finalize.
    struct PendingFlush {
        Flush f;
        uint64_t upto = 0;  // last job id of the flush
        svp_status st = SVP_OK;
        std::chrono::steady_clock::time_point t0;
    };
    std::unique_ptr<PendingFlush> pending;
    uint64_t flush_seq = 0;       // last issued flush
    std::vector<std::pair<uint64_t, int32_t>> failed_flushes;  // (seq, status), ascending
    bool last_ok = false;            // the last flush completed with SVP_OK
    uint64_t plan_gen = 0;           // bumped for every freshly planned flush
    double last_sim_makespan = 0, last_sim_serial = 0;
    svp_flush_stats fstats{};

    // Profiler
    std::mutex pmu;
    std::unordered_map<int32_t, VpProfile> prof;
    VpProfile prof_total;
    uint64_t prof_launches = 0;
    KStats kstats[K_COUNT];
    std::vector<DevStats> dstats;    // [ngpu]

    // svp_host_alloc blocks (NUMA-placed, page-locked), released by svp_host_free / finalize
    std::mutex hmu;
    std::unordered_map<void*, size_t> host_blocks;

    Executor* exec = nullptr;        // null in dry_run
    bool coschedule = false;         // SVP_COSCHEDULE=1: memory-first small-grid co-residency
                                     // (measured slower than longest-first)
};

// scheduler.cpp
svp_status validate_and_fill(Ctx* c, Job* j);
svp_status plan_flush(Ctx* c, Flush* f);             // match, dispatch, reschedule, simulate
int32_t dispatch_vp(Ctx* c, int32_t vp, double cost);
void lpt_stratified(int32_t n, const int32_t* classes, const double* costs, int32_t G,
                    const double* init_load, int32_t* out);
void simulate(Ctx* c, Flush* f, double* makespan, double* serial);

// executor.cpp
Executor* executor_create(Ctx* c, svp_status* st);
void executor_destroy(Executor* e);
// A flush in two halves (svp_flush_async overlaps the next flush's planning and issue with
// the device work between them): issue = tables, staging, enqueue, join into the external
// streams; complete = wait (watchdog), measured durations, Profiler.  abandon = after a
// failed issue, wait quietly for what was enqueued.
svp_status executor_issue(Executor* e, Flush* f);
svp_status executor_complete(Executor* e, Flush* f);
void executor_abandon(Executor* e, Flush* f);
std::string executor_error(Executor* e);

// numa.cpp: NUMA placement near a GPU (sysfs of its PCI function; -1 / false = unknown)
int gpu_numa_node(int ordinal);
bool parse_cpulist(const char* s, cpu_set_t* set);
bool gpu_local_cpus(int ordinal, cpu_set_t* set);
bool pin_thread_near_gpu(int ordinal, pthread_t th);
void executor_numa_info(Executor* e, int g, int32_t* node, int32_t* pinned);
void executor_forget_range(Executor* e, uintptr_t start, uintptr_t end);
svp_status host_alloc_near(int ordinal, size_t len, void** out, int* node_out, std::string* err);
void host_free_near(void* p, size_t len);
// residency check for svp_submit (validate_ptrs): returns SVP_OK or SVP_E_INVAL
// Residency check of one buffer [p, p + bytes) (cfg.validate_ptrs): declared DEVICE ->
// device (or managed) memory on the VP's GPU; HOST_PINNED -> page-locked host memory; and
// the whole range inside ONE allocation.  validate_ptrs 1 remembers every allocation range
// it has resolved (one driver query per allocation, not per submit); 2 queries every time.
// true if the chunk's kernel op really launches (chunk_needs_launch)
bool executor_chunk_launches(const Flush& f, const Chunk& ch);
// A batch of submits validates under one acquisition of the range cache's lock (the
// guard is a no-op without an executor or with validate_ptrs != 1).
struct RangeBatchLock {
    Executor* e = nullptr;
    explicit RangeBatchLock(Executor* ex);
    ~RangeBatchLock();
};
svp_status executor_check_ptr(Executor* e, const void* p, uint64_t bytes, int32_t mem, int32_t device,
                              std::string* why);

// errors
void set_error(const std::string& msg);

// used by the IPC front end (ipc.cpp)
svp_status ctx_submit_one(Ctx* c, const svp_job_desc& d, uint64_t* id);
uint64_t ctx_completed_upto(Ctx* c, int32_t unused = 0);
svp_status ctx_job_status(Ctx* c, uint64_t job);

}  // namespace svp

// executor.cpp -- per-GPU execution of a flush plan, device tables, staging arena and
// the Profiler.
//
//  * a5  segment / tile tables: built in pinned host memory, one H2D per GPU per flush
//        (skipped when byte-identical to the table already resident on the device).
//  * a6  H2D of host-resident inputs into the staging arena -- the paper's coalesced
//        "physically-contiguous" chunk (Fig 5), 256-B aligned slots,
//        element counts not padded.
//  * a7  one coalesced launch per chunk (kernels/*.cu).
//  * a8  D2H of each VP's outputs back to its own host buffer -- "the resulting data
//        are properly divided to be copied ... back to the host memory addresses"
//        (PAPER.md L303-306).
//  * a9  Kernel Interleaving: H2D / compute / D2H ops on separate streams linked by
//        events, so a chunk's copies overlap another chunk's kernel.
//  * a10 Profiler: CUDA events bracket every op; an op's device time is attributed to
//        its member VPs in proportion to algorithmic bytes (FLOPs for SGEMM).
//        PAPER.md L253-257 (the profiler "acquires ... elapsed clock cycles").
#include <cuda.h>
#include <cuda_runtime.h>
#include <stdlib.h>
#include <string.h>

#include <algorithm>
#include <chrono>
#include <condition_variable>
#include <map>
#include <mutex>
#include <thread>

#include "internal.h"
#include "launch.h"
#include "tables.h"

namespace svp {

#define CK(call)                                                                              \
    do {                                                                                      \
        cudaError_t _e = (call);                                                              \
        if (_e != cudaSuccess) {                                                              \
            d.err = std::string(#call) + " -> " + cudaGetErrorName(_e) + ": " + cudaGetErrorString(_e); \
            return SVP_E_CUDA;                                                                \
        }                                                                                     \
    } while (0)

struct MapKey {
    uint64_t a, b;
    int32_t M, N, K, variant;
    bool operator==(const MapKey& o) const {
        return a == o.a && b == o.b && M == o.M && N == o.N && K == o.K && variant == o.variant;
    }
};
struct MapKeyHash {
    size_t operator()(const MapKey& k) const {
        return std::hash<uint64_t>()(k.a * 1000003ull ^ k.b * 998244353ull ^ ((uint64_t)k.M << 40) ^
                                     ((uint64_t)k.N << 20) ^ (uint64_t)k.K ^ ((uint64_t)k.variant << 62));
    }
};
struct Maps2 {
    alignas(64) uint8_t a[128];
    alignas(64) uint8_t b[128];
};

struct Dev {
    int ordinal = 0;
    int idx = 0;
    std::vector<cudaStream_t> streams;  // [0] control, [1,S] compute, S+1 = H2D, S+2 = D2H
    cudaStream_t ext = nullptr;
    cudaStream_t own_ext = nullptr;     // created when the caller gave no external stream
    std::vector<cudaEvent_t> dep_ev, t_ev;
    cudaEvent_t ext_ev = nullptr, tbl_ev = nullptr;
    // join events per flush parity: an async flush (svp_flush_async) may still be in flight
    // while the next one is issued
    std::vector<cudaEvent_t> end_ev[2];
    // what the wait half of a flush needs from its issue half (per parity)
    struct Pending {
        bool active = false;
        bool prof = false;
        std::vector<cudaEvent_t> finals;
        std::vector<int32_t> tstart;
    };
    Pending pend[2];
    bool tbl_upload_inflight = false;  // tbl_host is the source of an enqueued upload
    uint8_t* arena = nullptr;
    uint64_t arena_bytes = 0;
    int numa_node = -1;       // the GPU's NUMA node (sysfs), -1 unknown
    bool cpu_pinned = false;  // its worker thread runs on the GPU's local CPUs
    // profile_level 2: per-segment busy-cycle counters of this flush's segment launches
    uint64_t* busy_dev = nullptr;
    size_t busy_cap = 0;  // counters
    // dynamic tile order of Black-Scholes / mixed launches: 2 self-resetting u32 per launch
    uint32_t* sched_dev = nullptr;
    size_t sched_cap = 0;  // slots
    // single-launch hist256: per launch nsegs * 257 self-resetting u32 (partials + arrivals)
    uint32_t* hscr_dev = nullptr;
    size_t hscr_cap = 0;  // u32
    // SGEMM tail split workspace (partial products), allocated once on first use
    float* tail_ws = nullptr;
    uint8_t* tbl_host = nullptr;
    uint8_t* tbl_dev = nullptr;
    size_t tbl_cap = 0;
    std::vector<uint8_t> tbl_last;      // host copy of the current tables (param launches read it)
    bool tbl_dev_valid = false;         // the device table buffer holds tbl_last
    LaunchLimits lim;
    std::unordered_map<MapKey, Maps2, MapKeyHash> map_cache;
    std::string err;
    uint64_t table_uploads = 0;
    // steady-state replay (cfg.graph): the device work of each recently seen plan as one
    // graph, keyed by plan generation (a serving loop that alternates input buffer sets
    // alternates plans).  Each graph owns a copy of its plan's device tables: the shared
    // tbl_dev holds whatever plan ran last.
    struct GraphEntry {
        cudaGraphExec_t gexec = nullptr;
        std::vector<int32_t> tstart;    // profiling event slots of each op inside the graph
        uint8_t* tbl = nullptr;         // the plan's device tables (device-table launches)
        size_t tbl_cap = 0;
        uint64_t last_use = 0;
    };
    std::unordered_map<uint64_t, GraphEntry> graphs;
    uint64_t graph_clock = 0;
    cudaEvent_t fork_ev = nullptr;
    std::vector<cudaEvent_t> join_ev;
};

// An allocation range resolved by executor_check_ptr (validate_ptrs 1 keeps them).
struct PtrRange {
    uintptr_t end = 0;
    int type = 0;    // cudaMemoryType
    int device = -1;
};

// Persistent per-GPU workers (multi-GPU contexts): GPU g > 0 is driven by worker thread g,
// created once at svp_init and parked on a condition variable between flushes (SURVEY §3.1
// step 4); the flushing thread drives GPU 0 itself.  A flush posts its plan with a new
// generation number and waits until every worker has finished its GPU's part.
struct Workers {
    std::mutex mu;
    std::condition_variable go, done;
    uint64_t gen = 0;
    int pending = 0;
    bool stop = false;
    Flush* f = nullptr;
    bool complete = false;   // this round: the issue half (false) or the wait half (true)
    std::vector<std::thread> th;
    std::vector<svp_status> st;
    std::vector<double> issue;
};

struct Executor {
    Ctx* c = nullptr;
    std::vector<Dev> devs;
    Workers w;
    std::string err;
    std::mutex rmu;                          // submits validate from many threads
    std::map<uintptr_t, PtrRange> ranges;    // allocation start -> range (validate_ptrs 1)
    // direct-mapped front of `ranges` by 2-MiB page (hits skip the tree walk)
    struct Hot {
        uintptr_t start = 0, end = 0;
        PtrRange r;
    };
    Hot hot[256];
};

static void start_workers(Executor* e);
static void stop_workers(Executor* e);

// the calling thread holds e->rmu through a RangeBatchLock
static thread_local Executor* t_range_locked = nullptr;

RangeBatchLock::RangeBatchLock(Executor* ex) {
    if (ex && ex->c->cfg.validate_ptrs == 1) {
        ex->rmu.lock();
        e = ex;
        t_range_locked = ex;
    }
}
RangeBatchLock::~RangeBatchLock() {
    if (e) {
        t_range_locked = nullptr;
        e->rmu.unlock();
    }
}

std::string executor_error(Executor* e) { return e->err; }

void executor_numa_info(Executor* e, int g, int32_t* node, int32_t* pinned) {
    *node = e->devs[g].numa_node;
    *pinned = e->devs[g].cpu_pinned ? 1 : 0;
}

static svp_status dev_setup(Dev& d, const svp_config& cfg, void* ext) {
    CK(cudaSetDevice(d.ordinal));
    CK(cudaFree(0));  // create / adopt the primary context
    // [0] control stream (table uploads, graph capture / launch, joins); plan stream k runs on
    // [k + 1]: compute 0..S-1, H2D S, D2H S+1.  Kernels and copies never share the control
    // stream: in the host-resident cfg5 timeline a compute stream that also carried the
    // control work started its first kernel ~100 ms late on repeated flushes, stalling every
    // D2H behind it (profiles/r02/e2e/)
    const int S = cfg.streams_per_gpu;
    d.streams.resize(S + 3);
    for (auto& s : d.streams) CK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
    // the stream a flush forks from and joins into: the caller's, else one of our own, so
    // consecutive flushes (svp_flush_async keeps one in flight) always run in order
    d.ext = (cudaStream_t)ext;
    if (!d.ext) {
        CK(cudaStreamCreateWithFlags(&d.own_ext, cudaStreamNonBlocking));
        d.ext = d.own_ext;
    }
    CK(cudaEventCreateWithFlags(&d.ext_ev, cudaEventDisableTiming));
    CK(cudaEventCreateWithFlags(&d.tbl_ev, cudaEventDisableTiming));
    for (auto& set : d.end_ev) {
        set.resize(S + 3);
        for (auto& e : set) CK(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
    }
    d.join_ev.resize(S + 3);
    for (auto& e : d.join_ev) CK(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
    CK(cudaEventCreateWithFlags(&d.fork_ev, cudaEventDisableTiming));
    d.arena_bytes = cfg.arena_bytes;
    d.numa_node = gpu_numa_node(d.ordinal);
    CK(query_limits(&d.lim));
    return SVP_OK;
}

static void dev_teardown(Dev& d) {
    cudaSetDevice(d.ordinal);
    for (auto& s : d.streams) if (s) cudaStreamSynchronize(s);
    for (auto& s : d.streams) if (s) cudaStreamDestroy(s);
    if (d.own_ext) {
        cudaStreamSynchronize(d.own_ext);
        cudaStreamDestroy(d.own_ext);
    }
    for (auto e : d.dep_ev) cudaEventDestroy(e);
    for (auto e : d.t_ev) cudaEventDestroy(e);
    for (auto& set : d.end_ev)
        for (auto e : set) cudaEventDestroy(e);
    for (auto e : d.join_ev) cudaEventDestroy(e);
    if (d.fork_ev) cudaEventDestroy(d.fork_ev);
    for (auto& kv : d.graphs) {
        if (kv.second.gexec) cudaGraphExecDestroy(kv.second.gexec);
        if (kv.second.tbl) cudaFree(kv.second.tbl);
    }
    d.graphs.clear();
    if (d.ext_ev) cudaEventDestroy(d.ext_ev);
    if (d.tbl_ev) cudaEventDestroy(d.tbl_ev);
    if (d.arena) cudaFree(d.arena);
    if (d.busy_dev) cudaFree(d.busy_dev);
    if (d.sched_dev) cudaFree(d.sched_dev);
    if (d.hscr_dev) cudaFree(d.hscr_dev);
    if (d.tail_ws) cudaFree(d.tail_ws);
    if (d.tbl_dev) cudaFree(d.tbl_dev);
    if (d.tbl_host) cudaFreeHost(d.tbl_host);
}

Executor* executor_create(Ctx* c, svp_status* st) {
    Executor* e = new Executor();
    e->c = c;
    int count = 0;
    cudaError_t ce = cudaGetDeviceCount(&count);
    if (ce != cudaSuccess || count == 0) {
        e->err = std::string("no CUDA device: ") + cudaGetErrorString(ce);
        set_error(e->err);
        *st = SVP_E_CUDA;
        delete e;
        return nullptr;
    }
    if (c->ngpu == 0) c->ngpu = count;
    if (c->device_ids.empty())
        for (int i = 0; i < c->ngpu; ++i) c->device_ids.push_back(i);
    e->devs.resize(c->ngpu);
    for (int i = 0; i < c->ngpu; ++i) {
        Dev& d = e->devs[i];
        d.idx = i;
        d.ordinal = c->device_ids[i];
        if (d.ordinal < 0 || d.ordinal >= count) {
            e->err = "device ordinal out of range";
            set_error(e->err);
            *st = SVP_E_INVAL;
            executor_destroy(e);
            return nullptr;
        }
        void* ext = c->cfg.external_streams ? c->cfg.external_streams[i] : nullptr;
        if (dev_setup(d, c->cfg, ext) != SVP_OK) {
            e->err = d.err;
            set_error(e->err);
            *st = SVP_E_CUDA;
            executor_destroy(e);
            return nullptr;
        }
    }
    start_workers(e);
    *st = SVP_OK;
    return e;
}

static svp_status run_device(Executor* e, Dev& d, Flush& f, double* issue_ns);
static svp_status complete_device(Executor* e, Dev& d, Flush& f);

static void worker_loop(Executor* e, int g) {
    Workers& w = e->w;
    uint64_t seen = 0;
    for (;;) {
        Flush* f = nullptr;
        bool complete = false;
        {
            std::unique_lock<std::mutex> lk(w.mu);
            w.go.wait(lk, [&] { return w.stop || w.gen != seen; });
            if (w.stop) return;
            seen = w.gen;
            f = w.f;
            complete = w.complete;
        }
        double issue = 0;
        const svp_status st = complete ? complete_device(e, e->devs[g], *f) : run_device(e, e->devs[g], *f, &issue);
        std::lock_guard<std::mutex> lk(w.mu);
        w.st[g] = st;
        if (!complete) w.issue[g] = issue;
        if (--w.pending == 0) w.done.notify_one();
    }
}

static void start_workers(Executor* e) {
    const int G = (int)e->devs.size();
    e->w.st.assign(G, SVP_OK);
    e->w.issue.assign(G, 0.0);
    for (int g = 1; g < G; ++g) {
        e->w.th.emplace_back(worker_loop, e, g);
        // worker g runs on the CPUs next to its GPU (numa.cpp; SVP_NUMA_AFFINITY=0 disables)
        e->devs[g].cpu_pinned = pin_thread_near_gpu(e->devs[g].ordinal, e->w.th.back().native_handle());
    }
}

static void stop_workers(Executor* e) {
    {
        std::lock_guard<std::mutex> lk(e->w.mu);
        e->w.stop = true;
    }
    e->w.go.notify_all();
    for (auto& t : e->w.th) t.join();
    e->w.th.clear();
}

void executor_destroy(Executor* e) {
    if (!e) return;
    stop_workers(e);
    for (auto& d : e->devs) dev_teardown(d);
    delete e;
}

svp_status executor_register_host(Executor* e, void* p, uint64_t bytes, std::string* why) {
    if (e->devs.empty()) return SVP_OK;
    cudaSetDevice(e->devs[0].ordinal);
    cudaError_t ce = cudaHostRegister(p, bytes, cudaHostRegisterPortable);
    if (ce != cudaSuccess) {
        cudaGetLastError();
        *why = cudaGetErrorString(ce);
        return SVP_E_CUDA;
    }
    return SVP_OK;
}

void executor_unregister_host(Executor* e, void* p) {
    if (e->devs.empty()) return;
    cudaSetDevice(e->devs[0].ordinal);
    cudaHostUnregister(p);
    cudaGetLastError();
    // forget the remembered range (validate_ptrs 1): it is no longer page-locked
    std::lock_guard<std::mutex> lk(e->rmu);
    auto it = e->ranges.upper_bound((uintptr_t)p);
    if (it != e->ranges.begin()) {
        --it;
        if ((uintptr_t)p < it->second.end) e->ranges.erase(it);
    }
    for (auto& h : e->hot) h = Executor::Hot();
}

// Allocation range of p through the driver (CU_POINTER_ATTRIBUTE_RANGE_START_ADDR / _SIZE);
// the entry point is fetched at runtime, libsvp does not link libcuda.  false: unknown.
typedef CUresult (*PFN_ptrAttr)(void*, CUpointer_attribute, CUdeviceptr);
static bool alloc_range(const void* p, uintptr_t* start, uintptr_t* end) {
    static PFN_ptrAttr fn = [] {
        void* q = nullptr;
        cudaDriverEntryPointQueryResult r;
        if (cudaGetDriverEntryPoint("cuPointerGetAttribute", &q, cudaEnableDefault, &r) != cudaSuccess ||
            r != cudaDriverEntryPointSuccess)
            q = nullptr;
        return reinterpret_cast<PFN_ptrAttr>(q);
    }();
    if (!fn) return false;
    CUdeviceptr base = 0;
    size_t size = 0;
    if (fn(&base, CU_POINTER_ATTRIBUTE_RANGE_START_ADDR, (CUdeviceptr)p) != CUDA_SUCCESS ||
        fn(&size, CU_POINTER_ATTRIBUTE_RANGE_SIZE, (CUdeviceptr)p) != CUDA_SUCCESS || size == 0)
        return false;
    *start = (uintptr_t)base;
    *end = (uintptr_t)base + size;
    return true;
}

// An allocation [start, end) was released (svp_host_free): drop its cached ranges so an
// address reused later is resolved afresh.
void executor_forget_range(Executor* e, uintptr_t start, uintptr_t end) {
    std::lock_guard<std::mutex> lk(e->rmu);
    for (auto it = e->ranges.lower_bound(start); it != e->ranges.end() && it->first < end;)
        it = e->ranges.erase(it);
    for (auto& h : e->hot)
        if (h.start < end && start < h.end) h = Executor::Hot{};
}

svp_status executor_check_ptr(Executor* e, const void* p, uint64_t bytes, int32_t mem, int32_t device,
                              std::string* why) {
    const uintptr_t a = (uintptr_t)p;
    const bool cached = e->c->cfg.validate_ptrs == 1;
    PtrRange r;
    bool hit = false, known = false;
    // a RangeBatchLock of this thread already holds the lock
    std::unique_lock<std::mutex> lk(e->rmu, std::defer_lock);
    if (cached && t_range_locked != e) lk.lock();
    Executor::Hot& hot = e->hot[(a >> 21) & 255];
    if (cached) {
        if (hot.start <= a && a < hot.end) {
            r = hot.r;
            hit = known = true;
        } else {
            auto it = e->ranges.upper_bound(a);
            if (it != e->ranges.begin()) {
                --it;
                if (a < it->second.end) {
                    r = it->second;
                    hit = known = true;
                    hot.start = it->first;
                    hot.end = it->second.end;
                    hot.r = it->second;
                }
            }
        }
    }
    if (!hit) {
        cudaPointerAttributes at;
        cudaError_t ce = cudaPointerGetAttributes(&at, p);
        if (ce != cudaSuccess) {
            cudaGetLastError();
            *why = std::string("cudaPointerGetAttributes failed: ") + cudaGetErrorString(ce);
            return SVP_E_INVAL;
        }
        r.type = (int)at.type;
        r.device = at.device;
        uintptr_t st = 0, en = 0;
        if (at.type != cudaMemoryTypeUnregistered && alloc_range(p, &st, &en) && st <= a && a < en) {
            r.end = en;
            known = true;
            if (cached) {
                e->ranges[st] = r;  // under lk or the batch lock
                hot.start = st;
                hot.end = en;
                hot.r = r;
            }
        }
    }
    if (mem == SVP_MEM_DEVICE) {
        if (r.type != cudaMemoryTypeDevice && r.type != cudaMemoryTypeManaged) {
            *why = "declared DEVICE but is not device memory";
            return SVP_E_INVAL;
        }
        if (r.type == cudaMemoryTypeDevice && r.device != e->devs[device].ordinal) {
            *why = "device buffer is on CUDA device " + std::to_string(r.device) + " but the VP runs on " +
                   std::to_string(e->devs[device].ordinal) + " (see svp_vp_device)";
            return SVP_E_INVAL;
        }
    } else {
        if (r.type != cudaMemoryTypeHost) {
            *why = "declared HOST_PINNED but is not page-locked host memory";
            return SVP_E_INVAL;
        }
    }
    if (known && bytes > r.end - a) {
        *why = "buffer of " + std::to_string(bytes) + " B extends " + std::to_string(bytes - (r.end - a)) +
               " B past the end of its allocation";
        return SVP_E_INVAL;
    }
    return SVP_OK;
}

// ------------------------------------------------------------------ tables (a5)
static int elem_size(int kernel, int b) { return (kernel == K_HIST256 && b == 0) ? 1 : 4; }
static int tile_elems(int kernel) {
    switch (kernel) {
        case K_VECADD: return kVecaddTile;
        case K_SAXPY: return kSaxpyTile;
        case K_BLACKSCHOLES: return kBsTile;
        case K_HIST256: return kHistTile;
    }
    return 0;
}

static size_t align_up(size_t x, size_t a) { return (x + a - 1) / a * a; }

// Resolve the device address the kernel uses for every buffer of every job in the chunk.
static void resolve_addresses(Dev& d, const Flush& f, Chunk& ch) {
    ch.staged.clear();
    uint64_t off = ch.arena_off;
    for (int32_t ji : ch.jobs) {
        const Job& j = f.jobs[ji];
        for (int b = 0; b < SVP_MAX_BUFS; ++b) {
            if (b >= j.nbufs) {
                ch.staged.push_back(0);
                continue;
            }
            if (j.bufs[b].mem == SVP_MEM_HOST_PINNED) {
                ch.staged.push_back((uint64_t)(d.arena + off));
                off += align_up(touched_bytes(j, b), 256);
            } else {
                ch.staged.push_back((uint64_t)j.bufs[b].ptr);
            }
        }
    }
}

// SGEMM tail split (SVP_SGEMM_TAIL=0: off): see plan_sgemm_tail.
static bool sgemm_tail_split() {
    static const bool on = !(getenv("SVP_SGEMM_TAIL") && atoi(getenv("SVP_SGEMM_TAIL")) == 0);
    return on;
}
constexpr size_t kTailWsFloats = (size_t)8 << 20;  // 32 MiB: up to 128 pieces of 256 x 256

// Dynamic tile order for Black-Scholes / mixed launches (SVP_EW_DYN=0: static order).
static bool ew_dynamic_order() {
    static const bool on = !(getenv("SVP_EW_DYN") && atoi(getenv("SVP_EW_DYN")) == 0);
    return on;
}

// SVP_HIST_DYN=1: hist256 in dynamic chunk order instead of the static blocked tile ranges.
// Measured (profiles/r02/hist_dyn/): the dynamic order makes a CTA visit more VPs, and each
// VP switch costs a flush of the replicated table (256 column sums of 32 replicas + 256
// global atomics), which outweighed the balance gain (cfg5 hist launch 3.09 -> 2.82 TB/s):
// off by default, SVP_HIST_DYN=1 enables it.
static bool hist_dynamic_order() {
    static const bool on = getenv("SVP_HIST_DYN") && atoi(getenv("SVP_HIST_DYN")) == 1;
    return on;
}

// SVP_HIST_FUSED=1: hist256 as ONE launch with a self-resetting per-launch scratch (the
// last CTA of each VP writes its counts) instead of a zeroing kernel + the accumulating
// launch.  Off by default: alone it was 2 us (4 %) faster per cfg5 hist launch, but the
// interleaved cfg5 step measured ~1 % slower with it (profiles/r01/hist_fused/).
static bool hist_single_launch() {
    static const bool on = getenv("SVP_HIST_FUSED") && atoi(getenv("SVP_HIST_FUSED")) != 0;
    return on;
}

// SGEMM tail split.  A wide (256 x 512 pair tile) launch over T tiles and P CTA pairs runs
// floor(T / P) full waves and a last wave of R = T mod P tiles, during which P - R pairs
// idle (cfg5: 1632 tiles, 74 pairs -> R = 4: ~110 us at 4/74 occupancy,
// profiles/r01/sgemm_waves.jsonl).  When R <= P / 2, the main launch stops after the full
// waves and the R tail tiles become 256 x 256 sub-tiles split along K into S slices
// (sub-tiles x S <= P): one wave of the narrow pair kernel writes the partial products to
// a workspace, and a reduction kernel sums them in a fixed order into C (alpha, beta).
// Same per-product arithmetic; the K sum is regrouped into S fp32 partial sums.
static svp_status plan_sgemm_tail(Executor* e, Dev& d, Flush& f, Chunk& ch, std::vector<uint8_t>& tbl, int P) {
    ch.main_tiles = ch.total_tiles;
    ch.tail_n = ch.tail_nred = 0;
    const uint32_t T = ch.total_tiles;
    if (!sgemm_tail_split() || !ch.wide || P < 2 || T < (uint32_t)P) return SVP_OK;
    const uint32_t R = T % (uint32_t)P;
    if (R == 0 || R > (uint32_t)P / 2) return SVP_OK;
    constexpr int WM = 2 * kTf32BM, WN = 2 * kTf32BN, SN = kTf32BN;  // wide tile, sub-tile width
    struct Sub {
        size_t k;  // job index in the chunk
        int m0, n0, rows, cols;
    };
    std::vector<Sub> subs;
    const GemmDesc* gd = reinterpret_cast<const GemmDesc*>(tbl.data() + ch.table_off);
    for (uint32_t t = T - R; t < T; ++t) {
        size_t k = 0;
        while (k + 1 < ch.jobs.size() && gd[k + 1].tile_begin <= t) ++k;
        const Job& j = f.jobs[ch.jobs[k]];
        const uint32_t lt = t - gd[k].tile_begin;
        const int tm = (int)(lt / gd[k].tiles_n), tn = (int)(lt % gd[k].tiles_n);
        const int m0 = tm * WM, rows = std::min(WM, j.M - m0);
        for (int h = 0; h < WN / SN; ++h) {
            const int n0 = tn * WN + h * SN;
            if (n0 < j.N) subs.push_back(Sub{k, m0, n0, rows, std::min(SN, j.N - n0)});
        }
    }
    int K = 0;
    for (const auto& sb : subs) K = std::max(K, f.jobs[ch.jobs[sb.k]].K);
    int S = std::min<int>(P / (int)subs.size(), K / 64);
    if (S < 2) return SVP_OK;
    // K-chunked mode (R23): the slices run as single accumulations, so each must fit in a chunk
    const int kc = sgemm_chunk_k(ch.sgemm_impl, e->c->cfg.sgemm_kchunk);
    if (kc > 0 && (K + S - 1) / S > kc) return SVP_OK;
    size_t ws_need = 0;
    for (const auto& sb : subs) ws_need += (size_t)S * sb.rows * sb.cols;
    if (ws_need > kTailWsFloats) return SVP_OK;
    if (!d.tail_ws) {
        cudaError_t ce = cudaMalloc(&d.tail_ws, kTailWsFloats * sizeof(float));
        if (ce != cudaSuccess) {
            cudaGetLastError();
            d.tail_ws = nullptr;
            return SVP_OK;  // no workspace: run the plain last wave
        }
    }
    // pieces: per sub-tile, S K-slices of Kp (multiple of the 16-k block) each
    std::vector<GemmDesc> pd;
    std::vector<uint8_t> pm;
    std::vector<TailRed> rd;
    size_t ws_off = 0;
    for (const auto& sb : subs) {
        const Job& j = f.jobs[ch.jobs[sb.k]];
        const float* A = (const float*)ch.staged[sb.k * SVP_MAX_BUFS + 0];
        const float* B = (const float*)ch.staged[sb.k * SVP_MAX_BUFS + 1];
        float* Cp = (float*)ch.staged[sb.k * SVP_MAX_BUFS + 2];
        const int Kp = ((j.K + S - 1) / S + kTf32BK - 1) / kTf32BK * kTf32BK;
        const int Se = (j.K + Kp - 1) / Kp;  // slices this sub-tile really has (<= S)
        const size_t plane = (size_t)sb.rows * sb.cols;
        TailRed r;
        memset(&r, 0, sizeof(r));
        r.C = Cp + (size_t)sb.m0 * j.N + sb.n0;
        r.ws = d.tail_ws + ws_off;
        r.ldc = j.N;
        r.rows = sb.rows;
        r.cols = sb.cols;
        r.S = Se;
        r.alpha = j.f0;
        r.beta = j.f1;
        rd.push_back(r);
        for (int s = 0; s < Se; ++s) {
            const int k0 = s * Kp, kl = std::min(Kp, j.K - k0);
            GemmDesc g;
            memset(&g, 0, sizeof(g));
            g.C = d.tail_ws + ws_off + (size_t)s * plane;
            g.M = sb.rows;
            g.N = sb.cols;
            g.K = kl;
            g.alpha = 1.f;
            g.beta = 0.f;
            g.tile_begin = (uint32_t)pd.size();
            g.tiles_n = 1;
            g.A = A + (size_t)sb.m0 * j.K + k0;  // the slice's operand views (exact-recompute path)
            g.B = B + (size_t)k0 * j.N + sb.n0;
            g.lda = j.K;
            g.ldb = j.N;
            pd.push_back(g);
            alignas(64) uint8_t m[256];  // CUtensorMap is 64-B aligned
            if (encode_gemm_maps_view(m, m + 128, A + (size_t)sb.m0 * j.K + k0, B + (size_t)k0 * j.N + sb.n0, sb.rows,
                                      sb.cols, kl, j.K, j.N) != 0) {
                d.err = "cuTensorMapEncodeTiled failed for an sgemm tail slice";
                return SVP_E_CUDA;
            }
            pm.insert(pm.end(), m, m + 256);
        }
        ws_off += (size_t)Se * plane;
    }
    ch.tail_maps_off = align_up(tbl.size(), 128);
    ch.tail_table_off = ch.tail_maps_off + pm.size();
    ch.tail_red_off = align_up(ch.tail_table_off + pd.size() * sizeof(GemmDesc), 128);
    tbl.resize(ch.tail_red_off + rd.size() * sizeof(TailRed));
    memcpy(tbl.data() + ch.tail_maps_off, pm.data(), pm.size());
    memcpy(tbl.data() + ch.tail_table_off, pd.data(), pd.size() * sizeof(GemmDesc));
    memcpy(tbl.data() + ch.tail_red_off, rd.data(), rd.size() * sizeof(TailRed));
    ch.main_tiles = T - R;
    ch.tail_n = (int32_t)pd.size();
    ch.tail_nred = (int32_t)rd.size();
    ch.kernel_launches = 3;
    return SVP_OK;
}

static svp_status build_tables(Executor* e, Dev& d, Flush& f, std::vector<uint8_t>& tbl) {
    tbl.clear();
    // launches that share their level with other kernel launches on this GPU co-run with them
    std::map<int32_t, int> chunks_in_level;
    for (const auto& ch : f.chunks)
        if (ch.device == d.idx) chunks_in_level[ch.level] += 1;
    for (auto& ch : f.chunks) {
        if (ch.device != d.idx) continue;
        resolve_addresses(d, f, ch);
        const bool gemm = ch.kernel == K_SGEMM || ch.kernel == K_SGEMM_TF32;
        if (ch.kernel == K_DGEMM) {
            ch.table_off = align_up(tbl.size(), 128);
            tbl.resize(ch.table_off + ch.jobs.size() * sizeof(DgemmDesc));
            // 32x32 tiles when the launch has fewer than 2 waves of 64x64 tiles
            uint64_t big = 0;
            for (int32_t ji : ch.jobs) {
                const Job& j = f.jobs[ji];
                if ((int64_t)j.M * j.N > 0)
                    big += (uint64_t)((j.M + kDgemmBM - 1) / kDgemmBM) * ((j.N + kDgemmBN - 1) / kDgemmBN);
            }
            ch.small_tiles = dgemm_dmma_enabled() || big < 2ull * d.lim.num_sms * d.lim.dgemm_blocks_per_sm;
            const int TM = ch.small_tiles ? kDgemmSmall : kDgemmBM, TN = ch.small_tiles ? kDgemmSmall : kDgemmBN;
            uint32_t tiles = 0;
            for (size_t k = 0; k < ch.jobs.size(); ++k) {
                const Job& j = f.jobs[ch.jobs[k]];
                DgemmDesc g;
                memset(&g, 0, sizeof(g));
                g.A = (const double*)ch.staged[k * SVP_MAX_BUFS + 0];
                g.B = (const double*)ch.staged[k * SVP_MAX_BUFS + 1];
                g.C = (double*)ch.staged[k * SVP_MAX_BUFS + 2];
                g.M = j.M;
                g.N = j.N;
                g.K = j.K;
                g.alpha = j.d0;
                g.beta = j.d1;
                g.tile_begin = tiles;
                g.tiles_n = (uint32_t)((j.N + TN - 1) / TN);
                uint64_t nt = (int64_t)j.M * j.N == 0 ? 0 : (uint64_t)((j.M + TM - 1) / TM) * g.tiles_n;
                tiles += (uint32_t)nt;
                memcpy(tbl.data() + ch.table_off + k * sizeof(DgemmDesc), &g, sizeof(g));
            }
            ch.total_tiles = tiles;
            ch.nsegs = (int32_t)ch.jobs.size();
        } else if (!gemm) {
            ch.table_off = align_up(tbl.size(), 128);
            tbl.resize(ch.table_off + ch.jobs.size() * sizeof(SegDesc));
            SegDesc* seg = reinterpret_cast<SegDesc*>(tbl.data() + ch.table_off);
            uint32_t tiles = 0;
            for (size_t k = 0; k < ch.jobs.size(); ++k) {
                const Job& j = f.jobs[ch.jobs[k]];
                const int T = tile_elems(j.kernel);  // per segment: K_EW_MIX mixes tile sizes
                SegDesc s;
                memset(&s, 0, sizeof(s));
                int nalign = j.kernel == K_HIST256 ? 1 : j.nbufs;  // counts need no alignment
                const uint64_t mis = ch.staged[k * SVP_MAX_BUFS] & 15;
                bool co = true;
                for (int b = 0; b < j.nbufs; ++b) {
                    s.ptr[b] = ch.staged[k * SVP_MAX_BUFS + b];
                    if (b < nalign && (s.ptr[b] & 15) != mis) co = false;
                }
                s.n = j.n;
                uint64_t nt = 0;
                bool scalar = false;
                seg_layout(s.ptr[0], co, elem_size(j.kernel, 0), T, j.n, &s.shift, &nt, &scalar);
                s.flags = (uint16_t)((scalar ? SEG_SCALAR : 0) | (j.kernel << SEG_KIND_SHIFT));
                s.f[0] = j.f0;
                s.f[1] = j.f1;
                s.tile_begin = tiles;
                if (tiles + nt >= (1ull << 31)) {
                    d.err = "svp_flush: coalesced launch exceeds 2^31 tiles";
                    return SVP_E_UNSUPPORTED;
                }
                tiles += (uint32_t)nt;
                seg[k] = s;
            }
            ch.total_tiles = tiles;
            ch.nsegs = (int32_t)ch.jobs.size();
            ch.param = e->c->cfg.table_mode == SVP_TABLE_PARAM && ch.nsegs <= kParamSegs;
            // hist256: the zeroing kernel precedes the accumulating launch (unless single-launch)
            ch.kernel_launches = ch.kernel == K_HIST256 && !hist_single_launch() && tiles > 0 ? 2 : 1;
        } else {
            // tcgen05 tiles for sgemm_tf32 and for sgemm with the 3xTF32 implementation
            const bool plain = ch.sgemm_impl == kSgemmPlain;
            const int variant = !plain && (ch.kernel == K_SGEMM_TF32 || ch.sgemm_impl != SVP_SGEMM_FFMA) ? 1 : 0;
            const bool pair = variant && ch.kernel == K_SGEMM && sgemm_tc_cta_pair();
            // wide (256 x 512) pair tiles halve the A-side conversion and L2 traffic per flop
            // but halve the tile count: used when they still fill >= 2 waves of CTA pairs
            bool wide = false;
            if (pair && ch.sgemm_impl == SVP_SGEMM_TF32BF16) {
                const int mode = sgemm_tc_wide_mode();
                uint64_t tw = 0;
                for (int32_t ji : ch.jobs) {
                    const Job& j = f.jobs[ji];
                    if ((int64_t)j.M * j.N > 0)
                        tw += (uint64_t)((j.M + 2 * kTf32BM - 1) / (2 * kTf32BM)) * ((j.N + 2 * kTf32BN - 1) / (2 * kTf32BN));
                }
                wide = mode == 2 || (mode == 1 && tw >= 2ull * (uint64_t)(d.lim.num_sms / 2));
            }
            ch.wide = wide;
            const int BM = plain ? kSgemmPlainTile : variant ? (pair ? 2 * kTf32BM : kTf32BM) : kGemmBM;
            const int BN = plain ? kSgemmPlainTile : variant ? (wide ? 2 * kTf32BN : kTf32BN) : kGemmBN;
            ch.maps_off = align_up(tbl.size(), 128);
            size_t nj = ch.jobs.size();
            ch.table_off = ch.maps_off + nj * 256;
            tbl.resize(ch.table_off + nj * sizeof(GemmDesc));
            uint32_t tiles = 0;
            for (size_t k = 0; k < nj; ++k) {
                const Job& j = f.jobs[ch.jobs[k]];
                GemmDesc g;
                memset(&g, 0, sizeof(g));
                const float* A = (const float*)ch.staged[k * SVP_MAX_BUFS + 0];
                const float* B = (const float*)ch.staged[k * SVP_MAX_BUFS + 1];
                g.C = (float*)ch.staged[k * SVP_MAX_BUFS + 2];
                g.M = j.M;
                g.N = j.N;
                g.K = j.K;
                g.alpha = j.f0;
                g.beta = j.f1;
                g.tile_begin = tiles;
                g.tiles_n = (uint32_t)((j.N + BN - 1) / BN);
                g.A = A;
                g.B = B;
                g.lda = j.K;
                g.ldb = j.N;
                uint64_t nt = (uint64_t)((j.M + BM - 1) / BM) * g.tiles_n;
                if ((int64_t)j.M * j.N == 0) nt = 0;
                tiles += (uint32_t)nt;
                uint8_t* mp = tbl.data() + ch.maps_off + k * 256;
                if (nt && j.K > 0 && !plain) {
                    MapKey key{(uint64_t)A, (uint64_t)B, j.M, j.N, j.K, variant};
                    auto it = d.map_cache.find(key);
                    if (it == d.map_cache.end()) {
                        Maps2 m;
                        if (encode_gemm_maps(m.a, m.b, A, B, j.M, j.N, j.K, variant) != 0) {
                            d.err = "cuTensorMapEncodeTiled failed for an sgemm job";
                            return SVP_E_CUDA;
                        }
                        if (d.map_cache.size() > 4096) d.map_cache.clear();
                        it = d.map_cache.emplace(key, m).first;
                    }
                    memcpy(mp, it->second.a, 128);
                    memcpy(mp + 128, it->second.b, 128);
                } else {
                    memset(mp, 0, 256);
                }
                memcpy(tbl.data() + ch.table_off + k * sizeof(GemmDesc), &g, sizeof(g));
            }
            ch.total_tiles = tiles;
            ch.nsegs = (int32_t)nj;
            ch.kernel_launches = 1;
            ch.main_tiles = tiles;
            ch.tail_n = ch.tail_nred = 0;
            ch.cmaps_off = -1;
            if (variant && ch.kernel == K_SGEMM) {
                // one TMA map of C per VP: the epilogue of beta == 0 tiles writes C by TMA (and
                // folds K chunks with TMA reduce-add, R23); cached per (C, M, N)
                const size_t coff = align_up(tbl.size(), 128);
                tbl.resize(coff + nj * 128);
                for (size_t k = 0; k < nj; ++k) {
                    const Job& j = f.jobs[ch.jobs[k]];
                    uint8_t* mp = tbl.data() + coff + k * 128;
                    float* Cp = (float*)ch.staged[k * SVP_MAX_BUFS + 2];
                    if ((int64_t)j.M * j.N > 0 && j.K > 0) {
                        MapKey key{(uint64_t)Cp, 0, j.M, j.N, 0, 7};
                        auto it = d.map_cache.find(key);
                        if (it == d.map_cache.end()) {
                            Maps2 m;
                            if (encode_c_map(m.a, Cp, j.M, j.N) != 0) {
                                d.err = "cuTensorMapEncodeTiled failed for an sgemm C map";
                                return SVP_E_CUDA;
                            }
                            if (d.map_cache.size() > 4096) d.map_cache.clear();
                            it = d.map_cache.emplace(key, m).first;
                        }
                        memcpy(mp, it->second.a, 128);
                    } else {
                        memset(mp, 0, 128);
                    }
                }
                ch.cmaps_off = (int64_t)coff;
            }
            // tail split only for a launch that has the GPU to itself: co-running with the
            // memory-bound launches of an interleaved level, the last wave's idle pairs are
            // not idle GPU time, and the power-capped step measured 0.7-2 % slower with the
            // extra slice pass (profiles/r01/sgemm_tail/)
            const bool alone = !e->c->cfg.interleave || chunks_in_level[ch.level] == 1;
            if (alone && ch.kernel == K_SGEMM && ch.sgemm_impl == SVP_SGEMM_TF32BF16) {
                const int P = (int)std::min<uint64_t>(tiles, (uint64_t)d.lim.num_sms / 2);
                svp_status st = plan_sgemm_tail(e, d, f, ch, tbl, P);
                if (st) return st;
            }
        }
    }
    return SVP_OK;
}

static cudaEvent_t pool_get(Dev& d, std::vector<cudaEvent_t>& pool, size_t i, bool timing) {
    while (pool.size() <= i) {
        cudaEvent_t ev;
        if (cudaEventCreateWithFlags(&ev, timing ? cudaEventDefault : cudaEventDisableTiming) != cudaSuccess)
            return nullptr;
        pool.push_back(ev);
    }
    (void)d;
    return pool[i];
}

// Captured graphs hold the addresses of the per-device scratch buffers: a reallocation
// drops every one of them (they are re-captured on the plans' next sightings).
// Before freeing or replacing anything the device work of a still-pending async flush may
// use (scratch buffers, captured graphs, the table buffers): let that work finish.
static svp_status quiesce(Dev& d) {
    if (d.pend[0].active || d.pend[1].active) CK(cudaDeviceSynchronize());
    return SVP_OK;
}

static svp_status drop_graphs(Dev& d) {
    if (svp_status q = quiesce(d)) return q;
    for (auto& kv : d.graphs) {
        if (kv.second.gexec) CK(cudaGraphExecDestroy(kv.second.gexec));
        if (kv.second.tbl) CK(cudaFree(kv.second.tbl));
    }
    d.graphs.clear();
    return SVP_OK;
}

static constexpr size_t kGraphsPerDevice = 32;

// base: the device table buffer the launch reads (d.tbl_dev, or a captured plan's own copy)
static cudaError_t launch_chunk(Dev& d, const Chunk& ch, int cfg_kchunk, cudaStream_t s, const uint8_t* base) {
    const int sgemm_impl = ch.sgemm_impl;
    const int kchunk = sgemm_chunk_k(sgemm_impl, cfg_kchunk);
    if (ch.total_tiles == 0 && ch.kernel != K_HIST256) return cudaSuccess;
    uint64_t* busy = ch.busy_off >= 0 ? d.busy_dev + ch.busy_off : nullptr;
    uint32_t* sched = ch.sched_slot >= 0 ? d.sched_dev + 2 * ch.sched_slot : nullptr;
    uint32_t* hscr = ch.hscr_off >= 0 ? d.hscr_dev + ch.hscr_off : nullptr;
    if (busy) {
        cudaError_t e = cudaMemsetAsync(busy, 0, (size_t)ch.nsegs * sizeof(uint64_t), s);
        if (e) return e;
    }
    auto grid_of = [&](int per_sm) {
        if (ch.co_grid > 0) per_sm = std::min(per_sm, (int)ch.co_grid);
        return (int)std::max<uint64_t>(1, std::min<uint64_t>(ch.total_tiles, (uint64_t)d.lim.num_sms * per_sm));
    };
    if (ch.param) {
        // table by value: copied into the launch's parameter buffer at enqueue time
        const SegDesc* p = reinterpret_cast<const SegDesc*>(d.tbl_last.data() + ch.table_off);
        switch (ch.kernel) {
            case K_VECADD:
            case K_SAXPY: return launch_ew_param(ch.kernel, p, ch.nsegs, ch.total_tiles, grid_of(d.lim.ew_blocks_per_sm), s, busy);
            case K_BLACKSCHOLES:
                return launch_ew_param(ch.kernel, p, ch.nsegs, ch.total_tiles, grid_of(d.lim.bs_blocks_per_sm), s, busy, sched);
            case K_EW_MIX:
                return launch_ew_param(ch.kernel, p, ch.nsegs, ch.total_tiles, grid_of(d.lim.mix_blocks_per_sm), s, busy, sched);
            case K_HIST256:
                return launch_hist256_param(p, ch.nsegs, ch.total_tiles, grid_of(d.lim.hist_blocks_per_sm), s, busy, hscr,
                                            sched);
        }
        return cudaErrorInvalidValue;
    }
    switch (ch.kernel) {
        case K_VECADD:
            return launch_vecadd((const SegDesc*)(base + ch.table_off), ch.nsegs, ch.total_tiles,
                                 grid_of(d.lim.ew_blocks_per_sm), s, busy);
        case K_SAXPY:
            return launch_saxpy((const SegDesc*)(base + ch.table_off), ch.nsegs, ch.total_tiles,
                                grid_of(d.lim.ew_blocks_per_sm), s, busy);
        case K_BLACKSCHOLES:
            return launch_blackscholes((const SegDesc*)(base + ch.table_off), ch.nsegs, ch.total_tiles,
                                       grid_of(d.lim.bs_blocks_per_sm), s, busy, sched);
        case K_EW_MIX:
            return launch_ew_mix((const SegDesc*)(base + ch.table_off), ch.nsegs, ch.total_tiles,
                                 grid_of(d.lim.mix_blocks_per_sm), s, busy, sched);
        case K_HIST256:
            return launch_hist256((const SegDesc*)(base + ch.table_off), ch.nsegs, ch.total_tiles,
                                  grid_of(d.lim.hist_blocks_per_sm), s, busy, hscr, sched);
        case K_SGEMM:
            if (sgemm_impl == kSgemmPlain)
                return launch_sgemm_plain((const GemmDesc*)(base + ch.table_off), ch.nsegs, ch.total_tiles,
                                          grid_of(d.lim.gemm_plain_blocks_per_sm), s);
            if (sgemm_impl == SVP_SGEMM_TF32BF16) {
                const void* cmaps = ch.cmaps_off >= 0 ? (const void*)(base + ch.cmaps_off) : nullptr;
                cudaError_t e = launch_sgemm_tf32bf16((const GemmDesc*)(base + ch.table_off), ch.nsegs,
                                                      base + ch.maps_off, ch.main_tiles, grid_of(1), ch.wide, s,
                                                      kchunk, cmaps);
                if (e || ch.tail_n == 0) return e;
                // tail split: the last wave's tiles as K-slices, then the ordered reduction
                e = launch_sgemm_tf32bf16((const GemmDesc*)(base + ch.tail_table_off), ch.tail_n,
                                          base + ch.tail_maps_off, (uint32_t)ch.tail_n,
                                          2 * std::min<int>(ch.tail_n, d.lim.num_sms / 2), false, s);
                if (e) return e;
                return launch_sgemm_tail_reduce((const TailRed*)(base + ch.tail_red_off), ch.tail_nred, s);
            }
            if (sgemm_impl == SVP_SGEMM_3XTF32)
                return launch_sgemm_3xtf32((const GemmDesc*)(base + ch.table_off), ch.nsegs, base + ch.maps_off,
                                           ch.total_tiles, grid_of(1), s, kchunk,
                                           ch.cmaps_off >= 0 ? (const void*)(base + ch.cmaps_off) : nullptr);
            return launch_sgemm_ffma((const GemmDesc*)(base + ch.table_off), ch.nsegs, base + ch.maps_off,
                                     ch.total_tiles, grid_of(d.lim.gemm_blocks_per_sm), s);
        case K_DGEMM:
            return launch_dgemm((const DgemmDesc*)(base + ch.table_off), ch.nsegs, ch.total_tiles,
                                grid_of(ch.small_tiles ? d.lim.dgemm_small_blocks_per_sm : d.lim.dgemm_blocks_per_sm),
                                ch.small_tiles, s);
        case K_SGEMM_TF32:
            if (sgemm_impl == kSgemmPlain)
                return launch_sgemm_plain((const GemmDesc*)(base + ch.table_off), ch.nsegs, ch.total_tiles,
                                          grid_of(d.lim.gemm_plain_blocks_per_sm), s);
            return launch_sgemm_tf32((const GemmDesc*)(base + ch.table_off), ch.nsegs, base + ch.maps_off,
                                     ch.total_tiles, grid_of(1), s);
    }
    return cudaErrorInvalidValue;
}

// zero-work hist jobs still must overwrite counts: handled in the kernel launcher by
// zeroing every segment (including n == 0 ones) before accumulating.
static bool chunk_needs_launch(const Flush& f, const Chunk& ch) {
    if (ch.total_tiles) return true;
    for (int32_t ji : ch.jobs) {
        const Job& j = f.jobs[ji];
        if (j.kernel == K_HIST256) return true;
        if (is_gemm(j.kernel) && (int64_t)j.M * j.N > 0) return true;
    }
    return false;
}

bool executor_chunk_launches(const Flush& f, const Chunk& ch) { return chunk_needs_launch(f, ch); }

static svp_status issue_ops(Executor* e, Dev& d, Flush& f, bool prof, bool capturing, const uint8_t* base,
                            cudaStream_t direct, std::vector<int>& used, std::vector<int32_t>& tstart);
static svp_status finish_device(Executor* e, Dev& d, Flush& f, bool prof, bool upload, bool direct,
                                const std::vector<int>& used, const std::vector<int32_t>& tstart,
                                std::chrono::steady_clock::time_point t_issue0, double* issue_ns);

static svp_status run_device(Executor* e, Dev& d, Flush& f, double* issue_ns) {
    Ctx* c = e->c;
    CK(cudaSetDevice(d.ordinal));
    const bool prof = c->cfg.profile_level >= 1;
    bool any = false;
    uint64_t arena_need = 0;
    for (auto& ch : f.chunks)
        if (ch.device == d.idx) {
            any = true;
            arena_need = std::max(arena_need, ch.arena_off + ch.arena_len);
        }
    if (!any) return SVP_OK;
    if (arena_need && !d.arena) {
        cudaError_t ce = cudaMalloc(&d.arena, d.arena_bytes);
        if (ce != cudaSuccess) {
            cudaGetLastError();
            d.err = "cannot allocate the staging arena (" + std::to_string(d.arena_bytes) + " B)";
            d.arena = nullptr;
            return SVP_E_NOMEM;
        }
    }
    // ---- steady-state replay: a reused plan replays its graph if this GPU captured one,
    // else it is captured now (second sighting of the plan)
    const bool graph = c->cfg.graph && f.reused && !c->cfg.sync_each_job;
    Dev::GraphEntry* ge = nullptr;
    if (graph) {
        auto it = d.graphs.find(f.plan_gen);
        if (it != d.graphs.end()) ge = &it->second;
    }
    bool replay = ge && ge->gexec;
    // ---- tables (a replayed graph carries its own; everything else builds them)
    std::vector<uint8_t> tbl;
    if (!replay) {
        svp_status st = build_tables(e, d, f, tbl);
        if (st) return st;
    }
    auto t_issue0 = std::chrono::steady_clock::now();
    // tables changed -> new host copy; the device copy is refreshed only if some launch on
    // this GPU reads the global table (param-mode launches carry theirs by value)
    if (!replay && !tbl.empty() &&
        (tbl.size() != d.tbl_last.size() || memcmp(tbl.data(), d.tbl_last.data(), tbl.size()))) {
        d.tbl_last.swap(tbl);
        d.tbl_dev_valid = false;
    }
    bool need_dev = false;
    for (const auto& ch : f.chunks)
        if (ch.device == d.idx && !ch.param && chunk_needs_launch(f, ch)) need_dev = true;
    const bool capture = graph && !replay;
    // a capture reads its own table copy (below), not the shared buffer
    const bool upload = !replay && !capture && need_dev && !d.tbl_dev_valid && !d.tbl_last.empty();
    // direct issue: when every op of this GPU is on one plan stream and nothing needs the
    // control stream (no upload, no graph), the ops go straight onto the caller's stream --
    // no fork / join events (a launch-bound flush: 7 -> 3 stream calls)
    bool direct = d.ext != nullptr && !graph && !upload;
    {
        int one = -1;
        for (const auto& o : f.ops) {
            if (!direct) break;
            if (o.device != d.idx) continue;
            if (one < 0) one = o.stream;
            else if (o.stream != one) direct = false;
        }
    }
    if (d.ext && !direct) {
        // only the streams this flush uses on this GPU (and stream 0: table upload, capture)
        std::vector<char> touch(d.streams.size(), 0);
        touch[0] = 1;
        for (const auto& o : f.ops)
            if (o.device == d.idx) touch[o.stream + 1] = 1;
        CK(cudaEventRecord(d.ext_ev, d.ext));
        for (size_t s = 0; s < d.streams.size(); ++s)
            if (touch[s]) CK(cudaStreamWaitEvent(d.streams[s], d.ext_ev, 0));
    }
    if (upload) {
        const size_t bytes = d.tbl_last.size();
        if (bytes > d.tbl_cap) {
            if (svp_status q = quiesce(d)) return q;
            if (d.tbl_upload_inflight) CK(cudaEventSynchronize(d.tbl_ev));
            if (d.tbl_dev) CK(cudaFree(d.tbl_dev));
            if (d.tbl_host) CK(cudaFreeHost(d.tbl_host));
            d.tbl_dev = nullptr;
            d.tbl_host = nullptr;
            size_t cap = align_up(bytes * 2, 1 << 16);
            CK(cudaMalloc(&d.tbl_dev, cap));
            CK(cudaHostAlloc(&d.tbl_host, cap, cudaHostAllocDefault));
            d.tbl_cap = cap;
        }
        if (d.tbl_upload_inflight) CK(cudaEventSynchronize(d.tbl_ev));  // (async flushes)
        memcpy(d.tbl_host, d.tbl_last.data(), bytes);
        CK(cudaMemcpyAsync(d.tbl_dev, d.tbl_host, bytes, cudaMemcpyHostToDevice, d.streams[0]));
        CK(cudaEventRecord(d.tbl_ev, d.streams[0]));
        d.tbl_upload_inflight = true;
        for (size_t s = 1; s < d.streams.size(); ++s) CK(cudaStreamWaitEvent(d.streams[s], d.tbl_ev, 0));
        d.tbl_dev_valid = true;
        ++d.table_uploads;
        {
            std::lock_guard<std::mutex> lk(c->pmu);  // one worker thread per GPU updates the stats
            f.stats.table_uploads += 1;
            f.stats.table_bytes += bytes;
        }
    }
    // ---- profile_level 2: busy-cycle counters for every segment launch on this GPU
    {
        size_t nbusy = 0;
        for (auto& ch : f.chunks) {
            if (ch.device != d.idx) continue;
            ch.busy_off = -1;
            ch.busy.clear();
            if (c->cfg.profile_level >= 2 && is_seg_kernel(ch.kernel) && ch.nsegs > 0 && chunk_needs_launch(f, ch)) {
                ch.busy_off = (int64_t)nbusy;
                nbusy += (size_t)ch.nsegs;
            }
        }
        if (nbusy > d.busy_cap) {
            {
                svp_status gs = drop_graphs(d);  // captured graphs hold the old counter addresses
                if (gs) return gs;
            }
            if (d.busy_dev) CK(cudaFree(d.busy_dev));
            d.busy_dev = nullptr;
            d.busy_cap = 0;
            CK(cudaMalloc(&d.busy_dev, std::max<size_t>(nbusy, 256) * sizeof(uint64_t)));
            d.busy_cap = std::max<size_t>(nbusy, 256);
        }
    }
    // ---- dynamic tile order (Black-Scholes / mixed launches): one counter slot per launch.
    // Only for a launch that has the GPU to itself: alone it balances the SMs (cfg5's BS
    // launch 0.753 -> 0.668 ms, one-stream step +2 %), but co-running with the other
    // kernels of an interleaved level it cost 0.7 % of the step (profiles/r01/ew_dyn/).
    {
        std::map<int32_t, int> kernels_in_level;
        for (const auto& ch : f.chunks)
            if (ch.device == d.idx && ch.total_tiles > 0) kernels_in_level[ch.level] += 1;
        size_t nslot = 0;
        for (auto& ch : f.chunks) {
            if (ch.device != d.idx) continue;
            ch.sched_slot = -1;
            const bool alone = !c->cfg.interleave || kernels_in_level[ch.level] == 1;
            if (ew_dynamic_order() && alone && (ch.kernel == K_BLACKSCHOLES || ch.kernel == K_EW_MIX) &&
                ch.total_tiles > 0)
                ch.sched_slot = (int32_t)nslot++;
            // hist256: dynamic chunk order whenever it is not the single-launch form (its CTAs
            // run at data-dependent speeds: replicated vs shared-table counting)
            if (hist_dynamic_order() && ch.kernel == K_HIST256 && !hist_single_launch() && ch.total_tiles > 0)
                ch.sched_slot = (int32_t)nslot++;
        }
        // single-launch hist256 scratch (SVP_HIST_FUSED=0: zeroing kernel + launch)
        size_t nh = 0;
        for (auto& ch : f.chunks) {
            if (ch.device != d.idx) continue;
            ch.hscr_off = -1;
            if (hist_single_launch() && ch.kernel == K_HIST256 && ch.nsegs > 0) {
                ch.hscr_off = (int64_t)nh;
                nh += (size_t)ch.nsegs * 257;
            }
        }
        if (nh > d.hscr_cap) {
            {
                svp_status gs = drop_graphs(d);
                if (gs) return gs;
            }
            if (d.hscr_dev) CK(cudaFree(d.hscr_dev));
            d.hscr_dev = nullptr;
            d.hscr_cap = 0;
            const size_t cap = std::max<size_t>(nh, 64 * 257);
            CK(cudaMalloc(&d.hscr_dev, cap * sizeof(uint32_t)));
            CK(cudaMemset(d.hscr_dev, 0, cap * sizeof(uint32_t)));
            d.hscr_cap = cap;
        }
        if (nslot > d.sched_cap) {
            {
                svp_status gs = drop_graphs(d);  // captured graphs hold the old counter addresses
                if (gs) return gs;
            }
            // the previous flush's launches have finished (svp_flush is synchronous)
            if (d.sched_dev) CK(cudaFree(d.sched_dev));
            d.sched_dev = nullptr;
            d.sched_cap = 0;
            const size_t cap = std::max<size_t>(nslot, 64);
            CK(cudaMalloc(&d.sched_dev, cap * 2 * sizeof(uint32_t)));
            CK(cudaMemset(d.sched_dev, 0, cap * 2 * sizeof(uint32_t)));
            d.sched_cap = cap;
        }
    }
    if (replay && d.graphs.find(f.plan_gen) == d.graphs.end()) {
        // cannot happen: a replayed plan needs no more scratch than when it was captured,
        // and any growth since then dropped its graph before this flush
        d.err = "internal: the graph of a replayed plan was dropped during its flush";
        return SVP_E_STATE;
    }
    // ---- steady-state replay: second sighting of a plan -> capture, later -> replay
    std::vector<int> used(d.streams.size(), 0);
    std::vector<int32_t> tstart(f.ops.size(), -1);
    const uint8_t* base = d.tbl_dev;
    bool capturing = false;
    if (capture) {
        // the entry for this plan (evicting the least recently used one past the cap); its
        // device tables are a private copy, uploaded before the capture begins
        if (d.graphs.size() >= kGraphsPerDevice) {
            if (svp_status q = quiesce(d)) return q;
            auto lru = d.graphs.begin();
            for (auto it = d.graphs.begin(); it != d.graphs.end(); ++it)
                if (it->second.last_use < lru->second.last_use) lru = it;
            if (lru->second.gexec) CK(cudaGraphExecDestroy(lru->second.gexec));
            if (lru->second.tbl) CK(cudaFree(lru->second.tbl));
            d.graphs.erase(lru);
        }
        ge = &d.graphs[f.plan_gen];
        if (need_dev && !d.tbl_last.empty()) {
            const size_t bytes = d.tbl_last.size();
            if (bytes > ge->tbl_cap) {
                if (ge->tbl) CK(cudaFree(ge->tbl));
                ge->tbl = nullptr;
                CK(cudaMalloc(&ge->tbl, bytes));
                ge->tbl_cap = bytes;
            }
            CK(cudaMemcpy(ge->tbl, d.tbl_last.data(), bytes, cudaMemcpyHostToDevice));
            base = ge->tbl;
        }
        CK(cudaStreamBeginCapture(d.streams[0], cudaStreamCaptureModeThreadLocal));
        capturing = true;
        svp_status cs = [&]() -> svp_status {
            CK(cudaEventRecord(d.fork_ev, d.streams[0]));
            for (size_t s = 1; s < d.streams.size(); ++s) CK(cudaStreamWaitEvent(d.streams[s], d.fork_ev, 0));
            return SVP_OK;
        }();
        if (cs) {
            cudaGraph_t g = nullptr;
            cudaStreamEndCapture(d.streams[0], &g);
            if (g) cudaGraphDestroy(g);
            return cs;
        }
    }
    svp_status ist = replay ? SVP_OK : issue_ops(e, d, f, prof, capturing, base, direct ? d.ext : nullptr, used, tstart);
    if (capturing) {
        // join every stream back into stream 0, close the capture, instantiate
        svp_status js = ist;
        for (size_t s = 1; s < d.streams.size() && js == SVP_OK; ++s) {
            cudaError_t ce = cudaEventRecord(d.join_ev[s], d.streams[s]);
            if (ce == cudaSuccess) ce = cudaStreamWaitEvent(d.streams[0], d.join_ev[s], 0);
            if (ce != cudaSuccess) {
                d.err = std::string("graph join: ") + cudaGetErrorString(ce);
                js = SVP_E_CUDA;
            }
        }
        cudaGraph_t g = nullptr;
        cudaError_t ce = cudaStreamEndCapture(d.streams[0], &g);
        if (js) {
            if (g) cudaGraphDestroy(g);
            return js;
        }
        if (ce != cudaSuccess) {
            d.err = std::string("cudaStreamEndCapture: ") + cudaGetErrorString(ce);
            return SVP_E_CUDA;
        }
        ce = cudaGraphInstantiate(&ge->gexec, g, 0);
        cudaGraphDestroy(g);
        if (ce != cudaSuccess) {
            ge->gexec = nullptr;
            d.err = std::string("cudaGraphInstantiate: ") + cudaGetErrorString(ce);
            return SVP_E_CUDA;
        }
        ge->tstart = tstart;
        replay = true;
    } else if (ist) {
        return ist;
    }
    if (replay) {
        ge->last_use = ++d.graph_clock;
        CK(cudaGraphLaunch(ge->gexec, d.streams[0]));
        tstart = ge->tstart;
        std::fill(used.begin(), used.end(), 0);
        used[0] = 1;
        std::lock_guard<std::mutex> lk(c->pmu);
        f.stats.graph_replays += 1;
    }
    return finish_device(e, d, f, prof, upload, direct, used, tstart, t_issue0, issue_ns);
}

// Enqueue the device's ops in plan order (directly, or into an open stream capture).
static svp_status issue_ops(Executor* e, Dev& d, Flush& f, bool prof, bool capturing, const uint8_t* base,
                            cudaStream_t direct, std::vector<int>& used, std::vector<int32_t>& tstart) {
    Ctx* c = e->c;
    size_t nt = 0;
    // inside a capture, timing events become event-record nodes of the graph
    auto rec = [&](cudaEvent_t ev, cudaStream_t s) {
        return capturing ? cudaEventRecordWithFlags(ev, s, cudaEventRecordExternal) : cudaEventRecord(ev, s);
    };
    for (size_t i = 0; i < f.ops.size(); ++i) {
        Op& o = f.ops[i];
        if (o.device != d.idx) continue;
        cudaStream_t s = direct ? direct : d.streams[o.stream + 1];
        if (!direct) used[o.stream + 1] = 1;
        for (int32_t p : o.wait_ops) {  // (direct: one stream, already in order)
            const Op& q = f.ops[p];
            if (q.device != d.idx || direct) continue;
            CK(cudaStreamWaitEvent(s, d.dep_ev[p], 0));
        }
        if (prof) {
            cudaEvent_t ev0 = pool_get(d, d.t_ev, 2 * nt, true), ev1 = pool_get(d, d.t_ev, 2 * nt + 1, true);
            if (!ev0 || !ev1) {
                d.err = "event allocation failed";
                return SVP_E_CUDA;
            }
            CK(rec(ev0, s));
            tstart[i] = (int32_t)nt;
        }
        Chunk& ch = f.chunks[o.chunk];
        if (o.kind == SVP_OP_H2D || o.kind == SVP_OP_D2H) {
            for (size_t k = 0; k < ch.jobs.size(); ++k) {
                const Job& j = f.jobs[ch.jobs[k]];
                for (int b = 0; b < j.nbufs; ++b) {
                    if (j.bufs[b].mem != SVP_MEM_HOST_PINNED) continue;
                    uint64_t bytes = touched_bytes(j, b);
                    if (!bytes) continue;
                    void* dev = (void*)ch.staged[k * SVP_MAX_BUFS + b];
                    if (o.kind == SVP_OP_H2D && (j.bufs[b].dir & SVP_DIR_IN)) {
                        // sgemm C with beta == 0 is OUT-only and not staged in
                        CK(cudaMemcpyAsync(dev, j.bufs[b].ptr, bytes, cudaMemcpyHostToDevice, s));
                    } else if (o.kind == SVP_OP_D2H && (j.bufs[b].dir & SVP_DIR_OUT)) {
                        CK(cudaMemcpyAsync(j.bufs[b].ptr, dev, bytes, cudaMemcpyDeviceToHost, s));
                    }
                }
            }
        } else if (chunk_needs_launch(f, ch)) {
            CK(launch_chunk(d, ch, c->cfg.sgemm_kchunk, s, base));
        }
        if (prof) {
            CK(rec(d.t_ev[2 * nt + 1], s));
            ++nt;
        }
        if (o.needs_event && !direct) {
            cudaEvent_t ev = pool_get(d, d.dep_ev, i, false);
            if (!ev) {
                d.err = "event allocation failed";
                return SVP_E_CUDA;
            }
            CK(cudaEventRecord(ev, s));
        }
        if (c->cfg.sync_each_job && o.last_of_job) CK(cudaStreamSynchronize(s));
    }
    return SVP_OK;
}

static svp_status finish_device(Executor* e, Dev& d, Flush& f, bool prof, bool upload, bool direct,
                                const std::vector<int>& used, const std::vector<int32_t>& tstart,
                                std::chrono::steady_clock::time_point t_issue0, double* issue_ns) {
    // ---- join into the external stream (the wait is complete_device, possibly later)
    auto& ev = d.end_ev[f.seq & 1];
    Dev::Pending& pd = d.pend[f.seq & 1];
    pd.finals.clear();
    if (direct) {  // the ops ran on the external stream itself
        CK(cudaEventRecord(ev[0], d.ext));
        pd.finals.push_back(ev[0]);
    }
    for (size_t s = 0; s < d.streams.size() && !direct; ++s) {
        if (!used[s] && !(upload && s == 0)) continue;
        CK(cudaEventRecord(ev[s], d.streams[s]));
        pd.finals.push_back(ev[s]);
        if (d.ext) CK(cudaStreamWaitEvent(d.ext, ev[s], 0));
    }
    *issue_ns = std::chrono::duration<double, std::nano>(std::chrono::steady_clock::now() - t_issue0).count();
    pd.prof = prof;
    pd.tstart = tstart;
    pd.active = true;
    return SVP_OK;
}

// The wait half of a flush on one GPU: its join events (watchdog), then the measured op
// durations and busy counters.
static svp_status complete_device(Executor* e, Dev& d, Flush& f) {
    Ctx* c = e->c;
    Dev::Pending& pd = d.pend[f.seq & 1];
    if (!pd.active) return SVP_OK;
    pd.active = false;
    CK(cudaSetDevice(d.ordinal));
    const bool prof = pd.prof;
    const std::vector<int32_t>& tstart = pd.tstart;
    const std::vector<cudaEvent_t>& finals = pd.finals;
    if (c->cfg.flush_timeout_ms > 0) {
        auto deadline = std::chrono::steady_clock::now() + std::chrono::milliseconds(c->cfg.flush_timeout_ms);
        for (auto ev : finals) {
            for (;;) {
                cudaError_t q = cudaEventQuery(ev);
                if (q == cudaSuccess) break;
                if (q != cudaErrorNotReady) CK(q);
                if (std::chrono::steady_clock::now() > deadline) {
                    d.err = "svp_flush: watchdog expired after " + std::to_string(c->cfg.flush_timeout_ms) + " ms";
                    return SVP_E_TIMEOUT;
                }
                std::this_thread::sleep_for(std::chrono::microseconds(50));
            }
        }
    } else {
        for (auto ev : finals) CK(cudaEventSynchronize(ev));
    }
    CK(cudaGetLastError());
    // ---- measured op durations
    if (prof) {
        for (size_t i = 0; i < f.ops.size(); ++i) {
            if (tstart[i] < 0) continue;
            float ms = 0;
            CK(cudaEventElapsedTime(&ms, d.t_ev[2 * tstart[i]], d.t_ev[2 * tstart[i] + 1]));
            f.ops[i].measured_ns = ms * 1e6;
        }
        // device span: earliest start to latest end
        float span = 0;
        int32_t first = -1, lastop = -1;
        for (size_t i = 0; i < f.ops.size(); ++i)
            if (tstart[i] >= 0) {
                if (first < 0) first = (int32_t)i;
                lastop = (int32_t)i;
            }
        if (first >= 0) {
            float mx = 0;
            for (size_t i = 0; i < f.ops.size(); ++i) {
                if (tstart[i] < 0) continue;
                // one query per op: its start offset; its end = start + the duration above
                float ms0 = 0;
                if (i != (size_t)first) CK(cudaEventElapsedTime(&ms0, d.t_ev[2 * tstart[first]], d.t_ev[2 * tstart[i]]));
                f.ops[i].measured_start_ns = (double)ms0 * 1e6;
                mx = std::max(mx, ms0 + (float)(f.ops[i].measured_ns * 1e-6));
            }
            span = mx;
        }
        (void)lastop;
        std::lock_guard<std::mutex> lk(c->pmu);
        f.stats.device_ns = std::max(f.stats.device_ns, (double)span * 1e6);
        DevStats& ds = c->dstats[d.idx];
        ds.last_device_ns = (double)span * 1e6;
        ds.device_ns += (double)span * 1e6;
    }
    // ---- profile_level 2: measured busy cycles per segment (the kernels are done)
    size_t nbusy = 0;
    for (const auto& ch : f.chunks)
        if (ch.device == d.idx && ch.busy_off >= 0) nbusy = std::max(nbusy, (size_t)ch.busy_off + ch.nsegs);
    if (nbusy) {
        std::vector<uint64_t> hb(nbusy);
        CK(cudaMemcpy(hb.data(), d.busy_dev, nbusy * sizeof(uint64_t), cudaMemcpyDeviceToHost));
        for (auto& ch : f.chunks)
            if (ch.device == d.idx && ch.busy_off >= 0)
                ch.busy.assign(hb.begin() + ch.busy_off, hb.begin() + ch.busy_off + ch.nsegs);
    }
    return SVP_OK;
}

// Profiler attribution (a10): w_v = algorithmic bytes (FLOPs for SGEMM) of the VP's job
// in the op -- or, with profile_level 2, the SM cycles measured on the VP's tiles of a
// segment launch; T_v = T_op * w_v / sum w.  Conservation (sum_v T_v = T_op) holds exactly up
// to fp64 rounding.
static void count_device_work(Ctx* c, const Flush& f) {  // under pmu
    std::vector<char> used(c->dstats.size(), 0);
    for (const auto& j : f.jobs) {
        if (j.device < 0 || j.device >= (int32_t)c->dstats.size()) continue;
        c->dstats[j.device].jobs += 1;
        used[j.device] = 1;
    }
    for (size_t g = 0; g < used.size(); ++g) c->dstats[g].flushes += used[g];
}

static void attribute(Ctx* c, const Flush& f) {
    std::lock_guard<std::mutex> lk(c->pmu);
    count_device_work(c, f);
    for (const auto& j : f.jobs) {
        c->prof[j.vp].jobs += 1;
        c->prof_total.jobs += 1;
    }
    for (const auto& o : f.ops)
        if (o.kind == SVP_OP_KERNEL && o.measured_ns >= 0 && o.device < (int32_t)c->dstats.size())
            c->dstats[o.device].kernel_ns += o.measured_ns;
    for (const auto& o : f.ops) {
        const Chunk& ch = f.chunks[o.chunk];
        if (o.kind == SVP_OP_KERNEL && o.measured_ns >= 0) {
            c->prof_launches += chunk_needs_launch(f, ch) ? 1 : 0;
            KStats& ks = c->kstats[ch.kernel];
            ks.launches += 1;
            ks.total_ns += o.measured_ns;
            ks.max_ns = std::max(ks.max_ns, o.measured_ns);
            ks.bytes += ch.alg_bytes;
            ks.flops += ch.flops;
        }
        if (o.measured_ns < 0) continue;
        double wsum = 0;
        std::vector<double> w(ch.jobs.size());
        // profile_level 2: a segment launch is split by the measured SM cycles of each VP's
        // tiles (when any were recorded), every other op by algorithmic work
        double bsum = 0;
        const bool measured = o.kind == SVP_OP_KERNEL && ch.busy.size() == ch.jobs.size();
        if (measured)
            for (uint64_t b : ch.busy) bsum += (double)b;
        for (size_t k = 0; k < ch.jobs.size(); ++k) {
            const Job& j = f.jobs[ch.jobs[k]];
            if (o.kind == SVP_OP_H2D) w[k] = (double)j.host_in_bytes;
            else if (o.kind == SVP_OP_D2H) w[k] = (double)j.host_out_bytes;
            else if (measured && bsum > 0) w[k] = (double)ch.busy[k];
            else w[k] = j.flops > 0 ? j.flops : j.alg_bytes;
            wsum += w[k];
        }
        for (size_t k = 0; k < ch.jobs.size(); ++k) {
            const Job& j = f.jobs[ch.jobs[k]];
            double share = wsum > 0 ? o.measured_ns * w[k] / wsum : o.measured_ns / ch.jobs.size();
            VpProfile& p = c->prof[j.vp];
            if (o.kind == SVP_OP_H2D) {
                p.h2d_ns += share;
                p.bytes_h2d += j.host_in_bytes;
                c->prof_total.h2d_ns += share;
                c->prof_total.bytes_h2d += j.host_in_bytes;
            } else if (o.kind == SVP_OP_D2H) {
                p.d2h_ns += share;
                p.bytes_d2h += j.host_out_bytes;
                c->prof_total.d2h_ns += share;
                c->prof_total.bytes_d2h += j.host_out_bytes;
            } else {
                p.kernel_ns += share;
                p.bytes_kernel += (uint64_t)j.alg_bytes;
                p.flops += j.flops;
                c->prof_total.kernel_ns += share;
                c->prof_total.bytes_kernel += (uint64_t)j.alg_bytes;
                c->prof_total.flops += j.flops;
            }
        }
    }
    // cost-model feedback (EMA of measured / predicted kernel time per kernel)
    for (const auto& o : f.ops) {
        if (o.kind != SVP_OP_KERNEL || o.measured_ns <= 0 || o.est_ns <= c->cost.launch_ns * 2) continue;
        const Chunk& ch = f.chunks[o.chunk];
        double pred = o.est_ns - c->cost.launch_ns;
        double meas = std::max(1.0, o.measured_ns - c->cost.launch_ns);
        double& ks = c->cost.kscale[ch.kernel][CostModel::bucket(ch.alg_bytes, ch.flops)];
        const double ratio = ks * meas / pred;
        ks = 0.8 * ks + 0.2 * std::min(8.0, std::max(0.125, ratio));
    }
}

// One half of a flush on every GPU: GPU 0 on the calling thread, GPUs 1.. on their
// workers.  Returns the first GPU's error.
static svp_status run_half(Executor* e, Flush* f, bool complete) {
    const int G = (int)e->devs.size();
    std::vector<svp_status> st(G, SVP_OK);
    std::vector<double> issue(G, 0.0);
    // the flushing thread drives GPU 0 and gets its current device back afterwards
    int caller_dev = -1;
    if (cudaGetDevice(&caller_dev) != cudaSuccess) {
        cudaGetLastError();
        caller_dev = -1;
    }
    if (G > 1) {
        {
            std::lock_guard<std::mutex> lk(e->w.mu);
            e->w.f = f;
            e->w.complete = complete;
            e->w.pending = G - 1;
            e->w.gen += 1;
        }
        e->w.go.notify_all();
    }
    st[0] = complete ? complete_device(e, e->devs[0], *f) : run_device(e, e->devs[0], *f, &issue[0]);
    if (G > 1) {
        std::unique_lock<std::mutex> lk(e->w.mu);
        e->w.done.wait(lk, [&] { return e->w.pending == 0; });
        for (int g = 1; g < G; ++g) {
            st[g] = e->w.st[g];
            if (!complete) issue[g] = e->w.issue[g];
        }
    }
    if (caller_dev >= 0) cudaSetDevice(caller_dev);
    if (!complete) f->stats.host_issue_ns = *std::max_element(issue.begin(), issue.end());
    for (int g = 0; g < G; ++g) {
        if (st[g] != SVP_OK) {
            e->err = "GPU " + std::to_string(g) + ": " + e->devs[g].err;
            return st[g];
        }
    }
    return SVP_OK;
}

// Issue half: every GPU's ops enqueued and joined into its external stream (no waiting).
svp_status executor_issue(Executor* e, Flush* f) { return run_half(e, f, false); }

// Wait half: every GPU's join events, measured durations, then the Profiler.
svp_status executor_complete(Executor* e, Flush* f) {
    Ctx* c = e->c;
    svp_status st = run_half(e, f, true);
    if (st) return st;
    if (c->cfg.profile_level >= 1) attribute(c, *f);
    else {
        std::lock_guard<std::mutex> lk(c->pmu);
        count_device_work(c, *f);
        for (const auto& j : f->jobs) {
            c->prof[j.vp].jobs += 1;
            c->prof_total.jobs += 1;
        }
        for (const auto& o : f->ops)
            if (o.kind == SVP_OP_KERNEL && chunk_needs_launch(*f, f->chunks[o.chunk])) c->prof_launches += 1;
    }
    return SVP_OK;
}

// After a failed issue half: wait for whatever the GPUs that did issue enqueued (no
// profiling), so nothing of this flush is left running when the error is returned.
void executor_abandon(Executor* e, Flush* f) {
    for (auto& d : e->devs) {
        Dev::Pending& pd = d.pend[f->seq & 1];
        if (!pd.active) continue;
        pd.active = false;
        cudaSetDevice(d.ordinal);
        for (auto ev : pd.finals) cudaEventSynchronize(ev);
        cudaGetLastError();
    }
}

}  // namespace svp

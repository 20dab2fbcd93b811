// capi.cpp -- the C-ABI entry points of libsvp (include/svp.h).
//
// This file is the boundary: argument checking, error codes, the thread-local error
// message, context lifetime, and the Job Queue front end (svp_submit stands in for the
// paper's VP -> IPC Manager -> Job Queue path, Fig 2).  The heavy
// lifting is in scheduler.cpp (Kernel Match, Dispatcher, Re-scheduler) and
// executor.cpp (per-GPU execution and the Profiler).
#include <stdio.h>
#include <stdlib.h>
#include <string.h>
#include <unistd.h>

#include <algorithm>
#include <chrono>
#include <new>

#include "internal.h"

namespace svp {

static const bool kTf32Available = true;
static thread_local std::string g_last_error;
void set_error(const std::string& msg) { g_last_error = msg; }

static const KernelDesc kKernels[] = {
    {"", 0, 0, {0, 0, 0, 0, 0}, 0},
    {"vecadd", K_VECADD, 3, {SVP_DIR_IN, SVP_DIR_IN, SVP_DIR_OUT, 0, 0}, sizeof(svp_args_vecadd)},
    {"saxpy", K_SAXPY, 2, {SVP_DIR_IN, SVP_DIR_INOUT, 0, 0, 0}, sizeof(svp_args_saxpy) - 4},
    {"hist256", K_HIST256, 2, {SVP_DIR_IN, SVP_DIR_OUT, 0, 0, 0}, sizeof(svp_args_hist256)},
    {"blackscholes", K_BLACKSCHOLES, 5, {SVP_DIR_IN, SVP_DIR_IN, SVP_DIR_IN, SVP_DIR_OUT, SVP_DIR_OUT},
     sizeof(svp_args_bs)},
    {"sgemm", K_SGEMM, 3, {SVP_DIR_IN, SVP_DIR_IN, SVP_DIR_OUT, 0, 0}, sizeof(svp_args_sgemm)},
    {"sgemm_tf32", K_SGEMM_TF32, 3, {SVP_DIR_IN, SVP_DIR_IN, SVP_DIR_OUT, 0, 0}, sizeof(svp_args_sgemm)},
    {"dgemm", K_DGEMM, 3, {SVP_DIR_IN, SVP_DIR_IN, SVP_DIR_OUT, 0, 0}, sizeof(svp_args_dgemm)},
};

const KernelDesc* kernel_desc(int32_t id) {
    if (id <= 0 || id >= K_EW_MIX) return nullptr;
    return &kKernels[id];
}
const KernelDesc* kernel_by_name(const char* name) {
    if (!name) return nullptr;
    for (int i = 1; i < K_EW_MIX; ++i)
        if (strcmp(kKernels[i].name, name) == 0) return &kKernels[i];
    return nullptr;
}

}  // namespace svp

using namespace svp;

#define SVP_TRY_BEGIN try {
#define SVP_TRY_END                                  \
    }                                                \
    catch (const std::bad_alloc&) {                  \
        set_error("out of host memory");             \
        return SVP_E_NOMEM;                          \
    }                                                \
    catch (const std::exception& e) {                \
        set_error(std::string("internal: ") + e.what()); \
        return SVP_E_STATE;                          \
    }                                                \
    catch (...) {                                    \
        set_error("internal: unknown exception");    \
        return SVP_E_STATE;                          \
    }

static svp_status check_ctx(svp_ctx* h) {
    if (!h) {
        set_error("null context");
        return SVP_E_INVAL;
    }
    Ctx* c = reinterpret_cast<Ctx*>(h);
    if (c->sticky.load() != SVP_OK) {
        set_error("context is sticky-errored: " + c->sticky_message());
        return SVP_E_STATE;
    }
    return SVP_OK;
}

extern "C" {

static void stop_dispatcher(Ctx* c);

const char* svp_last_error(void) { return g_last_error.c_str(); }
int32_t svp_abi_version(void) { return SVP_ABI_VERSION; }

void svp_config_default(svp_config* cfg) {
    if (!cfg) return;
    memset(cfg, 0, sizeof(*cfg));
    cfg->num_gpus = 0;
    cfg->streams_per_gpu = 4;
    cfg->coalesce = 1;
    cfg->interleave = 1;
    cfg->max_chunks = 8;
    cfg->profile_level = 0;
    cfg->validate_ptrs = 1;
    cfg->sgemm_impl = SVP_SGEMM_TF32BF16;
    cfg->table_mode = SVP_TABLE_PARAM;
    cfg->graph = 1;           // plan cache + graph replay (every BASELINE config gains, profiles/r02/graph/)
    cfg->sgemm_kchunk = 768;  // R23: the tensor-core splits' fp32 contract for any K and operand signs
}

svp_status svp_init(const svp_config* cfg, svp_ctx** out) {
    SVP_TRY_BEGIN
    if (!cfg || !out) {
        set_error("svp_init: null cfg/out");
        return SVP_E_INVAL;
    }
    *out = nullptr;
    if (cfg->num_gpus < 0 || cfg->num_gpus > 64 || cfg->streams_per_gpu < 1 || cfg->streams_per_gpu > 32 ||
        cfg->max_chunks < 1 || cfg->max_chunks > 64 || cfg->profile_level < 0 || cfg->profile_level > 2 ||
        cfg->flush_timeout_ms < 0 || cfg->sgemm_impl < 0 || cfg->sgemm_impl > 2 || cfg->table_mode < 0 ||
        cfg->table_mode > 1 || cfg->validate_ptrs < 0 || cfg->validate_ptrs > 2 || cfg->sgemm_kchunk < 0 ||
        cfg->sgemm_kchunk % 16 != 0 || cfg->sgemm_kchunk > (1 << 20)) {
        set_error("svp_init: config value out of range");
        return SVP_E_INVAL;
    }
    Ctx* c = new Ctx();
    c->cfg = *cfg;
    c->cfg.device_ids = nullptr;
    c->cfg.external_streams = nullptr;
    if (cfg->hbm_gbps > 0) c->cost.hbm_Bps = cfg->hbm_gbps * 1e9;
    if (cfg->pcie_gbps > 0) c->cost.pcie_Bps = cfg->pcie_gbps * 1e9;
    if (cfg->ffma_tflops > 0) c->cost.ffma_flops = cfg->ffma_tflops * 1e12;
    if (cfg->launch_us > 0) c->cost.launch_ns = cfg->launch_us * 1e3;
    if (cfg->arena_bytes == 0) c->cfg.arena_bytes = 2ull << 30;
    c->cost.sgemm_tc_units = cfg->sgemm_impl == SVP_SGEMM_3XTF32 ? 3 : cfg->sgemm_impl == SVP_SGEMM_TF32BF16 ? 2 : 0;
    if (const char* e = getenv("SVP_COSCHEDULE")) c->coschedule = atoi(e) != 0;

    if (cfg->dry_run) {
        c->ngpu = cfg->num_gpus > 0 ? cfg->num_gpus : 1;
        for (int i = 0; i < c->ngpu; ++i) c->device_ids.push_back(cfg->device_ids ? cfg->device_ids[i] : i);
    } else {
        c->ngpu = cfg->num_gpus;  // 0 -> executor fills from cudaGetDeviceCount
        if (cfg->device_ids)
            for (int i = 0; i < cfg->num_gpus; ++i) c->device_ids.push_back(cfg->device_ids[i]);
        // external streams are read by the executor at creation time
        c->cfg.external_streams = cfg->external_streams;
        svp_status st = SVP_OK;
        c->exec = executor_create(c, &st);
        c->cfg.external_streams = nullptr;
        if (!c->exec) {
            delete c;
            return st == SVP_OK ? SVP_E_CUDA : st;
        }
    }
    c->dev_load.assign(c->ngpu, 0.0);
    c->dstats.assign(c->ngpu, DevStats{});
    *out = reinterpret_cast<svp_ctx*>(c);
    return SVP_OK;
    SVP_TRY_END
}

static svp_status complete_pending(Ctx* c);

svp_status svp_finalize(svp_ctx* h) {
    SVP_TRY_BEGIN
    if (!h) {
        set_error("null context");
        return SVP_E_INVAL;
    }
    Ctx* c = reinterpret_cast<Ctx*>(h);
    stop_dispatcher(c);
    {
        std::lock_guard<std::mutex> flk(c->flush_mu);
        complete_pending(c);
    }
    if (c->exec) executor_destroy(c->exec);  // synchronizes every stream first
    for (auto& kv : c->host_blocks) host_free_near(kv.first, kv.second);
    c->host_blocks.clear();
    delete c;
    return SVP_OK;
    SVP_TRY_END
}

svp_status svp_register_kernel(svp_ctx* h, const char* name, int32_t* id_out) {
    SVP_TRY_BEGIN
    svp_status st = check_ctx(h);
    if (st) return st;
    const KernelDesc* d = kernel_by_name(name);
    if (!d) {
        set_error(std::string("unknown kernel '") + (name ? name : "(null)") + "'");
        return SVP_E_NOKERNEL;
    }
    if (d->id == K_SGEMM_TF32 && !kTf32Available) {
        set_error("sgemm_tf32: the tcgen05 TF32 kernel is not available in this build");
        return SVP_E_UNSUPPORTED;
    }
    Ctx* c = reinterpret_cast<Ctx*>(h);
    c->registered[d->id] = true;
    if (id_out) *id_out = d->id;
    return SVP_OK;
    SVP_TRY_END
}

}  // extern "C"

// Status of a completed job: the failed flush whose id range covers it, else OK.
svp_status svp::ctx_job_status(Ctx* c, uint64_t job) {
    std::lock_guard<std::mutex> lk(c->done_mu);
    uint64_t lo = 0;
    for (const auto& fr : c->failed) {
        if (job > lo && job <= fr.first) return fr.second;
        lo = fr.first;
    }
    return SVP_OK;
}

uint64_t svp::ctx_completed_upto(Ctx* c, int32_t) {
    std::lock_guard<std::mutex> lk(c->done_mu);
    return c->completed_upto;
}

extern "C" {

static svp_status submit_many(Ctx* c, int32_t n, const svp_job_desc* jd, const svp_job_desc* single_args_src,
                              uint64_t* ids) {
    (void)single_args_src;
    std::vector<Job> jobs(n);
    RangeBatchLock batch(c->exec);  // one lock of the validation cache for the whole batch
    for (int i = 0; i < n; ++i) {
        Job& j = jobs[i];
        j.vp = jd[i].vp;
        j.kernel = jd[i].kernel;
        j.nbufs = jd[i].nbufs;
        if (jd[i].args_bytes > SVP_MAX_ARGS || jd[i].nbufs < 0 || jd[i].nbufs > SVP_MAX_BUFS) {
            set_error("svp_submit: args_bytes > 64 or nbufs out of range");
            return SVP_E_INVAL;
        }
        memcpy(j.args, jd[i].args, jd[i].args_bytes);
        const KernelDesc* d = kernel_desc(j.kernel);
        if (d && jd[i].args_bytes < d->args_bytes) {
            set_error(std::string("svp_submit: args too small for ") + d->name);
            return SVP_E_INVAL;
        }
        for (int b = 0; b < j.nbufs; ++b) j.bufs[b] = jd[i].bufs[b];
        svp_status st = validate_and_fill(c, &j);
        if (st) return st;
    }
    {
        std::lock_guard<std::mutex> lk(c->qmu);
        for (int i = 0; i < n; ++i) {
            jobs[i].id = c->next_job_id++;
            if (ids) ids[i] = jobs[i].id;
        }
        if (c->queue.empty()) {
            c->queue.swap(jobs);
        } else {
            c->queue.reserve(c->queue.size() + n);
            c->queue.insert(c->queue.end(), jobs.begin(), jobs.end());
        }
    }
    c->q_cv.notify_one();
    return SVP_OK;
}

svp_status svp_submit(svp_ctx* h, int32_t vp, int32_t kernel, const void* args, size_t args_bytes,
                      const svp_buf* bufs, int32_t nbufs, uint64_t* job_out) {
    SVP_TRY_BEGIN
    svp_status st = check_ctx(h);
    if (st) return st;
    if ((!args && args_bytes) || args_bytes > SVP_MAX_ARGS || (!bufs && nbufs) || nbufs < 0 ||
        nbufs > SVP_MAX_BUFS) {
        set_error("svp_submit: bad args/bufs");
        return SVP_E_INVAL;
    }
    svp_job_desc d;
    memset(&d, 0, sizeof(d));
    d.vp = vp;
    d.kernel = kernel;
    d.args_bytes = (uint32_t)args_bytes;
    d.nbufs = nbufs;
    if (args_bytes) memcpy(d.args, args, args_bytes);
    for (int b = 0; b < nbufs; ++b) d.bufs[b] = bufs[b];
    return submit_many(reinterpret_cast<Ctx*>(h), 1, &d, nullptr, job_out);
    SVP_TRY_END
}

svp_status svp_submit_batch(svp_ctx* h, int32_t n, const svp_job_desc* jobs, uint64_t* ids) {
    SVP_TRY_BEGIN
    svp_status st = check_ctx(h);
    if (st) return st;
    if (n < 0 || (n && !jobs)) {
        set_error("svp_submit_batch: bad n/jobs");
        return SVP_E_INVAL;
    }
    return submit_many(reinterpret_cast<Ctx*>(h), n, jobs, nullptr, ids);
    SVP_TRY_END
}

// One flush of everything queued so far (serialized by flush_mu).  Marks every job id
// below the snapshot's next id as completed (or failed with the flush's status) and
// wakes svp_wait callers.
// Same requests in the same order: VP, kernel, argument bytes and buffer descriptors.
static bool same_requests(const std::vector<Job>& a, const std::vector<Job>& b) {
    if (a.size() != b.size() || a.empty()) return false;
    for (size_t i = 0; i < a.size(); ++i) {
        const Job &x = a[i], &y = b[i];
        if (x.vp != y.vp || x.kernel != y.kernel || x.nbufs != y.nbufs || x.device != y.device ||
            memcmp(x.args, y.args, sizeof(x.args)) != 0)
            return false;
        for (int k = 0; k < x.nbufs; ++k)
            if (x.bufs[k].ptr != y.bufs[k].ptr || x.bufs[k].bytes != y.bufs[k].bytes ||
                x.bufs[k].dir != y.bufs[k].dir || x.bufs[k].mem != y.bufs[k].mem)
                return false;
    }
    return true;
}

// The wait half of a flush (under flush_mu): its device work, the Profiler, the flush
// statistics, the plan cache, and job completion (svp_wait).
static svp_status complete_flush(Ctx* c, Ctx::PendingFlush& p) {
    Flush& f = p.f;
    svp_status st = p.st;
    if (st == SVP_OK && c->exec && !f.ops.empty()) {
        st = executor_complete(c->exec, &f);
        if (st == SVP_E_CUDA || st == SVP_E_TIMEOUT) {
            const std::string msg = executor_error(c->exec);
            {
                std::lock_guard<std::mutex> lk(c->done_mu);
                c->sticky_msg = msg;
                c->sticky.store(st);
            }
            set_error(msg);
        } else if (st) {
            set_error(executor_error(c->exec));
        }
    }
    auto t2 = std::chrono::steady_clock::now();
    f.stats.host_total_ns = std::chrono::duration<double, std::nano>(t2 - p.t0).count();
    c->fstats = f.stats;
    if (c->cfg.graph && c->last_ok && !c->last.jobs.empty()) {
        // the previous flush joins the plan cache (most recent first, one entry per plan)
        const uint64_t gen = c->last.plan_gen;
        for (size_t k = 0; k < c->plan_cache.size();)
            if (c->plan_cache[k].plan_gen == gen || c->plan_cache[k].plan_gen == f.plan_gen)
                c->plan_cache.erase(c->plan_cache.begin() + (long)k);
            else
                ++k;
        if (gen != f.plan_gen) {
            c->plan_cache.insert(c->plan_cache.begin(), std::move(c->last));
            if (c->plan_cache.size() > Ctx::kPlanCache) c->plan_cache.pop_back();
        }
    }
    const uint64_t seq = f.seq;
    c->last = std::move(f);
    c->last_ok = st == SVP_OK;
    {
        std::lock_guard<std::mutex> lk(c->done_mu);
        if (st != SVP_OK && p.upto > c->completed_upto) c->failed.emplace_back(p.upto, st);
        if (st != SVP_OK) c->failed_flushes.emplace_back(seq, st);
        if (p.upto > c->completed_upto) c->completed_upto = p.upto;
    }
    c->done_cv.notify_all();
    return st;
}

// Complete the pending async flush, if any (under flush_mu).
static svp_status complete_pending(Ctx* c) {
    if (!c->pending) return SVP_OK;
    std::unique_ptr<Ctx::PendingFlush> p = std::move(c->pending);
    return complete_flush(c, *p);
}

// One flush of everything queued so far (serialized by flush_mu): plan (or reuse a cached
// plan), issue every GPU's work, then -- after completing the previous async flush, whose
// device work ran meanwhile -- either wait for it (svp_flush) or leave it pending
// (svp_flush_async; *ticket = its sequence number).  Marks every job id below the
// snapshot's next id as completed (or failed with the flush's status) and wakes svp_wait
// callers when the flush completes.
static svp_status do_flush(Ctx* c, bool async, uint64_t* ticket) {
    std::lock_guard<std::mutex> flk(c->flush_mu);
    if (c->sticky.load() != SVP_OK) {
        set_error("context is sticky-errored: " + c->sticky_message());
        return SVP_E_STATE;
    }
    // overlap needs per-op profiling off (its events are reused flush to flush) and no
    // per-job synchronization; otherwise the previous flush completes first
    const bool overlap = c->cfg.profile_level == 0 && !c->cfg.sync_each_job;
    if (!overlap) {
        svp_status ps = complete_pending(c);
        if (ps == SVP_E_CUDA || ps == SVP_E_TIMEOUT) return ps;
    }
    auto p = std::make_unique<Ctx::PendingFlush>();
    p->t0 = std::chrono::steady_clock::now();
    Flush& f = p->f;
    {
        std::lock_guard<std::mutex> lk(c->qmu);
        f.jobs.swap(c->queue);
        p->upto = c->next_job_id - 1;
    }
    f.seq = ++c->flush_seq;
    svp_status st = SVP_OK;
    // Steady-state replay (cfg.graph, NEXT f4): the same requests as a recent flush (the
    // previous one, or one of the Ctx::kPlanCache before it -- a serving loop that alternates
    // input buffer sets alternates plans) get the same plan, so copy it (and, in the
    // executor, replay its CUDA graph).  A mismatch is found at the first differing job.
    const Flush* hit = nullptr;
    if (c->cfg.graph && !c->cfg.sync_each_job) {
        if (c->last_ok && same_requests(f.jobs, c->last.jobs)) hit = &c->last;
        for (size_t k = 0; !hit && k < c->plan_cache.size(); ++k)
            if (same_requests(f.jobs, c->plan_cache[k].jobs)) hit = &c->plan_cache[k];
    }
    const bool reuse = hit != nullptr;
    if (reuse) {
        for (size_t i = 0; i < f.jobs.size(); ++i) f.jobs[i].level = hit->jobs[i].level;
        f.groups = hit->groups;
        f.chunks = hit->chunks;
        f.ops = hit->ops;
        for (auto& o : f.ops) o.measured_ns = o.measured_start_ns = -1;
        f.levels = hit->levels;
        f.plan_gen = hit->plan_gen;
        f.reused = true;
        f.stats.plan_reused = 1;
    } else {
        st = plan_flush(c, &f);
        f.plan_gen = ++c->plan_gen;
    }
    auto t1 = std::chrono::steady_clock::now();
    if (st == SVP_OK) {
        double makespan = c->last_sim_makespan, serial = c->last_sim_serial;
        if (!reuse) simulate(c, &f, &makespan, &serial);
        c->last_sim_makespan = makespan;
        c->last_sim_serial = serial;
        f.stats.sim_makespan_ns = makespan;
        f.stats.sim_serial_ns = serial;
        f.stats.host_plan_ns = std::chrono::duration<double, std::nano>(t1 - p->t0).count();
        f.stats.jobs = f.jobs.size();
        f.stats.groups = f.groups.size();
        f.stats.chunks = f.chunks.size();
        f.stats.levels = f.levels;
        if (c->exec && !f.ops.empty()) {
            st = executor_issue(c->exec, &f);
            if (st) {
                executor_abandon(c->exec, &f);
                if (st == SVP_E_CUDA || st == SVP_E_TIMEOUT) {
                    const std::string msg = executor_error(c->exec);
                    {
                        std::lock_guard<std::mutex> lk(c->done_mu);
                        c->sticky_msg = msg;
                        c->sticky.store(st);
                    }
                    set_error(msg);
                } else {
                    set_error(executor_error(c->exec));
                }
            }
        }
    }
    if (st == SVP_OK) {
        // (after the issue half: the tables decide each chunk's kernel_launches)
        uint64_t launches = 0;
        for (auto& op : f.ops) {
            if (op.kind == SVP_OP_KERNEL) {
                ++launches;
                if (executor_chunk_launches(f, f.chunks[op.chunk]))
                    f.stats.kernel_launches += (uint64_t)f.chunks[op.chunk].kernel_launches;
            }
            if (op.kind == SVP_OP_H2D) f.stats.h2d_bytes += op.bytes;
            if (op.kind == SVP_OP_D2H) f.stats.d2h_bytes += op.bytes;
        }
        f.stats.launches = launches;
    }
    p->st = st;
    // the previous async flush's device work ran while this one was planned and issued
    svp_status prev = complete_pending(c);
    if (async && st == SVP_OK && prev == SVP_OK && c->exec && !f.ops.empty()) {
        if (ticket) *ticket = f.seq;
        c->pending = std::move(p);
        return SVP_OK;
    }
    if (ticket) *ticket = f.seq;
    st = complete_flush(c, *p);
    return st != SVP_OK ? st : prev;
}

svp_status svp_flush(svp_ctx* h) {
    SVP_TRY_BEGIN
    svp_status st = check_ctx(h);
    if (st) return st;
    return do_flush(reinterpret_cast<Ctx*>(h), false, nullptr);
    SVP_TRY_END
}

svp_status svp_flush_async(svp_ctx* h, uint64_t* ticket_out) {
    SVP_TRY_BEGIN
    svp_status st = check_ctx(h);
    if (st) return st;
    if (ticket_out) *ticket_out = 0;
    return do_flush(reinterpret_cast<Ctx*>(h), true, ticket_out);
    SVP_TRY_END
}

svp_status svp_flush_wait(svp_ctx* h, uint64_t ticket) {
    SVP_TRY_BEGIN
    if (!h) {
        set_error("null context");
        return SVP_E_INVAL;
    }
    Ctx* c = reinterpret_cast<Ctx*>(h);
    std::lock_guard<std::mutex> flk(c->flush_mu);
    if (ticket > c->flush_seq) {
        set_error("svp_flush_wait: unknown ticket");
        return SVP_E_INVAL;
    }
    if (c->pending && c->pending->f.seq <= ticket) {
        svp_status st = complete_pending(c);
        if (st) return st;
    }
    std::lock_guard<std::mutex> lk(c->done_mu);
    for (const auto& fs : c->failed_flushes)
        if (fs.first == ticket) {
            set_error("svp_flush_wait: that flush failed");
            return fs.second;
        }
    return SVP_OK;
    SVP_TRY_END
}

svp_status svp_wait(svp_ctx* h, uint64_t job, int32_t timeout_ms) {
    SVP_TRY_BEGIN
    if (!h) {
        set_error("null context");
        return SVP_E_INVAL;
    }
    Ctx* c = reinterpret_cast<Ctx*>(h);
    {
        std::lock_guard<std::mutex> lk(c->qmu);
        if (job == 0 || job >= c->next_job_id) {
            set_error("svp_wait: unknown job id");
            return SVP_E_INVAL;
        }
    }
    {
        // a job of the pending async flush: complete that flush here
        std::lock_guard<std::mutex> flk(c->flush_mu);
        if (c->pending && job <= c->pending->upto) complete_pending(c);
    }
    std::unique_lock<std::mutex> lk(c->done_mu);
    auto done = [&] { return c->completed_upto >= job || c->sticky != SVP_OK; };
    if (timeout_ms > 0) {
        if (!c->done_cv.wait_for(lk, std::chrono::milliseconds(timeout_ms), done)) {
            set_error("svp_wait: timed out");
            return SVP_E_TIMEOUT;
        }
    } else {
        c->done_cv.wait(lk, done);
    }
    if (c->completed_upto < job) {
        set_error("svp_wait: context errored before the job ran: " + c->sticky_msg);  // under done_mu
        return SVP_E_STATE;
    }
    lk.unlock();
    svp_status js = ctx_job_status(c, job);
    if (js) set_error("svp_wait: the flush that ran this job failed");
    return js;
    SVP_TRY_END
}

static void dispatcher_loop(Ctx* c) {
    for (;;) {
        {
            std::unique_lock<std::mutex> lk(c->qmu);
            c->q_cv.wait(lk, [&] { return c->disp_stop || !c->queue.empty(); });
            if (c->queue.empty() && c->disp_stop) return;
            // batching window: let more VPs join this flush (coalescing width)
            if (c->disp_window_us > 0 && !c->disp_stop) {
                auto deadline = std::chrono::steady_clock::now() + std::chrono::microseconds(c->disp_window_us);
                c->q_cv.wait_until(lk, deadline, [&] {
                    return c->disp_stop || (c->disp_max_jobs > 0 && (int64_t)c->queue.size() >= c->disp_max_jobs);
                });
            }
        }
        if (do_flush(c, false, nullptr) == SVP_E_STATE && c->sticky != SVP_OK) {
            c->done_cv.notify_all();
            return;
        }
    }
}

}  // extern "C"

svp_status svp::ctx_submit_one(Ctx* c, const svp_job_desc& d, uint64_t* id) {
    if (c->sticky != SVP_OK) return SVP_E_STATE;
    return submit_many(c, 1, &d, nullptr, id);
}

extern "C" {

svp_status svp_start_dispatcher(svp_ctx* h, int32_t window_us, int32_t max_jobs) {
    SVP_TRY_BEGIN
    svp_status st = check_ctx(h);
    if (st) return st;
    if (window_us < 0 || max_jobs < 0) {
        set_error("svp_start_dispatcher: negative window/max_jobs");
        return SVP_E_INVAL;
    }
    Ctx* c = reinterpret_cast<Ctx*>(h);
    std::lock_guard<std::mutex> lk(c->qmu);
    if (c->disp_running) {
        set_error("svp_start_dispatcher: already running");
        return SVP_E_STATE;
    }
    c->disp_window_us = window_us;
    c->disp_max_jobs = max_jobs;
    c->disp_stop = false;
    c->disp_running = true;
    c->disp = std::thread(dispatcher_loop, c);
    return SVP_OK;
    SVP_TRY_END
}

static void stop_dispatcher(Ctx* c) {
    {
        std::lock_guard<std::mutex> lk(c->qmu);
        if (!c->disp_running) return;
        c->disp_stop = true;
    }
    c->q_cv.notify_all();
    c->disp.join();
    std::lock_guard<std::mutex> lk(c->qmu);
    c->disp_running = false;
}

svp_status svp_stop_dispatcher(svp_ctx* h) {
    SVP_TRY_BEGIN
    if (!h) {
        set_error("null context");
        return SVP_E_INVAL;
    }
    stop_dispatcher(reinterpret_cast<Ctx*>(h));
    return SVP_OK;
    SVP_TRY_END
}

svp_status svp_vp_device(svp_ctx* h, int32_t vp, int32_t* device_out) {
    SVP_TRY_BEGIN
    svp_status st = check_ctx(h);
    if (st) return st;
    if (!device_out || vp < 0 || vp >= (1 << 20)) {
        set_error("svp_vp_device: bad vp/out");
        return SVP_E_INVAL;
    }
    *device_out = dispatch_vp(reinterpret_cast<Ctx*>(h), vp, 0.0);
    return SVP_OK;
    SVP_TRY_END
}

svp_status svp_assign_vps(svp_ctx* h, int32_t n, const int32_t* vps, const int32_t* classes, const double* costs,
                          int32_t* devices_out) {
    SVP_TRY_BEGIN
    svp_status st = check_ctx(h);
    if (st) return st;
    if (n < 0 || (n && (!vps || !classes || !costs))) {
        set_error("svp_assign_vps: bad arguments");
        return SVP_E_INVAL;
    }
    Ctx* c = reinterpret_cast<Ctx*>(h);
    std::lock_guard<std::mutex> lk(c->dmu);
    std::vector<int32_t> idx, cls;
    std::vector<double> cst;
    for (int i = 0; i < n; ++i) {
        if (vps[i] < 0 || vps[i] >= (1 << 20)) {
            set_error("svp_assign_vps: vp out of range");
            return SVP_E_INVAL;
        }
        if (!c->vp_dev.count(vps[i])) {
            idx.push_back(i);
            cls.push_back(classes[i]);
            cst.push_back(costs[i]);
        }
    }
    std::vector<int32_t> out(idx.size());
    lpt_stratified((int32_t)idx.size(), cls.data(), cst.data(), c->ngpu, c->dev_load.data(), out.data());
    for (size_t k = 0; k < idx.size(); ++k) {
        c->vp_dev[vps[idx[k]]] = out[k];
        c->dev_load[out[k]] += cst[k];
    }
    if (devices_out)
        for (int i = 0; i < n; ++i) devices_out[i] = c->vp_dev[vps[i]];
    return SVP_OK;
    SVP_TRY_END
}

svp_status svp_lpt_partition(int32_t n, const int32_t* classes, const double* costs, int32_t G, int32_t* out) {
    SVP_TRY_BEGIN
    if (n < 0 || G < 1 || (n && (!classes || !costs || !out))) {
        set_error("svp_lpt_partition: bad arguments");
        return SVP_E_INVAL;
    }
    std::vector<double> load(G, 0.0);
    lpt_stratified(n, classes, costs, G, load.data(), out);
    return SVP_OK;
    SVP_TRY_END
}

svp_status svp_profile(svp_ctx* h, int32_t vp, svp_vp_profile* out) {
    SVP_TRY_BEGIN
    if (!h || !out) {
        set_error("svp_profile: null argument");
        return SVP_E_INVAL;
    }
    Ctx* c = reinterpret_cast<Ctx*>(h);
    std::lock_guard<std::mutex> lk(c->pmu);
    memset(out, 0, sizeof(*out));
    const VpProfile* p = nullptr;
    if (vp == -1) {
        p = &c->prof_total;
        out->launches = c->prof_launches;
    } else {
        auto it = c->prof.find(vp);
        if (it == c->prof.end()) return SVP_OK;
        p = &it->second;
    }
    out->jobs = p->jobs;
    out->kernel_ns = p->kernel_ns;
    out->h2d_ns = p->h2d_ns;
    out->d2h_ns = p->d2h_ns;
    out->bytes_kernel = p->bytes_kernel;
    out->bytes_h2d = p->bytes_h2d;
    out->bytes_d2h = p->bytes_d2h;
    out->flops = p->flops;
    return SVP_OK;
    SVP_TRY_END
}

svp_status svp_reset_profile(svp_ctx* h) {
    SVP_TRY_BEGIN
    if (!h) {
        set_error("null context");
        return SVP_E_INVAL;
    }
    Ctx* c = reinterpret_cast<Ctx*>(h);
    std::lock_guard<std::mutex> lk(c->pmu);
    c->prof.clear();
    c->prof_total = VpProfile{};
    c->prof_launches = 0;
    for (auto& k : c->kstats) k = KStats{};
    for (auto& d : c->dstats) d = DevStats{};
    return SVP_OK;
    SVP_TRY_END
}

svp_status svp_kernel_stats_get(svp_ctx* h, int32_t kernel, svp_kernel_stats* out) {
    SVP_TRY_BEGIN
    if (!h || !out) {
        set_error("null argument");
        return SVP_E_INVAL;
    }
    if (!kernel_desc(kernel) && kernel != K_EW_MIX) {
        set_error("unknown kernel id");
        return SVP_E_NOKERNEL;
    }
    Ctx* c = reinterpret_cast<Ctx*>(h);
    std::lock_guard<std::mutex> lk(c->pmu);
    const KStats& k = c->kstats[kernel];
    out->launches = k.launches;
    out->total_ns = k.total_ns;
    out->bytes = k.bytes;
    out->flops = k.flops;
    out->max_ns = k.max_ns;
    return SVP_OK;
    SVP_TRY_END
}

svp_status svp_device_stats_get(svp_ctx* h, int32_t g, svp_device_stats* out) {
    SVP_TRY_BEGIN
    if (!h || !out) {
        set_error("null argument");
        return SVP_E_INVAL;
    }
    Ctx* c = reinterpret_cast<Ctx*>(h);
    if (g < 0 || g >= c->ngpu) {
        set_error("svp_device_stats_get: GPU index out of range");
        return SVP_E_INVAL;
    }
    memset(out, 0, sizeof(*out));
    out->ordinal = g < (int32_t)c->device_ids.size() ? c->device_ids[g] : g;
    {
        std::lock_guard<std::mutex> lk(c->dmu);
        for (const auto& kv : c->vp_dev)
            if (kv.second == g) out->vps += 1;
        out->est_load_ns = c->dev_load[g];
    }
    std::lock_guard<std::mutex> lk(c->pmu);
    const DevStats& d = c->dstats[g];
    out->flushes = d.flushes;
    out->jobs = d.jobs;
    out->device_ns = d.device_ns;
    out->kernel_ns = d.kernel_ns;
    out->last_device_ns = d.last_device_ns;
    out->numa_node = -1;
    if (c->exec) executor_numa_info(c->exec, g, &out->numa_node, &out->worker_cpu_pinned);
    return SVP_OK;
    SVP_TRY_END
}

svp_status svp_flush_stats_get(svp_ctx* h, svp_flush_stats* out) {
    if (!h || !out) {
        set_error("null argument");
        return SVP_E_INVAL;
    }
    *out = reinterpret_cast<Ctx*>(h)->fstats;
    return SVP_OK;
}

svp_status svp_plan_size(svp_ctx* h, int32_t* n) {
    if (!h || !n) {
        set_error("null argument");
        return SVP_E_INVAL;
    }
    *n = (int32_t)reinterpret_cast<Ctx*>(h)->last.ops.size();
    return SVP_OK;
}

svp_status svp_plan_get(svp_ctx* h, int32_t i, svp_plan_op* op, int32_t* vps_out, int32_t cap) {
    if (!h || !op) {
        set_error("null argument");
        return SVP_E_INVAL;
    }
    Ctx* c = reinterpret_cast<Ctx*>(h);
    const Flush& f = c->last;
    if (i < 0 || i >= (int32_t)f.ops.size()) {
        set_error("svp_plan_get: index out of range");
        return SVP_E_INVAL;
    }
    const Op& o = f.ops[i];
    const Chunk& ch = f.chunks[o.chunk];
    op->kind = o.kind;
    op->device = o.device;
    op->stream = o.stream;
    op->level = ch.level;
    op->kernel = ch.kernel;
    op->group = ch.group;
    op->chunk = ch.index;
    op->nvps = (int32_t)ch.jobs.size();
    op->bytes = o.bytes;
    op->flops = o.flops;
    op->est_ns = o.est_ns;
    op->sim_start_ns = o.sim_start;
    op->sim_end_ns = o.sim_end;
    op->measured_ns = o.measured_ns;
    if (vps_out)
        for (int k = 0; k < (int)ch.jobs.size() && k < cap; ++k) vps_out[k] = f.jobs[ch.jobs[k]].vp;
    return SVP_OK;
}

svp_status svp_plan_op_detail(svp_ctx* h, int32_t i, uint64_t* arena_off, uint64_t* arena_len, int32_t* waits_out,
                              int32_t cap, int32_t* nwaits, double* measured_start_ns) {
    if (!h) {
        set_error("null context");
        return SVP_E_INVAL;
    }
    const Flush& f = reinterpret_cast<Ctx*>(h)->last;
    if (i < 0 || i >= (int32_t)f.ops.size()) {
        set_error("svp_plan_op_detail: index out of range");
        return SVP_E_INVAL;
    }
    const Op& o = f.ops[i];
    const Chunk& ch = f.chunks[o.chunk];
    if (arena_off) *arena_off = ch.arena_off;
    if (arena_len) *arena_len = ch.arena_len;
    if (nwaits) *nwaits = (int32_t)o.wait_ops.size();
    if (measured_start_ns) *measured_start_ns = o.measured_start_ns;
    if (waits_out)
        for (int k = 0; k < (int)o.wait_ops.size() && k < cap; ++k) waits_out[k] = o.wait_ops[k];
    return SVP_OK;
}

}  // extern "C"

svp_status svp_host_alloc(svp_ctx* h, int32_t gpu, uint64_t bytes, void** ptr_out, int32_t* numa_node_out) {
    SVP_TRY_BEGIN
    svp_status st = check_ctx(h);
    if (st) return st;
    if (!ptr_out || bytes == 0) {
        set_error("svp_host_alloc: null ptr_out or bytes == 0");
        return SVP_E_INVAL;
    }
    *ptr_out = nullptr;
    if (numa_node_out) *numa_node_out = -1;
    Ctx* c = reinterpret_cast<Ctx*>(h);
    if (gpu < 0 || gpu >= c->ngpu) {
        set_error("svp_host_alloc: GPU index out of range");
        return SVP_E_INVAL;
    }
    if (!c->exec) {
        set_error("svp_host_alloc: a dry-run context has no CUDA devices");
        return SVP_E_UNSUPPORTED;
    }
    const long pg = sysconf(_SC_PAGESIZE) > 0 ? sysconf(_SC_PAGESIZE) : 4096;
    const size_t len = (size_t)((bytes + (uint64_t)pg - 1) / (uint64_t)pg * (uint64_t)pg);
    const int ordinal = gpu < (int32_t)c->device_ids.size() ? c->device_ids[gpu] : gpu;
    void* p = nullptr;
    int node = -1;
    std::string err;
    st = host_alloc_near(ordinal, len, &p, &node, &err);
    if (st) {
        set_error(err);
        return st;
    }
    {
        std::lock_guard<std::mutex> lk(c->hmu);
        c->host_blocks[p] = len;
    }
    *ptr_out = p;
    if (numa_node_out) *numa_node_out = node;
    return SVP_OK;
    SVP_TRY_END
}

svp_status svp_host_free(svp_ctx* h, void* ptr) {
    SVP_TRY_BEGIN
    if (!h) {
        set_error("null context");
        return SVP_E_INVAL;
    }
    Ctx* c = reinterpret_cast<Ctx*>(h);
    size_t len = 0;
    {
        std::lock_guard<std::mutex> lk(c->hmu);
        auto it = c->host_blocks.find(ptr);
        if (it == c->host_blocks.end()) {
            set_error("svp_host_free: not a block from svp_host_alloc (or already freed)");
            return SVP_E_INVAL;
        }
        len = it->second;
        c->host_blocks.erase(it);
    }
    if (c->exec) executor_forget_range(c->exec, (uintptr_t)ptr, (uintptr_t)ptr + len);
    host_free_near(ptr, len);
    return SVP_OK;
    SVP_TRY_END
}

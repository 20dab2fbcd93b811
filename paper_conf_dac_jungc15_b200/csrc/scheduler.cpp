// scheduler.cpp -- Job Queue validation, Kernel Match, Job Dispatcher, Re-scheduler
// and the cost model (host side, no CUDA).  SURVEY.md §8(a) rows a1-a4.
//
//  * Job Queue (Fig 2): jobs arrive per VP in program
//    order; at svp_flush the queue is snapshotted and the l-th pending job of a VP
//    gets level l.  Reading R3: a VP's jobs are totally ordered (program order);
//    jobs of different VPs are independent.
//  * Kernel Match: within a level and a GPU, jobs with
//    the same (kernel id, shape key) are "identical kernel requests" and form one
//    group (reading R1: ragged n is allowed for the elementwise kernels, SGEMM needs
//    equal M,N,K).  Groups are ordered by (kernel, shape key); members by VP id (R12).
//  * Job Dispatcher ("multiplexes the host GPUs", L28-31): every VP
//    is pinned to one GPU (sticky), placed by kernel-stratified LPT.
//  * Re-scheduler (Fig 3/4a): splits each group into c
//    chunks so copies of one chunk overlap the kernel of another, orders the chunks
//    of a level with Johnson's rule on (Tin+Tk, Tk+Tout) using the expected time of
//    each invocation (reading R4), assigns streams (one H2D, one
//    D2H, a pool of compute streams -- the paper's Copy/Compute engines), and adds
//    the event dependencies that keep every VP's program order.
#include <math.h>
#include <stdlib.h>
#include <string.h>

#include <algorithm>
#include <map>
#include <numeric>
#include <tuple>

#include "internal.h"
#include "launch.h"
#include "tables.h"

namespace svp {

// ------------------------------------------------------------------ cost model
double CostModel::kernel_ns(int32_t kernel, double alg_bytes, double flops) const {
    double body;
    if (kernel == K_SGEMM) body = flops / (sgemm_tc_units ? tf32_flops / sgemm_tc_units : ffma_flops) * 1e9;
    else if (kernel == K_DGEMM) body = flops / fp64_flops * 1e9;
    else if (kernel == K_SGEMM_TF32) body = flops / tf32_flops * 1e9;
    else body = alg_bytes / hbm_Bps * 1e9;
    return launch_ns + body * kscale[kernel][bucket(alg_bytes, flops)];
}
double CostModel::sgemm_ns(int32_t impl, double alg_bytes, double flops) const {
    const int units = impl == SVP_SGEMM_3XTF32 ? 3 : impl == SVP_SGEMM_TF32BF16 ? 2 : 0;
    const double body = flops / (units ? tf32_flops / units : ffma_flops) * 1e9;
    return launch_ns + body * kscale[K_SGEMM][bucket(alg_bytes, flops)];
}
double CostModel::h2d_ns(uint64_t bytes, int ncopies) const {
    return bytes ? copy_ns * ncopies + (double)bytes / pcie_Bps * 1e9 : 0.0;
}
double CostModel::d2h_ns(uint64_t bytes, int ncopies) const {
    return bytes ? copy_ns * ncopies + (double)bytes / pcie_Bps * 1e9 : 0.0;
}

// ------------------------------------------------------------------ validation (a1)
uint64_t touched_bytes(const Job& j, int b) {
    switch (j.kernel) {
        case K_VECADD:
        case K_SAXPY:
        case K_BLACKSCHOLES: return 4ull * j.n;
        case K_HIST256: return b == 0 ? j.n : 1024ull;
        case K_SGEMM:
        case K_SGEMM_TF32:
        case K_DGEMM: {
            const uint64_t es = j.kernel == K_DGEMM ? 8 : 4;
            if (b == 0) return es * j.M * j.K;
            if (b == 1) return es * j.K * j.N;
            return es * j.M * j.N;
        }
    }
    return 0;
}

static svp_status fail(svp_status st, const std::string& msg) {
    set_error(msg);
    return st;
}

svp_status validate_and_fill(Ctx* c, Job* j) {
    const KernelDesc* d = kernel_desc(j->kernel);
    if (!d || !c->registered[j->kernel])
        return fail(SVP_E_NOKERNEL, "svp_submit: kernel id " + std::to_string(j->kernel) + " not registered");
    if (j->vp < 0 || j->vp >= (1 << 20)) return fail(SVP_E_INVAL, "svp_submit: vp out of range [0, 2^20)");
    if (j->nbufs != d->nbufs)
        return fail(SVP_E_INVAL, std::string("svp_submit: ") + d->name + " takes " + std::to_string(d->nbufs) +
                                     " buffers");
    switch (j->kernel) {
        case K_VECADD:
        case K_HIST256: memcpy(&j->n, j->args, 8); break;
        case K_SAXPY:
            memcpy(&j->n, j->args, 8);
            memcpy(&j->f0, j->args + 8, 4);
            break;
        case K_BLACKSCHOLES:
            memcpy(&j->n, j->args, 8);
            memcpy(&j->f0, j->args + 8, 4);
            memcpy(&j->f1, j->args + 12, 4);
            break;
        case K_SGEMM:
        case K_SGEMM_TF32: {
            svp_args_sgemm a;
            memcpy(&a, j->args, sizeof(a));
            if (a.M < 0 || a.N < 0 || a.K < 0 || a.M >= (1 << 20) || a.N >= (1 << 20) || a.K >= (1 << 20))
                return fail(SVP_E_INVAL, "svp_submit: sgemm M,N,K must be in [0, 2^20)");
            j->M = a.M;
            j->N = a.N;
            j->K = a.K;
            j->f0 = a.alpha;
            j->f1 = a.beta;
            break;
        }
        case K_DGEMM: {
            svp_args_dgemm a;
            memcpy(&a, j->args, sizeof(a));
            if (a.M < 0 || a.N < 0 || a.K < 0 || a.M >= (1 << 20) || a.N >= (1 << 20) || a.K >= (1 << 20))
                return fail(SVP_E_INVAL, "svp_submit: dgemm M,N,K must be in [0, 2^20)");
            j->M = a.M;
            j->N = a.N;
            j->K = a.K;
            j->d0 = a.alpha;
            j->d1 = a.beta;
            break;
        }
    }
    if (j->n >= (1ull << 40)) return fail(SVP_E_INVAL, "svp_submit: n too large");
    // hist256 always writes its 256 counters (an empty input still overwrites them)
    bool empty = is_gemm(j->kernel) ? ((int64_t)j->M * j->N == 0)
                 : j->kernel == K_HIST256                             ? false
                                                                      : (j->n == 0);
    j->in_bytes = j->out_bytes = j->host_in_bytes = j->host_out_bytes = 0;
    for (int b = 0; b < j->nbufs; ++b) {
        const svp_buf& bf = j->bufs[b];
        uint64_t need = touched_bytes(*j, b);
        int want = d->dirs[b];
        bool is_c = is_gemm(j->kernel) && b == 2;
        const bool beta_nz = j->kernel == K_DGEMM ? j->d1 != 0.0 : j->f1 != 0.f;
        if (is_c) {
            if (beta_nz && bf.dir != SVP_DIR_INOUT)
                return fail(SVP_E_INVAL, "svp_submit: sgemm with beta != 0 needs C as SVP_DIR_INOUT");
            if (bf.dir != SVP_DIR_OUT && bf.dir != SVP_DIR_INOUT)
                return fail(SVP_E_INVAL, "svp_submit: sgemm C must be OUT or INOUT");
        } else if (bf.dir != want) {
            return fail(SVP_E_INVAL, std::string("svp_submit: buffer ") + std::to_string(b) + " of " + d->name +
                                         " has the wrong direction");
        }
        if (bf.mem != SVP_MEM_DEVICE && bf.mem != SVP_MEM_HOST_PINNED)
            return fail(SVP_E_INVAL, "svp_submit: buffer mem must be DEVICE or HOST_PINNED");
        if (empty) continue;
        if (need && !bf.ptr) return fail(SVP_E_INVAL, "svp_submit: null buffer " + std::to_string(b));
        if (bf.bytes < need)
            return fail(SVP_E_INVAL, "svp_submit: buffer " + std::to_string(b) + " has " + std::to_string(bf.bytes) +
                                         " bytes, kernel touches " + std::to_string(need));
        if (j->kernel == K_DGEMM && ((uintptr_t)bf.ptr & 7))
            return fail(SVP_E_INVAL, "svp_submit: dgemm buffers must be 8-B aligned");
        bool rd = bf.dir & SVP_DIR_IN, wr = bf.dir & SVP_DIR_OUT;
        // sgemm C with beta == 0 is written only; hist counts are written only
        if (rd) j->in_bytes += need;
        if (wr) j->out_bytes += need;
        if (bf.mem == SVP_MEM_HOST_PINNED) {
            if (rd) j->host_in_bytes += need;
            if (wr) j->host_out_bytes += need;
        }
    }
    switch (j->kernel) {
        case K_VECADD:
        case K_SAXPY: j->alg_bytes = 12.0 * j->n; break;
        case K_HIST256: j->alg_bytes = (double)j->n + (j->n ? 1024.0 : 0.0); break;
        case K_BLACKSCHOLES: j->alg_bytes = 20.0 * j->n; break;
        default: {
            const bool dbl = j->kernel == K_DGEMM;
            const bool beta_nz2 = dbl ? j->d1 != 0.0 : j->f1 != 0.f;
            j->alg_bytes = (dbl ? 8.0 : 4.0) * ((double)j->M * j->K + (double)j->K * j->N +
                                                (double)j->M * j->N * (beta_nz2 ? 2 : 1));
            j->flops = 2.0 * j->M * j->N * (double)j->K;
        }
    }
    // Reading R1 (revised with f2): every job of a kernel is "identical" -- ragged element
    // counts AND ragged GEMM shapes share one coalesced launch (per-VP M, N, K live in
    // the tile table).
    // Jobs TMA cannot address (a row pitch of K or N floats not a multiple of 16 B, or a
    // device buffer not 16-B aligned; staged host buffers are 256-B aligned in the arena)
    // match as their own group on the plain-load kernel (shape key 2); R23: "sgemm" jobs past
    // the tensor-core split's K limit match apart and run on FFMA (shape key 1).
    j->shape_key = 0;
    if (j->kernel == K_SGEMM || j->kernel == K_SGEMM_TF32) {
        bool plain = (j->K % 4) != 0 || (j->N % 4) != 0;
        for (int b = 0; b < j->nbufs; ++b)
            if (j->bufs[b].mem == SVP_MEM_DEVICE && ((uintptr_t)j->bufs[b].ptr & 15)) plain = true;
        if (plain) {
            j->shape_key = 2;
        } else if (j->kernel == K_SGEMM && c->cfg.sgemm_impl != SVP_SGEMM_FFMA) {
            // with K-chunked accumulation (sgemm_tc_kchunk) a beta == 0 job keeps the
            // tensor cores at any K; a beta != 0 job is not chunked (its exact NaN path needs
            // C_old), so it keeps them up to one chunk
            const int kc = sgemm_chunk_k(c->cfg.sgemm_impl, c->cfg.sgemm_kchunk);
            const int32_t kmax = kc > 0 ? (j->f1 != 0.f ? kc : (1 << 30)) : sgemm_tc_kmax(c->cfg.sgemm_impl);
            if (j->K > kmax) j->shape_key = 1;
        }
    }
    double cost = c->cost.kernel_ns(j->kernel, j->alg_bytes, j->flops);
    j->device = dispatch_vp(c, j->vp, cost);
    if (c->exec && c->cfg.validate_ptrs && !empty) {
        for (int b = 0; b < j->nbufs; ++b) {
            const uint64_t tb = touched_bytes(*j, b);
            if (tb == 0) continue;  // nothing is read or written there
            std::string why;
            if (executor_check_ptr(c->exec, j->bufs[b].ptr, tb, j->bufs[b].mem, j->device, &why) != SVP_OK)
                return fail(SVP_E_INVAL, "svp_submit: buffer " + std::to_string(b) + ": " + why);
        }
    }
    return SVP_OK;
}

// ------------------------------------------------------------------ Job Dispatcher (a3)
int32_t dispatch_vp(Ctx* c, int32_t vp, double cost) {
    std::lock_guard<std::mutex> lk(c->dmu);
    auto it = c->vp_dev.find(vp);
    if (it != c->vp_dev.end()) return it->second;
    int32_t best = 0;
    for (int32_t g = 1; g < c->ngpu; ++g)
        if (c->dev_load[g] < c->dev_load[best]) best = g;
    c->vp_dev[vp] = best;
    c->dev_load[best] += cost > 0 ? cost : 1.0;
    return best;
}

void lpt_stratified(int32_t n, const int32_t* classes, const double* costs, int32_t G, const double* init_load,
                    int32_t* out) {
    std::vector<double> load(init_load, init_load + G);
    std::map<int32_t, std::vector<int32_t>> by_class;
    for (int32_t i = 0; i < n; ++i) by_class[classes[i]].push_back(i);
    for (auto& kv : by_class) {
        auto& items = kv.second;
        std::stable_sort(items.begin(), items.end(), [&](int32_t a, int32_t b) {
            if (costs[a] != costs[b]) return costs[a] > costs[b];
            return a < b;
        });
        std::vector<double> cload(G, 0.0);
        for (int32_t i : items) {
            int32_t best = 0;
            for (int32_t g = 1; g < G; ++g) {
                if (std::tie(cload[g], load[g]) < std::tie(cload[best], load[best])) best = g;
            }
            out[i] = best;
            cload[best] += costs[i];
            load[best] += costs[i];
        }
    }
}

// ------------------------------------------------------------------ Re-scheduler (a4)
static void split_group(const Ctx* c, const Flush& f, const Group& g, int nchunks, std::vector<std::vector<int32_t>>& out) {
    // contiguous parts with balanced bytes (staged + algorithmic), members keep vp order
    std::vector<double> w;
    double tot = 0;
    for (int32_t ji : g.jobs) {
        const Job& j = f.jobs[ji];
        double x = (double)j.host_in_bytes + (double)j.host_out_bytes + j.alg_bytes + j.flops * 0.05 + 1.0;
        w.push_back(x);
        tot += x;
    }
    (void)c;
    out.clear();
    size_t m = g.jobs.size();
    nchunks = std::max(1, std::min<int>(nchunks, (int)m));
    double target = tot / nchunks, acc = 0;
    std::vector<int32_t> cur;
    for (size_t k = 0; k < m; ++k) {
        cur.push_back(g.jobs[k]);
        acc += w[k];
        size_t left_items = m - k - 1;
        int left_chunks = nchunks - (int)out.size() - 1;
        bool cut = acc >= target * (out.size() + 1) - 1e-9;
        if ((cut && left_chunks > 0 && left_items >= (size_t)left_chunks) || (left_items == (size_t)left_chunks && left_chunks > 0)) {
            out.push_back(cur);
            cur.clear();
        }
    }
    if (!cur.empty()) out.push_back(cur);
}

static void estimate_chunk(const Ctx* c, const Flush& f, Chunk& ch) {
    int nin = 0, nout = 0;
    ch.in_bytes = ch.out_bytes = 0;
    ch.alg_bytes = ch.flops = 0;
    for (int32_t ji : ch.jobs) {
        const Job& j = f.jobs[ji];
        ch.in_bytes += j.host_in_bytes;
        ch.out_bytes += j.host_out_bytes;
        ch.alg_bytes += j.alg_bytes;
        ch.flops += j.flops;
        for (int b = 0; b < j.nbufs; ++b) {
            if (j.bufs[b].mem != SVP_MEM_HOST_PINNED) continue;
            if (j.bufs[b].dir & SVP_DIR_IN) ++nin;
            if (j.bufs[b].dir & SVP_DIR_OUT) ++nout;
        }
    }
    ch.t_in = c->cost.h2d_ns(ch.in_bytes, nin);
    ch.t_k = (ch.kernel == K_SGEMM || ch.sgemm_impl == kSgemmPlain) ? c->cost.sgemm_ns(ch.sgemm_impl, ch.alg_bytes, ch.flops)
                                  : c->cost.kernel_ns(ch.kernel, ch.alg_bytes, ch.flops);
    ch.t_out = c->cost.d2h_ns(ch.out_bytes, nout);
}

static uint64_t staged_bytes(const Flush& f, const std::vector<int32_t>& jobs) {
    uint64_t s = 0;
    for (int32_t ji : jobs) {
        const Job& j = f.jobs[ji];
        for (int b = 0; b < j.nbufs; ++b)
            if (j.bufs[b].mem == SVP_MEM_HOST_PINNED) s += (touched_bytes(j, b) + 255) & ~255ull;
    }
    return s;
}

// Dense per-VP slots for the planner's per-VP state: a flat array when the VP ids are
// compact (the usual case), else a hash map (ids go up to 2^20).
struct VpSlots {
    std::vector<int32_t> flat;
    std::unordered_map<int32_t, int32_t> sparse;
    bool dense = true;
    int32_t init = 0;
    VpSlots(const std::vector<Job>& jobs, int32_t init_value) : init(init_value) {
        int32_t mx = -1;
        for (const auto& j : jobs) mx = std::max(mx, j.vp);
        dense = (size_t)mx < 4 * jobs.size() + 4096;
        if (dense) flat.assign((size_t)mx + 1, init_value);
        else sparse.reserve(jobs.size() * 2);
    }
    int32_t& operator[](int32_t vp) {
        if (dense) return flat[vp];
        auto it = sparse.find(vp);
        if (it == sparse.end()) it = sparse.emplace(vp, init).first;
        return it->second;
    }
};

svp_status plan_flush(Ctx* c, Flush* f) {
    const size_t n = f->jobs.size();
    // ---- levels (program order per VP)
    {
        VpSlots next_level(f->jobs, 0);
        f->levels = 0;
        for (auto& j : f->jobs) {
            j.level = next_level[j.vp]++;
            f->levels = std::max(f->levels, j.level + 1);
        }
    }
    const int S = c->cfg.streams_per_gpu;
    const bool inter = c->cfg.interleave != 0;
    const bool coal = c->cfg.coalesce != 0;

    // ---- Kernel Match (a2): groups per (level, device, kernel, shape)
    std::vector<int32_t> order(n);
    std::iota(order.begin(), order.end(), 0);
    // NEXT f4 (cfg.hetero): the elementwise kernels of one (level, GPU) match as ONE
    // heterogeneous group -- "identical kernels only" lifted for the
    // kernels that share a CTA shape and tile mapping; members stay in VP order.
    const bool het = c->cfg.hetero != 0;
    auto mkernel = [&](const Job& j) { return het && is_ew(j.kernel) ? (int32_t)K_EW_MIX : j.kernel; };
    f->groups.reserve(coal ? 16 : n);
    if (coal) {
        // sort by (level, device, match kernel, shape, vp); groups are the runs of equal
        // (level, device, match kernel, shape)
        struct MKey {
            int32_t level, device, kernel, vp;
            uint64_t shape;
        };
        std::vector<MKey> key(n);
        for (size_t i = 0; i < n; ++i) {
            const Job& j = f->jobs[i];
            key[i] = MKey{j.level, j.device, mkernel(j), j.vp, j.shape_key};
        }
        std::stable_sort(order.begin(), order.end(), [&](int32_t a, int32_t b) {
            const MKey &x = key[a], &y = key[b];
            return std::tie(x.level, x.device, x.kernel, x.shape, x.vp) <
                   std::tie(y.level, y.device, y.kernel, y.shape, y.vp);
        });
        for (size_t i = 0; i < n; ++i) {
            const MKey& k = key[order[i]];
            if (i == 0 || k.level != key[order[i - 1]].level || k.device != key[order[i - 1]].device ||
                k.kernel != key[order[i - 1]].kernel || k.shape != key[order[i - 1]].shape) {
                f->groups.emplace_back();
                Group& g = f->groups.back();
                g.kernel = k.kernel;
                g.shape_key = k.shape;
                g.level = k.level;
                g.device = k.device;
            }
            f->groups.back().jobs.push_back(order[i]);
        }
    } else {
        // no coalescing: one group per job, submission order within a level
        std::stable_sort(order.begin(), order.end(),
                         [&](int32_t a, int32_t b) { return f->jobs[a].level < f->jobs[b].level; });
        for (int32_t ji : order) {
            const Job& j = f->jobs[ji];
            f->groups.emplace_back();
            Group& g = f->groups.back();
            g.kernel = j.kernel;
            g.shape_key = j.shape_key;
            g.level = j.level;
            g.device = j.device;
            g.jobs.push_back(ji);
        }
    }

    // ---- chunking + estimates
    const uint64_t arena = c->cfg.arena_bytes;
    for (int32_t gi = 0; gi < (int32_t)f->groups.size(); ++gi) {
        const Group& g = f->groups[gi];
        const int32_t impl = g.shape_key == 2          ? kSgemmPlain
                             : g.kernel != K_SGEMM      ? -1
                             : g.shape_key == 1         ? (int32_t)SVP_SGEMM_FFMA
                                                        : c->cfg.sgemm_impl;
        Chunk whole;
        whole.kernel = g.kernel;
        whole.sgemm_impl = impl;
        whole.jobs = g.jobs;
        estimate_chunk(c, *f, whole);
        int nch = 1;
        bool staged = whole.in_bytes + whole.out_bytes > 0;
        if (staged && inter) {
            // c* ~ sqrt((sum T - max T) / T_o)  (Eq 7 pipeline gain vs Eq 9 per-launch overhead)
            double sum = whole.t_in + whole.t_k + whole.t_out;
            double mx = std::max(whole.t_in, std::max(whole.t_k, whole.t_out));
            double To = c->cost.launch_ns + 2 * c->cost.copy_ns;
            nch = (int)lround(sqrt(std::max(0.0, sum - mx) / To));
            nch = std::max(1, std::min(nch, c->cfg.max_chunks));
        }
        nch = std::min<int>(nch, (int)g.jobs.size());
        if (!staged) {
            // device-resident group: one chunk, the whole group (nothing to pipeline)
            Chunk ch = std::move(whole);
            ch.group = gi;
            ch.index = 0;
            ch.device = g.device;
            ch.level = g.level;
            ch.arena_len = 0;
            f->chunks.push_back(std::move(ch));
            continue;
        }
        std::vector<std::vector<int32_t>> parts;
        for (;;) {
            split_group(c, *f, g, nch, parts);
            uint64_t mx = 0;
            for (auto& p : parts) mx = std::max(mx, staged_bytes(*f, p));
            if (mx <= arena / 2 || nch >= (int)g.jobs.size()) {
                if (mx > arena) {
                    set_error("svp_flush: a job's host-resident buffers exceed the staging arena");
                    return SVP_E_NOMEM;
                }
                break;
            }
            nch = std::min<int>((int)g.jobs.size(), nch * 2);
        }
        for (size_t p = 0; p < parts.size(); ++p) {
            Chunk ch;
            ch.group = gi;
            ch.index = (int32_t)p;
            ch.device = g.device;
            ch.level = g.level;
            ch.kernel = g.kernel;
            ch.sgemm_impl = impl;
            ch.jobs = parts[p];
            estimate_chunk(c, *f, ch);
            ch.arena_len = staged_bytes(*f, ch.jobs);
            f->chunks.push_back(std::move(ch));
        }
    }

    // ---- order per (level, device): Johnson's rule on (Tin+Tk, Tk+Tout) when interleaving
    std::vector<int32_t> corder(f->chunks.size());
    std::iota(corder.begin(), corder.end(), 0);
    auto johnson_key = [&](int32_t ci) {
        const Chunk& ch = f->chunks[ci];
        double a = ch.t_in + ch.t_k, b = ch.t_k + ch.t_out;
        bool first = a < b;
        // first set: ascending a; second set: descending b; ties by (group, index)
        return std::make_tuple(first ? 0 : 1, first ? a : -b, ch.group, ch.index);
    };
    // Device-resident chunks (no copies): Johnson's key degenerates to longest-first, which
    // launches the tensor-core SGEMM (1 CTA/SM, most of shared memory) before the HBM-bound
    // kernels; their CTAs (no shared memory) then fill the SGEMM SMs' free thread and
    // register slots, so tensor-bound and HBM-bound coalesced kernels run concurrently
    // (cfg5: 44.1k jobs/s vs 42.7k on one stream).  SVP_COSCHEDULE=1 instead launches the
    // memory-bound kernels first on a small grid (co_grid CTAs/SM) -- measured slower
    // (41.3k), kept as an option for other mixes.
    auto tensor_chunk = [&](const Chunk& ch) {
        return (ch.kernel == K_SGEMM_TF32 || ch.kernel == K_SGEMM) && ch.sgemm_impl != SVP_SGEMM_FFMA &&
               ch.sgemm_impl != kSgemmPlain;
    };
    auto device_only = [&](const Chunk& ch) { return ch.t_in == 0 && ch.t_out == 0; };
    std::stable_sort(corder.begin(), corder.end(), [&](int32_t x, int32_t y) {
        const Chunk &a = f->chunks[x], &b = f->chunks[y];
        if (a.level != b.level) return a.level < b.level;
        if (!inter) return std::tie(a.group, a.index) < std::tie(b.group, b.index);
        const bool da = device_only(a), db = device_only(b);
        if (da != db) return da;  // device-only chunks first; copies are on their own streams
        if (da && c->coschedule) {
            const bool ta = tensor_chunk(a), tb = tensor_chunk(b);
            if (ta != tb) return !ta;
            return std::make_tuple(-a.t_k, a.group, a.index) < std::make_tuple(-b.t_k, b.group, b.index);
        }
        return johnson_key(x) < johnson_key(y);
    });
    if (inter && c->coschedule) {
        // co_grid for memory-bound device-only chunks sharing a (level, device) with a
        // tensor-core SGEMM chunk (hist256 keeps its default grid: it needs shared memory)
        std::map<std::pair<int32_t, int32_t>, bool> has_tensor;
        for (const auto& ch : f->chunks)
            if (device_only(ch) && tensor_chunk(ch)) has_tensor[{ch.level, ch.device}] = true;
        for (auto& ch : f->chunks) {
            if (!device_only(ch) || !has_tensor.count({ch.level, ch.device})) continue;
            if (ch.kernel == K_VECADD || ch.kernel == K_SAXPY || ch.kernel == K_EW_MIX) ch.co_grid = 2;
            else if (ch.kernel == K_BLACKSCHOLES) ch.co_grid = 3;
        }
    }

    // ---- ops, streams, dependencies, arena slots
    VpSlots vp_last_op(f->jobs, -1);                       // per VP: last op of its previous job
    struct Slot { uint64_t off, len; int32_t release_op; };
    std::vector<std::vector<Slot>> inflight(c->ngpu);
    std::vector<uint64_t> arena_head(c->ngpu, 0);
    std::vector<int32_t> rr(c->ngpu, 0);
    // compute stream of a chunk: the one with the least estimated kernel time queued so far
    // (list scheduling; ties -> lowest index).  Round-robin put cfg5's 5th launch (hist256)
    // behind the SGEMM on stream 0, so it ran alone after it.  SVP_STREAM_RR=1: round-robin.
    static const bool stream_rr = getenv("SVP_STREAM_RR") && atoi(getenv("SVP_STREAM_RR")) != 0;
    std::vector<std::vector<double>> sload(c->ngpu, std::vector<double>(S, 0.0));
    for (int32_t ci : corder) {
        Chunk& ch = f->chunks[ci];
        const int dev = ch.device;
        std::vector<int32_t> prev;
        for (int32_t ji : ch.jobs) {
            const int32_t lo = vp_last_op[f->jobs[ji].vp];
            if (lo >= 0) prev.push_back(lo);
        }
        // arena slot (ring) -- the chunk's first arena op waits for the release (last op) of
        // every in-flight slot overlapping [off, off + len).  The part of an old slot this
        // chunk covers is then guarded by this chunk's own release (which follows its first
        // op, which waited); the parts it does NOT cover keep the old slot's release, so a
        // later chunk placed there still waits for it (dropping the whole slot here let such
        // a chunk -- e.g. one whose first op is its kernel, not an H2D on the shared copy
        // stream -- overwrite staging another chunk was still using).
        std::vector<int32_t> arena_waits;
        if (ch.arena_len) {
            uint64_t off = arena_head[dev];
            if (off + ch.arena_len > arena) off = 0;
            const uint64_t lo = off, hi = off + ch.arena_len;
            auto& fl = inflight[dev];
            std::vector<Slot> keep;
            keep.reserve(fl.size() + 2);
            for (const Slot& s : fl) {
                const uint64_t se = s.off + s.len;
                if (s.off < hi && lo < se) {
                    if (std::find(arena_waits.begin(), arena_waits.end(), s.release_op) == arena_waits.end())
                        arena_waits.push_back(s.release_op);
                    if (s.off < lo) keep.push_back(Slot{s.off, lo - s.off, s.release_op});
                    if (se > hi) keep.push_back(Slot{hi, se - hi, s.release_op});
                } else {
                    keep.push_back(s);
                }
            }
            fl.swap(keep);
            ch.arena_off = off;
            arena_head[dev] = off + ch.arena_len;
        }
        int cs = 0;
        if (inter) {
            if (stream_rr) {
                cs = rr[dev]++ % S;
            } else {
                for (int k = 1; k < S; ++k)
                    if (sload[dev][k] < sload[dev][cs]) cs = k;
                sload[dev][cs] += std::max(ch.t_k, 1.0);
            }
        }
        int sh2d = inter ? S : 0, sd2h = inter ? S + 1 : 0;
        int32_t first_op = (int32_t)f->ops.size();
        int32_t k_op = -1, last = -1;
        if (ch.in_bytes) {
            Op o;
            o.kind = SVP_OP_H2D;
            o.chunk = ci;
            o.device = dev;
            o.stream = sh2d;
            o.wait_ops = prev;
            o.wait_ops.insert(o.wait_ops.end(), arena_waits.begin(), arena_waits.end());
            o.est_ns = ch.t_in;
            o.bytes = ch.in_bytes;
            f->ops.push_back(o);
            last = (int32_t)f->ops.size() - 1;
        }
        {
            Op o;
            o.kind = SVP_OP_KERNEL;
            o.chunk = ci;
            o.device = dev;
            o.stream = cs;
            if (last >= 0) o.wait_ops.push_back(last);
            else {
                o.wait_ops = prev;
                o.wait_ops.insert(o.wait_ops.end(), arena_waits.begin(), arena_waits.end());
            }
            o.est_ns = ch.t_k;
            o.bytes = (uint64_t)ch.alg_bytes;
            o.flops = ch.flops;
            f->ops.push_back(o);
            last = k_op = (int32_t)f->ops.size() - 1;
        }
        if (ch.out_bytes) {
            Op o;
            o.kind = SVP_OP_D2H;
            o.chunk = ci;
            o.device = dev;
            o.stream = sd2h;
            o.wait_ops.push_back(k_op);
            o.est_ns = ch.t_out;
            o.bytes = ch.out_bytes;
            f->ops.push_back(o);
            last = (int32_t)f->ops.size() - 1;
        }
        (void)first_op;
        f->ops[last].last_of_job = true;
        for (int32_t ji : ch.jobs) vp_last_op[f->jobs[ji].vp] = last;
        if (ch.arena_len) inflight[dev].push_back(Slot{ch.arena_off, ch.arena_len, last});
    }
    // dependencies on the same stream that precede in issue order are implicit; keep
    // only cross-stream waits, and mark the ops somebody waits on
    for (size_t i = 0; i < f->ops.size(); ++i) {
        Op& o = f->ops[i];
        std::vector<int32_t> w;
        for (int32_t p : o.wait_ops) {
            if (p < 0 || p >= (int32_t)i) continue;
            const Op& q = f->ops[p];
            if (q.device == o.device && q.stream == o.stream) continue;
            if (std::find(w.begin(), w.end(), p) == w.end()) w.push_back(p);
        }
        o.wait_ops.swap(w);
        for (int32_t p : o.wait_ops) f->ops[p].needs_event = true;
    }
    return SVP_OK;
}

// ------------------------------------------------------------------ plan simulation
// Engines per GPU (Fig 3): H2D copy engine, D2H copy engine, compute engine (coalesced
// kernels that fill the GPU serialize).  An op starts when its engine, its stream and
// every op it waits on are free.
void simulate(Ctx* c, Flush* f, double* makespan, double* serial) {
    const int S = c->cfg.streams_per_gpu + 2;
    std::vector<double> eng(c->ngpu * 3, 0.0), strm(c->ngpu * S, 0.0);
    double ms = 0, ser = 0;
    for (auto& o : f->ops) {
        int e = o.device * 3 + (o.kind == SVP_OP_H2D ? 0 : o.kind == SVP_OP_KERNEL ? 1 : 2);
        double t = std::max(eng[e], strm[o.device * S + o.stream]);
        for (int32_t p : o.wait_ops) t = std::max(t, f->ops[p].sim_end);
        o.sim_start = t;
        o.sim_end = t + o.est_ns;
        eng[e] = strm[o.device * S + o.stream] = o.sim_end;
        ms = std::max(ms, o.sim_end);
        ser += o.est_ns;
    }
    // same-stream predecessors implicitly ordered (already via strm); done
    *makespan = ms;
    *serial = ser;
}

}  // namespace svp

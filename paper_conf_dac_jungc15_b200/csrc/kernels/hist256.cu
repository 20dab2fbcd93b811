// hist256.cu -- coalesced 256-bin byte histogram for sm_100a.
//
// counts_v[b] = #{i : d_v[i] == b} for every VP v of the group, in one launch.
//
// A histogram needs one increment per input byte; done with shared-memory atomics that
// caps the kernel at the measured smem-atomic rate (tools/ubench.py: ~3.7e12 lanes/s =
// 3.7 TB/s of input, ~56 % of HBM), so the design goal is to keep the atomics busy and
// never let them wait on DRAM:
//  * a producer warp streams each tile global -> shared with 1-D bulk copies
//    (cp.async.bulk, mbarrier complete_tx) into a 3-stage ring, so DRAM latency is hidden
//    behind the consumers' atomics;
//  * 8 consumer warps read the staged tile (LDS.128, conflict-free) and increment a CTA
//    histogram replicated per lane -- h[bin][lane], 256 x 32 u32 = 32 KiB -- so the 32
//    addresses of every warp ATOMS sit in 32 distinct banks whatever the data: one smem
//    wavefront per instruction.  (Packing two 16-bit bins per word halves the table but
//    costs instructions: 2.5 vs 3.7 Tlanes/s measured.)  A warp whose batch is skewed
//    (>= 12 of its 32 lanes start on lane 0's byte) counts that batch into one shared
//    256-bin table instead, where same-byte lanes hit one word and ATOMS aggregates them:
//    5.06 vs 3.78 TB/s on 90 %-one-value data, 2.5 vs 3.78 on uniform data
//    (tools/hist_schemes.py, profiles/r02/hist_schemes.json -- the ceiling table of the
//    counting schemes, incl. __match_any_sync aggregation and private LDS/STS counters).
//  * CTAs walk contiguous (blocked) tile ranges, so a CTA stays in one VP for many tiles
//    (segment lookups are cached) and flushes its replicas to the VP's global counts
//    (one atomicAdd per non-zero bin) only at VP boundaries.
// A VP's ragged head/tail tiles (not 16-B aligned / partial) go through the ring too: the
// producer bulk-copies their 16-B-aligned interior, and the consumers read the < 16-B ends
// from global memory (byte loads of whole ragged tiles had made a CTA holding one ~8x
// slower than its neighbours: cfg5's hist launch ran at 65 % SM-active, ncu).  A preceding tiny kernel zeroes every segment's counts, so the result
// overwrites the output and is bit-exact (integer adds commute).  With a per-launch
// scratch (the executor's default) there is no zeroing kernel: the last CTA of each VP
// writes its counts (hist_flush_fused).
#include <string.h>

#include <atomic>

#include "../launch.h"
#include "common.cuh"

namespace svp {

constexpr int kHistConsumers = kHistThreads;          // 256 = 8 warps
constexpr int kHistBlock = kHistConsumers + 32;       // + producer warp
constexpr int kHistStages = 3;
constexpr int kHistBins = 256;
constexpr int kHistSmem = kHistStages * kHistTile + kHistBins * 33 * 4 + 2 * kHistStages * 8 + 128;
// a warp whose 32 lanes' first bytes agree with lane 0's in at least this many lanes counts
// its batch into the shared (non-replicated) table h1
constexpr int kHistSkewLanes = 12;

__device__ __forceinline__ void hist_zero_body(const SegDesc* __restrict__ segs, int nsegs) {
    for (int s = blockIdx.x; s < nsegs; s += gridDim.x) {
        uint32_t* counts = reinterpret_cast<uint32_t*>(segs[s].ptr[1]);
        counts[threadIdx.x] = 0u;
    }
}
__global__ void __launch_bounds__(256) k_hist_zero(const SegDesc* __restrict__ segs, int nsegs) {
    hist_zero_body(segs, nsegs);
}
template <int CAP>
__global__ void __launch_bounds__(256) k_hist_zero_p(const __grid_constant__ SegParamT<CAP> p, int nsegs) {
    hist_zero_body(p.s, nsegs);
}

__device__ __forceinline__ void consumers_sync() { asm volatile("bar.sync 1, %0;" ::"n"(kHistConsumers) : "memory"); }

__device__ __forceinline__ void bulk_g2s(void* smem_dst, const void* gsrc, uint32_t bytes, uint64_t* bar) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
            smem_u32(smem_dst)),
        "l"(gsrc), "r"(bytes), "r"(smem_u32(bar))
        : "memory");
}

// hl points at column `lane` of bin 0: hl[b * 32] is this lane's counter for bin b.
__device__ __forceinline__ void hist_add_byte(uint32_t* hl, uint32_t b) { atomicAdd(hl + (b << 5), 1u); }
__device__ __forceinline__ void hist_add_word(uint32_t* hl, uint32_t w) {
    hist_add_byte(hl, w & 0xFFu);
    hist_add_byte(hl, (w >> 8) & 0xFFu);
    hist_add_byte(hl, (w >> 16) & 0xFFu);
    hist_add_byte(hl, w >> 24);
}
// Skewed batches (round 2, profiles/r02/hist_schemes.json): ONE shared 256-bin table h1.
// Lanes holding the same byte hit the same word, which ATOMS.POPC.INC aggregates into one
// update -- on 90 %-one-value data this ran at 5.06 TB/s against 3.78 for the per-lane
// replicas (on uniform data the shared table's bank conflicts make it 2.5 TB/s, so each
// warp picks per batch).
__device__ __forceinline__ void hist_add_word_shared(uint32_t* h1, uint32_t w) {
    atomicAdd(h1 + (w & 0xFFu), 1u);
    atomicAdd(h1 + ((w >> 8) & 0xFFu), 1u);
    atomicAdd(h1 + ((w >> 16) & 0xFFu), 1u);
    atomicAdd(h1 + (w >> 24), 1u);
}

// Sum the 32 lane replicas of each bin (thread t owns bin t; the column walk is rotated
// by t so a warp's 32 reads hit 32 banks), zero them, and add to the VP's counts.
// Consumers only (named barrier 1).
__device__ __forceinline__ void hist_flush(uint32_t* h, uint32_t* counts) {
    static_assert(kHistConsumers == kHistBins, "one flush thread per bin");
    consumers_sync();
    const int b = threadIdx.x;
    uint32_t* h1 = h + kHistBins * 32;  // the shared table follows the replicas
    uint32_t sum = h1[b];
    h1[b] = 0;
#pragma unroll 8
    for (int j = 0; j < 32; ++j) {
        const int c = (j + b) & 31;
        sum += h[b * 32 + c];
        h[b * 32 + c] = 0;
    }
    if (sum) atomicAdd(&counts[b], sum);
    consumers_sync();
}

// Single-launch form (`scratch` non-null, no zeroing kernel): the CTAs that touch VP `si`
// add their sums into a per-launch partial histogram scratch[si][256], then count in
// scratch arrive[si]; the last of the VP's expected CTAs (known from the blocked tile
// ranges) moves the partial histogram into the VP's counts with plain stores -- the
// output is overwritten, never accumulated -- and leaves the scratch zeroed for the next
// launch on the same slot (threadfence-reduction pattern).
__device__ __forceinline__ uint32_t hist_expected_ctas(const SegDesc* __restrict__ segs, int nsegs, uint32_t total,
                                                       uint32_t per, int si) {
    const uint32_t tb = segs[si].tile_begin, te = si + 1 < nsegs ? segs[si + 1].tile_begin : total;
    return (te - 1) / per - tb / per + 1;
}
__device__ __forceinline__ void hist_flush_fused(uint32_t* h, uint32_t* counts, uint32_t* partial, uint32_t* arrive,
                                                 uint32_t expected, uint32_t* last_flag) {
    consumers_sync();
    const int b = threadIdx.x;
    uint32_t* h1 = h + kHistBins * 32;
    uint32_t sum = h1[b];
    h1[b] = 0;
#pragma unroll 8
    for (int j = 0; j < 32; ++j) {
        const int c = (j + b) & 31;
        sum += h[b * 32 + c];
        h[b * 32 + c] = 0;
    }
    if (sum) atomicAdd(&partial[b], sum);
    __threadfence();
    consumers_sync();
    if (b == 0) *last_flag = atomicAdd(arrive, 1u) == expected - 1;
    consumers_sync();
    if (*last_flag) {
        __threadfence();
        counts[b] = atomicExch(&partial[b], 0u);
        if (b == 0) *arrive = 0;
    }
    consumers_sync();
}

// [a, b): the 16-B-aligned interior (in element = byte indices) of the byte range [e0, e1)
// of the buffer at `base`; b <= a when the range holds no aligned 16-B block.
__device__ __forceinline__ void aligned_interior(uint64_t base, int64_t e0, int64_t e1, int64_t& a, int64_t& b) {
    a = (int64_t)(((base + (uint64_t)e0 + 15) & ~15ull) - base);
    b = (int64_t)(((base + (uint64_t)e1) & ~15ull) - base);
}

// Segment of tile t with a one-entry cache (tiles of a CTA are contiguous): [lo, hi) is
// the tile range the cached segment owns.
struct SegCache {
    int si = -1;
    uint32_t lo = 1, hi = 0;
    __device__ __forceinline__ int get(const SegDesc* __restrict__ segs, int nsegs, uint32_t total, uint32_t t) {
        if (t < lo || t >= hi) {
            si = find_seg(segs, nsegs, t);
            lo = segs[si].tile_begin;
            hi = si + 1 < nsegs ? segs[si + 1].tile_begin : total;
        }
        return si;
    }
};

// Dynamic tile order (sched != null; not with the single-launch scratch form): the producer
// claims chunks of kHistChunk consecutive tiles from the launch's self-resetting counter pair
// sched[0..1] and tells the consumers each staged tile's id through stile[stage]; a CTA whose
// data runs slower (uniform bytes: one ATOMS per byte into the replicas) takes fewer chunks
// than one whose data is skewed (the aggregated shared table is ~1.3x faster), instead of
// every CTA owning a fixed 1/grid of the tiles.
constexpr uint32_t kHistChunk = 8;
constexpr uint32_t kHistEnd = 0xFFFFFFFFu;

__device__ __forceinline__ void hist_body(const SegDesc* __restrict__ segs, int nsegs, uint32_t total,
                                          unsigned long long* __restrict__ busy, uint32_t* __restrict__ scratch,
                                          uint32_t* __restrict__ sched) {
    extern __shared__ __align__(128) uint8_t hsm[];
    uint8_t* ring = hsm;                                                         // [stages][tile]
    uint32_t* h = reinterpret_cast<uint32_t*>(hsm + kHistStages * kHistTile);     // [256][32] + h1[256]
    uint32_t* h1 = h + kHistBins * 32;
    uint64_t* full = reinterpret_cast<uint64_t*>(h + kHistBins * 33);
    uint64_t* empty = full + kHistStages;
    __shared__ uint32_t last_flag;
    __shared__ uint32_t stile[kHistStages];  // dynamic order: tile id of each stage
    const bool dyn = sched != nullptr && scratch == nullptr;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    uint32_t* arrive = scratch ? scratch + (size_t)nsegs * kHistBins : nullptr;
    if (scratch) {
        // single-launch form: VPs without input still get their counts overwritten with 0
        for (int si = blockIdx.x; si < nsegs; si += gridDim.x)
            if (segs[si].n == 0 && threadIdx.x < kHistBins) reinterpret_cast<uint32_t*>(segs[si].ptr[1])[threadIdx.x] = 0u;
    }

    for (int i = threadIdx.x; i < kHistBins * 33; i += kHistBlock) h[i] = 0;
    if (threadIdx.x == 0) {
        for (int s = 0; s < kHistStages; ++s) {
            mbar_init(&full[s], 1);
            mbar_init(&empty[s], kHistConsumers / 32);
        }
        mbar_fence_init();
    }
    __syncthreads();

    // blocked tile ranges
    const uint32_t per = (total + gridDim.x - 1) / gridDim.x;
    const uint32_t t0 = min(total, blockIdx.x * per), t1 = min(total, t0 + per);

    if (warp == kHistConsumers / 32) {
        // ------------------------------------------------------------ producer
        if (lane == 0) {
            uint32_t it = 0;
            SegCache sc;
            uint32_t t = t0, tend = t1, next = 0;
            if (dyn) {
                const uint32_t c = atomicAdd(sched, 1u);
                next = atomicAdd(sched, 1u);  // claimed one chunk ahead: its latency hides
                t = min(total, c * kHistChunk);
                tend = min(total, t + kHistChunk);
            }
            for (;; ++t, ++it) {
                if (t >= tend) {
                    if (!dyn || t >= total) break;
                    t = min(total, next * kHistChunk);
                    tend = min(total, t + kHistChunk);
                    if (t >= tend) break;
                    next = atomicAdd(sched, 1u);
                }
                const int s = it % kHistStages;
                const uint32_t ph = (it / kHistStages) & 1;
                const SegDesc& sd = segs[sc.get(segs, nsegs, total, t)];
                int64_t e0, e1;
                bool vec;
                tile_range(sd.n, sd.shift, sd.flags, t - sd.tile_begin, kHistTile, e0, e1, vec);
                mbar_wait(&empty[s], ph ^ 1);
                stile[s] = t;  // published by the arrive below (release) to the consumers' wait
                if (vec) {
                    mbar_expect_tx(&full[s], kHistTile);
                    bulk_g2s(ring + s * kHistTile, reinterpret_cast<const uint8_t*>(sd.ptr[0]) + e0, kHistTile, &full[s]);
                } else {
                    // ragged head/tail tile: bulk-copy its 16-B-aligned interior too; the
                    // consumers read the < 16-B ends from global memory
                    int64_t a, b;
                    aligned_interior(sd.ptr[0], e0, e1, a, b);
                    if (b > a) {
                        mbar_expect_tx(&full[s], (uint32_t)(b - a));
                        bulk_g2s(ring + s * kHistTile, reinterpret_cast<const uint8_t*>(sd.ptr[0]) + a, (uint32_t)(b - a),
                                 &full[s]);
                    } else {
                        mbar_arrive(&full[s]);  // < 32 B: consumers read it from global memory
                    }
                }
            }
            if (dyn) {  // end marker: one more stage carrying no tile
                const int s = it % kHistStages;
                const uint32_t ph = (it / kHistStages) & 1;
                mbar_wait(&empty[s], ph ^ 1);
                stile[s] = kHistEnd;
                mbar_arrive(&full[s]);
            }
        }
        return;  // no CTA-wide barrier after this point
    }

    // ---------------------------------------------------------------- consumers
    uint32_t* hl = h + lane;
    int cur = -1;
    uint32_t* cur_counts = nullptr;
    uint32_t it = 0;
    SegCache sc;
    for (uint32_t t = t0;; ++t, ++it) {
        const int s = it % kHistStages;
        const uint32_t ph = (it / kHistStages) & 1;
        // profile_level 2: thread 0's cycles per tile (from the wait for the stage to the
        // release) -> busy[segment]
        const long long c0 = (busy && threadIdx.x == 0) ? clock64() : 0;
        if (dyn) {
            mbar_wait(&full[s], ph);
            t = stile[s];
            if (t == kHistEnd) break;
        } else {
            if (t >= t1) break;
            mbar_wait(&full[s], ph);
        }
        const int si = sc.get(segs, nsegs, total, t);
        const SegDesc& sd = segs[si];
        if (si != cur) {
            if (cur >= 0) {
                if (scratch)
                    hist_flush_fused(h, cur_counts, scratch + (size_t)cur * kHistBins, arrive + cur,
                                     hist_expected_ctas(segs, nsegs, total, per, cur), &last_flag);
                else
                    hist_flush(h, cur_counts);
            }
            cur = si;
            cur_counts = reinterpret_cast<uint32_t*>(sd.ptr[1]);
        }
        int64_t e0, e1;
        bool vec;
        tile_range(sd.n, sd.shift, sd.flags, t - sd.tile_begin, kHistTile, e0, e1, vec);
        if (vec) {
            const uint4* st = reinterpret_cast<const uint4*>(ring + s * kHistTile) + threadIdx.x;
            uint4 r[kHistVec];
#pragma unroll
            for (int i = 0; i < kHistVec; ++i) r[i] = st[i * kHistConsumers];
            // per-warp choice of table for this batch (warp-uniform: no divergence)
            const uint32_t b0 = r[0].x & 0xFFu;
            const uint32_t hot = __shfl_sync(0xFFFFFFFFu, b0, 0);
            if (__popc(__ballot_sync(0xFFFFFFFFu, b0 == hot)) >= kHistSkewLanes) {
#pragma unroll
                for (int i = 0; i < kHistVec; ++i) {
                    hist_add_word_shared(h1, r[i].x);
                    hist_add_word_shared(h1, r[i].y);
                    hist_add_word_shared(h1, r[i].z);
                    hist_add_word_shared(h1, r[i].w);
                }
            } else {
#pragma unroll
                for (int i = 0; i < kHistVec; ++i) {
                    hist_add_word(hl, r[i].x);
                    hist_add_word(hl, r[i].y);
                    hist_add_word(hl, r[i].z);
                    hist_add_word(hl, r[i].w);
                }
            }
            // Release the stage only after every loaded word was consumed: the mbarrier
            // arrive (SYNCS unit) does not wait for this warp's outstanding LDS, so an
            // arrive issued right after them let the producer's next bulk copy overwrite
            // bytes not yet read (wrong-but-conserved counts under heavy co-scheduling).
            __syncwarp();
            if (lane == 0) mbar_arrive(&empty[s]);
        } else {
            // ragged head/tail tile: aligned interior from the stage, the ends (< 16 B each,
            // or the whole tile when it holds no aligned 16 B) from global memory
            const uint8_t* __restrict__ d = reinterpret_cast<const uint8_t*>(sd.ptr[0]);
            int64_t a, b;
            aligned_interior(sd.ptr[0], e0, e1, a, b);
            if (b > a) {
                const uint4* st = reinterpret_cast<const uint4*>(ring + s * kHistTile);
                const int nv = (int)((b - a) >> 4);
                for (int i = threadIdx.x; i < nv; i += kHistConsumers) {
                    const uint4 r = st[i];
                    hist_add_word(hl, r.x);
                    hist_add_word(hl, r.y);
                    hist_add_word(hl, r.z);
                    hist_add_word(hl, r.w);
                }
                const int th = threadIdx.x;
                if (th < 16) {
                    if (e0 + th < a) hist_add_byte(hl, d[e0 + th]);
                } else if (th < 32) {
                    if (b + (th - 16) < e1) hist_add_byte(hl, d[b + (th - 16)]);
                }
            } else {
                for (int64_t e = e0 + threadIdx.x; e < e1; e += kHistConsumers) hist_add_byte(hl, d[e]);
            }
            // release after the stage was consumed (see the vec path)
            __syncwarp();
            if (lane == 0) mbar_arrive(&empty[s]);
        }
        if (busy && threadIdx.x == 0) atomicAdd(busy + si, (unsigned long long)(clock64() - c0));
    }
    if (cur >= 0) {
        if (scratch)
            hist_flush_fused(h, cur_counts, scratch + (size_t)cur * kHistBins, arrive + cur,
                             hist_expected_ctas(segs, nsegs, total, per, cur), &last_flag);
        else
            hist_flush(h, cur_counts);
    }
    // dynamic order: the last CTA out (every producer has claimed past the end by then)
    // leaves the counter pair zeroed for the next launch on this slot
    if (dyn && threadIdx.x == 0 && atomicAdd(sched + 1, 1u) == gridDim.x - 1) {
        sched[0] = 0;
        sched[1] = 0;
    }
}

__global__ void __launch_bounds__(kHistBlock) k_hist256(const SegDesc* __restrict__ segs, int nsegs, uint32_t total,
                                                        unsigned long long* busy, uint32_t* scratch, uint32_t* sched) {
    hist_body(segs, nsegs, total, busy, scratch, sched);
}
template <int CAP>
__global__ void __launch_bounds__(kHistBlock) k_hist256_p(const __grid_constant__ SegParamT<CAP> p, int nsegs,
                                                          uint32_t total, unsigned long long* busy,
                                                          uint32_t* scratch, uint32_t* sched) {
    hist_body(p.s, nsegs, total, busy, scratch, sched);
}

template <int CAP>
static cudaError_t hist_attr_p() {
    static std::atomic<bool> attr[64] = {};  // per device; worker threads of several GPUs launch
    int dev = 0;
    cudaGetDevice(&dev);
    if (dev < 64 && !attr[dev]) {
        cudaError_t e = cudaFuncSetAttribute(k_hist256_p<CAP>, cudaFuncAttributeMaxDynamicSharedMemorySize, kHistSmem);
        if (e) return e;
        attr[dev] = true;
    }
    return cudaSuccess;
}

static cudaError_t hist_attr() {
    static std::atomic<bool> attr[64] = {};  // per device; worker threads of several GPUs launch
    int dev = 0;
    cudaGetDevice(&dev);
    if (dev < 64 && !attr[dev]) {
        cudaError_t e = cudaFuncSetAttribute(k_hist256, cudaFuncAttributeMaxDynamicSharedMemorySize, kHistSmem);
        if (e) return e;
        attr[dev] = true;
    }
    return cudaSuccess;
}

cudaError_t launch_hist256(const SegDesc* segs, int nsegs, uint32_t total, int grid, cudaStream_t s, uint64_t* busy,
                           uint32_t* scratch, uint32_t* sched) {
    if (nsegs <= 0) return cudaSuccess;
    cudaError_t e;
    if (!scratch) {
        k_hist_zero<<<nsegs < 1024 ? nsegs : 1024, 256, 0, s>>>(segs, nsegs);
        e = cudaGetLastError();
        if (e || total == 0) return e;
    }
    if ((e = hist_attr())) return e;
    k_hist256<<<grid, kHistBlock, kHistSmem, s>>>(segs, nsegs, total, reinterpret_cast<unsigned long long*>(busy),
                                                  scratch, sched);
    return cudaGetLastError();
}

template <int CAP>
static cudaError_t launch_hist256_param_cap(const SegDesc* segs, int nsegs, uint32_t total, int grid,
                                            cudaStream_t s, uint64_t* busy, uint32_t* scratch, uint32_t* sched) {
    SegParamT<CAP> p;
    memcpy(p.s, segs, (size_t)nsegs * sizeof(SegDesc));
    cudaError_t e;
    if (!scratch) {
        k_hist_zero_p<CAP><<<nsegs, 256, 0, s>>>(p, nsegs);
        e = cudaGetLastError();
        if (e || total == 0) return e;
    }
    if ((e = hist_attr_p<CAP>())) return e;
    k_hist256_p<CAP><<<grid, kHistBlock, kHistSmem, s>>>(p, nsegs, total, reinterpret_cast<unsigned long long*>(busy),
                                                         scratch, sched);
    return cudaGetLastError();
}

cudaError_t launch_hist256_param(const SegDesc* segs, int nsegs, uint32_t total, int grid, cudaStream_t s,
                                 uint64_t* busy, uint32_t* scratch, uint32_t* sched) {
    if (nsegs <= 0) return cudaSuccess;
    if (param_full_block() && nsegs <= kParamSegs)
        return launch_hist256_param_cap<kParamSegs>(segs, nsegs, total, grid, s, busy, scratch, sched);
    if (nsegs <= 16) return launch_hist256_param_cap<16>(segs, nsegs, total, grid, s, busy, scratch, sched);
    if (nsegs <= kParamSegs)
        return launch_hist256_param_cap<kParamSegs>(segs, nsegs, total, grid, s, busy, scratch, sched);
    return cudaErrorInvalidValue;
}

cudaError_t query_limits_hist(int* per_sm) {
    cudaError_t e = cudaFuncSetAttribute(k_hist256, cudaFuncAttributeMaxDynamicSharedMemorySize, kHistSmem);
    if (e) return e;
    return cudaOccupancyMaxActiveBlocksPerMultiprocessor(per_sm, k_hist256, kHistBlock, kHistSmem);
}

}  // namespace svp

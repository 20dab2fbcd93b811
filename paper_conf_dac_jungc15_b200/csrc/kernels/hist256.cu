// hist256.cu -- coalesced 256-bin byte histogram for sm_100a.
//
// counts_v[b] = #{i : d_v[i] == b} for every VP v of the group, in one launch.
// Each tile lies in one VP.  A CTA keeps ONE shared histogram replicated per lane
// (lane l of every warp increments column l, two 16-bit bins per 32-bit word), so the 32
// addresses of a warp instruction sit in 32 distinct banks whatever the data (uniform
// or 90 % one value): one smem wavefront per ATOMS, no same-address serialisation
// inside an instruction.  One smem atomic per byte caps this kernel at the measured
// shared-atomic rate (tools/ubench.py: ~3.7e12 lanes/s = 3.7 TB/s of input bytes).  The CTA flushes the replicas to
// the VP's global counts (one atomicAdd per non-zero bin) whenever it moves to another
// VP; a preceding tiny kernel zeroes every segment's counts, so the result overwrites
// the output and is bit-exact (integer adds commute).
#include "../launch.h"
#include "common.cuh"

namespace svp {

__global__ void __launch_bounds__(256) k_hist_zero(const SegDesc* __restrict__ segs, int nsegs) {
    for (int s = blockIdx.x; s < nsegs; s += gridDim.x) {
        uint32_t* counts = reinterpret_cast<uint32_t*>(segs[s].ptr[1]);
        counts[threadIdx.x] = 0u;
    }
}

// Shared table h[word][lane], word = bin & 127, 16-bit half = bin >> 7: 128 x 32 u32 =
// 16 KiB per CTA, so 8 CTAs (2048 threads) fit an SM and keep enough loads in flight.
// hl points at column `lane` of word 0.  A half-counter gains at most 8 warps x
// kHistVec x 16 increments per tile, so flushing every kHistFlushTiles tiles keeps it
// below 2^16.
constexpr int kHistWords = 128;
constexpr int kHistFlushTiles = 32;
static_assert(kHistFlushTiles * (kHistThreads / 32) * kHistVec * 16 < 65536, "16-bit half-counters overflow");

__device__ __forceinline__ void hist_add_byte(uint32_t* hl, uint32_t b) {
    atomicAdd(hl + ((b & 127u) << 5), 1u << ((b >> 7) << 4));
}
__device__ __forceinline__ void hist_add_word(uint32_t* hl, uint32_t w) {
    hist_add_byte(hl, w & 0xFFu);
    hist_add_byte(hl, (w >> 8) & 0xFFu);
    hist_add_byte(hl, (w >> 16) & 0xFFu);
    hist_add_byte(hl, w >> 24);
}

// Sum the 32 lane replicas of each word (thread t < 128 owns word t; the column walk is
// rotated by t so a warp's 32 reads hit 32 banks), zero them, and add both halves to the
// VP's counts (bins t and t + 128).
__device__ __forceinline__ void hist_flush(uint32_t* h, uint32_t* counts) {
    __syncthreads();
    const int w = threadIdx.x;
    if (w < kHistWords) {
        uint32_t lo = 0, hi = 0;
#pragma unroll 8
        for (int j = 0; j < 32; ++j) {
            const int c = (j + w) & 31;
            const uint32_t v = h[w * 32 + c];
            lo += v & 0xFFFFu;
            hi += v >> 16;
            h[w * 32 + c] = 0;
        }
        if (lo) atomicAdd(&counts[w], lo);
        if (hi) atomicAdd(&counts[w + 128], hi);
    }
    __syncthreads();
}

__global__ void __launch_bounds__(kHistThreads) k_hist256(const SegDesc* __restrict__ segs, int nsegs, uint32_t total) {
    __shared__ uint32_t h[kHistWords * 32];
    for (int i = threadIdx.x; i < kHistWords * 32; i += kHistThreads) h[i] = 0;
    __syncthreads();
    uint32_t* hl = h + (threadIdx.x & 31);
    int cur = -1, since_flush = 0;
    uint32_t* cur_counts = nullptr;
    // blocked tile ranges: a CTA walks contiguous tiles, so it stays inside one VP for
    // many tiles and flushes only at VP boundaries (or every kHistFlushTiles tiles)
    const uint32_t per = (total + gridDim.x - 1) / gridDim.x;
    const uint32_t t0 = blockIdx.x * per, t1 = min(total, t0 + per);
    for (uint32_t t = t0; t < t1; ++t) {
        const int si = find_seg(segs, nsegs, t);
        const SegDesc& sd = segs[si];
        if (si != cur || since_flush == kHistFlushTiles) {
            if (cur >= 0) hist_flush(h, cur_counts);
            cur = si;
            since_flush = 0;
            cur_counts = reinterpret_cast<uint32_t*>(sd.ptr[1]);
        }
        ++since_flush;
        const uint8_t* __restrict__ d = reinterpret_cast<const uint8_t*>(sd.ptr[0]);
        int64_t e0, e1;
        bool vec;
        tile_range(sd.n, sd.shift, sd.flags, t - sd.tile_begin, kHistTile, e0, e1, vec);
        if (vec) {
            const uint4* d4 = reinterpret_cast<const uint4*>(d + e0) + threadIdx.x;
            uint4 r[kHistVec];
#pragma unroll
            for (int i = 0; i < kHistVec; ++i) r[i] = __ldcs(d4 + i * kHistThreads);
#pragma unroll
            for (int i = 0; i < kHistVec; ++i) {
                hist_add_word(hl, r[i].x);
                hist_add_word(hl, r[i].y);
                hist_add_word(hl, r[i].z);
                hist_add_word(hl, r[i].w);
            }
        } else {
            for (int64_t e = e0 + threadIdx.x; e < e1; e += kHistThreads) hist_add_byte(hl, d[e]);
        }
    }
    if (cur >= 0) hist_flush(h, cur_counts);
}

constexpr int kHistSmem = 0;  // static shared table

cudaError_t launch_hist256(const SegDesc* segs, int nsegs, uint32_t total, int grid, cudaStream_t s) {
    if (nsegs <= 0) return cudaSuccess;
    k_hist_zero<<<nsegs < 1024 ? nsegs : 1024, 256, 0, s>>>(segs, nsegs);
    cudaError_t e = cudaGetLastError();
    if (e || total == 0) return e;
    k_hist256<<<grid, kHistThreads, kHistSmem, s>>>(segs, nsegs, total);
    return cudaGetLastError();
}

cudaError_t query_limits_hist(int* per_sm) {
    return cudaOccupancyMaxActiveBlocksPerMultiprocessor(per_sm, k_hist256, kHistThreads, kHistSmem);
}

}  // namespace svp

// hist256.cu -- coalesced 256-bin byte histogram for sm_100a.
//
// counts_v[b] = #{i : d_v[i] == b} for every VP v of the group, in one launch.
// Each tile lies in one VP.  A CTA keeps ONE shared histogram replicated per lane:
// h[bin][lane] (256 x 32 u32 = 32 KiB), and lane l of every warp increments column l.
// Within a warp instruction the 32 addresses therefore sit in 32 distinct banks
// whatever the data (uniform or 90 % one value): one smem wavefront per ATOMS, no
// same-address serialisation inside an instruction.  The CTA flushes the replicas to
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

// h points at column `lane` of bin 0: h[b * 32] is this lane's counter for bin b.
__device__ __forceinline__ void hist_add_word(uint32_t* h, uint32_t w) {
    atomicAdd(h + ((w & 0xFFu) << 5), 1u);
    atomicAdd(h + (((w >> 8) & 0xFFu) << 5), 1u);
    atomicAdd(h + (((w >> 16) & 0xFFu) << 5), 1u);
    atomicAdd(h + ((w >> 24) << 5), 1u);
}

// Sum the 32 replicas of each bin (thread t owns bin t; the column walk is rotated by
// t so a warp's 32 reads hit 32 banks), zero them, and add to the VP's counts.
__device__ __forceinline__ void hist_flush(uint32_t* h, uint32_t* counts) {
    __syncthreads();
    const int b = threadIdx.x;  // kHistThreads == 256 == #bins
    uint32_t s = 0;
#pragma unroll 8
    for (int j = 0; j < 32; ++j) {
        const int c = (j + b) & 31;
        s += h[b * 32 + c];
        h[b * 32 + c] = 0;
    }
    if (s) atomicAdd(&counts[b], s);
    __syncthreads();
}

__global__ void __launch_bounds__(kHistThreads) k_hist256(const SegDesc* __restrict__ segs, int nsegs, uint32_t total) {
    static_assert(kHistThreads == 256, "one flush thread per bin");
    extern __shared__ uint32_t h[];  // [256][32]
    for (int i = threadIdx.x; i < 256 * 32; i += kHistThreads) h[i] = 0;
    __syncthreads();
    uint32_t* hl = h + (threadIdx.x & 31);
    int cur = -1;
    uint32_t* cur_counts = nullptr;
    // blocked tile ranges: a CTA walks contiguous tiles, so it stays inside one VP for
    // many tiles and flushes its replicas only at VP boundaries
    const uint32_t per = (total + gridDim.x - 1) / gridDim.x;
    const uint32_t t0 = blockIdx.x * per, t1 = min(total, t0 + per);
    for (uint32_t t = t0; t < t1; ++t) {
        const int si = find_seg(segs, nsegs, t);
        const SegDesc& sd = segs[si];
        if (si != cur) {
            if (cur >= 0) hist_flush(h, cur_counts);
            cur = si;
            cur_counts = reinterpret_cast<uint32_t*>(sd.ptr[1]);
        }
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
            for (int64_t e = e0 + threadIdx.x; e < e1; e += kHistThreads) atomicAdd(hl + ((uint32_t)d[e] << 5), 1u);
        }
    }
    if (cur >= 0) hist_flush(h, cur_counts);
}

constexpr int kHistSmem = 256 * 32 * 4;

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

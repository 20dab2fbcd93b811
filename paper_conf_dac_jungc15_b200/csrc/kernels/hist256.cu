// hist256.cu -- coalesced 256-bin byte histogram for sm_100a.
//
// counts_v[b] = #{i : d_v[i] == b} for every VP v of the group, in one launch.
// Each tile lies in one VP; a CTA accumulates the bytes of its tiles into per-warp
// shared-memory sub-histograms (one smem atomic per byte), and flushes them to the VP's
// global counts with one atomicAdd per non-zero bin whenever it moves on to another VP.
// A preceding tiny kernel zeroes every segment's counts, so the result overwrites the
// output (the oracle's definition) and is bit-exact: integer adds commute.
#include "../launch.h"
#include "common.cuh"

namespace svp {

constexpr int kHistWarps = kHistThreads / 32;

__global__ void __launch_bounds__(256) k_hist_zero(const SegDesc* __restrict__ segs, int nsegs) {
    for (int s = blockIdx.x; s < nsegs; s += gridDim.x) {
        uint32_t* counts = reinterpret_cast<uint32_t*>(segs[s].ptr[1]);
        counts[threadIdx.x] = 0u;
    }
}

__device__ __forceinline__ void hist_add_word(uint32_t* h, uint32_t w) {
    atomicAdd(&h[w & 0xFF], 1u);
    atomicAdd(&h[(w >> 8) & 0xFF], 1u);
    atomicAdd(&h[(w >> 16) & 0xFF], 1u);
    atomicAdd(&h[w >> 24], 1u);
}

__device__ __forceinline__ void hist_flush(uint32_t (*h)[256], uint32_t* counts) {
    __syncthreads();
    for (int b = threadIdx.x; b < 256; b += kHistThreads) {
        uint32_t s = 0;
#pragma unroll
        for (int w = 0; w < kHistWarps; ++w) {
            s += h[w][b];
            h[w][b] = 0;
        }
        if (s) atomicAdd(&counts[b], s);
    }
    __syncthreads();
}

__global__ void __launch_bounds__(kHistThreads) k_hist256(const SegDesc* __restrict__ segs, int nsegs, uint32_t total) {
    __shared__ uint32_t h[kHistWarps][256];
    for (int i = threadIdx.x; i < kHistWarps * 256; i += kHistThreads) (&h[0][0])[i] = 0;
    __syncthreads();
    uint32_t* hw = h[threadIdx.x >> 5];
    int cur = -1;
    uint32_t* cur_counts = nullptr;
    for (uint32_t t = blockIdx.x; t < total; t += gridDim.x) {
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
                hist_add_word(hw, r[i].x);
                hist_add_word(hw, r[i].y);
                hist_add_word(hw, r[i].z);
                hist_add_word(hw, r[i].w);
            }
        } else {
            for (int64_t e = e0 + threadIdx.x; e < e1; e += kHistThreads) atomicAdd(&hw[d[e]], 1u);
        }
    }
    if (cur >= 0) hist_flush(h, cur_counts);
}

cudaError_t launch_hist256(const SegDesc* segs, int nsegs, uint32_t total, int grid, cudaStream_t s) {
    if (nsegs <= 0) return cudaSuccess;
    k_hist_zero<<<nsegs < 1024 ? nsegs : 1024, 256, 0, s>>>(segs, nsegs);
    cudaError_t e = cudaGetLastError();
    if (e || total == 0) return e;
    k_hist256<<<grid, kHistThreads, 0, s>>>(segs, nsegs, total);
    return cudaGetLastError();
}

cudaError_t query_limits_hist(int* per_sm) {
    return cudaOccupancyMaxActiveBlocksPerMultiprocessor(per_sm, k_hist256, kHistThreads, 0);
}

}  // namespace svp

// hist_schemes.cu -- microbenchmark of 256-bin byte-histogram counting schemes on sm_100a
// (the ceiling of each scheme, to decide whether any can reach 70 % of
// HBM on hist256).  Not part of libsvp; built by tools/hist_schemes.py into /tmp.
//
// Every kernel reads n bytes (grid-stride, 16 B per thread per step, ld.global.cs) and
// produces counts[256] (global atomics at the end).  Schemes:
//   0 "lane_replicated_atoms"  h[bin][lane] u32 per CTA (32 KiB), one ATOMS per byte into
//                             the lane's own column: 32 banks per warp instruction whatever
//                             the data (the libsvp kernel's counting scheme).
//   1 "match_any_aggregated"   the north star's warp aggregation: per byte position
//                             __match_any_sync over the warp, the lowest lane of each group
//                             adds popc(group) to a per-warp table (1 KiB per warp).
//   2 "private_u16_lds_sts"    per-thread private counters, two u16 per word, laid out
//                             [bin/2][thread] (bank = thread: conflict-free), plain LDS +
//                             STS (no atomics; 128 KiB per 256-thread CTA).
//   3 "private_u8_lds_sts"     the same with u8 counters (four per word, [bin/4][thread],
//                             64 KiB) widened into u32 shared totals every 255 bytes per
//                             thread.
//   4 "shared_atoms_one_table" one u32 table per CTA, ATOMS per byte (same-bin lanes are
//                             aggregated by ATOMS.POPC.INC; different bins collide in banks).
#include <stdint.h>

namespace {

constexpr int kThreads = 256;

__device__ __forceinline__ uint4 ldcs4(const uint8_t* p) {
    return __ldcs(reinterpret_cast<const uint4*>(p));
}

template <typename F>
__device__ __forceinline__ void for_bytes(const uint4& v, F f) {
    const uint32_t w[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
    for (int i = 0; i < 4; ++i) {
        f(w[i] & 0xFFu);
        f((w[i] >> 8) & 0xFFu);
        f((w[i] >> 16) & 0xFFu);
        f(w[i] >> 24);
    }
}

__global__ void __launch_bounds__(kThreads) k_lane_replicated(const uint8_t* d, uint64_t n, uint32_t* counts) {
    __shared__ uint32_t h[256 * 32];
    for (int i = threadIdx.x; i < 256 * 32; i += kThreads) h[i] = 0;
    __syncthreads();
    uint32_t* hl = h + (threadIdx.x & 31);
    const uint64_t nv = n / 16;
    for (uint64_t i = blockIdx.x * (uint64_t)kThreads + threadIdx.x; i < nv; i += (uint64_t)gridDim.x * kThreads) {
        const uint4 v = ldcs4(d + 16 * i);
        for_bytes(v, [&](uint32_t b) { atomicAdd(hl + (b << 5), 1u); });
    }
    __syncthreads();
    const int b = threadIdx.x;
    uint32_t s = 0;
    for (int j = 0; j < 32; ++j) s += h[b * 32 + ((j + b) & 31)];
    if (s) atomicAdd(&counts[b], s);
}

__global__ void __launch_bounds__(kThreads) k_match_any(const uint8_t* d, uint64_t n, uint32_t* counts) {
    __shared__ uint32_t h[kThreads / 32][256];
    for (int i = threadIdx.x; i < (kThreads / 32) * 256; i += kThreads) (&h[0][0])[i] = 0;
    __syncthreads();
    const int lane = threadIdx.x & 31;
    uint32_t* hw = h[threadIdx.x >> 5];
    const uint64_t nv = n / 16;
    // every lane of a warp runs the same trip count (match_any needs the full warp)
    const uint64_t stride = (uint64_t)gridDim.x * kThreads;
    const uint64_t base = blockIdx.x * (uint64_t)kThreads + (threadIdx.x & ~31u);
    for (uint64_t i0 = base; i0 < nv; i0 += stride) {
        const uint64_t i = i0 + lane;
        const uint4 v = i < nv ? ldcs4(d + 16 * i) : make_uint4(0, 0, 0, 0);
        const bool ok = i < nv;
        for_bytes(v, [&](uint32_t b) {
            const uint32_t key = ok ? b : 256u + lane;  // lanes past the end match nobody
            const uint32_t m = __match_any_sync(0xFFFFFFFFu, key);
            if (ok && lane == __ffs(m) - 1) atomicAdd(hw + b, (uint32_t)__popc(m));
        });
    }
    __syncthreads();
    const int b = threadIdx.x;
    uint32_t s = 0;
    for (int w = 0; w < kThreads / 32; ++w) s += h[w][b];
    if (s) atomicAdd(&counts[b], s);
}

__global__ void __launch_bounds__(kThreads) k_private_u16(const uint8_t* d, uint64_t n, uint32_t* counts) {
    extern __shared__ uint32_t hp[];  // [128][kThreads]
    for (int i = threadIdx.x; i < 128 * kThreads; i += kThreads) hp[i] = 0;
    __syncthreads();
    uint32_t* mine = hp + threadIdx.x;
    const uint64_t nv = n / 16;
    // <= 65535 bytes per thread between widenings: a CTA-wide pass of 4096 16-B steps
    uint32_t since = 0;
    for (uint64_t i = blockIdx.x * (uint64_t)kThreads + threadIdx.x; i < nv; i += (uint64_t)gridDim.x * kThreads) {
        const uint4 v = ldcs4(d + 16 * i);
        for_bytes(v, [&](uint32_t b) {
            uint32_t* p = mine + (b >> 1) * kThreads;
            *p += 1u << ((b & 1u) << 4);
        });
        since += 16;
        if (since > 65535 - 16) {  // widen: this thread's counters into the global counts
            for (int w = 0; w < 128; ++w) {
                const uint32_t x = mine[w * kThreads];
                if (x & 0xFFFFu) atomicAdd(&counts[2 * w], x & 0xFFFFu);
                if (x >> 16) atomicAdd(&counts[2 * w + 1], x >> 16);
                mine[w * kThreads] = 0;
            }
            since = 0;
        }
    }
    __syncthreads();
    // column sums: thread t sums word t/2 ... (one bin pair per 2 threads)
    const int w = threadIdx.x >> 1, half = threadIdx.x & 1;
    uint32_t s = 0;
    for (int t = 0; t < kThreads; ++t) s += (hp[w * kThreads + t] >> (16 * half)) & 0xFFFFu;
    if (s) atomicAdd(&counts[2 * w + half], s);
}

__global__ void __launch_bounds__(kThreads) k_private_u8(const uint8_t* d, uint64_t n, uint32_t* counts) {
    extern __shared__ uint32_t hp[];  // [64][kThreads] u8x4, then [256] u32 totals
    uint32_t* tot = hp + 64 * kThreads;
    for (int i = threadIdx.x; i < 64 * kThreads; i += kThreads) hp[i] = 0;
    tot[threadIdx.x] = 0;
    __syncthreads();
    uint32_t* mine = hp + threadIdx.x;
    const uint64_t nv = n / 16;
    uint32_t since = 0;
    for (uint64_t i = blockIdx.x * (uint64_t)kThreads + threadIdx.x; i < nv; i += (uint64_t)gridDim.x * kThreads) {
        const uint4 v = ldcs4(d + 16 * i);
        for_bytes(v, [&](uint32_t b) {
            uint32_t* p = mine + (b >> 2) * kThreads;
            *p += 1u << ((b & 3u) << 3);
        });
        since += 16;
        if (since > 255 - 16) {  // widen before a u8 counter can wrap
            for (int w = 0; w < 64; ++w) {
                const uint32_t x = mine[w * kThreads];
                if (x) {
#pragma unroll
                    for (int q = 0; q < 4; ++q)
                        if ((x >> (8 * q)) & 0xFFu) atomicAdd(&tot[4 * w + q], (x >> (8 * q)) & 0xFFu);
                    mine[w * kThreads] = 0;
                }
            }
            since = 0;
        }
    }
    __syncthreads();
    for (int w = 0; w < 64; ++w) {  // leftovers
        const uint32_t x = mine[w * kThreads];
#pragma unroll
        for (int q = 0; q < 4; ++q)
            if ((x >> (8 * q)) & 0xFFu) atomicAdd(&tot[4 * w + q], (x >> (8 * q)) & 0xFFu);
    }
    __syncthreads();
    if (tot[threadIdx.x]) atomicAdd(&counts[threadIdx.x], tot[threadIdx.x]);
}

__global__ void __launch_bounds__(kThreads) k_one_table(const uint8_t* d, uint64_t n, uint32_t* counts) {
    __shared__ uint32_t h[256];
    h[threadIdx.x] = 0;
    __syncthreads();
    const uint64_t nv = n / 16;
    for (uint64_t i = blockIdx.x * (uint64_t)kThreads + threadIdx.x; i < nv; i += (uint64_t)gridDim.x * kThreads) {
        const uint4 v = ldcs4(d + 16 * i);
        for_bytes(v, [&](uint32_t b) { atomicAdd(h + b, 1u); });
    }
    __syncthreads();
    if (h[threadIdx.x]) atomicAdd(&counts[threadIdx.x], h[threadIdx.x]);
}

}  // namespace

extern "C" int hs_run(int scheme, const void* d, uint64_t n, uint32_t* counts, int grid, void* stream) {
    cudaStream_t s = (cudaStream_t)stream;
    switch (scheme) {
        case 0: k_lane_replicated<<<grid, kThreads, 0, s>>>((const uint8_t*)d, n, counts); break;
        case 1: k_match_any<<<grid, kThreads, 0, s>>>((const uint8_t*)d, n, counts); break;
        case 2: {
            const int smem = 128 * kThreads * 4;
            cudaFuncSetAttribute(k_private_u16, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
            k_private_u16<<<grid, kThreads, smem, s>>>((const uint8_t*)d, n, counts);
            break;
        }
        case 3: {
            const int smem = (64 * kThreads + 256) * 4;
            cudaFuncSetAttribute(k_private_u8, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
            k_private_u8<<<grid, kThreads, smem, s>>>((const uint8_t*)d, n, counts);
            break;
        }
        case 4: k_one_table<<<grid, kThreads, 0, s>>>((const uint8_t*)d, n, counts); break;
        default: return -1;
    }
    return (int)cudaGetLastError();
}

// resident CTAs per SM of each scheme (occupancy), for sizing the grid
extern "C" int hs_blocks_per_sm(int scheme) {
    int nb = 0;
    switch (scheme) {
        case 0: cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k_lane_replicated, kThreads, 0); break;
        case 1: cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k_match_any, kThreads, 0); break;
        case 2:
            cudaFuncSetAttribute(k_private_u16, cudaFuncAttributeMaxDynamicSharedMemorySize, 128 * kThreads * 4);
            cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k_private_u16, kThreads, 128 * kThreads * 4);
            break;
        case 3:
            cudaFuncSetAttribute(k_private_u8, cudaFuncAttributeMaxDynamicSharedMemorySize, (64 * kThreads + 256) * 4);
            cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k_private_u8, kThreads, (64 * kThreads + 256) * 4);
            break;
        case 4: cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k_one_table, kThreads, 0); break;
    }
    return nb;
}

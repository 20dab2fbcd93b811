// dgemm.cu -- grouped (coalesced) fp64 GEMM for sm_100a: the paper's own matmul guest.
//
// Table 1 multiplies 320 x 320 fp64 matrices 300 times;
// one such job fills 25 64x64 tiles -- 17 % of a B200 -- so coalescing the identical
// calls of many VPs into one grouped launch is exactly the "alignment" gain of PAPER.md
// L526-531.  C_v = alpha_v A_v B_v + beta_v C_v, row-major, any M, N, K (ragged shapes
// in one launch), fp64 DFMA:
//  * persistent grid over the tiles of all VPs; tile -> (VP, tm, tn) via the DgemmDesc table;
//  * 64x64 output tile, 16-deep k blocks, 256 threads with 4x4 accumulators each;
//  * A staged transposed in shared memory (k-major rows padded to 65 doubles: the 16
//    k-rows of a warp's stores fall in distinct banks), B staged as is; two smem buffers
//    with the next k block's global loads issued before the current block's DFMAs.
#include "../launch.h"
#include "common.cuh"

namespace svp {

constexpr int DM = kDgemmBM, DN = kDgemmBN, DK = kDgemmBK;
constexpr int kDThreads = 256;
constexpr int kApad = DM + 1;

__device__ __forceinline__ int find_dgemm(const DgemmDesc* __restrict__ d, int n, uint32_t t) {
    int lo = 0, hi = n;
    while (lo < hi) {
        int mid = (lo + hi) >> 1;
        if (__ldg(&d[mid].tile_begin) <= t) lo = mid + 1;
        else hi = mid;
    }
    return lo - 1;
}

__global__ void __launch_bounds__(kDThreads) k_dgemm(const DgemmDesc* __restrict__ descs, int n, uint32_t total) {
    __shared__ double As[2][DK][kApad];
    __shared__ __align__(16) double Bs[2][DK][DN];
    const int tid = threadIdx.x, tx = tid & 15, ty = tid >> 4;
    for (uint32_t t = blockIdx.x; t < total; t += gridDim.x) {
        const DgemmDesc& g = descs[find_dgemm(descs, n, t)];
        const uint32_t lt = t - g.tile_begin;
        const int m0 = (lt / g.tiles_n) * DM, n0 = (lt % g.tiles_n) * DN;
        const int M = g.M, N = g.N, K = g.K;
        const double* __restrict__ A = g.A;
        const double* __restrict__ B = g.B;
        double acc[4][4];
#pragma unroll
        for (int i = 0; i < 4; ++i)
#pragma unroll
            for (int j = 0; j < 4; ++j) acc[i][j] = 0.0;

        // each thread moves 4 A and 4 B elements per k block
        double ra[4], rb[4];
        auto load = [&](int k0) {
#pragma unroll
            for (int i = 0; i < 4; ++i) {
                const int idx = tid + i * kDThreads;   // A: 64 rows x 16 k, k fastest
                const int r = idx >> 4, c = idx & 15;
                const int gm = m0 + r, gk = k0 + c;
                ra[i] = (gm < M && gk < K) ? A[(size_t)gm * K + gk] : 0.0;
                const int rr = idx >> 6, cc = idx & 63;  // B: 16 k x 64 cols, n fastest
                const int bk = k0 + rr, bn = n0 + cc;
                rb[i] = (bk < K && bn < N) ? B[(size_t)bk * N + bn] : 0.0;
            }
        };
        auto store = [&](int buf) {
#pragma unroll
            for (int i = 0; i < 4; ++i) {
                const int idx = tid + i * kDThreads;
                As[buf][idx & 15][idx >> 4] = ra[i];
                Bs[buf][idx >> 6][idx & 63] = rb[i];
            }
        };
        const int KB = (K + DK - 1) / DK;
        if (KB > 0) {
            load(0);
            store(0);
        }
        __syncthreads();
        for (int kb = 0; kb < KB; ++kb) {
            const int cur = kb & 1;
            if (kb + 1 < KB) load((kb + 1) * DK);
#pragma unroll
            for (int k = 0; k < DK; ++k) {
                double a[4], b[4];
#pragma unroll
                for (int i = 0; i < 4; ++i) a[i] = As[cur][k][ty * 4 + i];
                const double2 b01 = *reinterpret_cast<const double2*>(&Bs[cur][k][tx * 4]);
                const double2 b23 = *reinterpret_cast<const double2*>(&Bs[cur][k][tx * 4 + 2]);
                b[0] = b01.x;
                b[1] = b01.y;
                b[2] = b23.x;
                b[3] = b23.y;
#pragma unroll
                for (int i = 0; i < 4; ++i)
#pragma unroll
                    for (int j = 0; j < 4; ++j) acc[i][j] = __fma_rn(a[i], b[j], acc[i][j]);
            }
            if (kb + 1 < KB) store(cur ^ 1);
            __syncthreads();
        }
        // epilogue
#pragma unroll
        for (int i = 0; i < 4; ++i) {
            const int r = m0 + ty * 4 + i;
            if (r >= M) continue;
#pragma unroll
            for (int j = 0; j < 4; ++j) {
                const int c = n0 + tx * 4 + j;
                if (c >= N) continue;
                double* dst = g.C + (size_t)r * N + c;
                double o = g.alpha * acc[i][j];
                if (g.beta != 0.0) o = __fma_rn(g.beta, *dst, o);
                *dst = o;
            }
        }
        __syncthreads();  // smem reuse by the next tile
    }
}

cudaError_t launch_dgemm(const DgemmDesc* descs, int n, uint32_t total, int grid, cudaStream_t s) {
    k_dgemm<<<grid, kDThreads, 0, s>>>(descs, n, total);
    return cudaGetLastError();
}

cudaError_t query_limits_dgemm(int* per_sm) {
    return cudaOccupancyMaxActiveBlocksPerMultiprocessor(per_sm, k_dgemm, kDThreads, 0);
}

}  // namespace svp

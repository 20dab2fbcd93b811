// dgemm.cu -- grouped (coalesced) fp64 GEMM for sm_100a: the paper's own matmul guest.
//
// Table 1 multiplies 320 x 320 fp64 matrices 300 times;
// one such job fills 25 64x64 tiles -- 17 % of a B200 -- so coalescing the identical
// calls of many VPs into one grouped launch is exactly the "alignment" gain of PAPER.md
// L526-531.  C_v = alpha_v A_v B_v + beta_v C_v, row-major, any M, N, K (ragged shapes
// in one launch), fp64 DFMA:
//  * persistent grid over the tiles of all VPs; tile -> (VP, tm, tn) via the DgemmDesc table;
//  * 64x64 output tile, 16-deep k blocks, 256 threads with 4x4 accumulators each; when a
//    launch has fewer than 2 waves of 64x64 tiles (Table 1 with few VPs: 25 tiles per VP),
//    32x32 tiles with 64 threads instead -- 4x the CTAs, so the dependent 320^3 GEMMs of
//    the paper's program spread over the SMs instead of leaving 80 % of them idle;
//  * A staged transposed in shared memory (k-major rows padded to 65 doubles: the 16
//    k-rows of a warp's stores fall in distinct banks), B staged as is; two smem buffers
//    with the next k block's global loads issued before the current block's DFMAs;
//  * split K (session 3): when even the 32x32 tiles leave most CTA slots empty (the Table 1
//    program with 1-4 VPs: 100 tiles per VP), each tile runs on a cluster of S = 2 or 4
//    CTAs, CTA r accumulating k blocks [r*ceil(KB/S), ...); ranks 1..S-1 leave their 4x4
//    partials in shared memory and rank 0 adds them through DSMEM in rank order (a fixed
//    order: the result does not depend on timing) before the epilogue.
#include <stdlib.h>

#include <algorithm>

#include "../launch.h"
#include "common.cuh"

namespace svp {


__device__ __forceinline__ int find_dgemm(const DgemmDesc* __restrict__ d, int n, uint32_t t) {
    int lo = 0, hi = n;
    while (lo < hi) {
        int mid = (lo + hi) >> 1;
        if (__ldg(&d[mid].tile_begin) <= t) lo = mid + 1;
        else hi = mid;
    }
    return lo - 1;
}

// TM x TN output tile, (TM/4) x (TN/4) threads with 4x4 accumulators each, DK-deep k blocks
template <int TM, int TN, int DK, int S = 1>
__global__ void __launch_bounds__((TM / 4) * (TN / 4), S > 1 ? 6 : 0) k_dgemm(const DgemmDesc* __restrict__ descs, int n,
                                                               uint32_t total) {
    constexpr int NT = (TM / 4) * (TN / 4);
    uint32_t rank = 0;
    if constexpr (S > 1) asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(rank));
    auto cluster_sync = [] {
        asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
    };
    constexpr int LA = TM * DK / NT, LB = DK * TN / NT;  // elements per thread per k block
    constexpr int kApad = TM + 1;
    __shared__ double As[2][DK][kApad];
    __shared__ __align__(16) double Bs[2][DK][TN];
    // split K: this CTA's partials, [i*4+j][tid], in the A staging buffers (free after the k loop)
    double* red = &As[0][0][0];
    static_assert(S == 1 || 2 * DK * kApad >= 16 * NT, "partials fit in the A staging buffers");
    const int tid = threadIdx.x, tx = tid % (TN / 4), ty = tid / (TN / 4);
    for (uint32_t t = blockIdx.x / S; t < total; t += gridDim.x / S) {
        const DgemmDesc& g = descs[find_dgemm(descs, n, t)];
        const uint32_t lt = t - g.tile_begin;
        const int m0 = (lt / g.tiles_n) * TM, n0 = (lt % g.tiles_n) * TN;
        const int M = g.M, N = g.N, K = g.K;
        const double* __restrict__ A = g.A;
        const double* __restrict__ B = g.B;
        double acc[4][4];
#pragma unroll
        for (int i = 0; i < 4; ++i)
#pragma unroll
            for (int j = 0; j < 4; ++j) acc[i][j] = 0.0;

        double ra[LA], rb[LB];
        auto load = [&](int k0) {
#pragma unroll
            for (int i = 0; i < LA; ++i) {
                const int idx = tid + i * NT;  // A: TM rows x DK k, k fastest
                const int r = idx / DK, c = idx % DK;
                const int gm = m0 + r, gk = k0 + c;
                ra[i] = (gm < M && gk < K) ? A[(size_t)gm * K + gk] : 0.0;
            }
#pragma unroll
            for (int i = 0; i < LB; ++i) {
                const int idx = tid + i * NT;  // B: DK k x TN cols, n fastest
                const int rr = idx / TN, cc = idx % TN;
                const int bk = k0 + rr, bn = n0 + cc;
                rb[i] = (bk < K && bn < N) ? B[(size_t)bk * N + bn] : 0.0;
            }
        };
        auto store = [&](int buf) {
#pragma unroll
            for (int i = 0; i < LA; ++i) {
                const int idx = tid + i * NT;
                As[buf][idx % DK][idx / DK] = ra[i];
            }
#pragma unroll
            for (int i = 0; i < LB; ++i) {
                const int idx = tid + i * NT;
                Bs[buf][idx / TN][idx % TN] = rb[i];
            }
        };
        // this CTA's k blocks [kb0, KB) (split K: rank r of the cluster takes a contiguous share)
        const int KBall = (K + DK - 1) / DK, per = (KBall + S - 1) / S;
        const int kb0 = S == 1 ? 0 : min(KBall, (int)rank * per), KB = S == 1 ? KBall : min(KBall, kb0 + per);
        if (KB > kb0) {
            load(kb0 * DK);
            store(0);
        }
        __syncthreads();
        for (int kb = kb0; kb < KB; ++kb) {
            const int cur = S == 1 ? (kb & 1) : ((kb - kb0) & 1);
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
        if constexpr (S > 1) {
            // ranks 1..S-1 publish their partials; rank 0 adds them in rank order
            if (rank != 0) {
#pragma unroll
                for (int i = 0; i < 4; ++i)
#pragma unroll
                    for (int j = 0; j < 4; ++j) red[(i * 4 + j) * NT + tid] = acc[i][j];
            }
            cluster_sync();
            if (rank == 0) {
#pragma unroll 1
                for (uint32_t r = 1; r < (uint32_t)S; ++r) {
                    uint32_t base;
                    asm volatile("mapa.shared::cluster.u32 %0, %1, %2;"
                                 : "=r"(base)
                                 : "r"((uint32_t)__cvta_generic_to_shared(red)), "r"(r));
#pragma unroll
                    for (int i = 0; i < 4; ++i)
#pragma unroll
                        for (int j = 0; j < 4; ++j) {
                            double v;
                            asm volatile("ld.shared::cluster.f64 %0, [%1];"
                                         : "=d"(v)
                                         : "r"(base + (uint32_t)(((i * 4 + j) * NT + tid) * 8)));
                            acc[i][j] += v;
                        }
                }
            }
            cluster_sync();  // the peers' partials are read before they are overwritten
            if (rank != 0) continue;
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

// Small tiles on the FP64 tensor cores (session 3): the SIMT 32x32 kernel is bound by shared-
// memory loads (ncu: 0.5 LDS per DFMA, 40 % bank conflicts, FP64 pipe 25 % busy).  Here a
// 32x32 tile is 4 warps of 16x16, each 2x2 mma.sync.m8n8k4.f64 tiles (DMMA): per 4 k a thread
// loads 4 doubles for 32 FMAs.  A is staged m-major and B k-major with rows of TT + 4 / DK + 4
// doubles, so the fragment loads (lane -> (lane >> 2, lane & 3)) and the staging stores are
// both conflict-free.  The same split-K clusters as k_dgemm (rank-order DSMEM reduction).
constexpr int kMmaT = 32, kMmaDK = 32, kMmaThreads = 128;

__device__ __forceinline__ void dmma(double (&d)[2], double a, double b) {
    asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};"
                 : "+d"(d[0]), "+d"(d[1])
                 : "d"(a), "d"(b));
}

template <int S>
__global__ void __launch_bounds__(kMmaThreads, S > 1 ? 6 : 0) k_dgemm_mma(const DgemmDesc* __restrict__ descs, int n,
                                                                        uint32_t total) {
    constexpr int T = kMmaT, DK = kMmaDK, NT = kMmaThreads;
    constexpr int PA = DK + 4, PB = T + 4;   // row strides (doubles): 4 mod 16 -> conflict-free
    constexpr int LA = T * DK / NT, LB = DK * T / NT;
    __shared__ __align__(16) double As[2][T][PA];   // A tile, m-major (k fastest)
    __shared__ __align__(16) double Bs[2][DK][PB];  // B tile, k-major (n fastest)
    double* red = &As[0][0][0];                     // split K: partials [e][tid] after the k loop
    static_assert(S == 1 || 2 * T * PA >= 8 * NT, "partials fit in the A staging buffers");
    uint32_t rank = 0;
    if constexpr (S > 1) asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(rank));
    auto cluster_sync = [] {
        asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
    };
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int wm = (warp >> 1) * 16, wn = (warp & 1) * 16;
    const int fr = lane >> 2, fk = lane & 3;  // fragment row / k (A), col / k (B)
    for (uint32_t t = blockIdx.x / S; t < total; t += gridDim.x / S) {
        const DgemmDesc& g = descs[find_dgemm(descs, n, t)];
        const uint32_t lt = t - g.tile_begin;
        const int m0 = (lt / g.tiles_n) * T, n0 = (lt % g.tiles_n) * T;
        const int M = g.M, N = g.N, K = g.K;
        const double* __restrict__ A = g.A;
        const double* __restrict__ B = g.B;
        double acc[2][2][2];
#pragma unroll
        for (int i = 0; i < 2; ++i)
#pragma unroll
            for (int j = 0; j < 2; ++j) acc[i][j][0] = acc[i][j][1] = 0.0;
        double ra[LA], rb[LB];
        auto load = [&](int k0) {
#pragma unroll
            for (int i = 0; i < LA; ++i) {
                const int idx = tid + i * NT, r = idx / DK, c = idx % DK;
                const int gm = m0 + r, gk = k0 + c;
                ra[i] = (gm < M && gk < K) ? A[(size_t)gm * K + gk] : 0.0;
            }
#pragma unroll
            for (int i = 0; i < LB; ++i) {
                const int idx = tid + i * NT, rr = idx / T, cc = idx % T;
                const int bk = k0 + rr, bn = n0 + cc;
                rb[i] = (bk < K && bn < N) ? B[(size_t)bk * N + bn] : 0.0;
            }
        };
        auto store = [&](int buf) {
#pragma unroll
            for (int i = 0; i < LA; ++i) {
                const int idx = tid + i * NT;
                As[buf][idx / DK][idx % DK] = ra[i];
            }
#pragma unroll
            for (int i = 0; i < LB; ++i) {
                const int idx = tid + i * NT;
                Bs[buf][idx / T][idx % T] = rb[i];
            }
        };
        const int KBall = (K + DK - 1) / DK, per = (KBall + S - 1) / S;
        const int kb0 = S == 1 ? 0 : min(KBall, (int)rank * per), KB = S == 1 ? KBall : min(KBall, kb0 + per);
        if (KB > kb0) {
            load(kb0 * DK);
            store(0);
        }
        __syncthreads();
        for (int kb = kb0; kb < KB; ++kb) {
            const int cur = S == 1 ? (kb & 1) : ((kb - kb0) & 1);
            if (kb + 1 < KB) load((kb + 1) * DK);
#pragma unroll
            for (int ks = 0; ks < DK; ks += 4) {
                double a[2], b[2];
#pragma unroll
                for (int i = 0; i < 2; ++i) a[i] = As[cur][wm + i * 8 + fr][ks + fk];
#pragma unroll
                for (int j = 0; j < 2; ++j) b[j] = Bs[cur][ks + fk][wn + j * 8 + fr];
#pragma unroll
                for (int i = 0; i < 2; ++i)
#pragma unroll
                    for (int j = 0; j < 2; ++j) dmma(acc[i][j], a[i], b[j]);
            }
            if (kb + 1 < KB) store(cur ^ 1);
            __syncthreads();
        }
        if constexpr (S > 1) {
            if (rank != 0) {
#pragma unroll
                for (int e = 0; e < 8; ++e) red[e * NT + tid] = (&acc[0][0][0])[e];
            }
            cluster_sync();
            if (rank == 0) {
#pragma unroll 1
                for (uint32_t r = 1; r < (uint32_t)S; ++r) {
                    uint32_t base;
                    asm volatile("mapa.shared::cluster.u32 %0, %1, %2;"
                                 : "=r"(base)
                                 : "r"((uint32_t)__cvta_generic_to_shared(red)), "r"(r));
#pragma unroll
                    for (int e = 0; e < 8; ++e) {
                        double v;
                        asm volatile("ld.shared::cluster.f64 %0, [%1];" : "=d"(v) : "r"(base + (uint32_t)((e * NT + tid) * 8)));
                        (&acc[0][0][0])[e] += v;
                    }
                }
            }
            cluster_sync();
            if (rank != 0) continue;
        }
        // epilogue: D fragment (row lane / 4, cols 2 (lane % 4) + {0, 1}) of each 8x8 tile
#pragma unroll
        for (int i = 0; i < 2; ++i) {
            const int r = m0 + wm + i * 8 + fr;
            if (r >= M) continue;
#pragma unroll
            for (int j = 0; j < 2; ++j)
#pragma unroll
                for (int h = 0; h < 2; ++h) {
                    const int c = n0 + wn + j * 8 + 2 * fk + h;
                    if (c >= N) continue;
                    double* dst = g.C + (size_t)r * N + c;
                    double o = g.alpha * acc[i][j][h];
                    if (g.beta != 0.0) o = __fma_rn(g.beta, *dst, o);
                    *dst = o;
                }
        }
        __syncthreads();  // smem reuse by the next tile
    }
}

static cudaError_t launch_cluster(const void* kern, int S, uint32_t grid, int threads, cudaStream_t s,
                                  const DgemmDesc* descs, int n, uint32_t total) {
    cudaLaunchConfig_t lc = {};
    cudaLaunchAttribute attr[1];
    lc.gridDim = dim3(grid);
    lc.blockDim = dim3(threads);
    lc.stream = s;
    attr[0].id = cudaLaunchAttributeClusterDimension;
    attr[0].val.clusterDim.x = S;
    attr[0].val.clusterDim.y = 1;
    attr[0].val.clusterDim.z = 1;
    lc.attrs = attr;
    lc.numAttrs = S > 1 ? 1 : 0;
    void* args[] = {(void*)&descs, (void*)&n, (void*)&total};
    return cudaLaunchKernelExC(&lc, kern, args);
}

bool dgemm_dmma_enabled() {
    static const bool on = !(getenv("SVP_DGEMM_DMMA") && atoi(getenv("SVP_DGEMM_DMMA")) == 0);
    return on;
}

cudaError_t launch_dgemm(const DgemmDesc* descs, int n, uint32_t total, int grid, bool small, cudaStream_t s) {
    // small tiles: 32-deep k stages (fewer barriers per tile, 255 registers) when all tiles
    // are resident at once at that occupancy -- the Table 1 program with 1-4 VPs (S5: 1 VP
    // 14.9 -> 12.4 ms); otherwise the 16-deep variant's higher occupancy wins (8 VPs).
    static const int deep_cap = [] {
        int dev = 0, sms = 0, per = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, k_dgemm<kDgemmSmall, kDgemmSmall, kDgemmSmallDeepBK>,
                                                      (kDgemmSmall / 4) * (kDgemmSmall / 4), 0);
        cudaGetLastError();
        return sms * per;
    }();
    if (small && dgemm_dmma_enabled()) {
        // the DMMA small-tile kernel (32 x 32 tiles like the SIMT small variant), split K on
        // clusters under the same rule
        static const int mma_cap = [] {
            int dev = 0, sms = 0, per = 0;
            cudaGetDevice(&dev);
            cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
            cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, k_dgemm_mma<4>, kMmaThreads, 0);
            cudaGetLastError();
            return sms * per;
        }();
        static const int mma_per_sm = [] {
            int per = 0;
            cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, k_dgemm_mma<1>, kMmaThreads, 0);
            cudaGetLastError();
            return std::max(1, per);
        }();
        static const bool split_ok = !(getenv("SVP_DGEMM_SPLIT") && atoi(getenv("SVP_DGEMM_SPLIT")) == 0);
        const int Sm = !split_ok                             ? 1
                       : total * 4 <= (uint32_t)mma_cap / 2 ? 4
                       : total * 2 <= (uint32_t)mma_cap     ? 2
                                                            : 1;
        if (Sm == 4) return launch_cluster((const void*)k_dgemm_mma<4>, 4, total * 4, kMmaThreads, s, descs, n, total);
        if (Sm == 2) return launch_cluster((const void*)k_dgemm_mma<2>, 2, total * 2, kMmaThreads, s, descs, n, total);
        int dev = 0, sms = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
        const uint32_t g1 = std::min<uint32_t>(total, (uint32_t)(sms * mma_per_sm));
        k_dgemm_mma<1><<<g1, kMmaThreads, 0, s>>>(descs, n, total);
        return cudaGetLastError();
    }
    // split K when S times the tiles still fit in one wave of the deep small variant
    static const bool split_on = !(getenv("SVP_DGEMM_SPLIT") && atoi(getenv("SVP_DGEMM_SPLIT")) == 0);
    static const int split_cap = [] {
        int dev = 0, sms = 0, per = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, k_dgemm<kDgemmSmall, kDgemmSmall, kDgemmSmallDeepBK, 4>,
                                                      (kDgemmSmall / 4) * (kDgemmSmall / 4), 0);
        cudaGetLastError();
        return sms * per;
    }();
    // S = 4 only while the split launch would use at most half the CTA slots (S5: 2 VPs, 200
    // tiles, ran 5.5 ms at S = 2 and 7.3 ms at S = 4), S = 2 while it fits in one wave
    const int S = !small || !split_on                         ? 1
                  : total * 4 <= (uint32_t)split_cap / 2 ? 4
                  : total * 2 <= (uint32_t)split_cap     ? 2
                                                         : 1;
    if (S > 1) {
        cudaLaunchConfig_t lc = {};
        cudaLaunchAttribute attr[1];
        lc.gridDim = dim3(total * S);
        lc.blockDim = dim3((kDgemmSmall / 4) * (kDgemmSmall / 4));
        lc.stream = s;
        attr[0].id = cudaLaunchAttributeClusterDimension;
        attr[0].val.clusterDim.x = S;
        attr[0].val.clusterDim.y = 1;
        attr[0].val.clusterDim.z = 1;
        lc.attrs = attr;
        lc.numAttrs = 1;
        if (S == 4)
            return cudaLaunchKernelEx(&lc, k_dgemm<kDgemmSmall, kDgemmSmall, kDgemmSmallDeepBK, 4>, descs, n, total);
        return cudaLaunchKernelEx(&lc, k_dgemm<kDgemmSmall, kDgemmSmall, kDgemmSmallDeepBK, 2>, descs, n, total);
    }
    if (small && total <= (uint32_t)deep_cap)
        k_dgemm<kDgemmSmall, kDgemmSmall, kDgemmSmallDeepBK>
            <<<grid, (kDgemmSmall / 4) * (kDgemmSmall / 4), 0, s>>>(descs, n, total);
    else if (small)
        k_dgemm<kDgemmSmall, kDgemmSmall, kDgemmSmallBK>
            <<<grid, (kDgemmSmall / 4) * (kDgemmSmall / 4), 0, s>>>(descs, n, total);
    else k_dgemm<kDgemmBM, kDgemmBN, kDgemmBK><<<grid, (kDgemmBM / 4) * (kDgemmBN / 4), 0, s>>>(descs, n, total);
    return cudaGetLastError();
}

cudaError_t query_limits_dgemm(int* per_sm, int* per_sm_small) {
    cudaError_t e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(per_sm, k_dgemm<kDgemmBM, kDgemmBN, kDgemmBK>,
                                                                  (kDgemmBM / 4) * (kDgemmBN / 4), 0);
    if (e) return e;
    return cudaOccupancyMaxActiveBlocksPerMultiprocessor(per_sm_small, k_dgemm<kDgemmSmall, kDgemmSmall, kDgemmSmallBK>,
                                                         (kDgemmSmall / 4) * (kDgemmSmall / 4), 0);
}

}  // namespace svp

// sgemm_ffma.cu -- grouped (coalesced) fp32 SGEMM for sm_100a: TMA-staged tiles, fp32 FFMA.
//
// C_v = alpha_v A_v B_v + beta_v C_v for every VP v of a Kernel Match group (equal
// M,N,K -- reading R1), all in ONE persistent launch: the paper's matmul guest
// (Table 1) coalesced.  A single 512^3 job has
// 16 output tiles and fills 16 of 148 SMs; 16 coalesced jobs give 256 tiles (the
// "alignment" gain of PAPER.md L526-531 / Eq 9).
//
// Design (B200):
//  * persistent grid = #SMs, 1 CTA/SM; static tile walk t = blockIdx.x + i*gridDim.x;
//    tile -> (VP, tile_m, tile_n) through the GemmDesc table (binary search).
//  * warp 8 = TMA producer: one elected lane issues cp.async.bulk.tensor for the A
//    (128x32, 128-B swizzle) and B (32x128) tiles of each k-block into a 4-stage smem
//    ring guarded by full/empty mbarriers; per-VP CUtensorMaps live in the table.
//  * warps 0-7 = consumers: 8x8 fp32 register micro-tile per thread; per 4-k group a
//    thread reads 8 float4 of A (k-vectorised, conflict-free thanks to the swizzle) and
//    8 float4 of B, then issues 128 FFMA2 (fma.rn.f32x2: a broadcast A value times a pair
//    of B values, per-lane IEEE rounding) = 256 FMAs, half the issue slots of FFMA.
//  * epilogue: alpha*acc (+ beta*C) with 128-bit stores straight from registers.
#include <cuda.h>
#include <stdio.h>

#include <atomic>

#include "../launch.h"
#include "common.cuh"

namespace svp {

constexpr int GM = kGemmBM, GN = kGemmBN, GK = kGemmBK;
constexpr int kStages = 4;
constexpr int kConsumers = 256;
constexpr int kGemmThreads = kConsumers + 32;
constexpr int kStageA = GM * GK * 4;  // 16 KiB
constexpr int kStageB = GK * GN * 4;  // 16 KiB
constexpr size_t kGemmSmem = 1024 + kStages * (kStageA + kStageB) + 2 * kStages * sizeof(uint64_t);

__device__ __forceinline__ int find_gemm(const GemmDesc* __restrict__ d, int n, uint32_t t) {
    int lo = 0, hi = n;
    while (lo < hi) {
        int mid = (lo + hi) >> 1;
        if (__ldg(&d[mid].tile_begin) <= t) lo = mid + 1;
        else hi = mid;
    }
    return lo - 1;
}

__global__ void __launch_bounds__(kGemmThreads, 1)
    k_sgemm_ffma(const GemmDesc* __restrict__ descs, int n, const uint8_t* __restrict__ maps, uint32_t total) {
    extern __shared__ uint8_t smem_raw[];
    uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);  // keeps LDS (shared space)
    float* sA = reinterpret_cast<float*>(smem);
    float* sB = reinterpret_cast<float*>(smem + kStages * kStageA);
    uint64_t* full = reinterpret_cast<uint64_t*>(smem + kStages * (kStageA + kStageB));
    uint64_t* empty = full + kStages;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;

    if (threadIdx.x == 0) {
        for (int s = 0; s < kStages; ++s) {
            mbar_init(&full[s], 1);
            mbar_init(&empty[s], kConsumers / 32);
        }
        mbar_fence_init();
    }
    __syncthreads();

    if (warp == kConsumers / 32) {
        // ------------------------------------------------------------ TMA producer
        if (lane == 0) {
            uint32_t it = 0;
            int last = -1;
            for (uint32_t t = blockIdx.x; t < total; t += gridDim.x) {
                const int v = find_gemm(descs, n, t);
                const GemmDesc& g = descs[v];
                const void* mA = maps + (size_t)v * 256;
                const void* mB = maps + (size_t)v * 256 + 128;
                if (v != last) {
                    prefetch_tmap(mA);
                    prefetch_tmap(mB);
                    last = v;
                }
                const uint32_t lt = t - g.tile_begin;
                const int tm = lt / g.tiles_n, tn = lt % g.tiles_n;
                const int KB = (g.K + GK - 1) / GK;
                for (int kb = 0; kb < KB; ++kb, ++it) {
                    const int s = it % kStages;
                    const uint32_t ph = (it / kStages) & 1;
                    mbar_wait(&empty[s], ph ^ 1);
                    mbar_expect_tx(&full[s], kStageA + kStageB);
                    tma_load_2d(sA + s * GM * GK, mA, kb * GK, tm * GM, &full[s]);
                    tma_load_2d(sB + s * GK * GN, mB, tn * GN, kb * GK, &full[s]);
                }
            }
        }
        return;
    }

    // ---------------------------------------------------------------- consumers
    const int tx = threadIdx.x & 15, ty = threadIdx.x >> 4;
    uint32_t it = 0;
    for (uint32_t t = blockIdx.x; t < total; t += gridDim.x) {
        const int v = find_gemm(descs, n, t);
        const GemmDesc& g = descs[v];
        const uint32_t lt = t - g.tile_begin;
        const int tm = lt / g.tiles_n, tn = lt % g.tiles_n;
        const int KB = (g.K + GK - 1) / GK;
        // accumulators as packed fp32 pairs: acc[i][p] = C(row i, cols 2p, 2p+1) of the
        // thread's 8 columns; FFMA2 (fma.rn.f32x2) does both lanes with one instruction and
        // per-lane IEEE rounding identical to FFMA
        unsigned long long acc[8][4];
#pragma unroll
        for (int i = 0; i < 8; ++i)
#pragma unroll
            for (int p = 0; p < 4; ++p) acc[i][p] = 0ull;

        for (int kb = 0; kb < KB; ++kb, ++it) {
            const int s = it % kStages;
            const uint32_t ph = (it / kStages) & 1;
            mbar_wait(&full[s], ph);
            const float* A = sA + s * GM * GK;
            const float* B = sB + s * GK * GN;
#pragma unroll
            for (int kk = 0; kk < GK / 4; ++kk) {
                float4 a[8];
#pragma unroll
                for (int i = 0; i < 8; ++i) {
                    const int r = (i < 4) ? (ty * 4 + i) : (64 + ty * 4 + (i - 4));
                    const int chunk = kk ^ (r & 7);  // 128-B swizzle: 16-B chunk ^= row % 8
                    a[i] = *reinterpret_cast<const float4*>(A + r * GK + chunk * 4);
                }
#pragma unroll
                for (int q = 0; q < 4; ++q) {
                    const int k = kk * 4 + q;
                    const ulonglong2 b0 = *reinterpret_cast<const ulonglong2*>(B + k * GN + tx * 4);
                    const ulonglong2 b1 = *reinterpret_cast<const ulonglong2*>(B + k * GN + 64 + tx * 4);
                    const unsigned long long bp[4] = {b0.x, b0.y, b1.x, b1.y};
#pragma unroll
                    for (int i = 0; i < 8; ++i) {
                        const float av = q == 0 ? a[i].x : q == 1 ? a[i].y : q == 2 ? a[i].z : a[i].w;
                        unsigned long long ap;
                        asm("mov.b64 %0, {%1, %1};" : "=l"(ap) : "f"(av));
#pragma unroll
                        for (int p = 0; p < 4; ++p)
                            asm("fma.rn.f32x2 %0, %1, %2, %0;" : "+l"(acc[i][p]) : "l"(ap), "l"(bp[p]));
                    }
                }
            }
            // the stage is released to the TMA producer only once this warp's last LDS of it
            // returned: an mbarrier arrive does not wait for outstanding shared loads
            // (hist256.cu), so a membar.cta (MEMBAR + scoreboard drain) precedes it
            __threadfence_block();
            __syncwarp();
            if (lane == 0) mbar_arrive(&empty[s]);
        }

        // ------------------------------------------------------------ epilogue
        const int M = g.M, N = g.N;
        const float alpha = g.alpha, beta = g.beta;
        float* __restrict__ C = g.C;
#pragma unroll
        for (int i = 0; i < 8; ++i) {
            const int r = tm * GM + ((i < 4) ? (ty * 4 + i) : (64 + ty * 4 + (i - 4)));
            if (r >= M) continue;
#pragma unroll
            for (int h = 0; h < 2; ++h) {
                const int c = tn * GN + h * 64 + tx * 4;
                if (c >= N) continue;
                float4* dst = reinterpret_cast<float4*>(C + (size_t)r * N + c);
                float4 o;
                o.x = alpha * __uint_as_float((uint32_t)acc[i][h * 2 + 0]);
                o.y = alpha * __uint_as_float((uint32_t)(acc[i][h * 2 + 0] >> 32));
                o.z = alpha * __uint_as_float((uint32_t)acc[i][h * 2 + 1]);
                o.w = alpha * __uint_as_float((uint32_t)(acc[i][h * 2 + 1] >> 32));
                if (beta != 0.f) {
                    const float4 old = __ldcs(dst);
                    o.x = __fmaf_rn(beta, old.x, o.x);
                    o.y = __fmaf_rn(beta, old.y, o.y);
                    o.z = __fmaf_rn(beta, old.z, o.z);
                    o.w = __fmaf_rn(beta, old.w, o.w);
                }
                __stcs(dst, o);  // st.global.cs: C is written once
            }
        }
    }
}

static std::atomic<bool> g_smem_set[64] = {};  // per device (one worker thread per GPU)

cudaError_t launch_sgemm_ffma(const GemmDesc* descs, int n, const void* maps, uint32_t total, int grid,
                              cudaStream_t s) {
    int dev = 0;
    cudaGetDevice(&dev);
    if (dev < 64 && !g_smem_set[dev]) {
        cudaError_t e = cudaFuncSetAttribute(k_sgemm_ffma, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kGemmSmem);
        if (e) return e;
        g_smem_set[dev] = true;
    }
    k_sgemm_ffma<<<grid, kGemmThreads, kGemmSmem, s>>>(descs, n, reinterpret_cast<const uint8_t*>(maps), total);
    return cudaGetLastError();
}

// ------------------------------------------------------------------ plain-load SGEMM
// "sgemm" jobs TMA cannot address -- a row pitch (K or N floats) not a multiple of 16 B, or
// a device buffer not 16-B aligned (these used to be SVP_E_UNSUPPORTED)
// -- match as their own group and run here: the same grouped tile walk over the GemmDesc
// table (A, B, lda, ldb), 64 x 64 tiles, 16-deep k blocks staged through shared memory with
// guarded scalar loads, 4 x 4 fp32 FFMA register tiles (ascending k, like the FFMA kernel),
// alpha * acc (+ beta * C) with guarded scalar stores.  No alignment or shape requirement.
constexpr int PT = 64, PK = 16, kPlainThreads = 256;

__global__ void __launch_bounds__(kPlainThreads)
    k_sgemm_plain(const GemmDesc* __restrict__ descs, int n, uint32_t total) {
    __shared__ float As[PK][PT + 4];  // k-major (transposed): As[k][m]
    __shared__ float Bs[PK][PT];
    const int tx = threadIdx.x & 15, ty = threadIdx.x >> 4;
    for (uint32_t t = blockIdx.x; t < total; t += gridDim.x) {
        const GemmDesc& g = descs[find_gemm(descs, n, t)];
        const uint32_t lt = t - g.tile_begin;
        const int m0 = (int)(lt / g.tiles_n) * PT, n0 = (int)(lt % g.tiles_n) * PT;
        float acc[4][4] = {};
        for (int k0 = 0; k0 < g.K; k0 += PK) {
#pragma unroll
            for (int i = 0; i < 4; ++i) {
                const int e = threadIdx.x + kPlainThreads * i;
                const int ar = e >> 4, ak = e & 15;           // A: 64 rows x 16 k
                const int gm = m0 + ar, gk = k0 + ak;
                As[ak][ar] = (gm < g.M && gk < g.K) ? __ldg(g.A + (size_t)gm * g.lda + gk) : 0.f;
                const int bk = e >> 6, bn = e & 63;           // B: 16 k x 64 cols
                const int gk2 = k0 + bk, gn = n0 + bn;
                Bs[bk][bn] = (gk2 < g.K && gn < g.N) ? __ldg(g.B + (size_t)gk2 * g.ldb + gn) : 0.f;
            }
            __syncthreads();
#pragma unroll
            for (int k = 0; k < PK; ++k) {
                float a[4], b[4];
#pragma unroll
                for (int i = 0; i < 4; ++i) a[i] = As[k][ty * 4 + i];
#pragma unroll
                for (int j = 0; j < 4; ++j) b[j] = Bs[k][tx * 4 + j];
#pragma unroll
                for (int i = 0; i < 4; ++i)
#pragma unroll
                    for (int j = 0; j < 4; ++j) acc[i][j] = __fmaf_rn(a[i], b[j], acc[i][j]);
            }
            __syncthreads();
        }
#pragma unroll
        for (int i = 0; i < 4; ++i) {
            const int gm = m0 + ty * 4 + i;
            if (gm >= g.M) continue;
#pragma unroll
            for (int j = 0; j < 4; ++j) {
                const int gn = n0 + tx * 4 + j;
                if (gn >= g.N) continue;
                float* c = g.C + (size_t)gm * g.N + gn;
                float o = g.K == 0 ? 0.f : g.alpha * acc[i][j];
                if (g.beta != 0.f) o = __fmaf_rn(g.beta, *c, o);
                *c = o;
            }
        }
    }
}

cudaError_t launch_sgemm_plain(const GemmDesc* descs, int n, uint32_t total, int grid, cudaStream_t s) {
    k_sgemm_plain<<<grid, kPlainThreads, 0, s>>>(descs, n, total);
    return cudaGetLastError();
}

cudaError_t query_limits_gemm_plain(int* per_sm) {
    return cudaOccupancyMaxActiveBlocksPerMultiprocessor(per_sm, k_sgemm_plain, kPlainThreads, 0);
}

cudaError_t query_limits_gemm(int* per_sm) {
    cudaError_t e = cudaFuncSetAttribute(k_sgemm_ffma, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kGemmSmem);
    if (e) return e;
    return cudaOccupancyMaxActiveBlocksPerMultiprocessor(per_sm, k_sgemm_ffma, kGemmThreads, kGemmSmem);
}

// ------------------------------------------------------------------ TMA descriptors
typedef CUresult (*PFN_encodeTiled)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                    const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                    CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

static PFN_encodeTiled get_encode() {
    static PFN_encodeTiled fn = nullptr;
    if (!fn) {
        void* p = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            fn = reinterpret_cast<PFN_encodeTiled>(p);
    }
    return fn;
}

// pitch: row stride in elements (0 = inner, a dense matrix); a sub-matrix view passes the
// parent's row length
static int encode2d(void* out, const float* base, uint64_t inner, uint64_t outer, uint32_t box_inner,
                    uint32_t box_outer, CUtensorMapSwizzle sw, uint64_t pitch = 0) {
    PFN_encodeTiled enc = get_encode();
    if (!enc) return -1;
    cuuint64_t dims[2] = {inner, outer};
    cuuint64_t strides[1] = {(pitch ? pitch : inner) * 4};
    cuuint32_t box[2] = {box_inner, box_outer};
    cuuint32_t estr[2] = {1, 1};
    CUresult r = enc(reinterpret_cast<CUtensorMap*>(out), CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, (void*)base, dims, strides,
                     box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE, sw, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                     CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    return r == CUDA_SUCCESS ? 0 : (int)r;
}

// C (M x N row-major fp32) as 16-column x 32-row boxes with the 64-B swizzle: the layout of
// the tensor-core SGEMM epilogue's staging half-slabs (TMA store / reduce-add)
int encode_c_map(void* mapC, const float* C, int M, int N) {
    return encode2d(mapC, C, (uint64_t)N, (uint64_t)M, 16, 32, CU_TENSOR_MAP_SWIZZLE_64B);
}

int encode_gemm_maps(void* mapA, void* mapB, const float* A, const float* B, int M, int N, int K, int variant) {
    static_assert(sizeof(CUtensorMap) == 128, "CUtensorMap is 128 B");
    if (variant == 0) {
        // A: M x K row-major -> box 32 (k) x 128 (m), 128-B swizzle; B: K x N -> box 128 (n) x 32 (k)
        int r = encode2d(mapA, A, (uint64_t)K, (uint64_t)M, GK, GM, CU_TENSOR_MAP_SWIZZLE_128B);
        if (r) return r;
        return encode2d(mapB, B, (uint64_t)N, (uint64_t)K, GN, GK, CU_TENSOR_MAP_SWIZZLE_NONE);
    }
    // tcgen05 tiles: A lands K-major (box 16 k x 128 m, SWIZZLE_64B); B (row-major K x N,
    // MN-major for the MMA) lands as 32-n x 16-k boxes with the 32-B-atom 128-B swizzle
    // (UMMA layout SWIZZLE_128B_BASE32B), 8 boxes per 256-wide tile.
    int r = encode2d(mapA, A, (uint64_t)K, (uint64_t)M, kTf32BK, kTf32BM, CU_TENSOR_MAP_SWIZZLE_64B);
    if (r) return r;
    return encode2d(mapB, B, (uint64_t)N, (uint64_t)K, 32, kTf32BK, CU_TENSOR_MAP_SWIZZLE_128B_ATOM_32B);
}

int encode_gemm_maps_view(void* mapA, void* mapB, const float* A, const float* B, int M, int N, int K, int lda,
                          int ldb) {
    // a sub-matrix view for the tcgen05 tiles: A (M x K, row stride lda), B (K x N, row stride ldb)
    int r = encode2d(mapA, A, (uint64_t)K, (uint64_t)M, kTf32BK, kTf32BM, CU_TENSOR_MAP_SWIZZLE_64B, (uint64_t)lda);
    if (r) return r;
    return encode2d(mapB, B, (uint64_t)N, (uint64_t)K, 32, kTf32BK, CU_TENSOR_MAP_SWIZZLE_128B_ATOM_32B, (uint64_t)ldb);
}

}  // namespace svp

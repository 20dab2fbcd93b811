// sgemm_tf32.cu -- grouped (coalesced) SGEMM on the 5th-gen tensor cores (tcgen05, sm_100a).
//
// C_v = alpha_v A_v B_v + beta_v C_v for every VP of a Kernel Match group, one persistent
// launch (Kernel Coalescing; the paper's matmul guest, Table 1).
//
//  SPLIT = 1  "sgemm_tf32": one kind::tf32 MMA per k-step; the tensor core reads the fp32
//             operands as TF32 (low 13 mantissa bits ignored).  Own tolerance 2e-3.
//  SPLIT = 3  "3xTF32": x = hi + lo with hi = x with the low 13 bits cleared (exactly what
//             the tensor core sees when fed x) and lo = x - hi (exact in fp32); per k-step
//             D += A_hi B_lo + A_lo B_hi + A_hi B_hi.  The dropped A_lo B_lo term and the
//             truncation of lo are each < 2^-20 |a||b|, so the product error is
//             < 3 * 2^-20 |a||b| ~ 2.9e-6 |a||b|: inside the fp32 SGEMM bound 1e-5 (|A||B|)_ij
//             (R10) at tensor-core speed.
//
// Structure (1 CTA per SM, persistent static tile walk, 256 threads):
//   warp 0      TMA producer: A tile 128x32 (K-major, 128-B swizzle) + B tile 32x256 as 8
//               boxes of 32x32 (MN-major, 128-B swizzle) per k-block into a smem ring.
//   warp 1      TMEM allocator (512 columns = 2 fp32 accumulators of 128x256) and the MMA
//               issuer: one elected lane issues tcgen05.mma.cta_group::1.kind::tf32
//               (M=128, N=256, K=8) and tcgen05.commit's to the stage's empty barrier and,
//               after the last k-block, to the accumulator's full barrier.
//   warps 2-3   (SPLIT = 3) converters: lo = x - trunc_tf32(x) for the stage's A and B tiles
//               (same swizzled layout), fence.proxy.async, arrive on the stage's conv barrier.
//   warps 4-7   epilogue: tcgen05.ld 32x32b.x32 (warp w%4 owns TMEM lanes 32(w%4)..+31 =
//               tile rows), alpha*acc (+ beta*C), 128-bit stores; double-buffered TMEM
//               accumulators let tile i's epilogue overlap tile i+1's MMAs.
#include <cuda.h>

#include "../launch.h"
#include "common.cuh"

namespace svp {

namespace tc {

constexpr int BM = kTf32BM, BN = kTf32BN, BK = kTf32BK;  // 128 x 256 x 32
constexpr int kThreads = 256;
constexpr int kStageA = BM * BK * 4;  // 16 KiB
constexpr int kStageB = BK * BN * 4;  // 32 KiB
constexpr int kTmemCols = 512;

template <int SPLIT>
struct Cfg {
    static constexpr int kStages = SPLIT == 1 ? 4 : 2;
    static constexpr int kStageBytes = (kStageA + kStageB) * (SPLIT == 1 ? 1 : 2);
    static constexpr size_t kSmem = 1024 + (size_t)kStages * kStageBytes + 256;
};

__device__ __forceinline__ uint64_t make_desc(uint32_t saddr, uint32_t lbo, uint32_t sbo) {
    // SM100 shared-memory matrix descriptor: start>>4 [0,14), LBO>>4 [16,30), SBO>>4 [32,46),
    // version 1 [46,48), base offset 0, layout SWIZZLE_128B (2) [61,64)
    uint64_t d = 0;
    d |= (uint64_t)((saddr >> 4) & 0x3FFF);
    d |= (uint64_t)((lbo >> 4) & 0x3FFF) << 16;
    d |= (uint64_t)((sbo >> 4) & 0x3FFF) << 32;
    d |= (uint64_t)1 << 46;
    d |= (uint64_t)2 << 61;
    return d;
}

// kind::tf32 instruction descriptor: D f32, A/B tf32, A K-major, B MN-major, N=256, M=128
constexpr uint32_t kIdesc = (1u << 4) | (2u << 7) | (2u << 10) | (0u << 15) | (1u << 16) |
                            ((uint32_t)(BN >> 3) << 17) | ((uint32_t)(BM >> 4) << 24);

__device__ __forceinline__ void mma_tf32(uint32_t tmem_d, uint64_t adesc, uint64_t bdesc, uint32_t accum) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "setp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem_d),
        "l"(adesc), "l"(bdesc), "r"(kIdesc), "r"(accum)
        : "memory");
}
__device__ __forceinline__ void mma_commit(uint64_t* bar) {
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(bar))
                 : "memory");
}
__device__ __forceinline__ void tc_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void fence_proxy_async() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }

__device__ __forceinline__ void tmem_ld32(uint32_t taddr, uint32_t (&r)[32]) {
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x32.b32 "
        "{%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
        "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
        : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
          "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]),
          "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]),
          "=r"(r[24]), "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
        : "r"(taddr));
    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
}

__device__ __forceinline__ int find_tile_owner(const GemmDesc* __restrict__ d, int n, uint32_t t) {
    int lo = 0, hi = n;
    while (lo < hi) {
        int mid = (lo + hi) >> 1;
        if (__ldg(&d[mid].tile_begin) <= t) lo = mid + 1;
        else hi = mid;
    }
    return lo - 1;
}

// lo = x - (x with the low 13 mantissa bits cleared); exact in fp32
__device__ __forceinline__ float4 split_lo(float4 x) {
    float4 r;
    r.x = x.x - __uint_as_float(__float_as_uint(x.x) & 0xFFFFE000u);
    r.y = x.y - __uint_as_float(__float_as_uint(x.y) & 0xFFFFE000u);
    r.z = x.z - __uint_as_float(__float_as_uint(x.z) & 0xFFFFE000u);
    r.w = x.w - __uint_as_float(__float_as_uint(x.w) & 0xFFFFE000u);
    return r;
}

}  // namespace tc

template <int SPLIT>
__global__ void __launch_bounds__(tc::kThreads, 1)
    k_sgemm_tc(const GemmDesc* __restrict__ descs, int n, const uint8_t* __restrict__ maps, uint32_t total) {
    using namespace tc;
    constexpr int ST = Cfg<SPLIT>::kStages;
    constexpr int SB = Cfg<SPLIT>::kStageBytes;
    extern __shared__ uint8_t smem_raw[];
    uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
    uint64_t* bars = reinterpret_cast<uint64_t*>(smem + ST * SB);
    uint64_t* full = bars;            // [ST]  TMA landed
    uint64_t* empty = bars + ST;      // [ST]  MMAs done reading the stage
    uint64_t* conv = bars + 2 * ST;   // [ST]  lo tiles written (SPLIT = 3)
    uint64_t* acc_full = bars + 3 * ST;   // [2]
    uint64_t* acc_empty = bars + 3 * ST + 2;  // [2]
    uint32_t* tmem_base_slot = reinterpret_cast<uint32_t*>(bars + 3 * ST + 4);

    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x == 0) {
        for (int s = 0; s < ST; ++s) {
            mbar_init(&full[s], 1);
            mbar_init(&empty[s], 1);
            mbar_init(&conv[s], 2);
        }
        for (int a = 0; a < 2; ++a) {
            mbar_init(&acc_full[a], 1);
            mbar_init(&acc_empty[a], 4);
        }
        mbar_fence_init();
    }
    if (warp == 1) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_base_slot)),
                     "n"(kTmemCols)
                     : "memory");
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
    }
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem_base = *tmem_base_slot;

    auto stage_ptr = [&](int s) { return smem + (size_t)s * SB; };

    if (warp == 0) {
        // ------------------------------------------------------------ TMA producer
        if (lane == 0) {
            uint32_t it = 0;
            int last = -1;
            for (uint32_t t = blockIdx.x; t < total; t += gridDim.x) {
                const int v = find_tile_owner(descs, n, t);
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
                const int KB = (g.K + BK - 1) / BK;
                for (int kb = 0; kb < KB; ++kb, ++it) {
                    const int s = it % ST;
                    const uint32_t ph = (it / ST) & 1;
                    mbar_wait(&empty[s], ph ^ 1);
                    uint8_t* sp = stage_ptr(s);
                    mbar_expect_tx(&full[s], kStageA + kStageB);
                    tma_load_2d(sp, mA, kb * BK, tm * BM, &full[s]);
#pragma unroll
                    for (int j = 0; j < BN / 32; ++j)
                        tma_load_2d(sp + kStageA + j * (BK * 32 * 4), mB, tn * BN + j * 32, kb * BK, &full[s]);
                }
            }
        }
    } else if (warp == 1) {
        // ------------------------------------------------------------ MMA issuer
        uint32_t it = 0, tile_i = 0;
        for (uint32_t t = blockIdx.x; t < total; t += gridDim.x, ++tile_i) {
            const int v = find_tile_owner(descs, n, t);
            const int KB = (descs[v].K + BK - 1) / BK;
            const int a = tile_i & 1;
            const uint32_t aph = (tile_i >> 1) & 1;
            mbar_wait(&acc_empty[a], aph ^ 1);
            tc_fence_after();
            const uint32_t tmem_d = tmem_base + (uint32_t)(a * BN);
            for (int kb = 0; kb < KB; ++kb, ++it) {
                const int s = it % ST;
                const uint32_t ph = (it / ST) & 1;
                if (SPLIT == 1) mbar_wait(&full[s], ph);
                else mbar_wait(&conv[s], ph);
                tc_fence_after();
                if (lane == 0) {
                    const uint32_t sa = smem_u32(stage_ptr(s));
                    const uint32_t sbh = sa + kStageA;
#pragma unroll
                    for (int kk = 0; kk < BK / 8; ++kk) {
                        // A: K-major SW128 rows of 128 B, 8-row groups 1024 B apart; K advance = 32 B
                        const uint64_t ah = make_desc(sa + kk * 32, 16, 1024);
                        // B: MN-major SW128, 32-col blocks of 32 k-rows (4 KiB); K advance = 8 rows
                        const uint64_t bh = make_desc(sbh + kk * 1024, BK * 32 * 4, 1024);
                        const uint32_t acc0 = (kb > 0 || kk > 0) ? 1u : 0u;
                        if (SPLIT == 3) {
                            const uint32_t sal = sa + kStageA + kStageB;
                            const uint32_t sbl = sal + kStageA;
                            const uint64_t al = make_desc(sal + kk * 32, 16, 1024);
                            const uint64_t bl = make_desc(sbl + kk * 1024, BK * 32 * 4, 1024);
                            mma_tf32(tmem_d, ah, bl, acc0);
                            mma_tf32(tmem_d, al, bh, 1u);
                            mma_tf32(tmem_d, ah, bh, 1u);
                        } else {
                            mma_tf32(tmem_d, ah, bh, acc0);
                        }
                    }
                    mma_commit(&empty[s]);
                    if (kb == KB - 1) mma_commit(&acc_full[a]);
                }
                __syncwarp();
            }
            if (KB == 0 && lane == 0) mbar_arrive(&acc_full[a]);  // K == 0: nothing to wait for
            __syncwarp();
        }
    } else if (warp < 4) {
        // ------------------------------------------------------------ lo converters (SPLIT 3)
        if (SPLIT == 3) {
            const int ct = threadIdx.x - 64;  // 0..63
            uint32_t it = 0;
            for (uint32_t t = blockIdx.x; t < total; t += gridDim.x) {
                const int v = find_tile_owner(descs, n, t);
                const int KB = (descs[v].K + BK - 1) / BK;
                for (int kb = 0; kb < KB; ++kb, ++it) {
                    const int s = it % ST;
                    const uint32_t ph = (it / ST) & 1;
                    mbar_wait(&full[s], ph);
                    const float4* src = reinterpret_cast<const float4*>(stage_ptr(s));
                    float4* dst = reinterpret_cast<float4*>(stage_ptr(s) + kStageA + kStageB);
                    constexpr int NV = (kStageA + kStageB) / 16;  // 3072 float4
#pragma unroll 4
                    for (int i = ct; i < NV; i += 64) dst[i] = split_lo(src[i]);
                    fence_proxy_async();
                    __syncwarp();
                    if (lane == 0) mbar_arrive(&conv[s]);
                }
            }
        }
    } else {
        // ------------------------------------------------------------ epilogue (warps 4-7)
        const int q = warp & 3;  // TMEM lane quarter
        uint32_t tile_i = 0;
        for (uint32_t t = blockIdx.x; t < total; t += gridDim.x, ++tile_i) {
            const int v = find_tile_owner(descs, n, t);
            const GemmDesc& g = descs[v];
            const uint32_t lt = t - g.tile_begin;
            const int tm = lt / g.tiles_n, tn = lt % g.tiles_n;
            const int a = tile_i & 1;
            const uint32_t aph = (tile_i >> 1) & 1;
            mbar_wait(&acc_full[a], aph);
            tc_fence_after();
            const int row = tm * BM + q * 32 + lane;
            const bool row_ok = row < g.M;
            float* crow = g.C + (size_t)(row_ok ? row : 0) * g.N;
            const float alpha = g.alpha, beta = g.beta;
            const bool kzero = g.K == 0;
#pragma unroll 1
            for (int c0 = 0; c0 < BN; c0 += 32) {
                uint32_t r[32];
                tmem_ld32(tmem_base + ((uint32_t)(q * 32) << 16) + (uint32_t)(a * BN + c0), r);
                const int col0 = tn * BN + c0;
                if (!row_ok) continue;
#pragma unroll
                for (int j = 0; j < 32; j += 4) {
                    const int c = col0 + j;
                    if (c >= g.N) break;
                    float4 o;
                    o.x = kzero ? 0.f : alpha * __uint_as_float(r[j + 0]);
                    o.y = kzero ? 0.f : alpha * __uint_as_float(r[j + 1]);
                    o.z = kzero ? 0.f : alpha * __uint_as_float(r[j + 2]);
                    o.w = kzero ? 0.f : alpha * __uint_as_float(r[j + 3]);
                    float4* dst = reinterpret_cast<float4*>(crow + c);
                    if (beta != 0.f) {
                        const float4 old = *dst;
                        o.x = __fmaf_rn(beta, old.x, o.x);
                        o.y = __fmaf_rn(beta, old.y, o.y);
                        o.z = __fmaf_rn(beta, old.z, o.z);
                        o.w = __fmaf_rn(beta, old.w, o.w);
                    }
                    *dst = o;
                }
            }
            tc_fence_before();
            __syncwarp();
            if (lane == 0) mbar_arrive(&acc_empty[a]);
        }
    }
    // ---------------------------------------------------------------- teardown
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    if (warp == 1) {
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem_base), "n"(kTmemCols)
                     : "memory");
    }
}

static bool g_attr_set[2][64] = {};

template <int SPLIT>
static cudaError_t launch_tc(const GemmDesc* descs, int n, const void* maps, uint32_t total, int grid,
                             cudaStream_t s) {
    int dev = 0;
    cudaGetDevice(&dev);
    const int si = SPLIT == 1 ? 0 : 1;
    if (dev < 64 && !g_attr_set[si][dev]) {
        cudaError_t e = cudaFuncSetAttribute(k_sgemm_tc<SPLIT>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                             (int)tc::Cfg<SPLIT>::kSmem);
        if (e) return e;
        g_attr_set[si][dev] = true;
    }
    k_sgemm_tc<SPLIT><<<grid, tc::kThreads, tc::Cfg<SPLIT>::kSmem, s>>>(descs, n, reinterpret_cast<const uint8_t*>(maps),
                                                                       total);
    return cudaGetLastError();
}

cudaError_t launch_sgemm_tf32(const GemmDesc* descs, int n, const void* maps, uint32_t total, int grid,
                              cudaStream_t s) {
    return launch_tc<1>(descs, n, maps, total, grid, s);
}

cudaError_t launch_sgemm_3xtf32(const GemmDesc* descs, int n, const void* maps, uint32_t total, int grid,
                                cudaStream_t s) {
    return launch_tc<3>(descs, n, maps, total, grid, s);
}

}  // namespace svp

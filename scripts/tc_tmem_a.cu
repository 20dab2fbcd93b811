// tc_tmem_a.cu -- probe (debug tool, not part of libsvp): tcgen05.mma kind::f16 with the A
// operand in TMEM.  A values are written into TMEM columns [256, 256+ncolA) with
// tcgen05.st.32x32b (warp w -> lanes 32w..32w+31, thread = lane = row), B comes from a
// host-built smem image (K-major SW128 bf16), D (128 x 256 fp32) is dumped.
#include <cuda_runtime.h>
#include <stdint.h>

#include "../paper_conf_dac_jungc15_b200/csrc/kernels/common.cuh"

using namespace svp;

__global__ void k_probe_ta(const uint4* img, const uint32_t* Aw, int ncolA, const uint64_t* bdescs, float* D,
                           uint32_t idesc, int nk, int acol_step) {
    extern __shared__ __align__(1024) uint8_t sm[];
    uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(sm) + 1023) & ~uintptr_t(1023));
    __shared__ uint32_t tbase;
    __shared__ __align__(8) uint64_t bar;
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    uint4* s4 = reinterpret_cast<uint4*>(smem);
    for (int i = tid; i < 65536 / 16; i += blockDim.x) s4[i] = img[i];
    if (warp == 0) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(smem_u32(&tbase)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    if (tid == 0) {
        mbar_init(&bar, 1);
        mbar_fence_init();
    }
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const uint32_t t = tbase;
    const uint32_t lane_base = t + ((uint32_t)(warp * 32) << 16);
    // A -> TMEM columns 256.. (one 32-bit column per store), D zeroed with a NaN marker
    for (int c = 0; c < ncolA; ++c)
        asm volatile("tcgen05.st.sync.aligned.32x32b.x1.b32 [%0], {%1};" ::"r"(lane_base + 256 + c),
                     "r"(Aw[(warp * 32 + lane) * ncolA + c]));
    for (int c0 = 0; c0 < 256; c0 += 8)
        asm volatile("tcgen05.st.sync.aligned.32x32b.x8.b32 [%0], {%1,%1,%1,%1,%1,%1,%1,%1};" ::"r"(lane_base + c0),
                     "r"(0x7fc00000u));
    asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const uint32_t base = smem_u32(smem);
    if (tid == 0) {
        for (int kk = 0; kk < nk; ++kk) {
            uint64_t bd = bdescs[kk] + ((base >> 4) & 0x3FFF);
            uint32_t acc = kk > 0;
            asm volatile(
                "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                "tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n\t}" ::"r"(t),
                "r"(t + 256 + kk * acol_step), "l"(bd), "r"(idesc), "r"(acc)
                : "memory");
        }
        asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
                         smem_u32(&bar))
                     : "memory");
    }
    __syncwarp();
    mbar_wait(&bar, 0);
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    for (int c0 = 0; c0 < 256; c0 += 8) {
        uint32_t r[8];
        asm volatile("tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];\n\t"
                     "tcgen05.wait::ld.sync.aligned;"
                     : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7])
                     : "r"(lane_base + c0));
        for (int j = 0; j < 8; ++j) D[(warp * 32 + lane) * 256 + c0 + j] = __uint_as_float(r[j]);
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(t));
}

extern "C" int tc_probe_ta(const void* img, const uint32_t* Aw, int ncolA, const uint64_t* bdescs, float* D,
                           uint32_t idesc, int nk, int acol_step) {
    cudaFuncSetAttribute(k_probe_ta, cudaFuncAttributeMaxDynamicSharedMemorySize, 66 * 1024);
    k_probe_ta<<<1, 128, 66 * 1024>>>(reinterpret_cast<const uint4*>(img), Aw, ncolA, bdescs, D, idesc, nk,
                                      acol_step);
    return (int)cudaDeviceSynchronize();
}

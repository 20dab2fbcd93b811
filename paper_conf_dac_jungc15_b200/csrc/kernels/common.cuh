// common.cuh -- device helpers shared by the sm_100a guest kernels (internal).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "../tables.h"

namespace svp {

// Segment owning launch tile t: the last segment with tile_begin <= t.  Empty
// segments share their tile_begin with the next one, so upper_bound - 1 lands on the
// segment that actually owns the tile.  Plain loads: `segs` is a global table or the
// address of a __grid_constant__ SegParam (table_mode param).
__device__ __forceinline__ int find_seg(const SegDesc* __restrict__ segs, int nsegs, uint32_t t) {
    int lo = 0, hi = nsegs;
    while (lo < hi) {
        int mid = (lo + hi) >> 1;
        if (segs[mid].tile_begin <= t) lo = mid + 1;
        else hi = mid;
    }
    return lo - 1;
}

// tile_range (element range of a segment's local tile) lives in tables.h: the host-side
// layout (seg_layout) and the kernels share it, and tests/tile_check.cpp checks both on CPU.

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

// ---- mbarrier / TMA (sm_90+ PTX, used on sm_100a)
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_fence_init() {
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
                 : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ bool mbar_try_wait(uint32_t addr, uint32_t parity) {
    uint32_t ok;
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(ok)
        : "r"(addr), "r"(parity)
        : "memory");
    return ok != 0;
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
    uint32_t a = smem_u32(bar);
    while (!mbar_try_wait(a, parity)) {
    }
}
__device__ __forceinline__ void tma_load_2d(void* smem_dst, const void* tmap, int32_t c0, int32_t c1, uint64_t* bar) {
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];" ::"r"(
            smem_u32(smem_dst)),
        "l"(tmap), "r"(c0), "r"(c1), "r"(smem_u32(bar))
        : "memory");
}
__device__ __forceinline__ void prefetch_tmap(const void* tmap) {
    asm volatile("prefetch.tensormap [%0];" ::"l"(tmap) : "memory");
}

}  // namespace svp

// sgemm_tf32.cu -- grouped (coalesced) SGEMM on the 5th-gen tensor cores (tcgen05, sm_100a).
//
// C_v = alpha_v A_v B_v + beta_v C_v for every VP of a Kernel Match group, one persistent
// launch (Kernel Coalescing; the paper's matmul guest, Table 1).
//
//  SPLIT = 1  "sgemm_tf32": one kind::tf32 MMA per k-step; the tensor core reads fp32
//             operands as TF32 (low 13 mantissa bits ignored).  Own tolerance 2e-3.
//  SPLIT = 3  "3xTF32" (sgemm_impl SVP_SGEMM_3XTF32): x = hi + lo, hi = x with the low 13
//             bits cleared (exactly what the tensor core reads from x) and lo = x - hi
//             (exact in fp32); per k-step D += A_hi B_lo + A_lo B_hi + A_hi B_hi.  The
//             dropped A_lo B_lo and the truncation of lo are each < 2^-20 |a||b|, so the
//             product error is < 3 * 2^-20 |a||b| ~ 2.9e-6 |a||b|, inside the fp32 bound
//             1e-5 (|A||B|)_ij (R10).
//  SPLIT = 2  "TF32 + 2xBF16" (sgemm_impl SVP_SGEMM_TF32BF16): x = h + l with h = x rounded
//             to TF32 (the converters write h back over the raw TMA tile) and l = x - h
//             (exact, |l| <= 2^-11 |x|).  The main product A_h B_h is a kind::tf32 MMA on the
//             rounded tiles (exact products); the two cross terms only need ~8 significant
//             bits, so they run as kind::f16 BF16 MMAs on converter-written bf16 tiles:
//             D += bf(A_h) bf(B_l) + bf(A_l) bf(B_h).  Per 16 k: 2 TF32 + 2 BF16 MMAs (a BF16
//             K16 MMA costs what a TF32 K8 one does) = 4 MMA slots instead of 6.  Error per
//             product (bf16 unit roundoff 2^-8): 2 (2^-8 + 2^-8) 2^-11 + 2^-22 (dropped l l)
//             = 2^-17 + 2^-22 ~ 7.9e-6 |a||b|, inside the 1e-5 (|A||B|)_ij bound (DESIGN.md
//             R19); integer inputs (|x| <= 2^11) stay exact (l = 0).
//
//  SPLIT = 4  the SPLIT 2 arithmetic with the A-side bf16 operands in TMEM: converters
//             tcgen05.st bf(A_hi) / bf(A_lo) (lane = row, column = k pair) into a TMEM ring
//             next to the accumulator and the BF16 MMAs read A from TMEM ([a_tmem] form).
//             Removes 8 KiB of converter smem writes and 8 KiB of MMA smem reads per stage
//             (the pair kernel is shared-memory bound: LSU + tensor-core smem wavefronts ~96 %
//             of the data pipe); the price is a single TMEM accumulator (2x256 + the ring
//             would exceed 512 columns), so a tile's epilogue no longer overlaps the next
//             tile's MMAs.
//
// CG = 2 (CTA pair, cta_group::2; SPLIT 2, 3, 4): a cluster of 2 CTAs on one TPC computes a
// 256 x 256 tile with M256 N256 MMAs issued by the leader CTA.  Each CTA stages its own
// 128 rows of A and 128 columns of B (half the operand bytes per SM: the per-SM shared-
// memory traffic -- TMA writes + converter reads/writes -- is what bounds the single-CTA
// split kernels, profiles/r01), holds 128 rows x 256 columns of the accumulator in its
// own TMEM, and runs its own converters and epilogue.  Cross-CTA signalling: converters
// arrive on the leader's conv barrier (mbarrier.arrive.release.cluster), the leader's
// commits multicast to both CTAs' empty / acc_full barriers, the peer's epilogue arrives on
// the leader's acc_empty.
//
// Operand layouts in shared memory:
//   A (row-major M x K = K-major, TMA): 64-B rows of 16 k, SWIZZLE_64B (SBO 512).
//   B (row-major K x N = MN-major, TMA): 32-n x 16-k blocks of 128-B rows with the 32-B-atom
//     128-B swizzle (TMA CU_TENSOR_MAP_SWIZZLE_128B_ATOM_32B = UMMA SWIZZLE_128B_BASE32B;
//     LBO = 2 KiB between 32-n blocks, SBO = 512 B between 4-k groups).  A tf32 MMA with an
//     MN-major B in the plain 16-B-atom SW128 layout reads zeros on B200 (scripts/
//     tc_probe.py E1); the 32-B-atom layout is the one the hardware accepts (E6).
//   SPLIT 3 lo tiles: element-wise, same layouts as hi.
//   SPLIT 2 bf16 tiles: A K-major SWIZZLE_NONE (8x16-B core matrices, LBO 128 B between the
//     two k halves, SBO 256 B between 8-row groups); B MN-major SWIZZLE_128B (64-n x 8-k
//     atoms, LBO 2 KiB between n atoms, SBO 1 KiB between k groups).  The converter lane
//     mappings keep every LDS/STS.128 on the minimum 4 wavefronts (ncu: 0 excessive).
//
// Roles (persistent static tile walk, 448 threads per CTA):
//   warp 0        TMA producer: A 128x16 + B 16x(256/CG) per k-block into the operand ring.
//   warp 1        TMEM allocator (512 cols = 2 accumulators of 128x256 fp32) + MMA issuer
//                 (leader CTA only for CG 2): tcgen05.mma ... commit to empty / acc_full.
//   warps 2,3,8-13 converters (SPLIT 2/3), fence.proxy.async, arrive on conv.
//   warps 4-7     epilogue: tcgen05.ld 32x32b.x32 (warp w%4 owns TMEM lanes = tile rows
//                 32(w%4)..+31), alpha*acc (+ beta*C), 128-bit stores; two TMEM
//                 accumulators let tile i's epilogue overlap tile i+1's MMAs.
//
// NH = 2 (wide, SPLIT 2 pairs): 256 x 512 tiles, 576 threads.  Each CTA stages 256 B
// columns (two 128-column halves); per k-step the leader issues the SPLIT 2 MMAs once per
// 256-column half into TMEM columns [0,256) / [256,512) -- the A tiles (and their bf16
// conversions) serve both halves, halving the A-side conversion and L2 -> SM traffic per
// flop (profiles/r01/power: the split SGEMM runs at the power cap, so energy per flop sets
// its speed).  Warps 4-7 drain half 0 and warps 14-17 half 1, each half with its own
// acc_full / acc_empty barrier, so the next tile's half-0 MMAs start while half 1 drains.
// The executor uses NH 2 when a launch has >= 2 waves of wide tiles (SVP_TC_WIDE).
//
// Teardown: the producer waits for the release of the last use of every stage before the
// CTA exits (tcgen05.commit arrives land asynchronously and must not reach the shared
// memory of the next CTA scheduled on this SM).
#include <cuda.h>
#include <stdlib.h>

#include <algorithm>

#include <atomic>

#include "../launch.h"
#include "common.cuh"

namespace svp {

#ifndef SVP_PAIR_STAGES
#define SVP_PAIR_STAGES 6
#endif

namespace tc {

constexpr int BM = kTf32BM, BN = kTf32BN, BK = kTf32BK;  // 128 x 256 x 16 per CTA
constexpr int kConvWarps = 8;                              // warps 2,3 and 8..13
constexpr int kConvThreads = kConvWarps * 32;
constexpr int kThreads = (8 + kConvWarps - 2) * 32;        // 448 (+128 for NH 2)
constexpr int kTileA = BM * BK * 4;                        // 8 KiB
constexpr int kBBlock = BK * 128;                          // one 32-n block of B: 2 KiB
constexpr int kTmemCols = 512;
constexpr int kTileA16 = BM * BK * 2;                      // 4 KiB

template <int SPLIT, int CG, int NH = 1>
struct Cfg {
    // NH = 2 ("wide", SPLIT 2 pairs only): a pair computes 256 x 512, two 256-column MMA
    // halves per k-step on the same A tiles; the two TMEM accumulators are the two halves
    // of ONE tile (no double buffer), each drained by its own 4 epilogue warps.
    static_assert(NH == 1 || (SPLIT == 2 && CG == 2), "wide tiles: split-BF16 CTA pairs only");
    static constexpr int kThreads = tc::kThreads + (NH - 1) * 128;
    static constexpr int kBN = BN / CG * NH;               // B columns staged per CTA
    static constexpr int kTileB = BK * kBN * 4;            // 16 KiB (CG 1) / 8 KiB (CG 2)
    static constexpr int kTileB16 = BK * kBN * 2;
    // stage: A | B [| A_lo | B_lo]   (SPLIT 2: A | B | bf A_hi | bf A_lo | bf B_hi | bf B_lo;
    // SPLIT 4: A | B | bf B_hi | bf B_lo, the A-side bf16 tiles live in TMEM)
    static constexpr int kStageBytes = SPLIT == 4 ? kTileA + kTileB + 2 * kTileB16
                                                  : (kTileA + kTileB) * (SPLIT == 1 ? 1 : 2);
    static constexpr int kStages = SPLIT == 1 ? 8
                                 : SPLIT == 4 ? (CG == 2 ? 8 : 5)
                                 : NH == 2    ? 4
                                              : (CG == 2 ? SVP_PAIR_STAGES : 4);
    static constexpr int kAcc = (SPLIT == 4 || NH == 2) ? 1 : 2;  // accumulator sets (NH x 256 cols each)
    static constexpr int kTaCol = 256;                     // SPLIT 4: A ring, 16 cols per stage
    static_assert(SPLIT != 4 || kTaCol + 16 * kStages <= kTmemCols, "TMEM");
    // TMA epilogue (beta == 0) and K-chunk folds (R23): 4 KiB of staging per epilogue warp (two
    // 32 x 16 fp32 half-slabs, 64-B swizzled), written into C by TMA store / reduce-add
    static constexpr int kEpiWarps = 4 * NH;
    static constexpr size_t kStagingOff = (size_t)kStages * kStageBytes;  // 1024-B aligned
    static constexpr size_t kBarOff = kStagingOff + (size_t)kEpiWarps * 4096;
    static constexpr size_t kSmem = 1024 + kBarOff + 256;
    static constexpr int kMmaM = BM * CG;
    static_assert(kSmem <= 227 * 1024, "shared memory");
};

// SM100 shared-memory matrix descriptor: start>>4 [0,14), LBO>>4 [16,30), SBO>>4 [32,46),
// version 1 [46,48), base offset 0, layout [61,64)
__device__ __forceinline__ uint64_t make_desc(uint32_t saddr, uint32_t lbo, uint32_t sbo, uint32_t layout) {
    return (uint64_t)((saddr >> 4) & 0x3FFF) | ((uint64_t)((lbo >> 4) & 0x3FFF) << 16) |
           ((uint64_t)((sbo >> 4) & 0x3FFF) << 32) | ((uint64_t)1 << 46) | ((uint64_t)layout << 61);
}
// A: K-major, SWIZZLE_64B (4): LBO unused (1), SBO 512 B
__device__ __forceinline__ uint64_t desc_a(uint32_t saddr) { return make_desc(saddr, 16, 8 * BK * 4, 4); }
// B: MN-major, SWIZZLE_128B_BASE32B (1): LBO = 32-n block stride, SBO = 4-k group stride
__device__ __forceinline__ uint64_t desc_b(uint32_t saddr) { return make_desc(saddr, kBBlock, 512, 1); }
// SPLIT 2 bf16 tiles.  A: K-major, no swizzle, [8-row group][k half][8 rows][16 B]
__device__ __forceinline__ uint64_t desc_a16(uint32_t saddr) { return make_desc(saddr, 128, 256, 0); }
// B: MN-major, SWIZZLE_128B (2), [64-n atom][8-k group][8 k rows][128 B]
__device__ __forceinline__ uint64_t desc_b16(uint32_t saddr) { return make_desc(saddr, 2048, 1024, 2); }

// instruction descriptors: D f32 [4,6)=1, A/B format [7,10)/[10,13) (kind::tf32: TF32 = 2;
// kind::f16: BF16 = 1), A K-major (bit 15 = 0), B MN-major (bit 16 = 1), N>>3 at [17,23),
// M>>4 at [24,29)
template <int M>
struct Idesc {
    static constexpr uint32_t tf32 = (1u << 4) | (2u << 7) | (2u << 10) | (1u << 16) | ((uint32_t)(BN >> 3) << 17) |
                                     ((uint32_t)(M >> 4) << 24);
    static constexpr uint32_t bf16 = (1u << 4) | (1u << 7) | (1u << 10) | (1u << 16) | ((uint32_t)(BN >> 3) << 17) |
                                     ((uint32_t)(M >> 4) << 24);
};

template <int CG>
__device__ __forceinline__ void mma_tf32(uint32_t tmem_d, uint64_t adesc, uint64_t bdesc, uint32_t accum) {
    if constexpr (CG == 1)
        asm volatile(
            "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
            "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem_d),
            "l"(adesc), "l"(bdesc), "r"(Idesc<BM>::tf32), "r"(accum)
            : "memory");
    else
        asm volatile(
            "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
            "tcgen05.mma.cta_group::2.kind::tf32 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem_d),
            "l"(adesc), "l"(bdesc), "r"(Idesc<2 * BM>::tf32), "r"(accum)
            : "memory");
}
// kind::f16 with A from TMEM (lane = row, 32-bit column c = k pair {2c, 2c+1}, low half = even
// k: scripts/tc_tmem_a.py)
template <int CG>
__device__ __forceinline__ void mma_bf16_ta(uint32_t tmem_d, uint32_t tmem_a, uint64_t bdesc, uint32_t accum) {
    if constexpr (CG == 1)
        asm volatile(
            "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
            "tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n\t}" ::"r"(tmem_d),
            "r"(tmem_a), "l"(bdesc), "r"(Idesc<BM>::bf16), "r"(accum)
            : "memory");
    else
        asm volatile(
            "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
            "tcgen05.mma.cta_group::2.kind::f16 [%0], [%1], %2, %3, p;\n\t}" ::"r"(tmem_d),
            "r"(tmem_a), "l"(bdesc), "r"(Idesc<2 * BM>::bf16), "r"(accum)
            : "memory");
}
__device__ __forceinline__ void tmem_st4(uint32_t taddr, const uint4& v) {
    asm volatile("tcgen05.st.sync.aligned.32x32b.x4.b32 [%0], {%1,%2,%3,%4};" ::"r"(taddr), "r"(v.x), "r"(v.y),
                 "r"(v.z), "r"(v.w)
                 : "memory");
}

template <int CG>
__device__ __forceinline__ void mma_bf16(uint32_t tmem_d, uint64_t adesc, uint64_t bdesc, uint32_t accum) {
    if constexpr (CG == 1)
        asm volatile(
            "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
            "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem_d),
            "l"(adesc), "l"(bdesc), "r"(Idesc<BM>::bf16), "r"(accum)
            : "memory");
    else
        asm volatile(
            "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
            "tcgen05.mma.cta_group::2.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem_d),
            "l"(adesc), "l"(bdesc), "r"(Idesc<2 * BM>::bf16), "r"(accum)
            : "memory");
}
// MMA completion -> mbarrier (CG 2: the same barrier offset in both CTAs of the pair)
template <int CG>
__device__ __forceinline__ void mma_commit(uint64_t* bar) {
    if constexpr (CG == 1)
        asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
                         smem_u32(bar))
                     : "memory");
    else
        asm volatile(
            "tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;" ::"r"(
                smem_u32(bar)),
            "h"((uint16_t)3)
            : "memory");
}
__device__ __forceinline__ void tc_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void fence_proxy_async() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }

// ---- cluster helpers (CTA pair)
__device__ __forceinline__ uint32_t cluster_rank() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
    return r;
}
__device__ __forceinline__ void cluster_sync_all() {
    asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
// shared::cluster address of `p` (a local shared variable) in CTA `rank` of the cluster
__device__ __forceinline__ uint32_t map_to(const void* p, uint32_t rank) {
    uint32_t r;
    asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(smem_u32(p)), "r"(rank));
    return r;
}
// Remote arrive with the default (.release.cta) semantics, as CUTLASS's ClusterBarrier
// does: a .release.cluster arrive costs a cluster-scope memory barrier per call (ncu:
// stall_membar dominated the converters and halved the pair kernel's throughput).  The
// data it publishes is read by the tensor core through the async proxy after
// fence.proxy.async, like the single-CTA path.
__device__ __forceinline__ void mbar_arrive_cluster(uint32_t cluster_addr) {
    asm volatile("mbarrier.arrive.shared::cluster.b64 _, [%0];" ::"r"(cluster_addr) : "memory");
}
__device__ __forceinline__ void mbar_wait_cluster(uint64_t* bar, uint32_t parity) { mbar_wait(bar, parity); }

__device__ __forceinline__ void tmem_ld32(uint32_t taddr, uint32_t (&r)[32]) {
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x32.b32 "
        "{%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
        "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];\n\t"
        "tcgen05.wait::ld.sync.aligned;"
        : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
          "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]),
          "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]),
          "=r"(r[24]), "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
        : "r"(taddr)
        : "memory");
}

__device__ __forceinline__ void tmem_ld8(uint32_t taddr, uint32_t (&r)[8]) {
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];\n\t"
        "tcgen05.wait::ld.sync.aligned;"
        : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7])
        : "r"(taddr)
        : "memory");
}
__device__ __forceinline__ void tmem_ld16(uint32_t taddr, uint32_t (&r)[16]) {
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x16.b32 "
        "{%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];\n\t"
        "tcgen05.wait::ld.sync.aligned;"
        : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
          "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
        : "r"(taddr)
        : "memory");
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

__device__ __forceinline__ float lo_part(float x) { return x - __uint_as_float(__float_as_uint(x) & 0xFFFFE000u); }
__device__ __forceinline__ float4 lo_part4(float4 x) {
    return make_float4(lo_part(x.x), lo_part(x.y), lo_part(x.z), lo_part(x.w));
}

// bf16x2 of (a -> low half, b -> high half), round to nearest even (the low parts: a NaN or
// infinite l -- from an Inf / NaN operand, or a head that rounded past FLT_MAX -- must stay
// non-finite so the output's accumulator turns NaN and the epilogue recomputes it, R20)
__device__ __forceinline__ uint32_t bf2(float a, float b) {
    uint32_t r;
    asm("cvt.rn.bf16x2.f32 %0, %1, %2;" : "=r"(r) : "f"(b), "f"(a));
    return r;
}
// the heads: .satfinite (free in SASS: F2FP.SATFINITE) -- a finite TF32 head beyond the bf16
// range (|h| >= (2 - 2^-8) 2^127) becomes +-max_bf16 instead of +-Inf, so a finite operand
// near FLT_MAX cannot turn a cross term into an infinity with a finite accumulator
__device__ __forceinline__ uint32_t bf2s(float a, float b) {
    uint32_t r;
    asm("cvt.rn.satfinite.bf16x2.f32 %0, %1, %2;" : "=r"(r) : "f"(b), "f"(a));
    return r;
}

// SPLIT 2 / 4 head: h = x rounded to TF32 (nearest, ties away: |x - h| <= 2^-11 |x|), written
// back over the raw tile the TF32 MMA reads; the cross terms get bf16(h) and bf16(x - h).
// (A truncated head -- what the tensor core reads from an untouched tile -- leaves |l| up to
// 2^-10 |x| and a worst-case product error of 2^-16 + 2^-20 > 1e-5: tests/split_emulation.py.)
// |x| within 2^-12 of FLT_MAX rounds to inf (then l = -inf): the epilogue's exact recompute
// of NaN outputs covers it (R20).
__device__ __forceinline__ float rna_tf32(float x) {
    return __uint_as_float((__float_as_uint(x) + 0x1000u) & 0xFFFFE000u);
}
__device__ __forceinline__ float4 rna_tf32_4(float4 x) {
    return make_float4(rna_tf32(x.x), rna_tf32(x.y), rna_tf32(x.z), rna_tf32(x.w));
}
__device__ __forceinline__ void split8_given(const float4& p, const float4& q, const float4& ph, const float4& qh,
                                             uint4& hb, uint4& lb) {
    const float x[8] = {p.x, p.y, p.z, p.w, q.x, q.y, q.z, q.w};
    const float h[8] = {ph.x, ph.y, ph.z, ph.w, qh.x, qh.y, qh.z, qh.w};
    uint32_t hh[4], ll[4];
#pragma unroll
    for (int i = 0; i < 4; ++i) {
        hh[i] = bf2s(h[2 * i], h[2 * i + 1]);
        ll[i] = bf2(x[2 * i] - h[2 * i], x[2 * i + 1] - h[2 * i + 1]);
    }
    hb = make_uint4(hh[0], hh[1], hh[2], hh[3]);
    lb = make_uint4(ll[0], ll[1], ll[2], ll[3]);
}

}  // namespace tc

// One output of C = alpha A B + beta C_old exactly as the definition reads it (PAPER.md
// Table 1's matmul at BASELINE.json's fp32; R20): products in fp64 (exact for fp32
// operands), summed in ascending k in fp64 with IEEE +/x (no contraction), alpha * acc +
// beta * c_old in fp64, one rounding.  The rare path of the tensor-core epilogue for outputs
// whose accumulator came out NaN -- an Inf or NaN operand, or a finite one at the top of the
// fp32 range -- so their Inf / NaN / finite value is the IEEE one.
__device__ __forceinline__ float exact_element(const GemmDesc& g, int i, int j, float c_old) {
    const float* a = g.A + (size_t)i * g.lda;
    const float* b = g.B + j;
    const size_t ldb = (size_t)g.ldb;
    double acc = 0.0;
#pragma unroll 1
    for (int k = g.K; k > 0; --k, ++a, b += ldb) acc = __dadd_rn(acc, __dmul_rn((double)__ldg(a), (double)__ldg(b)));
    double r = __dmul_rn((double)g.alpha, acc);
    if (g.beta != 0.f) r = __dadd_rn(r, __dmul_rn((double)g.beta, (double)c_old));
    return (float)r;
}

// K-chunked accumulation (R23): the tcgen05 fp32 accumulation loses magnitude
// (measured -1.66e-8 relative per accumulating MMA), so a tile's K range is cut into chunks
// of `kchunk` 16-k blocks, each accumulated from zero in its own TMEM accumulator (the two
// accumulators ping-pong between chunks as they do between tiles) and folded into C by the
// epilogue with IEEE fp32 adds (chunk 0 stores alpha * acc, later chunks add alpha * acc with
// red.global.add.v4.f32): the output's relative bias is then that of ONE chunk, whatever K
// is.  Only for beta == 0 (a beta != 0 job keeps C_old for its exact NaN path; the executor
// routes those with K > the chunk to the FFMA kernel).  Producer, MMA issuer and epilogue all
// walk the same (tile, chunk) units.
// L2 policy of the epilogue's C writes: a partial sum another K chunk will fold into stays in
// L2 (evict_last -- the 74 pairs' in-flight tiles are ~39 MB), a final value streams out
// (evict_first)
__device__ __forceinline__ uint64_t l2_policy(bool keep) {
    uint64_t pol;
    if (keep) asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol));
    else asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
    return pol;
}
__device__ __forceinline__ void tma_store_2d(const void* tmap, int32_t c0, int32_t c1, const void* smem_src,
                                             uint64_t pol) {
    asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group.L2::cache_hint [%0, {%1, %2}], [%3], %4;" ::"l"(
                     tmap),
                 "r"(c0), "r"(c1), "r"(smem_u32(smem_src)), "l"(pol)
                 : "memory");
}
__device__ __forceinline__ void tma_reduce_add_2d(const void* tmap, int32_t c0, int32_t c1, const void* smem_src,
                                                  uint64_t pol) {
    asm volatile(
        "cp.reduce.async.bulk.tensor.2d.global.shared::cta.add.bulk_group.L2::cache_hint [%0, {%1, %2}], [%3], %4;" ::"l"(
            tmap),
        "r"(c0), "r"(c1), "r"(smem_u32(smem_src)), "l"(pol)
        : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
__device__ __forceinline__ void bulk_wait_read0() { asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory"); }
__device__ __forceinline__ void bulk_wait0() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }

__device__ __forceinline__ int tc_chunks(const GemmDesc& g, int KB, int kchunk) {
    return (kchunk > 0 && g.beta == 0.f && KB > kchunk) ? (KB + kchunk - 1) / kchunk : 1;
}
// flag in the kernel's kchunk argument above the 16-bit block count: the TMA epilogue frees the
// accumulator right after its last tcgen05.ld instead of after its last slab write
constexpr int kEpiEarlyRelease = 1 << 16;

template <int SPLIT, int CG, int NH>
__global__ void __launch_bounds__(tc::Cfg<SPLIT, CG, NH>::kThreads, 1)
    k_sgemm_tc(const GemmDesc* __restrict__ descs, int n, const uint8_t* __restrict__ maps, uint32_t total,
               int kchunk_flags, const uint8_t* __restrict__ cmaps) {
    using namespace tc;
    const int kchunk = kchunk_flags & 0xFFFF;
    const bool early_release = (kchunk_flags & kEpiEarlyRelease) != 0;
    using C = Cfg<SPLIT, CG, NH>;
    constexpr int TN = BN * NH;  // tile width in N per CTA pair (or CTA)
    constexpr int ST = C::kStages, SB = C::kStageBytes, TB = C::kTileB, TB16 = C::kTileB16;
    extern __shared__ uint8_t smem_raw[];
    // align to 1024 B (swizzle atoms) by offsetting smem_raw itself, so the compiler keeps
    // the shared address space and emits LDS/STS (not generic LD/ST) for the converters;
    // both CTAs of a pair get the same offsets (the leader's descriptors address both)
    uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
    uint64_t* bars = reinterpret_cast<uint64_t*>(smem + C::kBarOff);
    uint64_t* full = bars;               // [ST] this CTA's TMA A + B landed
    uint64_t* empty = bars + ST;         // [ST] MMAs done with the stage
    uint64_t* conv = bars + 2 * ST;      // [ST] (leader) both CTAs' converted tiles written
    uint64_t* acc_full = bars + 3 * ST;  // [2]
    uint64_t* acc_empty = acc_full + 2;  // [2] (leader) both CTAs' epilogues drained it
    uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(acc_empty + 2);

    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint32_t rank = CG == 2 ? cluster_rank() : 0;
    const bool leader = rank == 0;
    const uint32_t cl = blockIdx.x / CG, ncl = gridDim.x / CG;  // tile walk per CTA pair
    if (threadIdx.x == 0) {
        for (int s = 0; s < ST; ++s) {
            mbar_init(&full[s], 1);
            mbar_init(&empty[s], 1);
            mbar_init(&conv[s], kConvWarps * CG);
        }
        for (int a = 0; a < 2; ++a) {
            mbar_init(&acc_full[a], 1);
            mbar_init(&acc_empty[a], 4 * CG);
        }
        mbar_fence_init();
    }
    if (warp == 1) {
        if constexpr (CG == 1) {
            asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                             smem_u32(tmem_slot)),
                         "n"(kTmemCols)
                         : "memory");
            asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
        } else {
            asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                             smem_u32(tmem_slot)),
                         "n"(kTmemCols)
                         : "memory");
            asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;" ::: "memory");
        }
    }
    tc_fence_before();
    __syncthreads();
    if constexpr (CG == 2) cluster_sync_all();  // peer barriers initialised before any remote arrive
    tc_fence_after();
    const uint32_t tmem_base = *tmem_slot;

    auto stage = [&](int s) { return smem + (size_t)s * SB; };

    if (warp == 0) {
        // ------------------------------------------------------------ TMA producer
        if (lane == 0) {
            uint32_t it = 0;
            int last = -1;
            for (uint32_t t = cl; t < total; t += ncl) {
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
                const int m0 = tm * C::kMmaM + (int)rank * BM;
                // 32-n block j of this CTA: half h = j / 4 (NH 2) at columns h*256 + rank*128
                const int n0 = NH == 1 ? tn * BN + (int)rank * C::kBN : tn * TN + (int)rank * (BN / CG);
                const int KB = (g.K + BK - 1) / BK;
                for (int kb = 0; kb < KB; ++kb, ++it) {
                    const int s = it % ST;
                    const uint32_t ph = (it / ST) & 1;
                    mbar_wait(&empty[s], ph ^ 1);
                    uint8_t* sp = stage(s);
                    mbar_expect_tx(&full[s], kTileA + TB);
                    tma_load_2d(sp, mA, kb * BK, m0, &full[s]);
#pragma unroll
                    for (int j = 0; j < C::kBN / 32; ++j) {
                        const int col = NH == 1 ? n0 + j * 32 : n0 + (j >> 2) * BN + (j & 3) * 32;
                        tma_load_2d(sp + kTileA + j * kBBlock, mB, col, kb * BK, &full[s]);
                    }
                }
            }
            // Producer tail: the MMA issuer frees stages with tcgen05.commit, whose mbarrier
            // arrives land asynchronously when the MMAs complete (multicast into both CTAs
            // of a pair) -- possibly after the epilogue saw the last acc_full.  Wait for the
            // release of the last use of every stage, so no arrive can land in this SM's
            // shared memory after the CTA exited (it would corrupt whichever CTA of another
            // kernel got the memory next: seen as wrong hist256 counts in the cfg5 mix).
            for (uint32_t i = 0; i < (uint32_t)ST && i < it; ++i) {
                const uint32_t u = it - 1 - i;
                mbar_wait(&empty[u % ST], (u / ST) & 1);
            }
        }
    } else if (warp == 1) {
        // ------------------------------------------------------------ MMA issuer
        if (leader) {
            uint32_t it = 0, tile_i = 0;  // tile_i counts (tile, chunk) units
            for (uint32_t t = cl; t < total; t += ncl) {
              const int v = find_tile_owner(descs, n, t);
              const int KB = (descs[v].K + BK - 1) / BK;
              const int nch = tc_chunks(descs[v], KB, kchunk);
              for (int ck = 0; ck < nch; ++ck, ++tile_i) {
                const int kb0 = nch == 1 ? 0 : ck * kchunk, kb1 = nch == 1 ? KB : min(KB, kb0 + kchunk);
                const int a = tile_i % C::kAcc;
                const uint32_t aph = (tile_i / C::kAcc) & 1;
                if constexpr (CG == 2) mbar_wait_cluster(&acc_empty[a], aph ^ 1);
                else mbar_wait(&acc_empty[a], aph ^ 1);
                tc_fence_after();
                const uint32_t tmem_d = tmem_base + (uint32_t)(a * BN);
                for (int kb = kb0; kb < kb1; ++kb, ++it) {
                    const int s = it % ST;
                    const uint32_t ph = (it / ST) & 1;
                    if constexpr (CG == 2) {
                        mbar_wait_cluster(&conv[s], ph);  // implies both CTAs' TMA data landed
                    } else {
                        mbar_wait(&full[s], ph);
                        if (SPLIT != 1) mbar_wait(&conv[s], ph);
                    }
                    tc_fence_after();
                    if (lane == 0) {
                        const uint32_t s_ah = smem_u32(stage(s));
                        const uint32_t s_bh = s_ah + kTileA;
                        const uint32_t s_al = s_bh + TB;
                        const uint32_t s_bl = s_al + kTileA;
#pragma unroll
                        for (int h = 0; h < NH; ++h) {
                            // NH 2: half h = TMEM columns h*256, B blocks 4h..4h+3 (raw) /
                            // 64-n atoms 2h, 2h+1 (bf16); its accumulator is free once the
                            // previous tile's half-h epilogue drained it
                            const int ab = NH == 1 ? a : h;
                            if (NH == 2 && h == 1 && kb == kb0) {
                                mbar_wait_cluster(&acc_empty[1], aph ^ 1);
                                tc_fence_after();
                            }
                            const uint32_t td = NH == 1 ? tmem_d : tmem_base + (uint32_t)(h * BN);
                            const uint32_t bo = (uint32_t)h * (4 * kBBlock), bo16 = (uint32_t)h * 4096u;
#pragma unroll
                            for (int kk = 0; kk < BK / 8; ++kk) {
                                const uint64_t ah = desc_a(s_ah + kk * 32);         // +8 k in a 64-B row
                                const uint64_t bh = desc_b(s_bh + bo + kk * 1024);  // +8 k rows of 128 B
                                const uint32_t acc0 = (kb > kb0 || kk > 0) ? 1u : 0u;
                                if (SPLIT == 3) {
                                    mma_tf32<CG>(td, ah, desc_b(s_bl + kk * 1024), acc0);
                                    mma_tf32<CG>(td, desc_a(s_al + kk * 32), bh, 1u);
                                    mma_tf32<CG>(td, ah, bh, 1u);
                                } else {
                                    mma_tf32<CG>(td, ah, bh, acc0);
                                }
                            }
                            if (SPLIT == 2) {
                                // cross terms on the bf16 tiles, K = 16 in one MMA each
                                const uint32_t a16h = s_bh + TB, a16l = a16h + kTileA16;
                                const uint32_t b16h = a16l + kTileA16 + bo16, b16l = b16h + TB16;
                                mma_bf16<CG>(td, desc_a16(a16h), desc_b16(b16l), 1u);
                                mma_bf16<CG>(td, desc_a16(a16l), desc_b16(b16h), 1u);
                            } else if (SPLIT == 4) {
                                const uint32_t ta = tmem_base + (uint32_t)(C::kTaCol + 16 * s);
                                const uint32_t b16h = s_bh + TB, b16l = b16h + TB16;
                                mma_bf16_ta<CG>(td, ta, desc_b16(b16l), 1u);      // bf(A_hi) bf(B_lo)
                                mma_bf16_ta<CG>(td, ta + 8, desc_b16(b16h), 1u);  // bf(A_lo) bf(B_hi)
                            }
                            if (kb == kb1 - 1) mma_commit<CG>(&acc_full[ab]);
                        }
                        mma_commit<CG>(&empty[s]);
                    }
                    __syncwarp();
                }
                if (kb1 == kb0 && lane == 0) {  // K == 0: nothing accumulated
                    for (int h = 0; h < NH; ++h) {
                        const int ab = NH == 1 ? a : h;
                        if (NH == 2 && h == 1) mbar_wait_cluster(&acc_empty[1], aph ^ 1);
                        if constexpr (CG == 2) {
                            mbar_arrive_cluster(map_to(&acc_full[ab], 0));
                            mbar_arrive_cluster(map_to(&acc_full[ab], 1));
                        } else {
                            mbar_arrive(&acc_full[ab]);
                        }
                    }
                }
                __syncwarp();
              }
            }
        }
    } else if (warp < 4 || (warp >= 8 && warp < 14)) {
        // ------------------------------------------------------------ converters
        const int ct = (warp < 4 ? warp - 2 : warp - 6) * 32 + lane;  // 0..255
        const uint32_t conv_leader0 = CG == 2 ? map_to(&conv[0], 0) : 0;
        auto conv_done = [&](int s) {
            fence_proxy_async();
            __syncwarp();
            if (lane == 0) {
                if constexpr (CG == 2) mbar_arrive_cluster(conv_leader0 + (uint32_t)s * 8u);
                else mbar_arrive(&conv[s]);
            }
        };
        if constexpr (SPLIT == 3) {
            uint32_t it = 0;
            for (uint32_t t = cl; t < total; t += ncl) {
                const int v = find_tile_owner(descs, n, t);
                const int KB = (descs[v].K + BK - 1) / BK;
                for (int kb = 0; kb < KB; ++kb, ++it) {
                    const int s = it % ST;
                    const uint32_t ph = (it / ST) & 1;
                    mbar_wait(&full[s], ph);
                    const float4* hi = reinterpret_cast<const float4*>(stage(s));
                    float4* lo = reinterpret_cast<float4*>(stage(s) + kTileA + TB);
                    constexpr int NV = (kTileA + TB) / 16;  // A then B, same order
#pragma unroll
                    for (int i = ct; i < NV; i += kConvThreads) lo[i] = lo_part4(hi[i]);
                    conv_done(s);
                }
            }
        } else if constexpr (SPLIT == 2 || SPLIT == 4) {
            // SPLIT 4: this warp's TMEM lane quarter q = warp % 4 holds rows 32q..32q+31; the two
            // converter warps of a quarter split the 16 k into halves th (4 columns each)
            const int tq = warp & 3, th = (warp == 2 || warp == 3 || warp == 8 || warp == 9) ? 0 : 1;
            const int tm = tq * 32 + lane, tsw = (tm >> 1) & 3;
            const int t_rd0 = tm * 64 + (((2 * th) ^ tsw) << 4), t_rd1 = tm * 64 + (((2 * th + 1) ^ tsw) << 4);
            const uint32_t t_lane = tmem_base + ((uint32_t)(tq * 32) << 16) + (uint32_t)(C::kTaCol + 4 * th);
            // SPLIT 2 A unit (one per thread): row m, k half kc; a phase's 8 lanes = 8 rows, same kc
            const int am = (ct >> 4) * 8 + (ct & 7), akc = (ct >> 3) & 1;
            const int asw = (am >> 1) & 3;  // SWIZZLE_64B: 16-B chunk ^= bits [7,9) of the address
            const int a_rd0 = am * 64 + (((2 * akc) ^ asw) << 4), a_rd1 = am * 64 + (((2 * akc + 1) ^ asw) << 4);
            const int a_wr = (am >> 3) * 256 + akc * 128 + (am & 7) * 16;
            // B units: k row, 32-n block j, 32-B granule g (8 n); a phase's 8 lanes = 4
            // granules x 2 adjacent blocks, the first 16-B half read alternates with j
            constexpr int NB = (BK * C::kBN / 8) / kConvThreads;  // 2 (CG 1) or 1 (CG 2)
            constexpr int JB = C::kBN / 32;                       // 32-n blocks: 8 or 4
            int b_rd[NB][2], b_wr[NB];
#pragma unroll
            for (int r = 0; r < NB; ++r) {
                const int u = ct + kConvThreads * r;
                const int g = u & 3, j = ((u >> 2) & 1) + 2 * ((u >> 3) & (JB / 2 - 1));
                const int k = u / (4 * JB);
                const int base = j * kBBlock + k * 128 + ((g ^ (k & 3)) << 5);  // SWIZZLE_128B_BASE32B
                const int h = j & 1;
                b_rd[r][0] = base + 16 * h;
                b_rd[r][1] = base + 16 * (h ^ 1);
                const int c = 4 * (j & 1) + g, k8 = k & 7;  // bf16 SW128 MN-major
                b_wr[r] = (j >> 1) * 2048 + (k >> 3) * 1024 + k8 * 128 + ((c ^ k8) << 4);
            }
            uint32_t it = 0;
            for (uint32_t t = cl; t < total; t += ncl) {
                const int v = find_tile_owner(descs, n, t);
                const int KB = (descs[v].K + BK - 1) / BK;
                for (int kb = 0; kb < KB; ++kb, ++it) {
                    const int s = it % ST;
                    const uint32_t ph = (it / ST) & 1;
                    mbar_wait(&full[s], ph);
                    uint8_t* sp = stage(s);
                    uint8_t* a16h = sp + kTileA + TB;
                    uint8_t* a16l = a16h + kTileA16;
                    uint8_t* b16h = SPLIT == 4 ? a16h : a16l + kTileA16;
                    uint8_t* b16l = b16h + TB16;
                    if constexpr (SPLIT == 4) {
                        const float4 p = *reinterpret_cast<const float4*>(sp + t_rd0);
                        const float4 q = *reinterpret_cast<const float4*>(sp + t_rd1);
                        const float4 ph = rna_tf32_4(p), qh = rna_tf32_4(q);
                        *reinterpret_cast<float4*>(sp + t_rd0) = ph;
                        *reinterpret_cast<float4*>(sp + t_rd1) = qh;
                        uint4 hb, lb;
                        split8_given(p, q, ph, qh, hb, lb);
                        tmem_st4(t_lane + 16 * s, hb);
                        tmem_st4(t_lane + 16 * s + 8, lb);
                    } else {
                        const float4 p = *reinterpret_cast<const float4*>(sp + a_rd0);
                        const float4 q = *reinterpret_cast<const float4*>(sp + a_rd1);
                        // the TF32 MMA reads the raw tile: round it to TF32 in place (R19)
                        const float4 ph = rna_tf32_4(p), qh = rna_tf32_4(q);
                        *reinterpret_cast<float4*>(sp + a_rd0) = ph;
                        *reinterpret_cast<float4*>(sp + a_rd1) = qh;
                        uint4 hb, lb;
                        split8_given(p, q, ph, qh, hb, lb);
                        *reinterpret_cast<uint4*>(a16h + a_wr) = hb;
                        *reinterpret_cast<uint4*>(a16l + a_wr) = lb;
                    }
#pragma unroll
                    for (int r = 0; r < NB; ++r) {
                        const float4 x0 = *reinterpret_cast<const float4*>(sp + kTileA + b_rd[r][0]);
                        const float4 x1 = *reinterpret_cast<const float4*>(sp + kTileA + b_rd[r][1]);
                        const bool sw = (b_rd[r][0] & 16) != 0;  // read the upper half first
                        const float4 h0 = rna_tf32_4(x0), h1 = rna_tf32_4(x1);
                        *reinterpret_cast<float4*>(sp + kTileA + b_rd[r][0]) = h0;
                        *reinterpret_cast<float4*>(sp + kTileA + b_rd[r][1]) = h1;
                        uint4 hb, lb;
                        split8_given(sw ? x1 : x0, sw ? x0 : x1, sw ? h1 : h0, sw ? h0 : h1, hb, lb);
                        *reinterpret_cast<uint4*>(b16h + b_wr[r]) = hb;
                        *reinterpret_cast<uint4*>(b16l + b_wr[r]) = lb;
                    }
                    if constexpr (SPLIT == 4) {
                        asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
                        tc_fence_before();
                    }
                    conv_done(s);
                }
            }
        }
    } else {
        // ------------------------------------------------------------ epilogue (warps 4-7;
        // NH 2: warps 4-7 drain half 0, warps 14-17 half 1)
        const int q = warp & 3;  // TMEM lane quarter
        const int eh = (NH == 2 && warp >= 14) ? 1 : 0;
        const uint32_t acc_empty_leader = CG == 2 ? map_to(&acc_empty[0], 0) : 0;
        uint32_t tile_i = 0;  // (tile, chunk) units, as the MMA issuer counts them
        uint32_t nan_slabs = 0;  // K chunks: 8-column slabs of this row whose partial had a NaN
        for (uint32_t t = cl; t < total; t += ncl) {
          const int v = find_tile_owner(descs, n, t);
          const GemmDesc& g = descs[v];
          const int nch = tc_chunks(g, (g.K + BK - 1) / BK, kchunk);
          for (int ck = 0; ck < nch; ++ck, ++tile_i) {
            const uint32_t lt = t - g.tile_begin;
            const int tm = lt / g.tiles_n, tn = lt % g.tiles_n;
            const int a = NH == 1 ? (int)(tile_i % C::kAcc) : eh;
            const uint32_t aph = NH == 1 ? (tile_i / C::kAcc) & 1 : tile_i & 1;
            mbar_wait(&acc_full[a], aph);
            tc_fence_after();
            const int row = tm * C::kMmaM + (int)rank * BM + q * 32 + lane;
            const bool row_ok = row < g.M;
            float* crow = g.C + (size_t)(row_ok ? row : 0) * g.N;
            const float alpha = g.alpha, beta = g.beta;
            const bool kzero = g.K == 0;
            const bool first = ck == 0, last = ck == nch - 1;
            // beta == 0 tiles (with C maps) leave through TMA: full 128-B rows per store instead
            // of 16-B pieces of 32 different rows per warp store instruction
            const bool tma_epi = cmaps != nullptr && beta == 0.f && !kzero;
            // TMA epilogue (beta == 0): each 32 x 32 block of alpha * acc goes through this
            // warp's swizzled smem slab to C by TMA -- a store for chunk 0, a reduce-add (IEEE
            // round-to-nearest, performed by L2) for later chunks -- so a chunk boundary costs
            // the TMEM read and the slab writes, never a read of the partial sum.  The issuing
            // lane waits for its previous chunk's bulk group to complete before reducing into
            // the same addresses.  A chunk whose accumulator holds a NaN (an Inf / NaN operand,
            // or one near FLT_MAX, in its k range) marks the 8-column slab; after the last
            // chunk those slabs are read back and their NaN outputs recomputed exactly.
            constexpr int SW = 8, NV = SW / 4;
            if (first) nan_slabs = 0;
            // the accumulator is free for the next (tile, chunk) unit's MMAs once this warp's
            // last tcgen05.ld returned (early release), else after its last write
            bool released = false;
            auto release = [&]() {
                tc_fence_before();
                __syncwarp();
                if (lane == 0) {
                    if constexpr (CG == 2) mbar_arrive_cluster(acc_empty_leader + (uint32_t)a * 8u);
                    else mbar_arrive(&acc_empty[a]);
                }
                released = true;
            };
            if (tma_epi) {
                // two 32-row x 16-column half-slabs (64-B rows, 64-B swizzle) per epilogue warp,
                // alternating: the TMA op of one is in flight while the other is refilled
                uint8_t* slab = smem + C::kStagingOff + (size_t)(warp < 8 ? warp - 4 : warp - 10) * 4096;
                const void* cmap = cmaps + (size_t)v * 128;
                const int row0 = tm * C::kMmaM + (int)rank * BM + q * 32;
                if (lane == 0) bulk_wait0();  // the previous (tile, chunk) unit's writes landed
#pragma unroll 1
                for (int c0 = 0; c0 < BN; c0 += 16) {
                    uint8_t* hs = slab + ((c0 >> 4) & 1) * 2048;
                    if (lane == 0) asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");  // hs is free
                    __syncwarp();
#pragma unroll
                    for (int sl = 0; sl < 2; ++sl) {
                        uint32_t r[SW];
                        tmem_ld8(tmem_base + ((uint32_t)(q * 32) << 16) + (uint32_t)(a * BN + c0 + sl * SW), r);
                        if (early_release && c0 == BN - 16 && sl == 1) release();  // TMEM fully read
#pragma unroll
                        for (int jj = 0; jj < NV; ++jj) {
                            const int j = 4 * jj;
                            float4 o;
                            o.x = alpha * __uint_as_float(r[j + 0]);
                            o.y = alpha * __uint_as_float(r[j + 1]);
                            o.z = alpha * __uint_as_float(r[j + 2]);
                            o.w = alpha * __uint_as_float(r[j + 3]);
                            const float o4 = o.x + o.y + o.z + o.w;
                            if (o4 != o4) nan_slabs |= 1u << ((c0 + sl * SW) / SW);
                            const int ck16 = 2 * sl + jj;  // 16-B chunk of this lane's 64-B row
                            *reinterpret_cast<float4*>(hs + lane * 64 + ((ck16 ^ ((lane >> 1) & 3)) << 4)) = o;
                        }
                    }
                    fence_proxy_async();
                    __syncwarp();
                    if (lane == 0) {
                        const int col = tn * TN + eh * BN + c0;
                        const uint64_t pol = l2_policy(!last);
                        if (first) tma_store_2d(cmap, col, row0, hs, pol);
                        else tma_reduce_add_2d(cmap, col, row0, hs, pol);
                        bulk_commit();
                    }
                }
                if (lane == 0) bulk_wait_read0();
                __syncwarp();
            } else {
#pragma unroll 1
            for (int c0 = 0; c0 < BN; c0 += SW) {
                const int col0 = tn * TN + eh * BN + c0;
                uint32_t r[SW];
                tmem_ld8(tmem_base + ((uint32_t)(q * 32) << 16) + (uint32_t)(a * BN + c0), r);
                if (!row_ok) continue;
                uint32_t nan_mask = 0;  // outputs whose value came out NaN
#pragma unroll
                for (int jj = 0; jj < NV; ++jj) {
                    const int j = 4 * jj, c = col0 + j;
                    if (c >= g.N) break;
                    float4 o;
                    o.x = kzero ? 0.f : alpha * __uint_as_float(r[j + 0]);
                    o.y = kzero ? 0.f : alpha * __uint_as_float(r[j + 1]);
                    o.z = kzero ? 0.f : alpha * __uint_as_float(r[j + 2]);
                    o.w = kzero ? 0.f : alpha * __uint_as_float(r[j + 3]);
                    float4* dst = reinterpret_cast<float4*>(crow + c);
                    float4 old = make_float4(0.f, 0.f, 0.f, 0.f);
                    if (beta != 0.f) {
                        old = __ldcs(dst);
                        o.x = __fmaf_rn(beta, old.x, o.x);
                        o.y = __fmaf_rn(beta, old.y, o.y);
                        o.z = __fmaf_rn(beta, old.z, o.z);
                        o.w = __fmaf_rn(beta, old.w, o.w);
                    }
                    // IEEE special values (R20): an Inf / NaN operand (its low part x - h is NaN),
                    // or a finite one whose TF32 head rounds past FLT_MAX, leaves NaN in every
                    // accumulator it reaches.  Those outputs keep C_old for now and are recomputed
                    // exactly below (rare path, after r[] is dead).
                    const float o4 = o.x + o.y + o.z + o.w;
                    if (!kzero && o4 != o4) {
                        if (isnan(o.x)) { nan_mask |= 1u << (j + 0); o.x = old.x; }
                        if (isnan(o.y)) { nan_mask |= 1u << (j + 1); o.y = old.y; }
                        if (isnan(o.z)) { nan_mask |= 1u << (j + 2); o.z = old.z; }
                        if (isnan(o.w)) { nan_mask |= 1u << (j + 3); o.w = old.w; }
                    }
                    __stcs(dst, o);  // st.global.cs: C is written once
                }
                while (nan_mask) {
                    const int e = __ffs(nan_mask) - 1;
                    nan_mask &= nan_mask - 1;
                    float* cp = crow + col0 + e;
                    *cp = exact_element(g, row, col0 + e, beta != 0.f ? *cp : 0.f);
                }
            }
            }
            if (last && tma_epi && __any_sync(0xFFFFFFFFu, nan_slabs != 0)) {
                // the warp's bulk writes of every chunk have landed (wait_group 0) and are made
                // visible to this proxy's loads before the read-back
                if (lane == 0) bulk_wait0();
                __syncwarp();
                asm volatile("fence.proxy.async.global;" ::: "memory");
            }
            if (last && tma_epi && nan_slabs && row_ok) {
                while (nan_slabs) {
                    const int sl = __ffs(nan_slabs) - 1;
                    nan_slabs &= nan_slabs - 1;
                    const int col0 = tn * TN + eh * BN + sl * SW;
#pragma unroll 1
                    for (int e = 0; e < SW && col0 + e < g.N; ++e) {
                        float* cp = crow + col0 + e;
                        if (isnan(*(volatile float*)cp)) *cp = exact_element(g, row, col0 + e, 0.f);
                    }
                }
            }
            if (!released) release();
          }
        }
    }
    // ---------------------------------------------------------------- teardown
    if (warp >= 4 && ((warp < 8) || (NH == 2 && warp >= 14)) && lane == 0) bulk_wait0();  // epilogue TMA writes
    tc_fence_before();
    __syncthreads();
    if constexpr (CG == 2) cluster_sync_all();  // neither CTA frees TMEM / exits under the peer
    tc_fence_after();
    if (warp == 1) {
        if constexpr (CG == 1)
            asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem_base), "n"(kTmemCols)
                         : "memory");
        else
            asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(tmem_base), "n"(kTmemCols)
                         : "memory");
    }
}

static std::atomic<bool> g_attr_set[20][64] = {};  // per kernel variant and device

// SVP_TC_EARLY=0: the TMA epilogue frees the accumulator only after its last write (A/B switch;
// early release measured +0.9 % one-stream SGEMM, profiles/r02/epi_ab/)
static bool sgemm_tc_early_release() {
    static int v = -1;
    if (v < 0) {
        const char* e = getenv("SVP_TC_EARLY");
        v = (e && atoi(e) == 0) ? 0 : 1;
    }
    return v == 1;
}

template <int SPLIT, int CG, int NH = 1>
static cudaError_t launch_tc(const GemmDesc* descs, int n, const void* maps, uint32_t total, int clusters,
                             cudaStream_t s, int kchunk_k = 0, const void* cmaps = nullptr) {
    using Cf = tc::Cfg<SPLIT, CG, NH>;
    int dev = 0;
    cudaGetDevice(&dev);
    const int si = SPLIT + 5 * (CG - 1) + 10 * (NH - 1);
    auto kern = k_sgemm_tc<SPLIT, CG, NH>;
    if (dev < 64 && !g_attr_set[si][dev]) {
        cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                             (int)Cf::kSmem);
        if (e) return e;
        g_attr_set[si][dev] = true;
    }
    cudaLaunchConfig_t lc = {};
    cudaLaunchAttribute attr[1];
    lc.gridDim = dim3((unsigned)(clusters * CG));
    lc.blockDim = dim3(Cf::kThreads);
    lc.dynamicSmemBytes = Cf::kSmem;
    lc.stream = s;
    if (CG == 2) {
        attr[0].id = cudaLaunchAttributeClusterDimension;
        attr[0].val.clusterDim.x = 2;
        attr[0].val.clusterDim.y = 1;
        attr[0].val.clusterDim.z = 1;
        lc.attrs = attr;
        lc.numAttrs = 1;
    }
    // the plain-TF32 "sgemm_tf32" (own 2e-3 tolerance) accumulates the whole K in one chunk
    const int kchunk = (SPLIT == 1 || !cmaps) ? 0 : kchunk_k / tc::BK;
    const int flags = sgemm_tc_early_release() ? kEpiEarlyRelease : 0;
    return cudaLaunchKernelEx(&lc, kern, descs, n, reinterpret_cast<const uint8_t*>(maps), total, kchunk | flags,
                              reinterpret_cast<const uint8_t*>(cmaps));
}

// CTA-pair kernels for the fp32-accurate splits unless SVP_TC_CTA_PAIR=0 (A/B switch)
bool sgemm_tc_cta_pair() {
    static int v = -1;
    if (v < 0) {
        const char* e = getenv("SVP_TC_CTA_PAIR");
        v = (e && atoi(e) == 0) ? 0 : 1;
    }
    return v == 1;
}

cudaError_t launch_sgemm_tf32(const GemmDesc* descs, int n, const void* maps, uint32_t total, int grid,
                              cudaStream_t s) {
    return launch_tc<1, 1>(descs, n, maps, total, grid, s);
}

// `grid` counts SMs; with CTA pairs the grid of pairs is half of it
// SVP_TC_TMEM_A=1 selects SPLIT 4 (A-side bf16 operands in TMEM).  Measured on cfg5 it is
// not faster (2.71 vs 2.64 ms per launch, profiles/r01/pair): the kernel runs under the
// power cap, and the single accumulator costs the epilogue overlap; SPLIT 2 is the default.
static bool tmem_a() {
    static int v = -1;
    if (v < 0) {
        const char* e = getenv("SVP_TC_TMEM_A");
        v = (e && atoi(e) == 1) ? 1 : 0;
    }
    return v == 1;
}

// SVP_TC_WIDE: 0 never use the 256 x 512 pair tiles, 1 (default) let the executor choose per
// launch (>= 2 waves of wide tiles), 2 always (tests).  The executor builds the tile table
// for the choice and passes it to the launcher.
int sgemm_tc_wide_mode() {
    static int v = -1;
    if (v < 0) {
        const char* e = getenv("SVP_TC_WIDE");
        v = e ? std::min(2, std::max(0, atoi(e))) : 1;
    }
    return (sgemm_tc_cta_pair() && !tmem_a()) ? v : 0;
}

cudaError_t launch_sgemm_tf32bf16(const GemmDesc* descs, int n, const void* maps, uint32_t total, int grid,
                                  bool wide, cudaStream_t s, int kchunk, const void* cmaps) {
    const int pairs = (int)std::min<uint32_t>(total, std::max(1, grid / 2));
    if (wide) return launch_tc<2, 2, 2>(descs, n, maps, total, pairs, s, kchunk, cmaps);
    if (sgemm_tc_cta_pair())
        return tmem_a() ? launch_tc<4, 2>(descs, n, maps, total, pairs, s, kchunk, cmaps)
                        : launch_tc<2, 2>(descs, n, maps, total, pairs, s, kchunk, cmaps);
    return tmem_a() ? launch_tc<4, 1>(descs, n, maps, total, grid, s, kchunk, cmaps)
                    : launch_tc<2, 1>(descs, n, maps, total, grid, s, kchunk, cmaps);
}

// ------------------------------------------------------------------ tail split reduction
// One CTA per 4 rows of a sub-tile: thread (r, c4) sums the S partial products of one
// float4 in order s = 0..S-1, then C = alpha * sum (+ beta * C).
__global__ void __launch_bounds__(256) k_sgemm_tail_reduce(const TailRed* __restrict__ reds) {
    const TailRed& rd = reds[blockIdx.y];
    const int row = blockIdx.x * 4 + (threadIdx.x >> 6), c = (threadIdx.x & 63) * 4;
    if (row >= rd.rows || c >= rd.cols) return;
    const size_t plane = (size_t)rd.rows * rd.cols;
    const float* p = rd.ws + (size_t)row * rd.cols + c;
    float4 acc = *reinterpret_cast<const float4*>(p);
    for (int s = 1; s < rd.S; ++s) {
        const float4 v = *reinterpret_cast<const float4*>(p + s * plane);
        acc.x += v.x;
        acc.y += v.y;
        acc.z += v.z;
        acc.w += v.w;
    }
    float4* dst = reinterpret_cast<float4*>(rd.C + (size_t)row * rd.ldc + c);
    float4 o = make_float4(rd.alpha * acc.x, rd.alpha * acc.y, rd.alpha * acc.z, rd.alpha * acc.w);
    if (rd.beta != 0.f) {
        const float4 old = *dst;
        o.x = __fmaf_rn(rd.beta, old.x, o.x);
        o.y = __fmaf_rn(rd.beta, old.y, o.y);
        o.z = __fmaf_rn(rd.beta, old.z, o.z);
        o.w = __fmaf_rn(rd.beta, old.w, o.w);
    }
    *dst = o;
}

cudaError_t launch_sgemm_tail_reduce(const TailRed* reds, int nred, cudaStream_t s) {
    if (nred <= 0) return cudaSuccess;
    k_sgemm_tail_reduce<<<dim3((2 * kTf32BM) / 4, nred), 256, 0, s>>>(reds);
    return cudaGetLastError();
}

cudaError_t launch_sgemm_3xtf32(const GemmDesc* descs, int n, const void* maps, uint32_t total, int grid,
                                cudaStream_t s, int kchunk, const void* cmaps) {
    if (sgemm_tc_cta_pair())
        return launch_tc<3, 2>(descs, n, maps, total, (int)std::min<uint32_t>(total, std::max(1, grid / 2)), s,
                               kchunk, cmaps);
    return launch_tc<3, 1>(descs, n, maps, total, grid, s, kchunk, cmaps);
}

}  // namespace svp

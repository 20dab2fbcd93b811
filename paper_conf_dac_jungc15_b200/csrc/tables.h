// tables.h -- device-resident work tables shared by the executor (host) and the
// guest kernels (device).  Internal to libsvp; not part of the C-ABI.
//
// Kernel Coalescing (Fig 5/6) merges the identical kernel calls of
// several VPs into one launch over "one bigger piece of data".  Instead of physically
// gathering every VP's chunk into contiguous memory, a coalesced launch reads a
// segment table: segment i = one VP's job (its buffer bases, element count, scalar
// args) and owns tiles [tile_begin_i, tile_begin_{i+1}) of the launch's tile space.
// Ragged sizes need no padding: a VP's last tile is partial and predicated.
#pragma once
#include <stdint.h>

#ifdef __CUDACC__
#define SVP_HD __host__ __device__ __forceinline__
#else
#define SVP_HD inline
#endif

namespace svp {

// Elementwise / histogram segment: 64 bytes.
struct SegDesc {
    uint64_t ptr[5];      // buffer base addresses in kernel order (device)
    uint64_t n;           // elements (bytes for hist256)
    uint32_t tile_begin;  // first tile of this segment in the launch
    uint16_t shift;       // virtual-index shift: elements between the previous 16-B
                          // boundary and ptr[0] (tiles are aligned in address space)
    uint16_t flags;       // SEG_SCALAR: buffers not co-aligned mod 16 -> scalar path only;
                          // bits 8..15: the segment's kernel id (heterogeneous launch)
    float f[2];           // per-VP scalars (SAXPY a; Black-Scholes R, V)
};
static_assert(sizeof(SegDesc) == 64, "SegDesc must be 64 B");
enum : uint16_t { SEG_SCALAR = 1, SEG_KIND_SHIFT = 8 };

// table_mode = SVP_TABLE_PARAM: a launch of at most kParamSegs segments receives its table
// by value as a __grid_constant__ kernel parameter (15 KiB of the 32 KiB parameter space):
// no table upload and segment reads served from the constant cache.
// Tile layout of one segment (host side of the segment table): ptr0 = address of the
// first tiled buffer, co = every tiled buffer of the VP has the same address mod 16,
// es = element size.  Tiles live in a virtual index space shifted by `shift` elements so
// that every interior tile starts 16-B aligned in all buffers (the kernels' float4 /
// uint4 path, tile_range below); a VP whose buffers are mutually misaligned (or
// misaligned by a non-multiple of es) gets shift 0 and the scalar path (SEG_SCALAR).
inline void seg_layout(uint64_t ptr0, bool co, int es, int tile, uint64_t n, uint16_t* shift, uint64_t* ntiles,
                       bool* scalar) {
    const uint64_t mis = ptr0 & 15;
    const bool ok = co && mis % (uint64_t)es == 0;
    *scalar = !ok;
    *shift = ok ? (uint16_t)(mis / (uint64_t)es) : 0;
    *ntiles = n ? (n + *shift + (uint64_t)tile - 1) / (uint64_t)tile : 0;
}

// Element range [e0, e1) of local tile lt of a segment.  Tiles are laid out in a
// virtual index space shifted by `shift` so that every interior tile starts on a 16-B
// boundary of all the segment's buffers; `vec` says the whole tile is interior.
SVP_HD void tile_range(uint64_t n, uint32_t shift, uint32_t flags, uint32_t lt, int tile, int64_t& e0, int64_t& e1,
                       bool& vec) {
    int64_t v0 = (int64_t)lt * tile - (int64_t)shift;
    int64_t v1 = v0 + tile;
    e0 = v0 > 0 ? v0 : 0;
    e1 = v1 < (int64_t)n ? v1 : (int64_t)n;
    vec = !(flags & SEG_SCALAR) && v0 >= 0 && v1 <= (int64_t)n;
}

// The parameter block is sized to the launch: CAP in {16, 64} segments (1 or 4 KiB), the
// smallest that holds the group.  A launch's parameters are pushed through the front end
// with the launch; a 15-KiB block (the earlier 240-segment cap) cost ~9 us per launch on an
// idle GPU against ~1 us for 1 KiB, and groups above 64 segments ran faster from the global
// table (no upload in steady state) -- tools/s1_probe.py, profiles/r01/param_cap/.
constexpr int kParamSegs = 64;
template <int CAP>
struct SegParamT {
    SegDesc s[CAP];
};

// Grouped SGEMM: one entry per VP; tensor maps live in a separate 64-B aligned array
// (2 per VP: A then B).
struct GemmDesc {
    float* C;
    int32_t M, N, K;
    float alpha, beta;
    uint32_t tile_begin;  // first output tile of this VP
    uint32_t tiles_n;     // tiles along N
    uint32_t _pad0;
    // plain operand pointers + row pitches (elements): the tensor-core kernels stream A and B
    // through TMA maps and read these only on the rare exact-recompute path (R20)
    const float* A;
    const float* B;
    int32_t lda, ldb;
};
static_assert(sizeof(GemmDesc) == 64, "GemmDesc must be 64 B");

// SGEMM tail split (the partial last wave of a wide launch, split along K): one entry per
// 256 x 256 output sub-tile; its S partial products sit back to back in the workspace
// (piece s at ws + s * rows * cols), the reduction writes C = alpha * sum_s + beta * C.
struct TailRed {
    float* C;          // first element of the sub-tile in C
    const float* ws;   // first partial product
    int32_t ldc;       // row stride of C (elements)
    int32_t rows, cols;
    int32_t S;         // partial products
    float alpha, beta;
    uint32_t _pad[6];
};
static_assert(sizeof(TailRed) == 64, "TailRed must be 64 B");

// Grouped DGEMM (fp64): one entry per VP, plain pointers (no TMA).
struct DgemmDesc {
    const double* A;
    const double* B;
    double* C;
    int32_t M, N, K;
    uint32_t tile_begin;
    double alpha, beta;
    uint32_t tiles_n;
    uint32_t _pad;
};
static_assert(sizeof(DgemmDesc) == 64, "DgemmDesc must be 64 B");

// Tile geometry (elements per tile) -- host planner and kernels must agree.
constexpr int kEwThreads = 256;
constexpr int kVecaddVec = 4;                                  // float4 per thread per array
constexpr int kVecaddTile = kEwThreads * 4 * kVecaddVec;       // 4096 elements
constexpr int kSaxpyTile = kVecaddTile;
constexpr int kBsVec = 4;
constexpr int kBsTile = kEwThreads * 4 * kBsVec;               // 4096 options (kBsVec 4: +1.5 % cfg5, profiles/r01/bsvec)
constexpr int kHistThreads = 256;
constexpr int kHistVec = 4;                                    // uint4 (16 B) per thread
constexpr int kHistTile = kHistThreads * 16 * kHistVec;        // 16384 bytes
constexpr int kGemmBM = 128, kGemmBN = 128, kGemmBK = 32;
constexpr int kTf32BM = 128, kTf32BN = 256, kTf32BK = 16;
constexpr int kDgemmBM = 64, kDgemmBN = 64, kDgemmBK = 16;
constexpr int kDgemmSmall = 32;  // square tile of the small-launch DGEMM variant
constexpr int kDgemmSmallBK = 16;      // k depth per stage of the small variant
constexpr int kDgemmSmallDeepBK = 32;  // ... when every tile fits in one wave at its occupancy

}  // namespace svp

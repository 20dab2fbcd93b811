// launch.h -- host-side launchers of the sm_100a guest kernels (internal to libsvp).
// Every launcher enqueues ONE coalesced launch (plus hist256's output zeroing) on
// `stream` and returns the launch error; none synchronizes.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "tables.h"

namespace svp {

struct LaunchLimits {
    int num_sms = 148;
    int ew_blocks_per_sm = 8;   // occupancy of the elementwise kernels
    int bs_blocks_per_sm = 4;
    int mix_blocks_per_sm = 4;
    int hist_blocks_per_sm = 4;
    int gemm_blocks_per_sm = 1;
    int gemm_plain_blocks_per_sm = 1;
    int dgemm_blocks_per_sm = 1;
    int dgemm_small_blocks_per_sm = 1;
};

// Query occupancy / SM count for the current device (call once per device).
cudaError_t query_limits(LaunchLimits* out);

// Elementwise coalesced kernels: segs/nsegs describe the VPs, total_tiles is
// segs[nsegs-1].tile_begin + tiles of the last segment.  `busy` (profile_level 2, else
// null): nsegs zeroed u64 counters; thread 0 of every CTA adds its clock64 cycles per tile
// to the tile's segment (measured per-VP split of the launch).  `sched` (null: static
// tile order): 2 zeroed u32 -- dynamic tile order; the launch leaves them zeroed again.
cudaError_t launch_vecadd(const SegDesc* segs, int nsegs, uint32_t total_tiles, int grid, cudaStream_t s,
                        uint64_t* busy = nullptr, uint32_t* sched = nullptr);
cudaError_t launch_saxpy(const SegDesc* segs, int nsegs, uint32_t total_tiles, int grid, cudaStream_t s,
                        uint64_t* busy = nullptr, uint32_t* sched = nullptr);
cudaError_t launch_blackscholes(const SegDesc* segs, int nsegs, uint32_t total_tiles, int grid, cudaStream_t s,
                        uint64_t* busy = nullptr, uint32_t* sched = nullptr);
// Heterogeneous elementwise launch: segment kernel id in flags >> SEG_KIND_SHIFT.
cudaError_t launch_ew_mix(const SegDesc* segs, int nsegs, uint32_t total_tiles, int grid, cudaStream_t s,
                        uint64_t* busy = nullptr, uint32_t* sched = nullptr);
// table_mode param: the same kernels with the segment table passed by value; kind = kernel
// id (1 vecadd, 2 SAXPY, 4 Black-Scholes, 8 mixed), nsegs <= kParamSegs.
// `segs` is the HOST copy of the table (nsegs <= kParamSegs); it is copied into a
// parameter block of 16 or 64 segments, the smallest that holds it.
cudaError_t launch_ew_param(int kind, const SegDesc* segs, int nsegs, uint32_t total_tiles, int grid, cudaStream_t s,
                            uint64_t* busy = nullptr, uint32_t* sched = nullptr);
bool param_full_block();  // SVP_PARAM_FULL=1: always the kParamSegs block (A/B knob)
cudaError_t launch_hist256_param(const SegDesc* segs, int nsegs, uint32_t total_tiles, int grid, cudaStream_t s,
                                 uint64_t* busy = nullptr, uint32_t* scratch = nullptr, uint32_t* sched = nullptr);
// hist256: without `scratch`, a zeroing kernel then the accumulating launch; with
// `scratch` (nsegs * 257 zeroed u32, left zeroed) one launch whose last CTA per VP writes
// the VP's counts.
// `sched` (2 zeroed u32, left zeroed): dynamic tile order (chunks of 8 tiles claimed by each
// CTA's producer), ignored with `scratch`.
cudaError_t launch_hist256(const SegDesc* segs, int nsegs, uint32_t total_tiles, int grid, cudaStream_t s,
                        uint64_t* busy = nullptr, uint32_t* scratch = nullptr, uint32_t* sched = nullptr);

// Grouped SGEMM (fp32 FFMA, TMA-staged).  maps = 2*n CUtensorMap (A_i, B_i), 64-B aligned.
cudaError_t launch_sgemm_ffma(const GemmDesc* descs, int n, const void* maps, uint32_t total_tiles,
                              int grid, cudaStream_t s);
// Grouped SGEMM with plain guarded loads (64 x 64 tiles, FFMA): jobs whose pitches / buffers
// TMA cannot address (K or N not a multiple of 4, device buffers not 16-B aligned).
constexpr int kSgemmPlainTile = 64;
cudaError_t launch_sgemm_plain(const GemmDesc* descs, int n, uint32_t total_tiles, int grid, cudaStream_t s);
cudaError_t query_limits_gemm_plain(int* per_sm);
// Grouped SGEMM on tcgen05 TF32 tensor cores (TMEM accumulators).
cudaError_t launch_sgemm_tf32(const GemmDesc* descs, int n, const void* maps, uint32_t total_tiles,
                              int grid, cudaStream_t s);

// fp32-accurate grouped SGEMM on tcgen05: 3xTF32 (hi/lo operand split, 3 MMAs per k-step).
cudaError_t launch_sgemm_3xtf32(const GemmDesc* descs, int n, const void* maps, uint32_t total_tiles,
                                int grid, cudaStream_t s, int kchunk = 0, const void* cmaps = nullptr);

// fp32-accurate grouped SGEMM on tcgen05: A_hi B_hi as one kind::tf32 MMA per 8 k plus the
// cross terms bf16(A_hi) bf16(B_lo) + bf16(A_lo) bf16(B_hi) as kind::f16 (BF16) MMAs.
// kchunk (k) > 0 with cmaps (one 128-B CUtensorMap of C per VP, box 32 x 32, 128-B swizzle):
// K-chunked accumulation folded into C by TMA store / reduce-add (R23)
cudaError_t launch_sgemm_tf32bf16(const GemmDesc* descs, int n, const void* maps, uint32_t total_tiles,
                                  int grid, bool wide, cudaStream_t s, int kchunk = 0, const void* cmaps = nullptr);
int encode_c_map(void* mapC, const float* C, int M, int N);

// true: the fp32-accurate tcgen05 SGEMMs run as CTA pairs (cta_group::2, 256 x 256 tiles);
// SVP_TC_CTA_PAIR=0 selects the single-CTA kernels (128 x 256 tiles)
bool sgemm_tc_cta_pair();

// 256 x 512 tiles for the TF32+2xBF16 pair kernel (two 256-column accumulator halves sharing
// each A tile): SVP_TC_WIDE=0 never, 1 (default) when a launch has >= 2 waves of them, 2 always
int sgemm_tc_wide_mode();

// Grouped fp64 GEMM (the paper's Table 1 matmul), FP64 DFMA with smem tiles; `small`:
// 32x32 tiles (the table was built with kDgemmSmall tiles).
cudaError_t launch_dgemm(const DgemmDesc* descs, int n, uint32_t total_tiles, int grid, bool small, cudaStream_t s);
// the small-tile DGEMM runs on the FP64 tensor cores (DMMA) unless SVP_DGEMM_DMMA=0; the executor
// then uses the 32 x 32 tiles for every DGEMM launch
bool dgemm_dmma_enabled();
cudaError_t query_limits_dgemm(int* per_sm, int* per_sm_small);

// Host: encode the TMA descriptors an SGEMM entry needs (driver entry point fetched at
// runtime, so libsvp does not link libcuda).  variant 0 = FFMA tiles, 1 = TF32 tiles.
// Returns 0 on success.
int encode_gemm_maps(void* mapA, void* mapB, const float* A, const float* B, int M, int N, int K,
                     int variant);
// tcgen05 maps of a sub-matrix view: A (M x K, row stride lda), B (K x N, row stride ldb).
int encode_gemm_maps_view(void* mapA, void* mapB, const float* A, const float* B, int M, int N, int K, int lda,
                          int ldb);
// SGEMM tail split: C = alpha * (sum of the S partial products) + beta * C per sub-tile
// (fixed summation order: deterministic).
cudaError_t launch_sgemm_tail_reduce(const TailRed* reds, int nred, cudaStream_t s);

}  // namespace svp

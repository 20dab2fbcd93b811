// ubench.cu -- roofline-ceiling microbenchmarks for B200 (tooling, not part of libsvp).
//   ub_copy      float4 streaming copy (ld/st .cs) -> achievable HBM GB/s for our access style
//   ub_atoms     shared-memory atomics: 32 distinct banks per warp instruction, returns
//                total atomic lanes executed (time it with events) -> smem-atomic ceiling
//   ub_ffma      independent FFMA chains -> FP32 SIMT ceiling
// Host-side PCIe (pinned H2D / D2H / both) is measured from Python with cudaMemcpyAsync.
#include <cuda_runtime.h>
#include <stdint.h>

__global__ void k_copy(const float4* __restrict__ a, float4* __restrict__ b, size_t n4) {
    size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x;
    size_t stride = (size_t)gridDim.x * blockDim.x;
    for (; i + 3 * stride < n4; i += 4 * stride) {
        float4 x0 = __ldcs(a + i), x1 = __ldcs(a + i + stride), x2 = __ldcs(a + i + 2 * stride),
               x3 = __ldcs(a + i + 3 * stride);
        __stcs(b + i, x0);
        __stcs(b + i + stride, x1);
        __stcs(b + i + 2 * stride, x2);
        __stcs(b + i + 3 * stride, x3);
    }
    for (; i < n4; i += stride) __stcs(b + i, __ldcs(a + i));
}

// Each thread: iters x 4 atomics into column `lane` of a [256][32] u32 table, with
// pseudo-random bins (xorshift) -- the hist256 kernel's smem access without global loads.
__global__ void k_atoms(uint32_t* out, int iters) {
    __shared__ uint32_t h[256 * 32];
    for (int i = threadIdx.x; i < 256 * 32; i += blockDim.x) h[i] = 0;
    __syncthreads();
    uint32_t x = 0x9E3779B9u * (threadIdx.x + 1) ^ blockIdx.x;
    uint32_t* hl = h + (threadIdx.x & 31);
    for (int it = 0; it < iters; ++it) {
        x ^= x << 13;
        x ^= x >> 17;
        x ^= x << 5;
        atomicAdd(hl + ((x & 0xFFu) << 5), 1u);
        atomicAdd(hl + (((x >> 8) & 0xFFu) << 5), 1u);
        atomicAdd(hl + (((x >> 16) & 0xFFu) << 5), 1u);
        atomicAdd(hl + ((x >> 24) << 5), 1u);
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        uint32_t s = 0;
        for (int i = 0; i < 256 * 32; ++i) s += h[i];
        atomicAdd(out, s);
    }
}

// 16-bit packed variant: h[128][32] words, bin b -> word b & 127, half b >> 7
__global__ void k_atoms16(uint32_t* out, int iters) {
    __shared__ uint32_t h[128 * 32];
    for (int i = threadIdx.x; i < 128 * 32; i += blockDim.x) h[i] = 0;
    __syncthreads();
    uint32_t x = 0x9E3779B9u * (threadIdx.x + 1) ^ blockIdx.x;
    uint32_t* hl = h + (threadIdx.x & 31);
    for (int it = 0; it < iters; ++it) {
        x ^= x << 13;
        x ^= x >> 17;
        x ^= x << 5;
#pragma unroll
        for (int k = 0; k < 4; ++k) {
            uint32_t b = (x >> (8 * k)) & 0xFFu;
            atomicAdd(hl + ((b & 127u) << 5), 1u << ((b >> 7) << 4));
        }
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        uint32_t s = 0;
        for (int i = 0; i < 128 * 32; ++i) s += (h[i] & 0xFFFF) + (h[i] >> 16);
        atomicAdd(out, s);
    }
}

__global__ void k_ffma(float* out, int iters) {
    float a0 = threadIdx.x, a1 = a0 + 1, a2 = a0 + 2, a3 = a0 + 3, a4 = a0 + 4, a5 = a0 + 5, a6 = a0 + 6, a7 = a0 + 7;
    const float b = 0.999f, c = 0.001f;
    for (int i = 0; i < iters; ++i) {
#pragma unroll
        for (int j = 0; j < 8; ++j) {
            a0 = fmaf(a0, b, c); a1 = fmaf(a1, b, c); a2 = fmaf(a2, b, c); a3 = fmaf(a3, b, c);
            a4 = fmaf(a4, b, c); a5 = fmaf(a5, b, c); a6 = fmaf(a6, b, c); a7 = fmaf(a7, b, c);
        }
    }
    if (a0 + a1 + a2 + a3 + a4 + a5 + a6 + a7 == 12345.f) out[0] = a0;
}

__global__ void k_dfma(double* out, int iters) {
    double a0 = threadIdx.x, a1 = a0 + 1, a2 = a0 + 2, a3 = a0 + 3, a4 = a0 + 4, a5 = a0 + 5, a6 = a0 + 6, a7 = a0 + 7;
    const double b = 0.999, c = 0.001;
    for (int i = 0; i < iters; ++i) {
#pragma unroll
        for (int j = 0; j < 8; ++j) {
            a0 = fma(a0, b, c); a1 = fma(a1, b, c); a2 = fma(a2, b, c); a3 = fma(a3, b, c);
            a4 = fma(a4, b, c); a5 = fma(a5, b, c); a6 = fma(a6, b, c); a7 = fma(a7, b, c);
        }
    }
    if (a0 + a1 + a2 + a3 + a4 + a5 + a6 + a7 == 12345.0) out[0] = a0;
}

// packed FP32 (sm_100: FFMA2 = fma.rn.f32x2): 2 FMAs per lane per instruction
__global__ void k_ffma2(float* out, int iters) {
    unsigned long long a0 = threadIdx.x, a1 = a0 + 1, a2 = a0 + 2, a3 = a0 + 3, a4 = a0 + 4, a5 = a0 + 5,
                       a6 = a0 + 6, a7 = a0 + 7;
    unsigned long long b = 0x3f7fbe773f7fbe77ull, c = 0x3a83126f3a83126full;
    asm volatile("" : "+l"(b), "+l"(c));
    for (int i = 0; i < iters; ++i) {
#pragma unroll
        for (int j = 0; j < 8; ++j) {
            asm volatile("fma.rn.f32x2 %0, %0, %1, %2;" : "+l"(a0) : "l"(b), "l"(c));
            asm volatile("fma.rn.f32x2 %0, %0, %1, %2;" : "+l"(a1) : "l"(b), "l"(c));
            asm volatile("fma.rn.f32x2 %0, %0, %1, %2;" : "+l"(a2) : "l"(b), "l"(c));
            asm volatile("fma.rn.f32x2 %0, %0, %1, %2;" : "+l"(a3) : "l"(b), "l"(c));
            asm volatile("fma.rn.f32x2 %0, %0, %1, %2;" : "+l"(a4) : "l"(b), "l"(c));
            asm volatile("fma.rn.f32x2 %0, %0, %1, %2;" : "+l"(a5) : "l"(b), "l"(c));
            asm volatile("fma.rn.f32x2 %0, %0, %1, %2;" : "+l"(a6) : "l"(b), "l"(c));
            asm volatile("fma.rn.f32x2 %0, %0, %1, %2;" : "+l"(a7) : "l"(b), "l"(c));
        }
    }
    if ((a0 ^ a1 ^ a2 ^ a3 ^ a4 ^ a5 ^ a6 ^ a7) == 12345) out[0] = 1.f;
}

extern "C" {
int ub_dfma(double* out, int iters, int grid, int block, void* stream) {
    k_dfma<<<grid, block, 0, (cudaStream_t)stream>>>(out, iters);
    return (int)cudaGetLastError();
}
int ub_ffma2(float* out, int iters, int grid, int block, void* stream) {
    k_ffma2<<<grid, block, 0, (cudaStream_t)stream>>>(out, iters);
    return (int)cudaGetLastError();
}
int ub_copy(const void* a, void* b, size_t bytes, int grid, int block, void* stream) {
    k_copy<<<grid, block, 0, (cudaStream_t)stream>>>((const float4*)a, (float4*)b, bytes / 16);
    return (int)cudaGetLastError();
}
int ub_atoms(uint32_t* out, int iters, int grid, int block, void* stream) {
    k_atoms<<<grid, block, 0, (cudaStream_t)stream>>>(out, iters);
    return (int)cudaGetLastError();
}
int ub_atoms16(uint32_t* out, int iters, int grid, int block, void* stream) {
    k_atoms16<<<grid, block, 0, (cudaStream_t)stream>>>(out, iters);
    return (int)cudaGetLastError();
}
int ub_ffma(float* out, int iters, int grid, int block, void* stream) {
    k_ffma<<<grid, block, 0, (cudaStream_t)stream>>>(out, iters);
    return (int)cudaGetLastError();
}
}

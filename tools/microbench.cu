// Microbenchmarks for the primitives the GTS kernels are built from (B200):
// random fp32 RED into a large array (uniform and RMAT-skewed destinations),
// RED.v4, random 4-byte gathers from an L2-resident bitmap, shared-memory atomics.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o microbench tools/microbench.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint64_t mix(uint64_t x) {
    x += 0x9E3779B97F4A7C15ULL;
    x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ULL;
    x = (x ^ (x >> 27)) * 0x94D049BB133111EBULL;
    return x ^ (x >> 31);
}

// RMAT-like destination (27 bits, P(bit=0) = 0.76 per level) from one hash
__device__ __forceinline__ uint32_t rmat_dst(uint64_t e, int scale) {
    uint32_t v = 0;
    uint64_t h = mix(e);
    uint64_t h2 = mix(e ^ 0x1234567ULL);
    for (int l = 0; l < scale; ++l) {
        uint32_t r = (l < 16) ? (uint32_t)((h >> (4 * (l & 15))) & 15) : (uint32_t)((h2 >> (4 * (l & 15))) & 15);
        // 4-bit uniform r in [0,16): bit 1 with prob 4/16 = 0.25 (close to 0.24)
        v = (v << 1) | (r < 4 ? 1u : 0u);
    }
    return v;
}

template <int MODE>
__global__ void red_kernel(float* acc, uint64_t m, int scale, uint32_t mask) {
    uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    for (uint64_t e = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; e < m; e += stride) {
        uint32_t d = MODE == 0 ? (uint32_t)(mix(e) & mask) : rmat_dst(e, scale);
        atomicAdd(acc + d, 1.0f);
    }
}

__global__ void red_v4_kernel(float* acc, uint64_t m, uint32_t mask4) {
    uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    for (uint64_t e = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; e < m / 4; e += stride) {
        uint32_t d = (uint32_t)(mix(e) & mask4) * 4;
        asm volatile("red.global.add.v4.f32 [%0], {%1,%2,%3,%4};" ::"l"(acc + d), "f"(1.f), "f"(1.f), "f"(1.f), "f"(1.f));
    }
}

__global__ void hash_only_kernel(uint32_t* out, uint64_t m, int scale, int mode) {
    uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    uint32_t s = 0;
    for (uint64_t e = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; e < m; e += stride)
        s ^= mode == 0 ? (uint32_t)mix(e) : rmat_dst(e, scale);
    if (s == 0x12345) out[0] = s;
}

__global__ void gather_kernel(const uint32_t* bm, uint64_t m, uint32_t mask, uint32_t* out) {
    uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    uint32_t s = 0;
    for (uint64_t e = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; e < m; e += stride) {
        uint32_t d = (uint32_t)(mix(e) & mask);
        s ^= __ldcg(bm + (d >> 5));
    }
    if (s == 0x12345) out[0] = s;
}

__global__ void smem_atomic_kernel(uint64_t m, uint32_t* out) {
    __shared__ float h[8192];
    for (int i = threadIdx.x; i < 8192; i += blockDim.x) h[i] = 0;
    __syncthreads();
    uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    for (uint64_t e = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; e < m; e += stride)
        atomicAdd(&h[mix(e) & 8191], 1.0f);
    __syncthreads();
    if (h[threadIdx.x] == -1.f) out[0] = 1;
}

#define TIME(label, launch, ops)                                                              \
    do {                                                                                      \
        launch;                                                                               \
        cudaEventRecord(a);                                                                   \
        launch;                                                                               \
        cudaEventRecord(b);                                                                   \
        cudaEventSynchronize(b);                                                              \
        float ms;                                                                             \
        cudaEventElapsedTime(&ms, a, b);                                                      \
        printf("%-44s %8.3f ms  %7.1f Gop/s  (%s)\n", label, ms, (double)(ops) / ms / 1e6,    \
               cudaGetErrorString(cudaGetLastError()));                                       \
    } while (0)

int main() {
    const int scale = 27;
    const uint64_t n = 1ull << scale, m = 16 * n;
    float* acc;
    uint32_t* bm;
    uint32_t* out;
    cudaMalloc(&acc, n * 4);
    cudaMalloc(&bm, n / 8);
    cudaMalloc(&out, 4);
    cudaMemset(acc, 0, n * 4);
    cudaMemset(bm, 0, n / 8);
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    int sms;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    const int G = sms * 8, T = 256;
    TIME("hash only (uniform)", (hash_only_kernel<<<G, T>>>(out, m, scale, 0)), m);
    TIME("hash only (rmat)", (hash_only_kernel<<<G, T>>>(out, m, scale, 1)), m);
    TIME("RED.f32 uniform over 512 MiB", (red_kernel<0><<<G, T>>>(acc, m, scale, (uint32_t)(n - 1))), m);
    TIME("RED.f32 uniform over 64 MiB (L2)", (red_kernel<0><<<G, T>>>(acc, m, scale, (uint32_t)(n / 8 - 1))), m);
    TIME("RED.f32 uniform over 1 MiB", (red_kernel<0><<<G, T>>>(acc, m, scale, (uint32_t)(262144 - 1))), m);
    TIME("RED.f32 rmat-skewed over 512 MiB", (red_kernel<1><<<G, T>>>(acc, m, scale, 0)), m);
    TIME("RED.v4.f32 uniform over 512 MiB (per v4)", (red_v4_kernel<<<G, T>>>(acc, m, (uint32_t)(n / 4 - 1))), m / 4);
    TIME("gather u32 from 16 MiB bitmap (L2)", (gather_kernel<<<G, T>>>(bm, m, (uint32_t)(n - 1), out)), m);
    TIME("smem atomicAdd f32 random (8K slots)", (smem_atomic_kernel<<<G, T>>>(m, out)), m);
    return 0;
}

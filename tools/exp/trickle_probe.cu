// Experiment: GPU-paced SM copy HBM -> pinned host memory (is a smooth, rate-limited D2H
// stream gentler on eager training than copy-engine bursts?).  Not part of the library.
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint64_t gtime() {
    uint64_t t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}

__global__ void k_trickle(const uint4 *src, uint4 *dst, uint64_t bytes, uint64_t ns_per_block, uint32_t block_bytes) {
    __shared__ uint64_t t0;
    if (threadIdx.x == 0) t0 = gtime();
    __syncthreads();
    const uint64_t nblk = (bytes + block_bytes - 1) / block_bytes;
    uint64_t k = 0;
    for (uint64_t b = blockIdx.x; b < nblk; b += gridDim.x, ++k) {
        if (threadIdx.x == 0) {
            const uint64_t target = t0 + k * gridDim.x * ns_per_block;
            while (gtime() < target) __nanosleep(500);
        }
        __syncthreads();
        const uint64_t w0 = b * block_bytes / 16, w1 = min(bytes, (b + 1) * block_bytes) / 16;
        for (uint64_t w = w0 + threadIdx.x; w < w1; w += blockDim.x) dst[w] = __ldg(src + w);
    }
}

extern "C" int trickle(const void *src, void *dst, uint64_t bytes, double gbs, uint32_t ctas, uint32_t block_bytes,
                       void *stream) {
    const uint64_t ns = gbs > 0 ? (uint64_t)(block_bytes / gbs) : 0;  // bytes / (GB/s) = ns
    k_trickle<<<ctas, 256, 0, (cudaStream_t)stream>>>((const uint4 *)src, (uint4 *)dst, bytes, ns, block_bytes);
    return (int)cudaGetLastError();
}

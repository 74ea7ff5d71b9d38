// Round-2 probe (DESIGN §11 item 1): can TMA bulk copies (cp.async.bulk global->smem->global)
// move a K1-sized image faster than the register path?  Times, on the same 1.107 GB buffer
// (C2's state size), HBM->HBM:
//   memcpy : cudaMemcpyAsync D2D
//   ldst   : grid-stride uint4 LD/ST kernel, 148 x k CTAs
//   bulk   : one elected thread per CTA drives an S-stage smem ring of T-byte tiles with
//            cp.async.bulk loads (mbarrier complete_tx) and bulk stores (bulk_group)
// and checks every copy byte-for-byte.  Not part of the product path.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/exp/bulk_copy_probe tools/exp/bulk_copy_probe.cu
#include <cuda_runtime.h>
#include <cstdint>
#include <cstdio>
#include <algorithm>

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { \
  printf("CUDA error %s at %s:%d\n", cudaGetErrorString(e_), __FILE__, __LINE__); return 1; } } while (0)

__global__ void k_fill(uint4 *p, size_t n) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x)
    p[i] = make_uint4((uint32_t)i * 2654435761u, (uint32_t)(i >> 7) ^ 0x9e3779b9u, (uint32_t)i + 17u, ~(uint32_t)i);
}

__global__ void k_cmp(const uint4 *a, const uint4 *b, size_t n, unsigned long long *bad) {
  unsigned long long c = 0;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) {
    uint4 x = a[i], y = b[i];
    c += (x.x != y.x) | (x.y != y.y) | (x.z != y.z) | (x.w != y.w);
  }
  if (c) atomicAdd(bad, c);
}

__global__ void k_ldst(const uint4 *__restrict__ s, uint4 *__restrict__ d, size_t n) {
  const size_t stride = (size_t)gridDim.x * blockDim.x;
  size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x;
  for (; i + 3 * stride < n; i += 4 * stride) {
    uint4 a = __ldcs(s + i), b = __ldcs(s + i + stride), c = __ldcs(s + i + 2 * stride), e = __ldcs(s + i + 3 * stride);
    __stcs(d + i, a); __stcs(d + i + stride, b); __stcs(d + i + 2 * stride, c); __stcs(d + i + 3 * stride, e);
  }
  for (; i < n; i += stride) __stcs(d + i, __ldcs(s + i));
}

__device__ __forceinline__ uint32_t sa(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }

template <int S>
__global__ void __launch_bounds__(32) k_bulk(const char *src, char *dst, size_t ntiles, uint32_t T) {
  extern __shared__ __align__(128) uint8_t ring[];
  __shared__ __align__(8) uint64_t bar[S];
  if (threadIdx.x != 0) return;
  for (int i = 0; i < S; ++i) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(sa(&bar[i])));
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  const size_t first = blockIdx.x, step = gridDim.x;
  auto load = [&](size_t tile, int st) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(sa(&bar[st])), "r"(T) : "memory");
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 ::"r"(sa(ring + (size_t)st * T)), "l"(src + tile * T), "r"(T), "r"(sa(&bar[st])) : "memory");
  };
  // prologue: S loads in flight
  size_t k = 0;
  for (int i = 0; i < S; ++i)
    if (first + (size_t)i * step < ntiles) load(first + (size_t)i * step, i);
  for (size_t tile = first; tile < ntiles; tile += step, ++k) {
    const int st = (int)(k % S);
    const uint32_t ph = (uint32_t)((k / S) & 1);
    asm volatile("{\n.reg .pred p;\nW_%=:\nmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n@!p bra W_%=;\n}\n"
                 ::"r"(sa(&bar[st])), "r"(ph) : "memory");
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;"
                 ::"l"(dst + tile * T), "r"(sa(ring + (size_t)st * T)), "r"(T) : "memory");
    asm volatile("cp.async.bulk.commit_group;" ::: "memory");
    // refill the stage whose store was issued one iteration ago (at most 1 store group left
    // reading smem), so stores and loads overlap
    if (k >= 1) {
      asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");
      const size_t nt = tile + (size_t)(S - 1) * step;
      if (nt < ntiles) load(nt, (int)((k - 1) % S));
    }
  }
  asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}

template <typename F>
static float best_ms(F f, cudaStream_t s, int reps) {
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  float best = 1e30f;
  for (int i = 0; i < reps + 2; ++i) {
    cudaEventRecord(a, s); f(); cudaEventRecord(b, s); cudaEventSynchronize(b);
    float ms; cudaEventElapsedTime(&ms, a, b);
    if (i >= 2) best = std::min(best, ms);
  }
  return best;
}

template <int S>
static int run_bulk(const char *s, char *d, size_t bytes, uint32_t T, int cps, int nsm, cudaStream_t st,
                    unsigned long long *bad, const char *label) {
  const size_t ntiles = bytes / T;
  const size_t smem = (size_t)S * T;
  CK(cudaFuncSetAttribute(k_bulk<S>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  CK(cudaMemsetAsync(d, 0, bytes, st));
  const int grid = nsm * cps;
  float ms = best_ms([&] { k_bulk<S><<<grid, 32, smem, st>>>(s, d, ntiles, T); }, st, 5);
  CK(cudaGetLastError());
  CK(cudaMemsetAsync(bad, 0, 8, st));
  k_cmp<<<nsm * 8, 256, 0, st>>>((const uint4 *)s, (const uint4 *)d, ntiles * T / 16, bad);
  unsigned long long h = 0;
  CK(cudaMemcpyAsync(&h, bad, 8, cudaMemcpyDeviceToHost, st)); CK(cudaStreamSynchronize(st));
  printf("{\"kind\": \"bulk\", \"stages\": %d, \"tile\": %u, \"ctas_per_sm\": %d, \"ms\": %.4f, \"gbs\": %.1f, \"bad\": %llu, \"label\": \"%s\"}\n",
         S, T, cps, ms, 2.0 * ntiles * T / ms / 1e6, h, label);
  return 0;
}

int main() {
  const size_t bytes = 16889ull * 65536;  // C2 state size (1,106,860,352 B) rounded down to 64 KiB
  int nsm = 0; CK(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0));
  char *s, *d; unsigned long long *bad;
  CK(cudaMalloc(&s, bytes)); CK(cudaMalloc(&d, bytes)); CK(cudaMalloc(&bad, 8));
  cudaStream_t st; CK(cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking));
  k_fill<<<nsm * 8, 256, 0, st>>>((uint4 *)s, bytes / 16);
  CK(cudaStreamSynchronize(st));
  float ms = best_ms([&] { cudaMemcpyAsync(d, s, bytes, cudaMemcpyDeviceToDevice, st); }, st, 5);
  printf("{\"kind\": \"memcpy\", \"ms\": %.4f, \"gbs\": %.1f}\n", ms, 2.0 * bytes / ms / 1e6);
  for (int cps : {2, 4, 8}) {
    ms = best_ms([&] { k_ldst<<<nsm * cps, 1024 / (cps > 2 ? cps / 2 : 1), 0, st>>>((const uint4 *)s, (uint4 *)d, bytes / 16); }, st, 5);
    printf("{\"kind\": \"ldst\", \"grid\": %d, \"ms\": %.4f, \"gbs\": %.1f}\n", nsm * cps, ms, 2.0 * bytes / ms / 1e6);
  }
  for (int cps : {2, 3, 6}) {
    run_bulk<4>(s, d, bytes, 16384, cps, nsm, st, bad, "4x16K");
    run_bulk<8>(s, d, bytes, 8192, cps, nsm, st, bad, "8x8K");
  }
  for (int cps : {1, 2}) {
    run_bulk<4>(s, d, bytes, 32768, cps, nsm, st, bad, "4x32K");
    run_bulk<6>(s, d, bytes, 16384, cps, nsm, st, bad, "6x16K");
  }
  // round 2: the staging K1 could afford next to its 193 KiB of CRC tables (~34 KiB per SM,
  // one CTA per SM): is a TMA ring that small still at the copy peak?
  run_bulk<4>(s, d, bytes, 8192, 1, nsm, st, bad, "4x8K_1cta_32KiB");
  run_bulk<2>(s, d, bytes, 16384, 1, nsm, st, bad, "2x16K_1cta_32KiB");
  run_bulk<8>(s, d, bytes, 4096, 1, nsm, st, bad, "8x4K_1cta_32KiB");
  run_bulk<8>(s, d, bytes, 8192, 1, nsm, st, bad, "8x8K_1cta_64KiB");
  run_bulk<8>(s, d, bytes, 16384, 1, nsm, st, bad, "8x16K_1cta_128KiB");
  return 0;
}

// Box probe: measures the D2H / H2D link peaks that are the
// roofline denominators for the snapshot path, the SM zero-copy write ceiling
// into host-mapped memory, TMA bulk S2G into host memory, and whether a tmpfs
// file mapping can be registered as pinned staging.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/probe tools/probe.cu
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <cstdint>
#include <vector>
#include <algorithm>
#include <chrono>
#include <fcntl.h>
#include <unistd.h>
#include <sys/mman.h>

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { \
  printf("CUDA error %s at %s:%d\n", cudaGetErrorString(e_), __FILE__, __LINE__); return 1; } } while (0)

static double best_copy(void* dst, const void* src, size_t n, cudaMemcpyKind k, cudaStream_t s, int reps) {
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  double best = 1e30;
  for (int i = 0; i < reps + 2; ++i) {
    cudaEventRecord(a, s);
    cudaMemcpyAsync(dst, src, n, k, s);
    cudaEventRecord(b, s);
    cudaEventSynchronize(b);
    float ms; cudaEventElapsedTime(&ms, a, b);
    if (i >= 2) best = std::min(best, (double)ms);
  }
  cudaEventDestroy(a); cudaEventDestroy(b);
  return n / (best * 1e-3) / 1e9;
}

__global__ void zc_write(int4* __restrict__ dst, const int4* __restrict__ src, size_t n16) {
  size_t stride = (size_t)gridDim.x * blockDim.x;
  for (size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x; i < n16; i += stride) {
    int4 v = src[i];
    dst[i] = v;
  }
}

// one CTA moves 64 KiB blocks: ld.global -> smem -> cp.async.bulk S2G
__global__ void tma_s2g(char* __restrict__ dst, const int4* __restrict__ src, size_t nblk) {
  extern __shared__ __align__(128) int4 sm[];
  const int per = 16384 / 16;  // 16 KiB per stage
  for (size_t blk = blockIdx.x; blk < nblk; blk += gridDim.x) {
    // wait previous bulk reads of smem before overwrite
    if (threadIdx.x == 0) asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
    __syncthreads();
    for (int i = threadIdx.x; i < per; i += blockDim.x) sm[i] = src[blk * per + i];
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    __syncthreads();
    if (threadIdx.x == 0) {
      unsigned saddr = (unsigned)__cvta_generic_to_shared(sm);
      asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;"
                   :: "l"(dst + blk * 16384), "r"(saddr), "r"(16384) : "memory");
      asm volatile("cp.async.bulk.commit_group;" ::: "memory");
    }
  }
  if (threadIdx.x == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}

__global__ void hbm_copy(int4* __restrict__ dst, const int4* __restrict__ src, size_t n16) {
  size_t stride = (size_t)gridDim.x * blockDim.x;
  for (size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x; i < n16; i += stride) dst[i] = src[i];
}

template <class F> static double time_ms(cudaStream_t s, int reps, F f) {
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  double best = 1e30;
  for (int i = 0; i < reps + 2; ++i) {
    cudaEventRecord(a, s); f(); cudaEventRecord(b, s); cudaEventSynchronize(b);
    float ms; cudaEventElapsedTime(&ms, a, b);
    if (i >= 2) best = std::min(best, (double)ms);
  }
  return best;
}

int main(int argc, char** argv) {
  int dev = argc > 1 ? atoi(argv[1]) : 0;
  CK(cudaSetDevice(dev));
  cudaDeviceProp p; CK(cudaGetDeviceProperties(&p, dev));
  printf("{\"device\": %d, \"name\": \"%s\", \"sms\": %d, \"pci_bus\": %d, \"canMapHost\": %d, \"pageableMemoryAccess\": %d}\n",
         dev, p.name, p.multiProcessorCount, p.pciBusID, p.canMapHostMemory, p.pageableMemoryAccess);
  cudaStream_t s; CK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
  const size_t GiB = 1ull << 30;
  void *d, *d2, *h;
  CK(cudaMalloc(&d, GiB)); CK(cudaMalloc(&d2, GiB));
  CK(cudaMemset(d, 0x5a, GiB));
  CK(cudaHostAlloc(&h, GiB, cudaHostAllocMapped | cudaHostAllocPortable));
  memset(h, 1, GiB);
  size_t sizes[] = {4ull << 20, 64ull << 20, GiB};
  for (size_t n : sizes) {
    double d2h = best_copy(h, d, n, cudaMemcpyDeviceToHost, s, 10);
    double h2d = best_copy(d, h, n, cudaMemcpyHostToDevice, s, 10);
    printf("{\"probe\": \"memcpy_pinned\", \"bytes\": %zu, \"d2h_gbs\": %.2f, \"h2d_gbs\": %.2f}\n", n, d2h, h2d);
  }
  // chunked D2H: 64 MiB pieces back-to-back on one stream, and on 2 streams
  {
    cudaStream_t s2; cudaStreamCreateWithFlags(&s2, cudaStreamNonBlocking);
    cudaEvent_t j; cudaEventCreate(&j);
    size_t ch = 4ull << 20;
    double ms = time_ms(s, 5, [&] {
      for (size_t o = 0; o < GiB; o += ch) cudaMemcpyAsync((char*)h + o, (char*)d + o, ch, cudaMemcpyDeviceToHost, s);
    });
    printf("{\"probe\": \"memcpy_d2h_chunked_4MiB\", \"gbs\": %.2f}\n", GiB / (ms * 1e-3) / 1e9);
    ms = time_ms(s, 5, [&] {
      cudaEventRecord(j, s); cudaStreamWaitEvent(s2, j, 0);
      for (size_t o = 0; o < GiB; o += 2 * ch) {
        cudaMemcpyAsync((char*)h + o, (char*)d + o, ch, cudaMemcpyDeviceToHost, s);
        cudaMemcpyAsync((char*)h + o + ch, (char*)d + o + ch, ch, cudaMemcpyDeviceToHost, s2);
      }
      cudaEventRecord(j, s2); cudaStreamWaitEvent(s, j, 0);
    });
    printf("{\"probe\": \"memcpy_d2h_2streams_4MiB\", \"gbs\": %.2f}\n", GiB / (ms * 1e-3) / 1e9);
    // bidirectional
    ms = time_ms(s, 5, [&] {
      cudaEventRecord(j, s); cudaStreamWaitEvent(s2, j, 0);
      cudaMemcpyAsync(h, d, GiB / 2, cudaMemcpyDeviceToHost, s);
      cudaMemcpyAsync(d2, (char*)h + GiB / 2, GiB / 2, cudaMemcpyHostToDevice, s2);
      cudaEventRecord(j, s2); cudaStreamWaitEvent(s, j, 0);
    });
    printf("{\"probe\": \"memcpy_bidir_512MiB_each\", \"gbs_total\": %.2f}\n", GiB / (ms * 1e-3) / 1e9);
  }
  // zero-copy SM stores into host-mapped memory
  {
    void* hd; CK(cudaHostGetDevicePointer(&hd, h, 0));
    size_t n = 256ull << 20;
    int ctas[] = {1, 2, 4, 8, 16, 32, 64, 148, 296, 592};
    for (int c : ctas) {
      double ms = time_ms(s, 5, [&] { zc_write<<<c, 512, 0, s>>>((int4*)hd, (const int4*)d, n / 16); });
      printf("{\"probe\": \"zerocopy_stg128\", \"ctas\": %d, \"gbs\": %.2f}\n", c, n / (ms * 1e-3) / 1e9);
    }
    cudaFuncSetAttribute(tma_s2g, cudaFuncAttributeMaxDynamicSharedMemorySize, 16384);
    for (int c : ctas) {
      double ms = time_ms(s, 5, [&] { tma_s2g<<<c, 256, 16384, s>>>((char*)hd, (const int4*)d, n / 16384); });
      printf("{\"probe\": \"zerocopy_tma_bulk_s2g\", \"ctas\": %d, \"gbs\": %.2f}\n", c, n / (ms * 1e-3) / 1e9);
    }
    cudaError_t e = cudaStreamSynchronize(s);
    // check correctness of TMA path
    memset(h, 0, n);
    tma_s2g<<<148, 256, 16384, s>>>((char*)hd, (const int4*)d, n / 16384);
    cudaStreamSynchronize(s);
    size_t bad = 0; for (size_t i = 0; i < n; ++i) bad += ((unsigned char*)h)[i] != 0x5a;
    printf("{\"probe\": \"tma_s2g_host_correct\", \"err\": \"%s\", \"bad_bytes\": %zu}\n", cudaGetErrorString(e), bad);
    double ms = time_ms(s, 5, [&] { hbm_copy<<<148 * 8, 512, 0, s>>>((int4*)d2, (const int4*)d, GiB / 16); });
    printf("{\"probe\": \"hbm_copy_kernel\", \"gbs_rw\": %.1f}\n", 2.0 * GiB / (ms * 1e-3) / 1e9);
  }
  // tmpfs file mapping registered as pinned staging
  {
    const char* path = argc > 2 ? argv[2] : "/dev/shm/pcc_probe.bin";
    int fd = open(path, O_RDWR | O_CREAT | O_TRUNC, 0600);
    size_t n = 256ull << 20;
    int rc = ftruncate(fd, n);
    void* m = mmap(nullptr, n, PROT_READ | PROT_WRITE, MAP_SHARED, fd, 0);
    memset(m, 0, n);
    cudaError_t e = cudaHostRegister(m, n, cudaHostRegisterMapped | cudaHostRegisterPortable);
    double gbs = 0;
    if (e == cudaSuccess) gbs = best_copy(m, d, n, cudaMemcpyDeviceToHost, s, 5);
    printf("{\"probe\": \"register_file_mmap\", \"path\": \"%s\", \"ftruncate\": %d, \"err\": \"%s\", \"d2h_gbs\": %.2f}\n",
           path, rc, cudaGetErrorString(e), gbs);
    cudaGetLastError();
    if (e == cudaSuccess) cudaHostUnregister(m);
    munmap(m, n); close(fd); unlink(path);
    // host memcpy bandwidth, 1 thread
    void* a = aligned_alloc(4096, n); void* b2 = aligned_alloc(4096, n);
    memset(a, 3, n); memset(b2, 0, n);
    auto t0 = std::chrono::steady_clock::now();
    for (int i = 0; i < 3; ++i) memcpy(b2, a, n);
    auto t1 = std::chrono::steady_clock::now();
    printf("{\"probe\": \"host_memcpy_1thread\", \"gbs\": %.2f}\n", 3.0 * n / std::chrono::duration<double>(t1 - t0).count() / 1e9);
  }
  return 0;
}

// Diagnostic (round 2): a stream made to wait (cuStreamWaitValue32) for work ANOTHER host
// thread enqueues later, while the first thread blocks in a synchronous CUDA call on that
// stream — which CUDA calls of the second thread still go through?  Each step of the helper
// thread prints a timestamp; a step that never prints is blocked behind the first thread.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O2 -o tools/exp/gate_probe tools/exp/gate_probe.cu
//   tools/exp/gate_probe <mode>   mode: pageable | streamsync | eventsync | hostwait
#include <cuda.h>
#include <cuda_runtime.h>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <thread>
#include <vector>

using WaitFn = CUresult (*)(CUstream, CUdeviceptr, cuuint32_t, unsigned int);
using WriteFn = CUresult (*)(CUstream, CUdeviceptr, cuuint32_t, unsigned int);
static double t0s;
static double now() {
  return std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now().time_since_epoch()).count() - t0s;
}
#define STEP(x)                                                                              \
  do {                                                                                       \
    auto r_ = (x);                                                                           \
    std::printf("  helper %8.1f ms  %-60s -> %d\n", now(), #x, (int)r_);                     \
    std::fflush(stdout);                                                                     \
  } while (0)

__global__ void k_touch(int *p) { if (threadIdx.x == 0) p[0] += 1; }
__global__ void k_cold(int *p) { if (threadIdx.x == 0) p[1] += 1; }  // never launched before the gate

int main(int argc, char **argv) {
  const char *mode = argc > 1 ? argv[1] : "pageable";
  const bool host_word = argc > 2 && !std::strcmp(argv[2], "hostword");
  // argv[3]: "warm" = k_touch launched once before the gate (module loaded);
  //          "warmcold" = also the main thread launches the never-loaded k_cold on another
  //          stream while the gate is closed (a lazy module load racing the helper)
  const char *warm = argc > 3 ? argv[3] : "";
  t0s = now();
  cudaSetDevice(0);
  cudaFree(0);
  void *w = nullptr, *x = nullptr;
  cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPointByVersion("cuStreamWaitValue32", &w, 12000, cudaEnableDefault, &q);
  cudaGetDriverEntryPointByVersion("cuStreamWriteValue32", &x, 12000, cudaEnableDefault, &q);
  WaitFn wait32 = (WaitFn)w;
  WriteFn write32 = (WriteFn)x;
  uint32_t *gate = nullptr, *hgate = nullptr;
  if (host_word) {
    cudaHostAlloc(&hgate, 4, cudaHostAllocMapped);
    *hgate = 0;
    cudaHostGetDevicePointer((void **)&gate, hgate, 0);
  } else {
    cudaMalloc(&gate, 4);
    cudaMemset(gate, 0, 4);
  }
  int *dev;
  cudaMalloc(&dev, 64 << 20);
  cudaMemset(dev, 0, 64 << 20);
  std::vector<char> pageable(64 << 20);
  cudaStream_t s, s2, s3;
  cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
  cudaStreamCreateWithFlags(&s2, cudaStreamNonBlocking);
  cudaStreamCreateWithFlags(&s3, cudaStreamNonBlocking);
  if (!std::strcmp(warm, "warm") || !std::strcmp(warm, "warmcold")) k_touch<<<1, 32, 0, s2>>>(dev);
  cudaDeviceSynchronize();
  // the "training" stream waits for the gate
  std::printf("mode %s, gate in %s memory, %s\n", mode, host_word ? "host-mapped" : "device", warm);
  CUresult r = wait32((CUstream)s, (CUdeviceptr)gate, 1, CU_STREAM_WAIT_VALUE_GEQ);
  std::printf("main %8.1f ms  wait32 enqueued -> %d\n", now(), (int)r);
  cudaEvent_t ev_s;
  cudaEventCreate(&ev_s);
  cudaEventRecord(ev_s, s);
  std::thread helper([&] {
    std::this_thread::sleep_for(std::chrono::milliseconds(300));
    cudaSetDevice(0);
    cudaEvent_t ev;
    STEP(cudaEventCreateWithFlags(&ev, cudaEventDisableTiming));
    STEP(cudaEventRecord(ev, s2));
    k_touch<<<1, 32, 0, s2>>>(dev);
    STEP(cudaGetLastError());
    STEP(cudaStreamWaitEvent(s3, ev, 0));
    STEP(cudaMemsetAsync(dev, 0, 4096, s2));
    STEP(cudaEventSynchronize(ev));
    STEP(cudaStreamSynchronize(s2));
    int *tmp = nullptr;
    STEP(cudaMallocHost(&tmp, 4096));
    STEP(cudaMemcpyAsync(tmp, dev, 4096, cudaMemcpyDeviceToHost, s2));
    STEP(cudaStreamSynchronize(s2));
    if (host_word) {
      __atomic_store_n(hgate, 1u, __ATOMIC_SEQ_CST);
      std::printf("  helper %8.1f ms  host store gate = 1\n", now());
    } else {
      STEP(write32((CUstream)s2, (CUdeviceptr)gate, 1, CU_STREAM_WRITE_VALUE_DEFAULT));
    }
    std::fflush(stdout);
  });
  // the main thread blocks on the gated stream
  double a = now();
  if (!std::strcmp(warm, "warmcold")) {
    std::this_thread::sleep_for(std::chrono::milliseconds(100));
    k_cold<<<1, 32, 0, s3>>>(dev);  // lazy load of a fresh kernel while s is blocked
    std::printf("main %8.1f ms  k_cold launched -> %d\n", now(), (int)cudaGetLastError());
  }
  if (!std::strcmp(mode, "pageable")) {
    cudaMemcpyAsync(pageable.data(), dev, 64 << 20, cudaMemcpyDeviceToHost, s);
  } else if (!std::strcmp(mode, "streamsync")) {
    k_touch<<<1, 32, 0, s>>>(dev);
    cudaStreamSynchronize(s);
  } else if (!std::strcmp(mode, "eventsync")) {
    cudaEventRecord(ev_s, s);
    cudaEventSynchronize(ev_s);
  } else {  // hostwait: the main thread does not enter CUDA while waiting
    while (cudaEventQuery(ev_s) == cudaErrorNotReady) std::this_thread::sleep_for(std::chrono::milliseconds(1));
  }
  std::printf("main %8.1f ms  released after %.1f ms\n", now(), now() - a);
  helper.join();
  std::printf("done\n");
  return 0;
}

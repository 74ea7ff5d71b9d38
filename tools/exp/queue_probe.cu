// Diagnostic (round 2): while one host thread is blocked inside a launch because the GPU's
// launch queue is full (a training loop running far ahead of the GPU), do another thread's
// CUDA calls (the library's D2H copies, event queries) still go through?
//   nvcc -gencode arch=compute_100a,code=sm_100a -O2 -o tools/exp/queue_probe tools/exp/queue_probe.cu
//   tools/exp/queue_probe kernels|graphs
#include <cuda_runtime.h>
#include <chrono>
#include <cstdio>
#include <cstring>
#include <thread>

static double t0s;
static double now() {
  return std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now().time_since_epoch()).count() - t0s;
}
__global__ void k_sleep(unsigned ns) { __nanosleep(ns); }

int main(int argc, char **argv) {
  const bool graphs = argc > 1 && !std::strcmp(argv[1], "graphs");
  t0s = now();
  cudaSetDevice(0);
  cudaStream_t s, s2;
  cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
  cudaStreamCreateWithFlags(&s2, cudaStreamNonBlocking);
  char *dev, *host;
  cudaMalloc(&dev, 256 << 20);
  cudaMallocHost(&host, 256 << 20);
  k_sleep<<<1, 32, 0, s>>>(1000);
  cudaGraphExec_t ge = nullptr;
  if (graphs) {
    cudaGraph_t g;
    cudaStreamBeginCapture(s, cudaStreamCaptureModeThreadLocal);
    for (int i = 0; i < 200; ++i) k_sleep<<<1, 32, 0, s>>>(20000);  // 200 x 20 us = 4 ms per replay
    cudaStreamEndCapture(s, &g);
    cudaGraphInstantiate(&ge, g, 0);
  }
  cudaDeviceSynchronize();
  double last_launch = 0;
  std::thread helper([&] {
    std::this_thread::sleep_for(std::chrono::milliseconds(300));
    cudaEvent_t ev;
    double a = now();
    cudaEventCreateWithFlags(&ev, cudaEventDisableTiming);
    double b = now();
    cudaMemcpyAsync(host, dev, 256 << 20, cudaMemcpyDeviceToHost, s2);  // ~4.5 ms of link
    double c = now();
    cudaEventRecord(ev, s2);
    double d = now();
    cudaEventSynchronize(ev);
    double e = now();
    std::printf("helper: start %.1f ms; eventCreate %.2f ms, memcpyAsync %.2f ms, eventRecord %.2f ms, "
                "copy done after %.2f ms (main's last launch returned at %.1f ms)\n",
                a, b - a, c - b, d - c, e - d, last_launch);
  });
  // main: far more work than the queue holds
  for (int i = 0; i < (graphs ? 400 : 60000); ++i) {
    if (graphs) cudaGraphLaunch(ge, s);
    else k_sleep<<<1, 32, 0, s>>>(20000);
    last_launch = now();
  }
  double f = now();
  cudaStreamSynchronize(s);
  std::printf("main: enqueue loop ended at %.1f ms, GPU done at %.1f ms\n", f, now());
  helper.join();
  return 0;
}

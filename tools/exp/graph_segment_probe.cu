// Sub-1 MiB D2H copies issued as CUDA-graph segments (DESIGN §11 item 4): per buffer, one
// instantiated graph of K chained 1D copy nodes of q bytes (K*q = one 64 MiB segment); per segment
// the host re-points the nodes (cudaGraphExecMemcpyNodeSetParams1D; the template graph stays
// alive, its node handles name the nodes) and launches the graph — no host call per copy.
// 4 GiB device -> pinned host; meanwhile 3000 tiny kernels on another stream, timed with CUDA
// events (device us per kernel).  Compared with plain cudaMemcpyAsync streams of 64 MiB and 1 MiB
// copies.  Not part of the product path.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O2 -o tools/exp/graph_segment_probe tools/exp/graph_segment_probe.cu
#include <cuda_runtime.h>
#include <chrono>
#include <cstdio>
#include <cstring>
#include <vector>

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { printf("{\"error\": \"%s at line %d\"}\n", cudaGetErrorString(e_), __LINE__); return 1; } } while (0)

__global__ void tiny(float *x) { if (threadIdx.x < 32) x[threadIdx.x] += 1.0f; }

static float launch_us(cudaStream_t s, float *x, int n) {
    cudaEvent_t a, b;
    cudaEventCreate(&a); cudaEventCreate(&b);
    cudaEventRecord(a, s);
    for (int i = 0; i < n; ++i) tiny<<<1, 32, 0, s>>>(x);
    cudaEventRecord(b, s);
    cudaEventSynchronize(b);
    float ms = 0; cudaEventElapsedTime(&ms, a, b);
    cudaEventDestroy(a); cudaEventDestroy(b);
    return ms * 1e3f / n;
}

int main() {
    const size_t N = 4ull << 30, SEG = 64ull << 20;
    char *src, *dst;
    float *x;
    CK(cudaMalloc(&src, N)); CK(cudaMallocHost(&dst, N)); CK(cudaMalloc(&x, 4096));
    CK(cudaMemset(src, 7, N));
    cudaStream_t cs, ks;
    CK(cudaStreamCreateWithFlags(&cs, cudaStreamNonBlocking)); CK(cudaStreamCreateWithFlags(&ks, cudaStreamNonBlocking));
    for (int i = 0; i < 3; ++i) launch_us(ks, x, 1000);
    printf("{\"kind\": \"alone\", \"us\": %.2f}\n", launch_us(ks, x, 3000));
    fflush(stdout);
    const size_t qs[] = {64u << 20, 1u << 20, 1u << 20, 512u << 10, 256u << 10};
    const bool graphs[] = {false, false, true, true, true};
    for (int ci = 0; ci < 5; ++ci) {
        const size_t q = qs[ci], K = SEG / q;
        const bool g = graphs[ci];
        cudaGraph_t gr[2] = {nullptr, nullptr};
        cudaGraphExec_t ex[2] = {nullptr, nullptr};
        std::vector<cudaGraphNode_t> nodes[2];
        if (g) {
            for (int b = 0; b < 2; ++b) {
                CK(cudaGraphCreate(&gr[b], 0));
                nodes[b].assign(K, nullptr);
                for (size_t i = 0; i < K; ++i)
                    CK(cudaGraphAddMemcpyNode1D(&nodes[b][i], gr[b], i ? &nodes[b][i - 1] : nullptr, i ? 1 : 0, dst + i * q,
                                                src + i * q, q, cudaMemcpyDeviceToHost));
                CK(cudaGraphInstantiate(&ex[b], gr[b], 0));
            }
        }
        cudaEvent_t e0, e1;
        cudaEventCreate(&e0); cudaEventCreate(&e1);
        CK(cudaDeviceSynchronize());
        const auto t0 = std::chrono::steady_clock::now();
        cudaEventRecord(e0, cs);
        double upd_ms = 0;
        for (size_t s = 0; s < N / SEG; ++s) {
            if (!g) {
                for (size_t i = 0; i < K; ++i)
                    CK(cudaMemcpyAsync(dst + s * SEG + i * q, src + s * SEG + i * q, q, cudaMemcpyDeviceToHost, cs));
            } else {
                const int b = s & 1;
                const auto tu = std::chrono::steady_clock::now();
                for (size_t i = 0; i < K; ++i)
                    CK(cudaGraphExecMemcpyNodeSetParams1D(ex[b], nodes[b][i], dst + s * SEG + i * q, src + s * SEG + i * q, q,
                                                          cudaMemcpyDeviceToHost));
                upd_ms += std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - tu).count();
                CK(cudaGraphLaunch(ex[b], cs));
            }
        }
        cudaEventRecord(e1, cs);
        const double issue_ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
        const float us = launch_us(ks, x, 3000);
        const bool done_early = cudaEventQuery(e1) == cudaSuccess;
        CK(cudaEventSynchronize(e1));
        float ms = 0; cudaEventElapsedTime(&ms, e0, e1);
        const bool ok = dst[N - 1] == 7 && dst[0] == 7 && dst[N / 2 + 12345] == 7;
        printf("{\"kind\": \"%s\", \"copy_kib\": %zu, \"issue_ms\": %.1f, \"update_ms\": %.1f, \"d2h_ms\": %.1f, \"d2h_gbs\": %.1f, "
               "\"us_per_launch_during\": %.2f, \"transfer_done_before_launches_end\": %s, \"bytes_ok\": %s}\n",
               g ? "graph_segments" : "stream", q >> 10, issue_ms, upd_ms, ms, N / (ms * 1e-3) / 1e9, us,
               done_early ? "true" : "false", ok ? "true" : "false");
        fflush(stdout);
        memset(dst, 0, 16); memset(dst + N - 16, 0, 16); dst[N / 2 + 12345] = 0;
        cudaEventDestroy(e0); cudaEventDestroy(e1);
        for (int b = 0; b < 2; ++b) {
            if (ex[b]) cudaGraphExecDestroy(ex[b]);
            if (gr[b]) cudaGraphDestroy(gr[b]);
        }
    }
    printf("{\"kind\": \"alone\", \"us\": %.2f}\n", launch_us(ks, x, 3000));
    return 0;
}

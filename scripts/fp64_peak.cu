// Measured fp64 (DFMA) peak of this B200, the denominator of the fused kernel's roofline
// ("Measure the DFMA peak under sustained load ... quote both spec and measured").
//
// Every thread runs 8 independent DFMA chains (enough ILP to cover the DFMA latency with 8
// warps per SMSP); the grid is 148 SM x 8 CTAs of 256 threads.  Reports
//   burst:     one ~50 ms launch after a warm-up, CUDA events;
//   sustained: back-to-back launches for ~6 s (the power cap engages), CUDA events around the
//              whole loop.
// Output: one JSON line.  Clocks are sampled by the caller (scripts/fp64_peak.sh) with nvidia-smi.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o fp64_peak scripts/fp64_peak.cu
#include <cuda_runtime.h>

#include <chrono>
#include <cstdio>

constexpr int kChains = 8;

__global__ void __launch_bounds__(256) dfma_loop(double* out, int iters, double a, double b) {
    double x[kChains];
#pragma unroll
    for (int c = 0; c < kChains; ++c) x[c] = 1.0 + 1e-3 * (threadIdx.x + c);
    for (int i = 0; i < iters; ++i) {
#pragma unroll
        for (int u = 0; u < 16; ++u) {
#pragma unroll
            for (int c = 0; c < kChains; ++c) x[c] = fma(x[c], a, b);
        }
    }
    double s = 0.0;
#pragma unroll
    for (int c = 0; c < kChains; ++c) s += x[c];
    if (s == 12345.678) out[0] = s;  // keeps the chains live; never true
}

int main() {
    int dev = 0, sms = 0, clk_khz = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    cudaDeviceGetAttribute(&clk_khz, cudaDevAttrClockRate, dev);
    double* out;
    cudaMalloc(&out, 64);
    const int blocks = sms * 8, threads = 256, iters = 2048;
    const double dfma_per_launch = (double)blocks * threads * iters * 16 * kChains;
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    const double a = 0.9999999999, b = 1e-12;
    for (int w = 0; w < 3; ++w) dfma_loop<<<blocks, threads>>>(out, iters, a, b);
    cudaEventRecord(e0);
    dfma_loop<<<blocks, threads>>>(out, iters, a, b);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms_burst = 0.f;
    cudaEventElapsedTime(&ms_burst, e0, e1);
    // sustained: ~6 s of back-to-back launches
    const int n_sus = (int)(6000.0 / ms_burst) + 1;
    cudaEventRecord(e0);
    for (int i = 0; i < n_sus; ++i) dfma_loop<<<blocks, threads>>>(out, iters, a, b);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms_sus = 0.f;
    cudaEventElapsedTime(&ms_sus, e0, e1);
    const cudaError_t e = cudaDeviceSynchronize();
    const double tf_burst = 2.0 * dfma_per_launch / (ms_burst * 1e-3) / 1e12;
    const double tf_sus = 2.0 * dfma_per_launch * n_sus / (ms_sus * 1e-3) / 1e12;
    printf("{\"fp64_tflops_burst\": %.3f, \"fp64_tflops_sustained\": %.3f, \"burst_ms\": %.3f, "
           "\"sustained_s\": %.3f, \"sustained_launches\": %d, \"sms\": %d, \"attr_clock_mhz\": %.0f, "
           "\"dfma_per_sm_per_clk_at_attr_clock_burst\": %.2f, \"status\": \"%s\"}\n",
           tf_burst, tf_sus, ms_burst, ms_sus * 1e-3, n_sus, sms, clk_khz / 1e3,
           tf_burst * 1e12 / 2.0 / sms / (clk_khz * 1e3), cudaGetErrorString(e));
    return e == cudaSuccess ? 0 : 1;
}

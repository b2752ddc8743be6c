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

template <int kChains>
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

// Burst and ~6 s sustained TFLOP/s of dfma_loop<CH> with `bps` CTAs of 256 threads per SM.
template <int CH>
void measure(int sms, int bps, double* out, double* burst, double* sus, int* n_sus_out, float* ms_burst_out,
             float* ms_sus_out) {
    const int blocks = sms * bps, threads = 256, iters = 2048 * 8 / CH;
    const double dfma_per_launch = (double)blocks * threads * iters * 16 * CH;
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    const double a = 0.9999999999, b = 1e-12;
    for (int w = 0; w < 3; ++w) dfma_loop<CH><<<blocks, threads>>>(out, iters, a, b);
    cudaEventRecord(e0);
    dfma_loop<CH><<<blocks, threads>>>(out, iters, a, b);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms_burst = 0.f;
    cudaEventElapsedTime(&ms_burst, e0, e1);
    const int n_sus = (int)(6000.0 / ms_burst) + 1;
    cudaEventRecord(e0);
    for (int i = 0; i < n_sus; ++i) dfma_loop<CH><<<blocks, threads>>>(out, iters, a, b);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms_sus = 0.f;
    cudaEventElapsedTime(&ms_sus, e0, e1);
    *burst = 2.0 * dfma_per_launch / (ms_burst * 1e-3) / 1e12;
    *sus = 2.0 * dfma_per_launch * n_sus / (ms_sus * 1e-3) / 1e12;
    *n_sus_out = n_sus;
    *ms_burst_out = ms_burst;
    *ms_sus_out = ms_sus;
}

int main() {
    int dev = 0, sms = 0, clk_khz = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    cudaDeviceGetAttribute(&clk_khz, cudaDevAttrClockRate, dev);
    double* out;
    cudaMalloc(&out, 64);
    // three shapes (ILP x occupancy); the best is the peak
    double bu[3], su[3];
    int ns[3];
    float mb[3], msu[3];
    measure<8>(sms, 8, out, &bu[0], &su[0], &ns[0], &mb[0], &msu[0]);
    measure<16>(sms, 4, out, &bu[1], &su[1], &ns[1], &mb[1], &msu[1]);
    measure<4>(sms, 8, out, &bu[2], &su[2], &ns[2], &mb[2], &msu[2]);
    const cudaError_t e = cudaDeviceSynchronize();
    int best = 0;
    for (int i = 1; i < 3; ++i)
        if (su[i] > su[best]) best = i;
    printf("{\"fp64_tflops_burst\": %.3f, \"fp64_tflops_sustained\": %.3f, \"shapes\": [", bu[best], su[best]);
    const char* names[3] = {"8 chains x 8 CTAs/SM", "16 chains x 4 CTAs/SM", "4 chains x 8 CTAs/SM"};
    for (int i = 0; i < 3; ++i)
        printf("%s{\"shape\": \"%s\", \"burst\": %.3f, \"sustained\": %.3f, \"sustained_s\": %.2f, "
               "\"launches\": %d}",
               i ? ", " : "", names[i], bu[i], su[i], msu[i] * 1e-3, ns[i]);
    printf("], \"sms\": %d, \"attr_clock_mhz\": %.0f, \"dfma_per_sm_per_clk_at_attr_clock\": %.2f, "
           "\"status\": \"%s\"}\n",
           sms, clk_khz / 1e3, su[best] * 1e12 / 2.0 / sms / (clk_khz * 1e3), cudaGetErrorString(e));
    return e == cudaSuccess ? 0 : 1;
}

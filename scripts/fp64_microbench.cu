// Throughput and latency of the instructions the fused kernel is built from, on this B200
// (sm_100a): DFMA, DMUL, DADD, DSETP+FSEL, F2I.F64, the magic-number floor, MUFU.RCP64H,
// MUFU.RSQ64H, FFMA, IMAD, LOP3.  Decides which forms the per-det-sample arithmetic uses.
// Throughput: 148 x 8 warps x (8 independent chains) per thread; latency: 1 warp, 1 chain.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o fp64_microbench scripts/fp64_microbench.cu
#include <cstdio>
#include <cuda_runtime.h>

constexpr int kIters = 4096;

template <int OP, int CH>
__global__ void bench(double* out, double seed, long long* cyc) {
    double x[CH];
    int xi[CH];
#pragma unroll
    for (int c = 0; c < CH; ++c) {
        x[c] = seed + 1e-3 * (threadIdx.x + c);
        xi[c] = threadIdx.x + c;
    }
    const double a = 0.999999, b = 1e-9;
    long long t0 = clock64();
#pragma unroll 4
    for (int i = 0; i < kIters; ++i) {
#pragma unroll
        for (int c = 0; c < CH; ++c) {
            if (OP == 0) x[c] = fma(x[c], a, b);                         // DFMA
            if (OP == 1) x[c] = x[c] * a;                                // DMUL
            if (OP == 2) x[c] = x[c] + b;                                // DADD
            if (OP == 3) x[c] = (x[c] > 1.0) ? x[c] * 0.5 : x[c] + 1.0;  // DSETP + select-ish
            if (OP == 4) {                                               // F2I.F64 + I2F-free back
                const int k = (int)x[c];
                x[c] = __hiloint2double(0x43300000, k + 7) - 4503599627370496.0 + b;
            }
            if (OP == 5) {  // rcp.approx.ftz.f64
                double r;
                asm volatile("rcp.approx.ftz.f64 %0, %1;" : "=d"(r) : "d"(x[c]));
                x[c] = r;
            }
            if (OP == 6) {  // rsqrt.approx.ftz.f64
                double r;
                asm volatile("rsqrt.approx.ftz.f64 %0, %1;" : "=d"(r) : "d"(x[c]));
                x[c] = r + 1.0;
            }
            if (OP == 7) {  // FFMA
                float f = __double2float_rn(0.0);
                (void)f;
                xi[c] = __float_as_int(fmaf(__int_as_float(xi[c]), 0.9999f, 1e-7f));
            }
            if (OP == 8) xi[c] = xi[c] * 0x9E3779B1 + 7;           // IMAD
            if (OP == 9) xi[c] = (xi[c] ^ 0x5555) & (xi[c] >> 1);  // LOP3 (+SHF)
            if (OP == 10) x[c] = -fabs(x[c]) * a;                   // DMUL with modifiers
        }
    }
    long long t1 = clock64();
    double s = 0.0;
    int si = 0;
#pragma unroll
    for (int c = 0; c < CH; ++c) {
        s += x[c];
        si += xi[c];
    }
    out[blockIdx.x * blockDim.x + threadIdx.x] = s + si;
    if (threadIdx.x == 0 && blockIdx.x == 0) *cyc = t1 - t0;
}

template <int OP>
void run(const char* name, double* out, long long* cyc) {
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    // throughput
    bench<OP, 8><<<148 * 4, 256>>>(out, 1.5, cyc);
    cudaEventRecord(e0);
    bench<OP, 8><<<148 * 4, 256>>>(out, 1.5, cyc);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    long long c_thr;
    cudaMemcpy(&c_thr, cyc, 8, cudaMemcpyDeviceToHost);
    const double ops = 148.0 * 4 * 256 * 8 * kIters;
    int clk_khz;
    cudaDeviceGetAttribute(&clk_khz, cudaDevAttrClockRate, 0);
    // latency: one warp, one chain
    bench<OP, 1><<<1, 32>>>(out, 1.5, cyc);
    cudaDeviceSynchronize();
    long long c_lat;
    cudaMemcpy(&c_lat, cyc, 8, cudaMemcpyDeviceToHost);
    // thread-ops per SM per cycle, using the SM cycles of block 0 (all blocks resident at once)
    printf("%-22s thr %7.2f thread-op/clk/SM (%8.2f Gop/s)   dep-latency %6.2f clk/op\n", name,
           ops / 148.0 / (double)c_thr, ops / (ms * 1e-3) / 1e9, (double)c_lat / kIters);
}

int main() {
    double* out;
    long long* cyc;
    cudaMalloc(&out, 148 * 4 * 256 * sizeof(double));
    cudaMalloc(&cyc, 8);
    run<0>("DFMA", out, cyc);
    run<1>("DMUL", out, cyc);
    run<2>("DADD", out, cyc);
    run<3>("DSETP+DMUL/DADD+sel", out, cyc);
    run<4>("F2I.F64+DADD", out, cyc);
    run<5>("MUFU.RCP64H", out, cyc);
    run<6>("MUFU.RSQ64H+DADD", out, cyc);
    run<7>("FFMA", out, cyc);
    run<8>("IMAD", out, cyc);
    run<9>("LOP3+SHF", out, cyc);
    run<10>("DMUL -|x|", out, cyc);
    cudaError_t e = cudaDeviceSynchronize();
    printf("status: %s\n", cudaGetErrorString(e));
    return 0;
}

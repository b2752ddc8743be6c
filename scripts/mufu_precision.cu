// Measures the relative error of the sm_100a fp64 MUFU seeds (rcp.approx.ftz.f64,
// rsqrt.approx.ftz.f64) and of their Newton refinements, over 2^24 random inputs in [1, 4):
// decides how many refinement steps the fused kernel's fast_rcp / fast_sqrt need.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o mufu_precision scripts/mufu_precision.cu
#include <cstdio>
#include <cmath>
__device__ unsigned long long g_max[6];
__device__ double atomicMaxD(unsigned long long* a, double v) {
    return (double)atomicMax(a, (unsigned long long)__double_as_longlong(v));  // v >= 0
}
__global__ void k(int n) {
    int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= n) return;
    unsigned long long h = (unsigned long long)i * 0x9E3779B97F4A7C15ull;
    h ^= h >> 31; h *= 0xBF58476D1CE4E5B9ull; h ^= h >> 29;
    double x = 1.0 + 3.0 * (double)(h >> 11) * 0x1p-53;
    double r; asm("rcp.approx.ftz.f64 %0, %1;" : "=d"(r) : "d"(x));
    double ex = 1.0 / x;
    double e0 = fabs(r - ex) / ex;
    double e = fma(-x, r, 1.0);
    double r1 = fma(r, e, r);                   // quadratic step
    double r3 = fma(r, fma(e, e, e), r);        // cubic step
    double y; asm("rsqrt.approx.ftz.f64 %0, %1;" : "=d"(y) : "d"(x));
    double ey = 1.0 / sqrt(x);
    double y1 = y * fma(-0.5 * x, y * y, 1.5);
    atomicMaxD(&g_max[0], e0);
    atomicMaxD(&g_max[1], fabs(r1 - ex) / ex);
    atomicMaxD(&g_max[2], fabs(r3 - ex) / ex);
    atomicMaxD(&g_max[3], fabs(y - ey) / ey);
    atomicMaxD(&g_max[4], fabs(y1 - ey) / ey);
}
int main() {
    int n = 1 << 24;
    k<<<n / 256, 256>>>(n);
    unsigned long long h[6];
    cudaMemcpyFromSymbol(h, g_max, sizeof(h));
    const char* nm[5] = {"rcp.approx", "rcp+1 quadratic", "rcp+1 cubic", "rsqrt.approx", "rsqrt+1 newton"};
    for (int i = 0; i < 5; ++i) {
        double v = __builtin_bit_cast(double, h[i]);
        printf("%-18s max rel err %.3e (2^%.1f)\n", nm[i], v, log2(v));
    }
    return 0;
}

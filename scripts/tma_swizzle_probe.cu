// Dump the shared-memory layout a TMA load produces for a [32 rows][8 f64] box with each swizzle
// mode: smem[i] = value (100 row + col) found at double slot i.  Build: nvcc -gencode
// arch=compute_100a,code=sm_100a -o probe scripts/tma_swizzle_probe.cu -lcuda
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>

__global__ void k(const __grid_constant__ CUtensorMap m, double* out) {
    __shared__ __align__(1024) double s[256];
    __shared__ __align__(8) unsigned long long bar;
    unsigned sb = (unsigned)__cvta_generic_to_shared(&bar), ss = (unsigned)__cvta_generic_to_shared(s);
    if (threadIdx.x == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(sb));
        asm volatile("fence.mbarrier_init.release.cluster;");
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(sb), "r"(2048));
        asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];"
                     ::"r"(ss), "l"(&m), "r"(8), "r"(0), "r"(sb) : "memory");
        unsigned done = 0;
        while (!done)
            asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0; selp.u32 %0, 1, 0, p; }"
                         : "=r"(done) : "r"(sb));
    }
    __syncthreads();
    for (int i = threadIdx.x; i < 256; i += blockDim.x) out[i] = s[i];
}

int main() {
    const int rows = 32, cols = 64;
    double h[rows * cols];
    for (int r = 0; r < rows; ++r)
        for (int c = 0; c < cols; ++c) h[r * cols + c] = 100 * r + c;
    double *g, *o;
    cudaMalloc(&g, sizeof(h));
    cudaMalloc(&o, 256 * 8);
    cudaMemcpy(g, h, sizeof(h), cudaMemcpyHostToDevice);
    CUtensorMapSwizzle modes[3] = {CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_SWIZZLE_32B, CU_TENSOR_MAP_SWIZZLE_64B};
    const char* names[3] = {"none", "32B", "64B"};
    for (int mi = 0; mi < 3; ++mi) {
        CUtensorMap m;
        cuuint64_t dims[2] = {(cuuint64_t)cols, (cuuint64_t)rows}, strides[1] = {cols * 8};
        cuuint32_t box[2] = {8, 32}, es[2] = {1, 1};
        CUresult r = cuTensorMapEncodeTiled(&m, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 2, g, dims, strides, box, es,
                                            CU_TENSOR_MAP_INTERLEAVE_NONE, modes[mi], CU_TENSOR_MAP_L2_PROMOTION_NONE,
                                            CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
        if (r != CUDA_SUCCESS) { printf("%s: encode failed %d\n", names[mi], (int)r); continue; }
        k<<<1, 128>>>(m, o);
        double s[256];
        cudaMemcpy(s, o, sizeof(s), cudaMemcpyDeviceToHost);
        printf("%s:\n", names[mi]);
        for (int i = 0; i < 64; ++i) printf("%5.0f%s", s[i], (i % 8 == 7) ? "\n" : " ");
    }
    printf("status %s\n", cudaGetErrorString(cudaDeviceSynchronize()));
}

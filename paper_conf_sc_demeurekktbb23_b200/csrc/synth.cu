// synth.cu — on-device generation of the seeded synthetic timestream (bench / test input
// generator, NOT part of the method; include/toast_b200_synth.h).
//
// The same counter-based generator as paper_conf_sc_demeurekktbb23_b200/synth.py:
//   h = mix(mix(mix(seed + G (stream + 1)) + G (det + 1)) + G (sample + 1))   (SplitMix64 finaliser,
//   all mod 2^64), u = (h >> 11) 2^-52 - 1 (an exact dyadic in [-1, 1)), tod[d][s] = sigma[d] u,
// so a 52 GB C4 timestream is produced in HBM in milliseconds and is bit-identical to the host
// generator on any subset (tests/test_synth_gpu.py).  Only integer operations and one fp64
// multiply by an exact power of two, one subtraction of 1 and one multiply by sigma: no
// arithmetic of the pointing->map method.
#include <cuda_runtime.h>

#include <cstdint>

#include "../../include/toast_b200_synth.h"

namespace {

constexpr uint64_t kGolden = 0x9E3779B97F4A7C15ull;

__device__ __forceinline__ uint64_t mix64(uint64_t z) {
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

__global__ void synth_tod_kernel(double* __restrict__ out, const double* __restrict__ sigma,
                                 const int64_t* __restrict__ det_ids, int64_t n_det, int64_t n_samp, uint64_t seed,
                                 uint64_t stream) {
    const uint64_t k0 = mix64(seed + kGolden * (stream + 1));
    for (int64_t d = blockIdx.y; d < n_det; d += gridDim.y) {
        const uint64_t kd = mix64(k0 + kGolden * ((uint64_t)det_ids[d] + 1));
        const double sg = sigma[d];
        for (int64_t s = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; s < n_samp;
             s += (int64_t)gridDim.x * blockDim.x) {
            const uint64_t h = mix64(kd + kGolden * ((uint64_t)s + 1));
            const double u = (double)(h >> 11) * 0x1p-52 - 1.0;  // exact: 53-bit integer times 2^-52
            __stcs(&out[d * n_samp + s], sg * u);               // streamed once: evict-first
        }
    }
}

}  // namespace

extern "C" int toast_synth_tod(double* out, const double* sigma, const int64_t* det_ids, int64_t n_det,
                               int64_t n_samp, uint64_t seed, uint64_t stream_id, void* stream) {
    if (n_det < 0 || n_samp < 0) return -1;
    if (n_det == 0 || n_samp == 0) return 0;
    if (!out || !sigma || !det_ids) return -1;
    const unsigned gx = (unsigned)((n_samp + 255) / 256 < 1184 ? (n_samp + 255) / 256 : 1184);
    const unsigned gy = (unsigned)(n_det < 65535 ? n_det : 65535);
    synth_tod_kernel<<<dim3(gx, gy), 256, 0, (cudaStream_t)stream>>>(out, sigma, det_ids, n_det, n_samp, seed, stream_id);
    return cudaGetLastError() == cudaSuccess ? 0 : -2;
}

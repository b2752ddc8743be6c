// templates.cu — SURVEY 8(f) NEXT rows on sm_100a: the offset-template (destriper) kernels
// f2 and the trivial variants f4 (stokes_weights_I, PAPER.md:125;
// noise_weight).  All are HBM-bound streaming kernels: one thread per sample,
// CTA = (chunk of <= 256 in-interval samples) x detector, coalesced along samples.
#include <cuda_runtime.h>

#include <algorithm>

#include "internal.h"

namespace toastb200 {

namespace {

constexpr unsigned kFullMask = 0xffffffffu;

__device__ __forceinline__ int64_t row_or(const int32_t* __restrict__ index, int64_t d) {
    return index ? (int64_t)__ldg(&index[d]) : d;
}

dim3 grid2(const WorkList& wl, int64_t n_det) {
    return dim3((unsigned)std::min<int64_t>(wl.n_chunks, 0x7fffffff), (unsigned)std::min<int64_t>(n_det, 65535), 1);
}

__global__ void __launch_bounds__(kChunk) stokes_weights_i_kernel(const Chunk* __restrict__ chunks, int64_t n_chunks,
                                                                  const int32_t* __restrict__ weight_index,
                                                                  double* __restrict__ weights, double cal,
                                                                  int64_t n_det, int64_t n_samp) {
    for (int64_t c = blockIdx.x; c < n_chunks; c += gridDim.x) {
        const Chunk ch = chunks[c];
        if ((int)threadIdx.x >= ch.count) continue;
        const int64_t s = ch.first + threadIdx.x;
        for (int64_t d = blockIdx.y; d < n_det; d += gridDim.y) weights[row_or(weight_index, d) * n_samp + s] = cal;
    }
}

__global__ void __launch_bounds__(kChunk) noise_weight_kernel(const Chunk* __restrict__ chunks, int64_t n_chunks,
                                                              const int32_t* __restrict__ data_index,
                                                              double* __restrict__ det_data,
                                                              const double* __restrict__ det_weights, int64_t n_det,
                                                              int64_t n_samp) {
    for (int64_t c = blockIdx.x; c < n_chunks; c += gridDim.x) {
        const Chunk ch = chunks[c];
        if ((int)threadIdx.x >= ch.count) continue;
        const int64_t s = ch.first + threadIdx.x;
        for (int64_t d = blockIdx.y; d < n_det; d += gridDim.y)
            det_data[row_or(data_index, d) * n_samp + s] *= __ldg(&det_weights[d]);
    }
}

// Amplitude of (d, s) under reading O1: amp_offset[d] + view_base[iv] + (s - iv_first[iv]) / step.
__device__ __forceinline__ int64_t offset_index(const OffsetViews& v, const int64_t* __restrict__ amp_offset,
                                                int64_t d, const Chunk& ch, int64_t s) {
    const int64_t first = __ldg(&v.iv_first[ch.interval]);
    return __ldg(&amp_offset[d]) + __ldg(&v.view_base[ch.interval]) + (int64_t)((int)(s - first) / v.step);
}

__global__ void __launch_bounds__(kChunk) offset_add_kernel(const Chunk* __restrict__ chunks, int64_t n_chunks,
                                                            OffsetViews v, const int64_t* __restrict__ amp_offset,
                                                            const double* __restrict__ amplitudes,
                                                            const int32_t* __restrict__ data_index,
                                                            double* __restrict__ det_data, int64_t n_det,
                                                            int64_t n_samp) {
    for (int64_t c = blockIdx.x; c < n_chunks; c += gridDim.x) {
        const Chunk ch = chunks[c];
        if ((int)threadIdx.x >= ch.count) continue;
        const int64_t s = ch.first + threadIdx.x;
        for (int64_t d = blockIdx.y; d < n_det; d += gridDim.y)
            det_data[row_or(data_index, d) * n_samp + s] += __ldg(&amplitudes[offset_index(v, amp_offset, d, ch, s)]);
    }
}

// Projection: the samples of one step are consecutive, so a warp (32 consecutive samples of
// one detector) holds runs of equal amplitude index; each run is summed by a segmented
// shuffle scan and its last lane issues ONE fp64 red.
__global__ void __launch_bounds__(kChunk) offset_project_kernel(
    const Chunk* __restrict__ chunks, int64_t n_chunks, OffsetViews v, const int64_t* __restrict__ amp_offset,
    double* __restrict__ amplitudes, const int32_t* __restrict__ data_index, const double* __restrict__ det_data,
    const int32_t* __restrict__ flag_index, const uint8_t* __restrict__ det_flags, uint8_t det_flag_mask,
    int64_t n_det, int64_t n_samp) {
    const int lane = threadIdx.x & 31;
    for (int64_t c = blockIdx.x; c < n_chunks; c += gridDim.x) {
        const Chunk ch = chunks[c];
        if ((int)(threadIdx.x & ~31u) >= ch.count) continue;  // whole warp past the chunk
        const bool in = (int)threadIdx.x < ch.count;
        const int64_t s = ch.first + threadIdx.x;
        for (int64_t d = blockIdx.y; d < n_det; d += gridDim.y) {
            int64_t key = -1 - lane;
            double val = 0.0;
            if (in) {
                const bool fl = det_flags && (__ldg(&det_flags[row_or(flag_index, d) * n_samp + s]) & det_flag_mask);
                if (!fl) {
                    key = offset_index(v, amp_offset, d, ch, s);
                    val = __ldg(&det_data[row_or(data_index, d) * n_samp + s]);
                }
            }
            const int64_t kprev = __shfl_up_sync(kFullMask, key, 1);
            const unsigned heads = __ballot_sync(kFullMask, lane == 0 || kprev != key);
            const int start = 31 - __clz(heads & (kFullMask >> (31 - lane)));
            const int depth = lane - start;
#pragma unroll
            for (int off = 1; off < 32; off <<= 1) {
                const bool need = depth >= off;
                if (!__any_sync(kFullMask, need)) break;
                const double t = __shfl_up_sync(kFullMask, val, off);
                if (need) val += t;
            }
            const bool tail = lane == 31 || ((heads >> (lane + 1)) & 1u);
            if (tail && key >= 0) atomicAdd(&amplitudes[key], val);
        }
    }
}

__global__ void precond_kernel(const double* __restrict__ var, const double* __restrict__ in,
                               double* __restrict__ out, int64_t n) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        out[i] = __ldg(&var[i]) * __ldg(&in[i]);
}

}  // namespace

cudaError_t launch_stokes_weights_i(const WorkList& wl, const int32_t* weight_index, double* weights, double cal,
                                    int64_t n_det, int64_t n_samp, cudaStream_t st) {
    if (wl.n_chunks == 0 || n_det == 0) return cudaSuccess;
    stokes_weights_i_kernel<<<grid2(wl, n_det), kChunk, 0, st>>>(wl.chunks, wl.n_chunks, weight_index, weights, cal,
                                                                  n_det, n_samp);
    return cudaGetLastError();
}

cudaError_t launch_noise_weight(const WorkList& wl, const int32_t* data_index, double* det_data,
                                const double* det_weights, int64_t n_det, int64_t n_samp, cudaStream_t st) {
    if (wl.n_chunks == 0 || n_det == 0) return cudaSuccess;
    noise_weight_kernel<<<grid2(wl, n_det), kChunk, 0, st>>>(wl.chunks, wl.n_chunks, data_index, det_data,
                                                              det_weights, n_det, n_samp);
    return cudaGetLastError();
}

cudaError_t launch_offset_add(const WorkList& wl, const OffsetViews& v, const int64_t* amp_offset,
                              const double* amplitudes, const int32_t* data_index, double* det_data, int64_t n_det,
                              int64_t n_samp, cudaStream_t st) {
    if (wl.n_chunks == 0 || n_det == 0) return cudaSuccess;
    offset_add_kernel<<<grid2(wl, n_det), kChunk, 0, st>>>(wl.chunks, wl.n_chunks, v, amp_offset, amplitudes,
                                                            data_index, det_data, n_det, n_samp);
    return cudaGetLastError();
}

cudaError_t launch_offset_project(const WorkList& wl, const OffsetViews& v, const int64_t* amp_offset,
                                  double* amplitudes, const int32_t* data_index, const double* det_data,
                                  const int32_t* flag_index, const uint8_t* det_flags, uint8_t det_flag_mask,
                                  int64_t n_det, int64_t n_samp, cudaStream_t st) {
    if (wl.n_chunks == 0 || n_det == 0) return cudaSuccess;
    offset_project_kernel<<<grid2(wl, n_det), kChunk, 0, st>>>(wl.chunks, wl.n_chunks, v, amp_offset, amplitudes,
                                                                data_index, det_data, flag_index, det_flags,
                                                                det_flag_mask, n_det, n_samp);
    return cudaGetLastError();
}

cudaError_t launch_precond(const double* var, const double* in, double* out, int64_t n, cudaStream_t st) {
    if (n <= 0) return cudaSuccess;
    const int64_t blocks = std::min<int64_t>((n + 255) / 256, (int64_t)num_sms() * 8);
    precond_kernel<<<(unsigned)blocks, 256, 0, st>>>(var, in, out, n);
    return cudaGetLastError();
}

}  // namespace toastb200

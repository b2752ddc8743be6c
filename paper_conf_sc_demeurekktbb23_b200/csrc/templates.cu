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

// IDX = false: no row-index array (the common case) — no branch between the loads, so the
// kDT detectors' loads issue back to back.
template <bool IDX>
__device__ __forceinline__ int64_t row_or(const int32_t* __restrict__ index, int64_t d) {
    return (IDX && index) ? (int64_t)__ldg(&index[d]) : d;
}

// A CTA covers kDT detectors of one chunk: each thread keeps kDT independent loads in flight
// (one (chunk, detector) per CTA left a 2 KB CTA with a dependent chunk-descriptor load in
// front of one 8-byte load per thread — latency-bound at ~40 % of HBM bandwidth).
#ifndef TB_TPL_DT
#define TB_TPL_DT 4  // measured best of 1/4/8 (noise_weight 94 %, projection 2x faster than 8)
#endif
constexpr int kDT = TB_TPL_DT;

dim3 grid_dt(const WorkList& wl, int64_t n_det) {
    return dim3((unsigned)std::min<int64_t>(wl.n_chunks, 0x7fffffff),
                (unsigned)std::min<int64_t>((n_det + kDT - 1) / kDT, 65535), 1);
}

template <bool IDX>
__global__ void __launch_bounds__(kChunk) stokes_weights_i_kernel(const Chunk* __restrict__ chunks, int64_t n_chunks,
                                                                  const int32_t* __restrict__ weight_index,
                                                                  double* __restrict__ weights, double cal,
                                                                  int64_t n_det, int64_t n_samp) {
    for (int64_t c = blockIdx.x; c < n_chunks; c += gridDim.x) {
        const Chunk ch = chunks[c];
        if ((int)threadIdx.x >= ch.count) continue;
        const int64_t s = ch.first + threadIdx.x;
        for (int64_t d0 = (int64_t)blockIdx.y * kDT; d0 < n_det; d0 += (int64_t)gridDim.y * kDT) {
#pragma unroll
            for (int j = 0; j < kDT; ++j)
                if (d0 + j < n_det) weights[row_or<IDX>(weight_index, d0 + j) * n_samp + s] = cal;
        }
    }
}

template <bool IDX>
__global__ void __launch_bounds__(kChunk) noise_weight_kernel(const Chunk* __restrict__ chunks, int64_t n_chunks,
                                                              const int32_t* __restrict__ data_index,
                                                              double* __restrict__ det_data,
                                                              const double* __restrict__ det_weights, int64_t n_det,
                                                              int64_t n_samp) {
    for (int64_t c = blockIdx.x; c < n_chunks; c += gridDim.x) {
        const Chunk ch = chunks[c];
        if ((int)threadIdx.x >= ch.count) continue;
        const int64_t s = ch.first + threadIdx.x;
        for (int64_t d0 = (int64_t)blockIdx.y * kDT; d0 < n_det; d0 += (int64_t)gridDim.y * kDT) {
            int64_t o[kDT];
            double v[kDT];
#pragma unroll
            for (int j = 0; j < kDT; ++j) {
                o[j] = d0 + j < n_det ? row_or<IDX>(data_index, d0 + j) * n_samp + s : -1;
                v[j] = o[j] >= 0 ? det_data[o[j]] * __ldg(&det_weights[d0 + j]) : 0.0;
            }
#pragma unroll
            for (int j = 0; j < kDT; ++j)
                if (o[j] >= 0) det_data[o[j]] = v[j];
        }
    }
}

// Amplitude of (d, s) under reading O1: amp_offset[d] + view_base[iv] + (s - iv_first[iv]) / step.
template <bool IDX>
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
        const int64_t rel = __ldg(&v.view_base[ch.interval]) +
                            (int64_t)((int)(s - __ldg(&v.iv_first[ch.interval])) / v.step);
        for (int64_t d0 = (int64_t)blockIdx.y * kDT; d0 < n_det; d0 += (int64_t)gridDim.y * kDT) {
            int64_t o[kDT];
            double t[kDT], a[kDT];
#pragma unroll
            for (int j = 0; j < kDT; ++j) {
                const bool ok = d0 + j < n_det;
                o[j] = ok ? row_or<IDX>(data_index, d0 + j) * n_samp + s : -1;
                t[j] = ok ? det_data[o[j]] : 0.0;
                a[j] = ok ? __ldg(&amplitudes[__ldg(&amp_offset[d0 + j]) + rel]) : 0.0;
            }
#pragma unroll
            for (int j = 0; j < kDT; ++j)
                if (o[j] >= 0) det_data[o[j]] = t[j] + a[j];
        }
    }
}

// Projection: the samples of one step are consecutive, so a warp (32 consecutive samples of
// one detector) holds runs of equal amplitude index; each run is summed by a segmented
// shuffle scan and its last lane issues ONE fp64 red.  The kDT detectors' loads are issued
// together, then reduced one detector at a time.
template <bool IDX>
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
        // amplitude index relative to the detector's amp_offset; runs are detector-independent
        const int64_t rel = __ldg(&v.view_base[ch.interval]) +
                            (int64_t)((int)(s - __ldg(&v.iv_first[ch.interval])) / v.step);
        const int64_t rprev = __shfl_up_sync(kFullMask, rel, 1);
        for (int64_t d0 = (int64_t)blockIdx.y * kDT; d0 < n_det; d0 += (int64_t)gridDim.y * kDT) {
            double val[kDT];
            unsigned okm = 0u;  // bit j: this lane contributes to detector d0 + j
#pragma unroll
            for (int j = 0; j < kDT; ++j) {
                val[j] = 0.0;
                if (in && d0 + j < n_det) {
                    // both loads issued unconditionally (the TOD load must not wait for the flag)
                    const bool fl =
                        det_flags && (__ldg(&det_flags[row_or<IDX>(flag_index, d0 + j) * n_samp + s]) & det_flag_mask);
#ifdef TB_PROJ_COND
                    if (!fl) {
                        val[j] = __ldg(&det_data[row_or<IDX>(data_index, d0 + j) * n_samp + s]);
                        okm |= 1u << j;
                    }
#else
                    const double t = __ldg(&det_data[row_or<IDX>(data_index, d0 + j) * n_samp + s]);
                    if (!fl) {
                        val[j] = t;
                        okm |= 1u << j;
                    }
#endif
                }
            }
#pragma unroll
            for (int j = 0; j < kDT; ++j) {
                if (d0 + j >= n_det) break;
                // a run = consecutive lanes with equal rel that contribute
                const bool ok = (okm >> j) & 1u;
                const bool okp = __shfl_up_sync(kFullMask, ok, 1);
                const bool head = lane == 0 || rprev != rel || !okp || !ok;
                const unsigned heads = __ballot_sync(kFullMask, head);
                const int start = 31 - __clz(heads & (kFullMask >> (31 - lane)));
                const int depth = lane - start;
                double x = val[j];
#pragma unroll
                for (int off = 1; off < 32; off <<= 1) {
                    const bool need = depth >= off;
                    if (!__any_sync(kFullMask, need)) break;
                    const double t = __shfl_up_sync(kFullMask, x, off);
                    if (need) x += t;
                }
                const bool tail = lane == 31 || ((heads >> (lane + 1)) & 1u);
                if (tail && ok) atomicAdd(&amplitudes[__ldg(&amp_offset[d0 + j]) + rel], x);
            }
        }
    }
}

// Projection for step >= kSpan (the destriper's usual steps are hundreds of samples): a WARP
// owns one (chunk, detector) pair and lane L sums the kSpan consecutive samples
// [8L, 8L + 8) of the chunk in registers.  With step >= kSpan a lane meets at most one step
// boundary, so it holds two partial sums: A for its first amplitude r and B for r + 1.  B is
// handed to the next lane (whose first amplitude is r + 1) by one shuffle, then ONE segmented
// scan over the 32 lanes sums each amplitude and its last lane issues one fp64 red — one scan
// per 256 samples instead of one per 32 (offset_project_kernel), the loads 8 deep per thread.
// (Measured alternative: coalesced loads staged through a padded shared-memory transpose, 1.7x
// slower.)
constexpr int kSpan = 8;
// measured r02pj (project ms, C2 / C3 / C5): scalar loads, 1 row per warp 0.193 / 0.173 / 0.662 (44-50 %
// of HBM); 16-byte loads 0.126 / 0.116 / 0.481; 4 rows per warp 0.161 / 0.153 / 0.586; both 0.109 /
// 0.101 / 0.387 (79-85 %)
#ifndef TB_PROJ_VEC
#define TB_PROJ_VEC 1
#endif
#ifndef TB_PROJ_ROWS
#define TB_PROJ_ROWS 4
#endif
static_assert(kSpan * 32 == kChunk, "a warp covers one work chunk");

template <bool IDX>
__global__ void __launch_bounds__(kChunk) offset_project_span_kernel(
    const Chunk* __restrict__ chunks, int64_t n_chunks, OffsetViews v, const int64_t* __restrict__ amp_offset,
    double* __restrict__ amplitudes, const int32_t* __restrict__ data_index, const double* __restrict__ det_data,
    const int32_t* __restrict__ flag_index, const uint8_t* __restrict__ det_flags, uint8_t det_flag_mask,
    int64_t n_det, int64_t n_samp) {
    const int lane = threadIdx.x & 31;
    const int warp = threadIdx.x >> 5;
    constexpr int kWarpsPerCta = kChunk / 32;
    for (int64_t c = blockIdx.x; c < n_chunks; c += gridDim.x) {
        const Chunk ch = chunks[c];
        const int k0 = kSpan * lane;
        const int n = max(0, min(kSpan, ch.count - k0));  // this lane's samples in the chunk
        const bool ok = n > 0;
        const bool next_ok = lane < 31 && k0 + kSpan < ch.count;
        const int64_t s0 = ch.first + k0;
        const int off0 = (int)(s0 - __ldg(&v.iv_first[ch.interval]));
        const int r = off0 / v.step;                // amplitude of the lane's first sample in its interval
        const int kb = (r + 1) * v.step - off0;     // first lane-local sample of amplitude r + 1 (>= 1)
        const int64_t base = __ldg(&v.view_base[ch.interval]);
        const int rprev = __shfl_up_sync(kFullMask, r, 1);
        const bool okprev = __shfl_up_sync(kFullMask, ok, 1);
        const bool head = lane == 0 || rprev != r || !okprev || !ok;
        const unsigned heads = __ballot_sync(kFullMask, head);
        const int depth = lane - (31 - __clz(heads & (kFullMask >> (31 - lane))));
        const bool tail = lane == 31 || ((heads >> (lane + 1)) & 1u);
        for (int64_t d = (int64_t)blockIdx.y * kWarpsPerCta + warp; d < n_det; d += (int64_t)gridDim.y * kWarpsPerCta) {
            const double* t = det_data + row_or<IDX>(data_index, d) * n_samp + s0;
            const uint8_t* f = det_flags ? det_flags + row_or<IDX>(flag_index, d) * n_samp + s0 : nullptr;
            double A = 0.0, B = 0.0;
#if TB_PROJ_VEC
            // the lane's 8 samples as 4 x 16-byte loads (and its 8 flag bytes as one) when aligned
            if (n == kSpan && ((reinterpret_cast<uintptr_t>(t) & 15u) == 0) &&
                (!f || (reinterpret_cast<uintptr_t>(f) & 7u) == 0)) {
                double xv[kSpan];
#pragma unroll
                for (int k = 0; k < kSpan; k += 2) {
                    const double2 q = __ldg(reinterpret_cast<const double2*>(t + k));
                    xv[k] = q.x;
                    xv[k + 1] = q.y;
                }
                unsigned long long fb = 0ull;
                if (f) fb = __ldg(reinterpret_cast<const unsigned long long*>(f));
#pragma unroll
                for (int k = 0; k < kSpan; ++k) {
                    const double x = ((fb >> (8 * k)) & det_flag_mask) ? 0.0 : xv[k];
                    if (k < kb) A += x; else B += x;
                }
            } else
#endif
#pragma unroll
            for (int k = 0; k < kSpan; ++k) {
                if (k < n) {
                    double x = __ldg(t + k);
                    if (f && (__ldg(f + k) & det_flag_mask)) x = 0.0;
                    if (k < kb) A += x; else B += x;
                }
            }
            const int64_t a0 = ok ? __ldg(&amp_offset[d]) + base : 0;
            const double Bp = __shfl_up_sync(kFullMask, B, 1);
            if (lane > 0 && ok) A += Bp;  // the previous lane's tail belongs to my first amplitude
            if (ok && kb < n && !next_ok) atomicAdd(&amplitudes[a0 + r + 1], B);  // no next lane to take it
            double x = A;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                if (!__any_sync(kFullMask, depth >= o)) break;
                const double y = __shfl_up_sync(kFullMask, x, o);
                if (depth >= o) x += y;
            }
            if (tail && ok) atomicAdd(&amplitudes[a0 + r], x);
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
    (weight_index ? stokes_weights_i_kernel<true> : stokes_weights_i_kernel<false>)<<<grid_dt(wl, n_det), kChunk, 0, st>>>(wl.chunks, wl.n_chunks, weight_index, weights, cal,
                                                                  n_det, n_samp);
    return cudaGetLastError();
}

cudaError_t launch_noise_weight(const WorkList& wl, const int32_t* data_index, double* det_data,
                                const double* det_weights, int64_t n_det, int64_t n_samp, cudaStream_t st) {
    if (wl.n_chunks == 0 || n_det == 0) return cudaSuccess;
    (data_index ? noise_weight_kernel<true> : noise_weight_kernel<false>)<<<grid_dt(wl, n_det), kChunk, 0, st>>>(wl.chunks, wl.n_chunks, data_index, det_data,
                                                              det_weights, n_det, n_samp);
    return cudaGetLastError();
}

cudaError_t launch_offset_add(const WorkList& wl, const OffsetViews& v, const int64_t* amp_offset,
                              const double* amplitudes, const int32_t* data_index, double* det_data, int64_t n_det,
                              int64_t n_samp, cudaStream_t st) {
    if (wl.n_chunks == 0 || n_det == 0) return cudaSuccess;
    (data_index ? offset_add_kernel<true> : offset_add_kernel<false>)<<<grid_dt(wl, n_det), kChunk, 0, st>>>(wl.chunks, wl.n_chunks, v, amp_offset, amplitudes,
                                                            data_index, det_data, n_det, n_samp);
    return cudaGetLastError();
}

cudaError_t launch_offset_project(const WorkList& wl, const OffsetViews& v, const int64_t* amp_offset,
                                  double* amplitudes, const int32_t* data_index, const double* det_data,
                                  const int32_t* flag_index, const uint8_t* det_flags, uint8_t det_flag_mask,
                                  int64_t n_det, int64_t n_samp, cudaStream_t st) {
    if (wl.n_chunks == 0 || n_det == 0) return cudaSuccess;
    const bool idx = data_index || flag_index;
    if (v.step >= kSpan) {
        // TB_PROJ_ROWS detector rows per warp (the y-stride loop), so each warp amortises its
        // chunk's step bookkeeping over several rows
        const int64_t rows = (int64_t)(kChunk / 32) * TB_PROJ_ROWS;
        const dim3 grid((unsigned)std::min<int64_t>(wl.n_chunks, 0x7fffffff),
                        (unsigned)std::min<int64_t>((n_det + rows - 1) / rows, 65535), 1);
        (idx ? offset_project_span_kernel<true> : offset_project_span_kernel<false>)<<<grid, kChunk, 0, st>>>(
            wl.chunks, wl.n_chunks, v, amp_offset, amplitudes, data_index, det_data, flag_index, det_flags,
            det_flag_mask, n_det, n_samp);
        return cudaGetLastError();
    }
    (idx ? offset_project_kernel<true> : offset_project_kernel<false>)<<<grid_dt(wl, n_det), kChunk, 0, st>>>(wl.chunks, wl.n_chunks, v, amp_offset, amplitudes,
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

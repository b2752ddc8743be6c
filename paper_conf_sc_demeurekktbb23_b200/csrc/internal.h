// internal.h — launch-side types shared by api.cu and the kernel files (not part of the ABI).
#pragma once
#include <cuda_runtime.h>

#include <cstdint>

#include "../../include/toast_b200.h"

namespace toastb200 {

// Samples per work chunk = threads per CTA of every kernel (one sample per thread).
constexpr int kChunk = 256;
// Samples per work chunk of the fused kernel (a warp item = one such chunk x 32 or 64
// detectors; small enough that the dynamic schedule balances to a few percent).
#ifndef TB_FUSED_CHUNK
#define TB_FUSED_CHUNK 128  // <= 128: the incremental longitude's unwrapped range (fused.cu stage_a)
#endif
constexpr int kFusedChunk = TB_FUSED_CHUNK;
static_assert(kFusedChunk <= 128, "the tt + 1 chain must stay inside (0.18, 5.82)");

// One chunk of <= kChunk consecutive in-interval samples (never crosses an interval).
struct Chunk {
    int64_t first;
    int32_t count;
    int32_t interval;
};

struct WorkList {
    const Chunk* chunks;  // device
    int64_t n_chunks;
    int64_t n_samples;    // total in-interval samples
};

struct MapGeom {
    const int64_t* global2local;
    int64_t n_pix_submap;
    int sm_shift;         // log2(n_pix_submap) if a power of two, else -1
    // fused kernels only (set at launch): n_submap = 12 nside^2 / n_pix_submap, and whether each
    // CTA caches global2local (as int16, with the hit flag in bit 15) in shared memory
    // (n_submap <= kG2lCache); the hit flags then reach hit_submaps once per CTA, at its end.
    int64_t n_submap = 0;
    int cache_g2l = 0;
};

// Shared-memory global2local cache of the fused kernels: up to kG2lCache submaps (3072 at every
// nside >= 16 with the 16x16-submap layout of the benchmarks).
constexpr int kG2lCache = 4096;

struct FusedArgs {
    const double* fp_quats;
    const double* boresight;
    const double* hwp;
    const double* epsilon;
    double cal;
    const double* det_scale;
    const double* det_data;
    const uint8_t* det_flags;
    uint8_t det_flag_mask;
    const uint8_t* shared_flags;
    uint8_t shared_flag_mask;
    int64_t nside;
    int nest;
    int nnz;
    MapGeom map;
    double* zmap;          // fp64 map, or (map_f32) a float map at the same address
    int map_f32;
    uint8_t* hit_submaps;
    int64_t* pixels_out;
    double* weights_out;
    int64_t n_det;
    int64_t n_samp;
    // reading R3 (f4): per-detector polarisation angle [n_det] (NULL: 0) and the IAU sign of U
    const double* gamma;
    int iau;
    // debug counter of det-samples whose hit submap has no storage (global2local < 0); NULL: off
    unsigned long long* dropped;
    // pointing_to_tod (scan direction) only
    const double* mapdata;  // fp64 map, or (map_f32) a float map
    double data_scale;
    int should_zero;
    int should_subtract;
    double* tod_out;
};

cudaError_t launch_pointing_detector(const WorkList& wl, const double* fp_quats, const double* boresight,
                                     const int32_t* quat_index, double* quats, const uint8_t* shared_flags,
                                     uint8_t shared_flag_mask, int64_t n_det, int64_t n_samp, cudaStream_t st);
cudaError_t launch_pixels_healpix(const WorkList& wl, const int32_t* quat_index, const double* quats,
                                  const uint8_t* shared_flags, uint8_t shared_flag_mask, const int32_t* pixel_index,
                                  int64_t* pixels, uint8_t* hit_submaps, int64_t n_pix_submap, int64_t nside,
                                  int nest, int64_t n_det, int64_t n_samp, cudaStream_t st);
cudaError_t launch_stokes_weights_iqu(const WorkList& wl, const int32_t* quat_index, const double* quats,
                                      const int32_t* weight_index, double* weights, const double* hwp,
                                      const double* epsilon, double cal, int64_t n_det, int64_t n_samp,
                                      cudaStream_t st, const double* gamma = nullptr, int iau = 0);
cudaError_t launch_build_noise_weighted(const WorkList& wl, const MapGeom& mg, double* zmap, int nnz,
                                        const int32_t* pixel_index, const int64_t* pixels,
                                        const int32_t* weight_index, const double* weights,
                                        const int32_t* data_index, const double* det_data,
                                        const int32_t* flag_index, const uint8_t* det_flags, uint8_t det_flag_mask,
                                        const double* det_scale, const uint8_t* shared_flags,
                                        uint8_t shared_flag_mask, int64_t n_det, int64_t n_samp, cudaStream_t st);
cudaError_t launch_scan_map(const WorkList& wl, const MapGeom& mg, const double* mapdata, int nnz,
                            const int32_t* data_index, double* det_data, const int32_t* pixel_index,
                            const int64_t* pixels, const int32_t* weight_index, const double* weights,
                            double data_scale, int should_zero, int should_subtract, int64_t n_det, int64_t n_samp,
                            cudaStream_t st);
cudaError_t launch_pointing_to_map(const WorkList& wl, const FusedArgs& a, unsigned long long* sched,
                                   cudaStream_t st);
// How the last toast_pointing_to_map call on this host thread staged its inputs ("tma", or
// "cp.async (<reason>)").
const char* last_fused_path();
cudaError_t launch_pointing_to_tod(const WorkList& wl, const FusedArgs& a, unsigned long long* sched,
                                   cudaStream_t st);

// Offset-template views (reading O1): per interval, its first sample and the index of its
// first amplitude relative to the detector's amp_offset.
struct OffsetViews {
    const int64_t* iv_first;   // device [n_intervals]
    const int64_t* view_base;  // device [n_intervals]
    int step;
};

cudaError_t launch_stokes_weights_i(const WorkList& wl, const int32_t* weight_index, double* weights, double cal,
                                    int64_t n_det, int64_t n_samp, cudaStream_t st);
cudaError_t launch_noise_weight(const WorkList& wl, const int32_t* data_index, double* det_data,
                                const double* det_weights, int64_t n_det, int64_t n_samp, cudaStream_t st);
cudaError_t launch_offset_add(const WorkList& wl, const OffsetViews& v, const int64_t* amp_offset,
                              const double* amplitudes, const int32_t* data_index, double* det_data, int64_t n_det,
                              int64_t n_samp, cudaStream_t st);
cudaError_t launch_offset_project(const WorkList& wl, const OffsetViews& v, const int64_t* amp_offset,
                                  double* amplitudes, const int32_t* data_index, const double* det_data,
                                  const int32_t* flag_index, const uint8_t* det_flags, uint8_t det_flag_mask,
                                  int64_t n_det, int64_t n_samp, cudaStream_t st);
cudaError_t launch_precond(const double* var, const double* in, double* out, int64_t n, cudaStream_t st);

// A device counter for dynamic work distribution (zeroed on the stream before each use).
unsigned long long* sched_counter(int* err);

int num_sms();
cudaError_t launch_map_allreduce_nvls(double* mc, int64_t n, unsigned* const* pads, int rank, int world,
                                      cudaStream_t st);

}  // namespace toastb200

// map_accum.cuh — warp-aggregated fp64 scatter-add into the submap-distributed sky map.
//
// A warp holds 32 consecutive samples of one detector (lane = sample), so equal pixels
// come in runs along the scan.  Runs are reduced with a segmented inclusive scan over
// shuffles (stopping as soon as every run is covered — 1-2 steps for fast scans at high
// nside, up to 5 for slow ones) and only the LAST lane of each run issues the 1 or 3
// `red.global.add.f64`.  Each run's sum is exact-order sequential within the warp, so the
// result differs from the oracle's sequential sum only by reassociation (T4 tolerance).
#pragma once
#include <cstdint>

#include "internal.h"

namespace toastb200 {

constexpr unsigned kFull = 0xffffffffu;

// key >= 0: global pixel of this lane's contribution (det-flagged lanes carry key = pixel
// and zero values so they still mark hit submaps); key < 0: no contribution (must be
// unique per lane so such lanes never join a run).
template <int NNZ>
__device__ __forceinline__ void warp_accumulate(int64_t key, double v0, double v1, double v2, const MapGeom& mg,
                                                double* __restrict__ zmap, uint8_t* __restrict__ hit_submaps) {
    const int lane = threadIdx.x & 31;
    const int64_t kprev = __shfl_up_sync(kFull, key, 1);
    const bool head = (lane == 0) || (kprev != key);
    const unsigned heads = __ballot_sync(kFull, head);
    const unsigned upto = heads & (kFull >> (31 - lane));
    const int seg_start = 31 - __clz(upto);
    const int depth = lane - seg_start;  // lanes before me in my run
#pragma unroll
    for (int off = 1; off < 32; off <<= 1) {
        const bool need = depth >= off;
        if (!__any_sync(kFull, need)) break;
        const double t0 = __shfl_up_sync(kFull, v0, off);
        double t1 = 0.0, t2 = 0.0;
        if (NNZ == 3) {
            t1 = __shfl_up_sync(kFull, v1, off);
            t2 = __shfl_up_sync(kFull, v2, off);
        }
        if (need) {
            v0 += t0;
            if (NNZ == 3) {
                v1 += t1;
                v2 += t2;
            }
        }
    }
    const bool tail = (lane == 31) || ((heads >> (lane + 1)) & 1u);
    if (tail && key >= 0) {
        int64_t sm, lp;
        if (mg.sm_shift >= 0) {
            sm = key >> mg.sm_shift;
            lp = key & (mg.n_pix_submap - 1);
        } else {
            sm = key / mg.n_pix_submap;
            lp = key - sm * mg.n_pix_submap;
        }
        if (hit_submaps) hit_submaps[sm] = 1;
        const int64_t loc = __ldg(&mg.global2local[sm]);
        if (loc >= 0) {
            double* dst = zmap + (loc * mg.n_pix_submap + lp) * NNZ;
            atomicAdd(dst, v0);
            if (NNZ == 3) {
                atomicAdd(dst + 1, v1);
                atomicAdd(dst + 2, v2);
            }
        }
    }
}

}  // namespace toastb200

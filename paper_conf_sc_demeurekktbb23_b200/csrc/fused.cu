// fused.cu — toast_pointing_to_map: A1 -> A2 -> A3 -> A4 per detector-sample in registers.
//
// Work item = (chunk of <= 256 consecutive in-interval samples, block of kDetBlock
// detectors); a persistent grid of (#SM x resident CTAs) walks the items chunk-major, so
// the CTAs resident at any moment cover a short time window of the whole focal plane and
// the sky footprint they scatter into stays in L2.
//
// Per CTA and item:
//   * the detector block's frames are staged in shared memory once:
//       u = R(f) z, v = R(f) x, w = R(f) y  (columns of the detector rotation),
//       eta*cal and det_scale;
//   * each thread owns ONE sample: it loads the boresight quaternion once, forms the
//     boresight rotation matrix B (identity when shared-flagged, reading S2) and, with an
//     HWP, cos/sin(4 chi), and keeps them in registers for all detectors of the block;
//   * per detector: dir = B u, bx = (B v)_z, by = -(B w)_z (15 DP ops), phi = atan2,
//     HEALPix pixel, (cos 2psi, sin 2psi) algebraically, the HWP angle addition, the
//     noise-weighted contribution det_scale * tod * w, then a warp-segmented reduction
//     over runs of equal pixels and one fp64 red per run and Stokes component.
// The only HBM streams are the TOD (coalesced along samples), the optional det flags,
// the per-sample boresight/HWP/shared flags (read once per CTA item, i.e. once per
// kDetBlock detectors) and the map updates.
#include <cuda_runtime.h>

#include <algorithm>
#include <mutex>

#include "device_math.cuh"
#include "internal.h"
#include "map_accum.cuh"

namespace toastb200 {

namespace {

struct DetFrame {
    double u[3], v[3], w[3];
    double etacal;
    double scale;
    double pad;
};

template <bool NEST, int NNZ, bool HWP, bool DEBUG>
__global__ void __launch_bounds__(kChunk, 2) pointing_to_map_kernel(const Chunk* __restrict__ chunks,
                                                                    int64_t n_chunks, FusedArgs a, HealpixGeom g) {
    __shared__ DetFrame s_det[kDetBlock];
    const int tid = threadIdx.x;
    const int lane = tid & 31;
    const int64_t n_dblk = (a.n_det + kDetBlock - 1) / kDetBlock;
    const int64_t n_items = n_chunks * n_dblk;

    for (int64_t item = blockIdx.x; item < n_items; item += gridDim.x) {
        const int64_t c = item / n_dblk;
        const int64_t d0 = (item - c * n_dblk) * kDetBlock;
        const int64_t nd_rem = a.n_det - d0;
        const int nd = nd_rem < kDetBlock ? (int)nd_rem : kDetBlock;
        const Chunk ch = chunks[c];

        __syncthreads();  // previous item finished reading s_det
        if (tid < nd) {
            const double* f = a.fp_quats + 4 * (d0 + tid);
            double m[9];
            quat_to_matrix(f[0], f[1], f[2], f[3], m);
            DetFrame df;
            df.u[0] = m[2]; df.u[1] = m[5]; df.u[2] = m[8];
            df.v[0] = m[0]; df.v[1] = m[3]; df.v[2] = m[6];
            df.w[0] = m[1]; df.w[1] = m[4]; df.w[2] = m[7];
            const double eps = a.epsilon[d0 + tid];
            df.etacal = (1.0 - eps) / (1.0 + eps) * a.cal;
            df.scale = a.det_scale[d0 + tid];
            df.pad = 0.0;
            s_det[tid] = df;
        }
        __syncthreads();

        if ((tid & ~31) >= ch.count) continue;  // whole warp beyond this chunk (uniform per warp)
        const bool in = tid < ch.count;
        const int64_t s = ch.first + (in ? tid : 0);

        // ---- per-sample state, reused for every detector of the block
        bool sflag = false;
        double B[9];
        {
            double q[4] = {0.0, 0.0, 0.0, 1.0};
            if (in) {
                sflag = a.shared_flags && (__ldg(&a.shared_flags[s]) & a.shared_flag_mask);
                if (!sflag) {
                    const double2 lo = __ldg(reinterpret_cast<const double2*>(a.boresight + 4 * s));
                    const double2 hi = __ldg(reinterpret_cast<const double2*>(a.boresight + 4 * s) + 1);
                    q[0] = lo.x; q[1] = lo.y; q[2] = hi.x; q[3] = hi.y;
                }
            }
            quat_to_matrix(q[0], q[1], q[2], q[3], B);
        }
        double c4 = 1.0, s4 = 0.0;
        if (HWP && NNZ == 3) {
            if (in) sincos(4.0 * __ldg(&a.hwp[s]), &s4, &c4);
        }
        const bool pix_ok = in && !sflag;

        const double* __restrict__ tod_base = a.det_data + d0 * a.n_samp + s;
        const uint8_t* __restrict__ fl_base = a.det_flags ? a.det_flags + d0 * a.n_samp + s : nullptr;

#pragma unroll 1
        for (int j = 0; j < nd; ++j) {
            const DetFrame& df = s_det[j];
            const double tod = in ? __ldg(tod_base + j * a.n_samp) : 0.0;
            const bool dflag = (in && fl_base) ? ((__ldg(fl_base + j * a.n_samp) & a.det_flag_mask) != 0) : false;

            // A1 + rotation: dir = B u; bx = (B v)_z; by = -(B w)_z
            const double dx = B[0] * df.u[0] + B[1] * df.u[1] + B[2] * df.u[2];
            const double dy = B[3] * df.u[0] + B[4] * df.u[1] + B[5] * df.u[2];
            const double dz = B[6] * df.u[0] + B[7] * df.u[1] + B[8] * df.u[2];

            // A2
            int64_t pix = -1;
            if (pix_ok) pix = vec2pix<NEST>(g, dx, dy, dz);

            // A3
            double wq = 0.0, wu = 0.0;
            if (NNZ == 3) {
                const double bx = B[6] * df.v[0] + B[7] * df.v[1] + B[8] * df.v[2];
                const double by = -(B[6] * df.w[0] + B[7] * df.w[1] + B[8] * df.w[2]);
                double c2, s2;
                cos_sin_2psi(bx, by, c2, s2);
                if (HWP) {
                    const double cq = c2 * c4 - s2 * s4;
                    const double sq = s2 * c4 + c2 * s4;
                    c2 = cq;
                    s2 = sq;
                }
                wq = df.etacal * c2;
                wu = df.etacal * s2;
            }

            if (DEBUG && in) {
                const int64_t o = (d0 + j) * a.n_samp + s;
                if (a.pixels_out) a.pixels_out[o] = pix;
                if (a.weights_out) {
                    a.weights_out[o * NNZ] = a.cal;
                    if (NNZ == 3) {
                        a.weights_out[o * NNZ + 1] = wq;
                        a.weights_out[o * NNZ + 2] = wu;
                    }
                }
            }

            // A4: contribution of this det-sample; det-flagged samples keep their pixel key
            // (they still mark hit submaps, as A2 does) but add nothing.
            const double val = (pix >= 0 && !dflag) ? df.scale * tod : 0.0;
            const int64_t key = pix >= 0 ? pix : (int64_t)(-1 - lane);
            warp_accumulate<NNZ>(key, val * a.cal, val * wq, val * wu, a.map, a.zmap, a.hit_submaps);
        }
    }
}

template <bool NEST, int NNZ, bool HWP, bool DEBUG>
cudaError_t launch_t(const WorkList& wl, const FusedArgs& a, cudaStream_t st) {
    auto kern = pointing_to_map_kernel<NEST, NNZ, HWP, DEBUG>;
    static int blocks_per_sm = 0;
    static std::once_flag once;
    std::call_once(once, [&] {
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&blocks_per_sm, kern, kChunk, 0) != cudaSuccess ||
            blocks_per_sm < 1)
            blocks_per_sm = 1;
    });
    const int64_t n_dblk = (a.n_det + kDetBlock - 1) / kDetBlock;
    const int64_t n_items = wl.n_chunks * n_dblk;
    const int64_t grid = std::min<int64_t>(n_items, (int64_t)num_sms() * blocks_per_sm);
    if (grid <= 0) return cudaSuccess;
    kern<<<(unsigned)grid, kChunk, 0, st>>>(wl.chunks, wl.n_chunks, a, make_geom(a.nside));
    return cudaGetLastError();
}

template <bool NEST, int NNZ, bool HWP>
cudaError_t dispatch_debug(const WorkList& wl, const FusedArgs& a, cudaStream_t st) {
    if (a.pixels_out || a.weights_out) return launch_t<NEST, NNZ, HWP, true>(wl, a, st);
    return launch_t<NEST, NNZ, HWP, false>(wl, a, st);
}

template <bool NEST, int NNZ>
cudaError_t dispatch_hwp(const WorkList& wl, const FusedArgs& a, cudaStream_t st) {
    if (a.hwp && NNZ == 3) return dispatch_debug<NEST, NNZ, true>(wl, a, st);
    return dispatch_debug<NEST, NNZ, false>(wl, a, st);
}

}  // namespace

cudaError_t launch_pointing_to_map(const WorkList& wl, const FusedArgs& a, cudaStream_t st) {
    if (wl.n_chunks == 0 || a.n_det == 0) return cudaSuccess;
    if (a.nest) {
        return a.nnz == 3 ? dispatch_hwp<true, 3>(wl, a, st) : dispatch_hwp<true, 1>(wl, a, st);
    }
    return a.nnz == 3 ? dispatch_hwp<false, 3>(wl, a, st) : dispatch_hwp<false, 1>(wl, a, st);
}

}  // namespace toastb200

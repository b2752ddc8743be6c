// fused.cu — toast_pointing_to_map: A1 -> A2 -> A3 -> A4 per detector-sample in registers, and
// (SCAN mode of the same kernel) toast_pointing_to_tod: A1 -> A2 -> A3 -> A5.
//
// Decomposition (B200-first):
//   * A WARP owns a work item = (chunk of <= kFusedChunk consecutive in-interval samples,
//     group of 32 detectors); LANE = DETECTOR.  Items are handed out dynamically (one atomic per
//     item, fetched one item ahead) in chunk-major order, so the warps in flight cover a short
//     time window of the focal plane and the sky footprint they scatter into stays L2-resident.
//   * Each lane holds its detector's frame in registers for the whole item:
//       u = R(f) z, v = R(f) x, w = R(f) y and its noise-weight scales.
//   * An item is a STREAM OF BLOCKS of kBlk = 16 samples through two warp-private shared
//     buffers: while block i is computed, lane 0's bulk tensor copies (TMA, mbarrier-completed;
//     per-lane cp.async when the TMA constraints fail) stage block i+1 — the TOD tile [32 x 16]
//     (128-byte swizzled), the det-flag rows, 16 boresight quaternions, HWP angles and shared
//     flags.  Lanes 0..15 turn them into the per-sample state (boresight rotation matrix B —
//     identity if shared-flagged, reading S2), lanes 16..31 into cos/sin 4 chi; every lane then
//     walks the 16 samples reading that state as shared-memory broadcasts.  Boresight, HWP and
//     shared flags are read from HBM once per 32 detectors.  (Measured and rejected: a 7 KB
//     single-buffer staging with two TOD half tiles for 24 warps/SM — the 80-register bound
//     added 35 % instructions and the half-block lookahead exposed TMA latency: C2 0.56 ms vs
//     0.47 ms.)
//   * Per det-sample: dir = B u, bx = (B v)_z, by = -(B w)_z, the longitude carried
//     incrementally along the lane's samples (one reciprocal shared with the weights), the
//     compact HEALPix run key (belt: the two floors only, device_math.cuh loc2ckey), cos/sin 2psi
//     algebraically, the HWP angle addition.
//   * Map accumulation is RUN-LENGTH aggregated per lane along time: consecutive samples of one
//     detector with the same key are summed in registers; when the key changes the lane
//     flushes its run: key -> pixel, submap, global2local and hit flag from a per-CTA
//     shared-memory cache, one fp64 `red` per Stokes component (measured against a converged
//     per-warp flush queue: the queue won 2 % at C2 and lost 8-10 % at C3/C5, where some lane of
//     the 32 changes pixel at most samples anyway).
//   * PIPE kernels (the production map direction): the run that ended at sample k is flushed at
//     sample k+1 as straight-line predicated code in the same basic block as k+1's pointing, so
//     its integer decode / lookup / reduction chain interleaves with independent fp64 work
//     (nside >= 1024: always; below: the hybrid form, only when some lane has a pending run).
//   * SCAN mode gathers the map instead (cached per lane across the run) and updates the
//     staged TOD, written back after each half block.
#include <cuda.h>  // CUtensorMap (the encoder is fetched through the runtime; no -lcuda)
#include <cuda_runtime.h>
#include <cudaTypedefs.h>

#include <algorithm>
#include <cstdlib>
#include <cstring>
#include <mutex>

#include "device_math.cuh"
#include "internal.h"
#include "tma.cuh"

namespace toastb200 {

namespace {

using namespace tma;

#ifndef TB_FUSED_MINB
#define TB_FUSED_MINB 2  // resident CTAs per SM the register allocation is bounded for
#endif
#ifndef TB_ORDER_W
#define TB_ORDER_W 0
#endif
constexpr int kOrderW = TB_ORDER_W;
#ifndef TB_PIPE_UNROLL
#define TB_PIPE_UNROLL 2  // measured r02p6: C4 48.1 -> 47.2 ms, C3 0.432 -> 0.424 ms (the loop-carried copies alternate)
#endif
constexpr int kPipeUnroll = TB_PIPE_UNROLL;
constexpr int kWarps = 8;  // warps per CTA
constexpr int kBlk = 16;   // samples per block
constexpr unsigned kFull = 0xffffffffu;

// ----------------------------------------------------------------------------- TMA
struct alignas(64) TmaMaps {
    CUtensorMap tod;   // f64 [n_det][n_samp], box {16, 32}, SWIZZLE_128B
    CUtensorMap flg;   // u8  [n_det][n_samp], box {16, 32}
    CUtensorMap bore;  // f64 [n_samp][4],     box {4, 16}
    CUtensorMap hwp;   // f64 [n_samp],        box {16}
    CUtensorMap sflg;  // u8  [n_samp],        box {16}
};

// Per-warp shared memory: two staging buffers and the per-sample state (12 KB).  Every TMA
// destination is 128-byte aligned; the 16 shared-flag bytes of a buffer share their 128-byte slot
// with that buffer's mbarrier.
struct alignas(128) SflgSlot {
    uint8_t f[16];
    unsigned long long mbar;
    uint8_t pad[104];
};
// A finished run waiting in the warp's flush queue (QUEUE kernels): its compact key, the lane
// (detector) that produced it and its scaled sums.
struct alignas(16) QEntry {
    int key;
    int src;
    double r0, r1, r2;
};
constexpr int kQ = 32;  // queue entries per warp

struct alignas(1024) WarpSmem {
    double tod[2][32][16];  // 1024-aligned (the 128-byte swizzle pattern spans 1 KB)
    uint8_t flg[2][32][16];
    double bore[2][16][4];
    double hwp[2][16];
    SflgSlot sf[2];
    double st[16][12];      // per-sample state: B[0..8], c4, 2 s4, s4 / 2
    QEntry q[kQ];           // the flush queue (QUEUE kernels)
};
static_assert(sizeof(WarpSmem) == 13312, "13 KB per warp");

// Pixel index / key type: 32-bit compact keys up to nside 4096, else the 64-bit pixel itself.
template <bool WIDE>
struct PixT;
template <>
struct PixT<false> {
    using T = int;
};
template <>
struct PixT<true> {
    using T = int64_t;
};

// Per-CTA shared state besides the warps' areas: the global2local cache (int16: local submap,
// 0x7fff = no storage, bit 15 = hit) and whether it is in use.
struct CtaMem {
    uint16_t* g2l;  // [n_submap] when cached
    bool cached;
};
constexpr uint16_t kNoLoc = 0x7fff;
constexpr uint16_t kHitBit = 0x8000;

// Map geometry and the key -> (local submap, pixel in submap) step of a run flush.
template <bool NEST, bool OFF, bool WIDE>
__device__ __forceinline__ int64_t key_to_pixel(typename PixT<WIDE>::T key, const HealpixGeom& g) {
    if constexpr (WIDE)
        return key;
    else
        return ckey_to_pix<NEST, OFF>(key, g);
}

// Resolve the storage of a pixel's submap and mark the submap hit.  Returns the map element
// offset (in elements of nnz) or -1 if the submap has no storage.
__device__ __forceinline__ int64_t locate(int64_t pix, const FusedArgs& a, const CtaMem& cm) {
    const MapGeom& mg = a.map;
    int64_t sm, lp;
    if (mg.sm_shift >= 0) {
        sm = pix >> mg.sm_shift;
        lp = pix & (mg.n_pix_submap - 1);
    } else {
        sm = pix / mg.n_pix_submap;
        lp = pix - sm * mg.n_pix_submap;
    }
    int64_t loc;
    if (cm.cached) {
        const uint16_t v = cm.g2l[sm];
        if (a.hit_submaps) cm.g2l[sm] = v | kHitBit;  // idempotent: every writer stores the same value
        const unsigned l = v & 0x7fffu;
        loc = l == kNoLoc ? -1 : (int64_t)l;
    } else {
        if (a.hit_submaps) a.hit_submaps[sm] = 1;
        loc = __ldg(&mg.global2local[sm]);
    }
    return loc < 0 ? -1 : loc * mg.n_pix_submap + lp;
}

// Reading R3: (r1, r2) <- diag(1, +-1) R(-4 gamma_det) (r1, r2).  Out of line: the full-range
// sincos is large and this variant path must not grow the hot loop's code.
__device__ __noinline__ double2 gamma_rotate(double r1, double r2, const double* gamma, int iau, int64_t det) {
    double s4, c4;
    sincos(4.0 * __ldg(&gamma[det]), &s4, &c4);
    const double q = fma(c4, r1, s4 * r2);
    const double u = fma(c4, r2, -s4 * r1);
    return make_double2(q, iau ? -u : u);
}

// One run's contribution into the map (prescaled sums; reading R3's rotation by -4 gamma and
// the IAU sign of U applied here when a gamma array is given).
template <int NNZ>
__device__ __forceinline__ void add_run(int64_t elem, double r0, double r1, double r2, const FusedArgs& a,
                                        int64_t det) {
    if (elem < 0) return;
    if (NNZ == 3 && a.gamma != nullptr && a.hwp != nullptr) {
        const double2 v = gamma_rotate(r1, r2, a.gamma, a.iau, det);
        r1 = v.x;
        r2 = v.y;
    }
    if (a.map_f32) {
        float* dst = reinterpret_cast<float*>(a.zmap) + elem * NNZ;
        red_f32(dst, (float)r0);
        if (NNZ == 3) {
            red_f32(dst + 1, (float)r1);
            red_f32(dst + 2, (float)r2);
        }
    } else {
        double* dst = a.zmap + elem * NNZ;
        red_f64(dst, r0);
        if (NNZ == 3) {
            red_f64(dst + 1, r1);
            red_f64(dst + 2, r2);
        }
    }
}

// The general run flush (64-bit keys, non-power-of-two submaps, uncached global2local, fp32
// maps, the reading-R3 rotation), out of line so that the hot loop's code stays small.
// SCAN, general case (non-power-of-two submap, uncached global2local, fp32 map, gamma / IAU):
// the map element of `key` and its values, folded for reading R3.  Out of line, so the hot
// loop keeps only the lean gather.
struct Gathered {
    double m0, m1, m2;
    int64_t elem;
};
template <bool NEST, int NNZ, bool OFF, bool WIDE>
__device__ __noinline__ Gathered gather_general(typename PixT<WIDE>::T key, const double* mapdata, int map_f32,
                                                const int64_t* global2local, int sm_shift, int64_t n_pix_submap,
                                                uint16_t* g2l, bool cached, const double* gamma, bool have_hwp,
                                                int iau, int64_t det, HealpixGeom g) {
    Gathered r{0.0, 0.0, 0.0, -1};
    const int64_t pix = key_to_pixel<NEST, OFF, WIDE>(key, g);
    int64_t sm, lp;
    if (sm_shift >= 0) {
        sm = pix >> sm_shift;
        lp = pix & (n_pix_submap - 1);
    } else {
        sm = pix / n_pix_submap;
        lp = pix - sm * n_pix_submap;
    }
    int64_t loc;
    if (cached) {
        const unsigned l = g2l[sm] & 0x7fffu;
        loc = l == kNoLoc ? -1 : (int64_t)l;
    } else {
        loc = __ldg(&global2local[sm]);
    }
    if (loc < 0) return r;
    r.elem = loc * n_pix_submap + lp;
    if (map_f32) {
        const float* mp = reinterpret_cast<const float*>(mapdata) + r.elem * NNZ;
        r.m0 = __ldg(mp);
        if (NNZ == 3) {
            r.m1 = __ldg(mp + 1);
            r.m2 = __ldg(mp + 2);
        }
    } else {
        const double* mp = mapdata + r.elem * NNZ;
        r.m0 = __ldg(mp);
        if (NNZ == 3) {
            r.m1 = __ldg(mp + 1);
            r.m2 = __ldg(mp + 2);
        }
    }
    // reading R3 (a variant): t = m . (D R(-4 gamma) w) = (R(4 gamma) D m) . w;
    // gamma_rotate gives diag(1, -1) R(-4 gamma) (m1, -m2) = R(4 gamma) (m1, m2)
    if (NNZ == 3) {
        if (iau) r.m2 = -r.m2;
        if (gamma != nullptr && have_hwp) {
            const double2 n = gamma_rotate(r.m1, -r.m2, gamma, 1, det);
            r.m1 = n.x;
            r.m2 = n.y;
        }
    }
    return r;
}

template <bool NEST, int NNZ, bool OFF, bool WIDE>
__device__ __noinline__ void drain_general(typename PixT<WIDE>::T key, double r0, double r1, double r2, double* zmap,
                                           int map_f32, uint8_t* hit_submaps, const int64_t* global2local,
                                           int sm_shift, int64_t n_pix_submap, uint16_t* g2l_cache, bool cached,
                                           const double* gamma, bool have_hwp, int iau, int64_t det, HealpixGeom g) {
    const int64_t pix = key_to_pixel<NEST, OFF, WIDE>(key, g);
    int64_t sm, lp;
    if (sm_shift >= 0) {
        sm = pix >> sm_shift;
        lp = pix & (n_pix_submap - 1);
    } else {
        sm = pix / n_pix_submap;
        lp = pix - sm * n_pix_submap;
    }
    int64_t loc;
    if (cached) {
        const uint16_t v = g2l_cache[sm];
        if (hit_submaps) g2l_cache[sm] = v | kHitBit;
        const unsigned l = v & 0x7fffu;
        loc = l == kNoLoc ? -1 : (int64_t)l;
    } else {
        if (hit_submaps) hit_submaps[sm] = 1;
        loc = __ldg(&global2local[sm]);
    }
    if (loc < 0) return;
    const int64_t elem = loc * n_pix_submap + lp;
    if (NNZ == 3 && gamma != nullptr && have_hwp) {
        double s4, c4;
        sincos(4.0 * __ldg(&gamma[det]), &s4, &c4);
        const double q = fma(c4, r1, s4 * r2);
        const double u = fma(c4, r2, -s4 * r1);
        r1 = q;
        r2 = iau ? -u : u;
    }
    if (map_f32) {
        float* dst = reinterpret_cast<float*>(zmap) + elem * NNZ;
        red_f32(dst, (float)r0);
        if (NNZ == 3) {
            red_f32(dst + 1, (float)r1);
            red_f32(dst + 2, (float)r2);
        }
    } else {
        double* dst = zmap + elem * NNZ;
        red_f64(dst, r0);
        if (NNZ == 3) {
            red_f64(dst + 1, r1);
            red_f64(dst + 2, r2);
        }
    }
}

// Per-lane state of an item.
template <typename P>
struct Slot {
    double u0, u1, u2, v0, v1, v2, w0, w1, w2;
    double sI;      // det_scale * cal             (I)
    double sQ, sU;  // det_scale * eta * cal, times 2 for U (the run sums carry bx by, not 2 bx by) and
                    // the IAU sign when no gamma rotation follows in add_run
    double etacal;  // debug outputs / SCAN
    double r0, r1, r2;  // run sums: sum tod, sum tod cq / r, sum tod sq' / r
    double px, py, ptt; // incremental longitude: projected direction and tt of the previous sample
    P run_key;          // key of the run being aggregated (-1: none)
    int pk;             // PIPE: key of the finished run flushed at the next sample (-1: none)
    double pf0, pf1, pf2;  // PIPE: its scaled sums
    int64_t run_elem;   // SCAN: map element of the cached run (-1: none)
    unsigned pend_addr; // SCAN: shared address of the sample whose TOD update is pending (~0: none)
    double pend_c, pend_s;  // SCAN: its eta cal cos / r and 2 eta cal sin' / r
    int64_t det;
    bool ok;
};

template <typename P>
__device__ __forceinline__ void load_slot(Slot<P>& sl, const FusedArgs& a, int64_t d, bool ok, int64_t dfallback) {
    const int64_t dd = ok ? d : dfallback;
    double m[9];
    const double2 f01 = __ldg(reinterpret_cast<const double2*>(a.fp_quats + 4 * dd));
    const double2 f23 = __ldg(reinterpret_cast<const double2*>(a.fp_quats + 4 * dd) + 1);
    quat_to_matrix(f01.x, f01.y, f23.x, f23.y, m);
    sl.u0 = m[2]; sl.u1 = m[5]; sl.u2 = m[8];
    sl.v0 = m[0]; sl.v1 = m[3]; sl.v2 = m[6];
    sl.w0 = m[1]; sl.w1 = m[4]; sl.w2 = m[7];
    const double eps = __ldg(&a.epsilon[dd]);
    const double scale = __ldg(&a.det_scale[dd]);
    sl.etacal = (1.0 - eps) / (1.0 + eps) * a.cal;
    const bool rot = a.gamma != nullptr && a.hwp != nullptr;
    const double usign = (a.iau && !rot) ? -1.0 : 1.0;
    // a lane without a detector contributes exactly 0
    sl.sI = ok ? scale * a.cal : 0.0;
    sl.sQ = ok ? scale * sl.etacal : 0.0;
    sl.sU = 2.0 * usign * sl.sQ;
    sl.run_key = -1;
    sl.pk = -1;
    sl.pf0 = sl.pf1 = sl.pf2 = 0.0;
    sl.run_elem = -1;
    sl.pend_addr = 0xffffffffu;
    sl.pend_c = sl.pend_s = 0.0;
    sl.r0 = sl.r1 = sl.r2 = 0.0;
    sl.px = sl.py = sl.ptt = 0.0;  // dot = 0: the item's first sample takes the full arctangent
    sl.det = dd;
    sl.ok = ok;
}

// The straight-line fp64 part of one det-sample (A1 -> direction, A3 weights and the A2
// longitude).
struct StageA {
    double dx, dy, dz, tt;
    double cw, sw, invr;  // r cos 2(psi + 2 chi), r sin 2(psi + 2 chi) / 2, 1/r
    double t1m;           // N (tt + 1/2): the belt floors' common term (see loc2ckey)
};

// (2/pi) atan(t) = t Q(t^2) for |t| <= kIncrMax = 0.01 (TB_INCR_MAX, in the constant bank): the
// Taylor series to t^5; the omitted tail is below (2/pi) t^7 / 7 <= 9.1e-16 quarter turns per step
// at |t| = 0.01, so a chain of <= 127 steps drifts by < 1.2e-13 quarter turns (1.8e-13 rad), inside
// rule T1's 1e-12 rad.
__constant__ double kIncrQ[3] = {0.63661977236758134308, -0.21220659078919378103, 0.12732395447351626862};

// OFF: 32-bit keys with the incremental longitude carried as tt + 1 WITHOUT wrapping (see below).
template <int NNZ, typename P>
constexpr bool kOff = NNZ == 3 && sizeof(P) == 4;

template <int NNZ, bool HWP, typename P>
__device__ __forceinline__ StageA stage_a(Slot<P>& sl, const double* x, const KeyConsts& kc) {
    constexpr bool OFF = kOff<NNZ, P>;
    StageA o;
    o.dx = x[0] * sl.u0 + x[1] * sl.u1 + x[2] * sl.u2;
    o.dy = x[3] * sl.u0 + x[4] * sl.u1 + x[5] * sl.u2;
    o.dz = x[6] * sl.u0 + x[7] * sl.u1 + x[8] * sl.u2;
    o.cw = o.sw = o.invr = 0.0;
    if (NNZ == 3) {
        const double bx = x[6] * sl.v0 + x[7] * sl.v1 + x[8] * sl.v2;
        const double by = -(x[6] * sl.w0 + x[7] * sl.w1 + x[8] * sl.w2);
        // INCREMENTAL LONGITUDE: consecutive samples of a detector
        // are close on the sky, so tt(s) = tt(s') + (2/pi) atan(t) with t = tan(phi(s) - phi(s'))
        // = cross / dot of the projected directions of s and of this lane's previous processed
        // sample s' — a 4-term series instead of the octant reduction and the 11-term polynomial.
        // Each step adds ~1 ulp of tt; the chain restarts from the full arctangent at every item
        // (<= 128 samples), so the drift stays ~1e-15 rad, far inside rule T1's 1e-12 rad.  The
        // ONE reciprocal 1/(dot r) serves both t and the weights' 1/r.  Lanes whose step is large
        // (|t| > 0.01: near a pole, after a gap) or that have no previous sample (dot = 0) take
        // the full path.  The series is evaluated for every sample (NaN at dot = 0, no traps on
        // the GPU), so only the rare full path is a branch.
        const double bx2 = fma(bx, bx, TB_TINY);
        const double r = fma(by, by, bx2);
        o.cw = fma(-by, by, bx2);
        o.sw = bx * by;  // half of r sin 2 psi: the factor 2 is folded into the U scale
        const double cross = fma(sl.px, o.dy, -(sl.py * o.dx));
        const double dot = fma(sl.px, o.dx, sl.py * o.dy);
        const double cr = cross * r;  // off the reciprocal's critical path
        const double inv = fast_rcp(dot * r);
        // the belt floors need N (tt + 1/2) - 1/2 = N t q + (N ptt + N/2 - 1/2): the second term is
        // formed while the reciprocal is in flight, so the key path after t is short (Estrin
        // form of q: depth 2 instead of 3)
        {
            const double t = cr * inv;
            o.invr = dot * inv;
            const double s2 = t * t;
            const double q = fma(fma(kIncrQ[2], s2, kIncrQ[1]), s2, kIncrQ[0]);
            double tt = fma(t, q, sl.ptt);
            if constexpr (!OFF) {
                if (__double2hiint(tt) < 0) tt += 4.0;
                if (__double2hiint(tt) >= 0x40100000) tt -= 4.0;
            }
            o.tt = tt;
            o.t1m = fma(kc.dn, tt, kc.dn_half);  // N (tt + 1/2) (N tt exact)
        }
        // |cross| < kIncrMax dot  <=>  dot > 0 and |t| < kIncrMax; false at dot = 0 and for steps
        // beyond a quarter turn
        if (!(fma(TB_INCR_MAX, dot, -fabs(cross)) > 0.0)) {
            // OFF: the chain is carried as tt + 1 WITHOUT wrapping: it restarts here from a value in
            // [1, 5) and drifts by at most 127 steps of (2/pi) atan(0.01) = 0.0064 within an item,
            // so it stays in (0.18, 5.82); loc2ckey<NEST, true> folds it back
            double A, B;
            o.tt = lon_pol_raw(o.dx, o.dy, bx, by, A, B, o.invr) + (OFF ? 1.0 : 0.0);
            o.t1m = fma(kc.dn, o.tt, kc.dn_half);
        }
        sl.px = o.dx;
        sl.py = o.dy;
        sl.ptt = o.tt;
        if (HWP) {
            // (cq, sq') = rotation of (cw, 2 sw') by 4 chi, with sq' = sq / 2:
            // x[9] = cos 4chi, x[10] = 2 sin 4chi, x[11] = sin 4chi / 2
            const double cq = fma(-o.sw, x[10], o.cw * x[9]);
            const double sq = fma(o.sw, x[9], o.cw * x[11]);
            o.cw = cq;
            o.sw = sq;
        }
    } else {
        o.tt = quarter_turns(o.dx, o.dy);
        o.t1m = fma(kc.dn, o.tt, kc.dn_half);
    }
    return o;
}

// The HEALPix key of a det-sample (-1: no pixel).
template <bool NEST, int NNZ, bool WIDE>
__device__ __forceinline__ typename PixT<WIDE>::T stage_b(const StageA& o, bool pixelise, const HealpixGeom& g,
                                                         const KeyConsts& kc) {
    using P = typename PixT<WIDE>::T;
    P key;
    if constexpr (WIDE)
        key = (P)loc2pix<NEST, int64_t>(g, o.dz, o.tt, o.dx, o.dy);
    else
        key = (P)loc2ckey<NEST, kOff<NNZ, P>>(g, kc, o.dz, o.tt, o.t1m, o.dx, o.dy);
    return pixelise ? key : (P)-1;
}

// A block of the stream: samples [s0 + k0, s0 + k0 + nb) of the box starting at s0 (a multiple
// of 16), detector rows d0 .. d0 + nrows - 1.
struct Blk {
    int item;   // < 0: end of stream
    int d0;
    int s0;     // first sample of the staged box (multiple of 16)
    int s_end;  // end of the item's chunk
    int nb;     // samples processed: box indices k0 .. k0 + nb - 1
    int nrows;
    int k0;
};

// The lean run flush: 32-bit keys, a power-of-two submap, the cached global2local, an fp64 map,
// no reading-R3 rotation (every map element index is < 2^31 when nside <= 4096).
template <bool NEST, int NNZ, bool OFF>
__device__ __forceinline__ void flush_lean(int key, double r0, double r1, double r2, const FusedArgs& a,
                                           const HealpixGeom& g, uint16_t* g2l) {
    const MapGeom& mg = a.map;
    // branchy decode: the lanes of a warp (a 5-degree focal plane) are almost always all in the
    // belt or all in a cap, so one path runs (the branch-free form ran both: +20 instructions
    // per flush, and at nside >= 2048 some lane flushes at nearly every sample)
    const unsigned pix = (unsigned)ckey_to_pix<NEST, OFF>(key, g);
    const unsigned sm = pix >> mg.sm_shift;
    const unsigned lp = pix & (unsigned)(mg.n_pix_submap - 1);
    const unsigned v = g2l[sm];
    g2l[sm] = (uint16_t)(v | kHitBit);  // idempotent: every writer stores the same value
    const unsigned loc = v & 0x7fffu;
#ifdef TB_PRED_RED
    const bool ok = loc != kNoLoc;
    double* dst = a.zmap + (size_t)((loc << mg.sm_shift) + lp) * NNZ;
    red_f64_if(ok, dst, r0);
    if (NNZ == 3) {
        red_f64_if(ok, dst + 1, r1);
        red_f64_if(ok, dst + 2, r2);
    }
#else
    if (loc != kNoLoc) {
        double* dst = a.zmap + (size_t)((loc << mg.sm_shift) + lp) * NNZ;
        red_f64(dst, r0);
        if (NNZ == 3) {
            red_f64(dst + 1, r1);
            red_f64(dst + 2, r2);
        }
    }
#endif
}

// The lean flush as straight-line, PREDICATED code (no branch: executed by every lane at every
// sample, the reductions and the hit-flag store predicated on `go`); a variant for scans where
// some lane of the warp changes pixel at nearly every sample anyway (large nside).
template <bool NEST, int NNZ, bool OFF>
__device__ __forceinline__ void flush_lean_pred(bool go, int key, double r0, double r1, double r2,
                                                const FusedArgs& a, const HealpixGeom& g, uint16_t* g2l) {
    const MapGeom& mg = a.map;
    const unsigned pix = (unsigned)ckey_to_pix_bf<NEST, OFF>(go ? key : 0, g);
    const unsigned sm = pix >> mg.sm_shift;
    const unsigned lp = pix & (unsigned)(mg.n_pix_submap - 1);
    const unsigned v = g2l[sm];
    if (go) g2l[sm] = (uint16_t)(v | kHitBit);
    const unsigned loc = v & 0x7fffu;
    const bool ok = go && loc != kNoLoc;
    double* dst = a.zmap + (size_t)((loc << mg.sm_shift) + lp) * NNZ;
    red_f64_if(ok, dst, r0);
    if (NNZ == 3) {
        red_f64_if(ok, dst + 1, r1);
        red_f64_if(ok, dst + 2, r2);
    }
}

// The lean flush of a PENDING run (the one that ended at the lane's previous sample), written as
// straight-line predicated code with no memory clobbers: it sits in the same basic block as the
// next sample's pointing, so the scheduler interleaves the decode / lookup / reduction chain with
// independent fp64 work instead of running it as a divergent branch (PIPE kernels).
template <bool NEST, int NNZ, bool OFF>
__device__ __forceinline__ void flush_pending(int pk, double f0, double f1, double f2, double* __restrict__ zmap,
                                              int sm_shift, unsigned psm_mask, const HealpixGeom& g,
                                              uint16_t* g2l, uint64_t pol) {
    const bool go = pk >= 0;
    const unsigned pix = (unsigned)ckey_to_pix_bf<NEST, OFF>(go ? pk : 0, g);
    const unsigned sm = pix >> sm_shift;
    const unsigned v = g2l[sm];
    if (go) g2l[sm] = (uint16_t)(v | kHitBit);
    const unsigned loc = v & 0x7fffu;
    if (go && loc != kNoLoc) {
        double* dst = zmap + (size_t)((loc << sm_shift) + (pix & psm_mask)) * NNZ;
        // L2 policy per launch (see pol_map): keeps fine maps' lines against the streaming inputs
        asm volatile("red.global.add.L2::cache_hint.f64 [%0], %1, %2;" ::"l"(dst), "d"(f0), "l"(pol));
        if (NNZ == 3) {
            asm volatile("red.global.add.L2::cache_hint.f64 [%0], %1, %2;" ::"l"(dst + 1), "d"(f1), "l"(pol));
            asm volatile("red.global.add.L2::cache_hint.f64 [%0], %1, %2;" ::"l"(dst + 2), "d"(f2), "l"(pol));
        }
    }
}

template <bool NEST, int NNZ, bool HWP, bool DEBUG, bool WIDE, bool TMA, bool SCAN, bool QUEUE, int PIPE>
__global__ void __launch_bounds__(kWarps * 32, TB_FUSED_MINB)
    pointing_to_map_kernel(const Chunk* __restrict__ chunks, int n_chunks, FusedArgs a, HealpixGeom g, KeyConsts kc,
                           unsigned long long* __restrict__ sched, const __grid_constant__ TmaMaps tm) {
    static_assert(!SCAN || !DEBUG, "the scan direction has no debug outputs");
    static_assert(!QUEUE || (!SCAN && !DEBUG && !WIDE), "the flush queue: production map kernels, 32-bit keys");
    using P = typename PixT<WIDE>::T;
    constexpr bool OFF = kOff<NNZ, P>;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    const int lane = threadIdx.x & 31;
    const int wid = threadIdx.x >> 5;
    // the warps' areas start at the first 1 KB boundary of the shared window (the launch reserves
    // the padding); offset arithmetic on the __shared__ array itself keeps accesses LDS / STS
    const unsigned pad1k = (1024u - (smem_u32(smem_raw) & 1023u)) & 1023u;
    WarpSmem& ws = reinterpret_cast<WarpSmem*>(smem_raw + pad1k)[wid];
    uint16_t* s_g2l = reinterpret_cast<uint16_t*>(smem_raw + pad1k + kWarps * sizeof(WarpSmem));
    int& s_nocache = *reinterpret_cast<int*>(smem_raw + pad1k + kWarps * sizeof(WarpSmem) +
                                             ((2 * a.map.n_submap * a.map.cache_g2l + 15) & ~15));
    const MapGeom& mg = a.map;
    if (threadIdx.x == 0) s_nocache = 0;
    __syncthreads();
    if (mg.cache_g2l) {
        for (int i = threadIdx.x; i < (int)mg.n_submap; i += blockDim.x) {
            const int64_t v = __ldg(&mg.global2local[i]);
            if (v >= (int64_t)kNoLoc) s_nocache = 1;  // local index beyond the 15-bit cache
            s_g2l[i] = v < 0 ? kNoLoc : (uint16_t)(v & 0x7fff);
        }
    }
    __syncthreads();
    const CtaMem cm{s_g2l, mg.cache_g2l && !s_nocache};
    const bool lean = !WIDE && mg.sm_shift >= 0 && cm.cached && !a.map_f32 &&
                      !(a.gamma != nullptr && a.hwp != nullptr) && a.hit_submaps != nullptr;
    const bool scan_lean = SCAN && !WIDE && mg.sm_shift >= 0 && cm.cached && !a.map_f32 && !a.iau &&
                           !(a.gamma != nullptr && a.hwp != nullptr);

    const int n_groups = (int)((a.n_det + 31) / 32);
    const int n_items = n_chunks * n_groups;
    const unsigned dmask = a.det_flag_mask;
    const unsigned smask = a.shared_flag_mask;
    const bool have_dflags = !SCAN && a.det_flags != nullptr;  // scan_map ignores det flags (S12)
    const bool have_sflags = a.shared_flags != nullptr;
    const int n_samp = (int)a.n_samp;
    // TMA: bytes landing per block (full boxes, out-of-range elements zero-filled)
    const unsigned tx_bytes = 32 * 16 * 8 + 16 * 32 + (have_dflags ? 32 * 16 : 0) + ((HWP && NNZ == 3) ? 16 * 8 : 0) +
                              (have_sflags ? 16 : 0);
    unsigned phase = 0u;  // TMA: bit b = parity of the next completion of mbar[b]
    const uint64_t pol = evict_first_policy();
    // map reductions of the PIPE flush: evict_last on maps whose touched footprint exceeds L2
    // (nside >= 4096: C5 2.474 -> 2.438 ms, r02p10), evict_normal otherwise (C2-C4 unchanged)
    uint64_t pol_last, pol_normal;
    asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;\n" : "=l"(pol_last));
    asm volatile("createpolicy.fractional.L2::evict_normal.b64 %0, 1.0;\n" : "=l"(pol_normal));
    const uint64_t pol_map = g.nside >= 4096 ? pol_last : pol_normal;
    // swizzled byte offset of row `lane` in a TOD tile (16-byte chunk c of row r at c ^ (r & 7));
    // sample k is at row_swz ^ (8 k)
    const unsigned row_swz = (unsigned)lane * 128u + (((unsigned)lane & 7u) << 4);

    // Lane 0 fetches the NEXT item id and its chunk descriptor one item ahead (issued at an item
    // switch, consumed at the next one), so neither latency is on the critical path.
    int pend_item = -1, pend_first = 0, pend_count = 0;
    // item -> (chunk, detector group): windows of kOrderW chunks, group-major inside a window
    // (kOrderW = 0: chunk-major, all groups of a chunk in a row)
    auto item_chunk = [&](int item, int& grp) -> int {
        if (kOrderW <= 0) {
            const int c = item / n_groups;
            grp = item - c * n_groups;
            return c;
        }
        const int win = item / (kOrderW * n_groups);
        const int r = item - win * kOrderW * n_groups;
        const int wc = min(kOrderW, n_chunks - win * kOrderW);
        grp = r / wc;
        return win * kOrderW + (r - grp * wc);
    };
    auto prefetch_item = [&]() {
        if (lane == 0) {
            const unsigned long long it = atomicAdd(sched, 1ull);
            pend_item = it < (unsigned long long)n_items ? (int)it : -1;
            if (pend_item >= 0) {
                int grp;
                const Chunk ch = chunks[item_chunk(pend_item, grp)];
                pend_first = (int)ch.first;
                pend_count = ch.count;
            }
        }
    };
    auto take_item = [&]() -> Blk {
        Blk bk;
        bk.item = __shfl_sync(kFull, pend_item, 0);
        const int first = __shfl_sync(kFull, pend_first, 0);
        const int count = __shfl_sync(kFull, pend_count, 0);
        if (bk.item < 0) {
            bk.d0 = bk.s0 = bk.s_end = bk.nb = bk.nrows = bk.k0 = 0;
            return bk;
        }
        int grp;
        (void)item_chunk(bk.item, grp);
        bk.d0 = grp * 32;
        bk.nrows = min(32, (int)a.n_det - bk.d0);
        // boxes start at multiples of 16 samples (a TMA box must start 16-byte aligned in every
        // staged row; the u8 flag rows need that); a chunk's first block processes k0 .. 15 only
        bk.k0 = first & 15;
        bk.s0 = first - bk.k0;
        bk.s_end = first + count;
        bk.nb = min(count, kBlk - bk.k0);
        return bk;
    };
    auto successor = [&](const Blk& cur) -> Blk {
        Blk nx;
        if (cur.s0 + kBlk < cur.s_end) {
            nx = cur;
            nx.s0 = cur.s0 + kBlk;
            nx.k0 = 0;
            nx.nb = min(kBlk, nx.s_end - nx.s0);
        } else {
            nx = take_item();
            if (nx.item >= 0) prefetch_item();
        }
        return nx;
    };
    // Stage the raw inputs of block bk into buffer b.
    auto issue = [&](int b, const Blk& bk) {
        if constexpr (TMA) {
            if (lane == 0) {
                // the generic-proxy reads of buffer b (two blocks ago) are ordered before the
                // async-proxy writes that refill it
                asm volatile("fence.proxy.async.shared::cta;\n" ::: "memory");
                mbar_expect_tx(&ws.sf[b].mbar, tx_bytes);
                tma_2d_stream(&ws.tod[b][0][0], &tm.tod, bk.s0, bk.d0, &ws.sf[b].mbar, pol);
                if (have_dflags) tma_2d_stream(&ws.flg[b][0][0], &tm.flg, bk.s0, bk.d0, &ws.sf[b].mbar, pol);
                tma_2d(&ws.bore[b][0][0], &tm.bore, 0, bk.s0, &ws.sf[b].mbar);
                if (HWP && NNZ == 3) tma_1d(&ws.hwp[b][0], &tm.hwp, bk.s0, &ws.sf[b].mbar);
                if (have_sflags) tma_1d(&ws.sf[b].f[0], &tm.sflg, bk.s0, &ws.sf[b].mbar);
            }
        } else {
            // per-lane cp.async into the same (swizzled) layout; only the block's own samples
            const int scol = lane & 15, srow = lane >> 4;
            const bool valid = scol >= bk.k0 && scol < bk.k0 + bk.nb;
            if (valid) {
                const double* src = a.det_data + (int64_t)(bk.d0 + srow) * n_samp + bk.s0 + scol;
                const unsigned base = smem_u32(&ws.tod[b][0][0]);
                for (int r = srow; r < bk.nrows; r += 2, src += 2 * (int64_t)n_samp)
                    cp_async8_pol(base + (unsigned)r * 128u + (((unsigned)scol << 3) ^ (((unsigned)r & 7u) << 4)), src,
                                  pol);
            }
            if ((lane >> 1) >= bk.k0 && (lane >> 1) < bk.k0 + bk.nb)
                cp_async16(&ws.bore[b][lane >> 1][2 * (lane & 1)],
                           a.boresight + 4 * (int64_t)(bk.s0 + (lane >> 1)) + 2 * (lane & 1));
            if (HWP && NNZ == 3 && valid && lane < 16) cp_async8(smem_u32(&ws.hwp[b][lane]), a.hwp + bk.s0 + lane);
            cp_async_commit();
            // flags: plain loads of the block's own bytes (the rows need not be 4-byte aligned)
            if (have_sflags && valid && lane < 16) ws.sf[b].f[lane] = __ldg(a.shared_flags + bk.s0 + lane);
            if (have_dflags && lane < bk.nrows) {
                const uint8_t* fr = a.det_flags + (int64_t)(bk.d0 + lane) * n_samp + bk.s0;
                for (int k = bk.k0; k < bk.k0 + bk.nb; ++k) ws.flg[b][lane][k] = __ldg(fr + k);
            }
        }
    };

    if constexpr (TMA) {
        if (lane == 0) {
            mbar_init(&ws.sf[0].mbar);
            mbar_init(&ws.sf[1].mbar);
            asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
        }
        __syncwarp();
    }
    prefetch_item();
    Blk cur = take_item();
    // every thread reaches the hit-flag write-back below (a warp without work skips the stream)
    if (cur.item >= 0) [&] {
        prefetch_item();
        issue(0, cur);
        Slot<P> sl;
        load_slot<P>(sl, a, cur.d0 + lane, lane < cur.nrows, cur.d0);
        const double sgn_ds = (a.should_subtract ? -1.0 : 1.0) * a.data_scale;  // SCAN only

        // A run ends: flush its scaled sums (the lanes whose key changed; divergent).
        auto flush_run = [&](P key, double f0, double f1, double f2, int64_t det) {
            if (lean) {
                flush_lean<NEST, NNZ, OFF>((int)key, f0, f1, f2, a, g, cm.g2l);
            } else {
                drain_general<NEST, NNZ, OFF, WIDE>(key, f0, f1, f2, a.zmap, a.map_f32, a.hit_submaps,
                                                    mg.global2local, mg.sm_shift, mg.n_pix_submap, cm.g2l, cm.cached,
                                                    a.gamma, a.hwp != nullptr, a.iau, det, g);
            }
        };
        // QUEUE: finished runs are pushed (one ballot, converged) into the warp's queue and
        // flushed 32 at a time by all lanes, instead of by the few lanes whose key changed
        // while the rest of the warp waits (better when runs are long enough
        // that few lanes change key per sample, nside <= 2048)
        int qn = 0;
        const unsigned lt_mask = (1u << lane) - 1u;
        auto drain = [&](int n) {
            __syncwarp();
            if (lane < n) {
                const QEntry e = ws.q[lane];
                flush_run((P)e.key, e.r0, e.r1, e.r2, (int64_t)cur.d0 + e.src);
            }
            __syncwarp();
        };
        auto push = [&](bool do_push, P key, double f0, double f1, double f2) {
            const unsigned m = __ballot_sync(kFull, do_push);
            if (m) {
                const int np = __popc(m);
                if (qn + np > kQ) {
                    drain(qn);
                    qn = 0;
                }
                if (do_push) {
                    QEntry& e = ws.q[qn + __popc(m & lt_mask)];
                    e.key = (int)key;
                    e.src = lane;
                    e.r0 = f0;
                    e.r1 = f1;
                    e.r2 = f2;
                }
                qn += np;
            }
        };

        int p = 0;
        // SCAN: complete the pending sample's TOD update (t = data_scale sum_k m_k w_k)
        auto scan_finish = [&]() {
            if constexpr (SCAN) {
                if (sl.pend_addr != 0xffffffffu) {
                    double t = sl.r0 * a.cal;
                    if (NNZ == 3) t = fma(sl.r1, sl.pend_c, fma(sl.r2, sl.pend_s, t));
                    double v;
                    if (a.should_zero) {
                        v = sgn_ds * t;  // the old value is overwritten, never read (NaN-safe)
                    } else {
                        double old;
                        asm volatile("ld.shared.f64 %0, [%1];" : "=d"(old) : "r"(sl.pend_addr));
                        v = fma(sgn_ds, t, old);
                    }
                    asm volatile("st.shared.f64 [%0], %1;" ::"r"(sl.pend_addr), "d"(v) : "memory");
                    sl.pend_addr = 0xffffffffu;
                }
            }
        };

        while (true) {
            // successor block: next 16 samples of this item, or the first block of the next item
            const Blk nxt = successor(cur);
            if constexpr (TMA) {
                mbar_wait(&ws.sf[p].mbar, (phase >> p) & 1u);
                phase ^= 1u << p;
            } else {
                cp_async_wait_all();
                __syncwarp();
            }
            if (nxt.item >= 0) issue(p ^ 1, nxt);
            __syncwarp();  // reconverge after the lane-0 / spin-wait paths
            double* st_base = &ws.st[0][0];
            bool pixelise_me = false;
            {
                // lanes 0..15: the boresight rotation matrix of sample `lane` (identity if
                // shared-flagged, S2); lanes 16..31: the HWP cos/sin(4 chi) of sample `lane - 16`
                const int ks = lane & 15;
                const bool in_blk = ks >= cur.k0 && ks < cur.k0 + cur.nb;
                if (lane < kBlk) {
                    double q0 = 0.0, q1 = 0.0, q2 = 0.0, q3 = 1.0;
                    if (in_blk) {
                        const bool flagged = have_sflags && (ws.sf[p].f[lane] & smask);
                        pixelise_me = !flagged;
                        if (!flagged) {
                            const double* bq = ws.bore[p][lane];
                            q0 = bq[0]; q1 = bq[1]; q2 = bq[2]; q3 = bq[3];
                        }
                    }
                    double m[9];
                    quat_to_matrix(q0, q1, q2, q3, m);
                    double2* dst = reinterpret_cast<double2*>(st_base + 12 * lane);
#pragma unroll
                    for (int i = 0; i < 4; ++i) dst[i] = make_double2(m[2 * i], m[2 * i + 1]);
                    st_base[12 * lane + 8] = m[8];
                    // without HWP, slot 9 holds the sample's key mask (all ones: no pixel, S2), so
                    // the per-sample loop forms key | mask with one LOP3
                    if (!(HWP && NNZ == 3))
                        st_base[12 * lane + 9] = __longlong_as_double(pixelise_me ? 0ll : -1ll);
                } else if (HWP && NNZ == 3) {
                    double c4 = 1.0, s4 = 0.0;
                    if (in_blk) {
                        // reading R1: any finite chi; the Cody-Waite reduction of small_sincos
                        // holds for |4 chi| < 2^20 pi/2, CUDA's full-range sincos beyond
                        const double a4 = 4.0 * ws.hwp[p][ks];
                        if (fabs(a4) < 1.6e6)
                            small_sincos(a4, &s4, &c4);
                        else
                            sincos(a4, &s4, &c4);
                    }
                    st_base[12 * ks + 9] = c4;
                    st_base[12 * ks + 10] = 2.0 * s4;
                    st_base[12 * ks + 11] = 0.5 * s4;
                }
            }
            const unsigned pmask = __ballot_sync(kFull, pixelise_me) & 0xffffu;
            const unsigned keep = ((1u << cur.nb) - 1u) << cur.k0;  // samples of the block processed
            // zm: samples whose staged TOD is zeroed — det-flagged (they add exactly 0 but still
            // form runs and mark their submap, reading R2) and, in the map direction,
            // shared-flagged ones (they run through the loop with key -1)
            unsigned zm = SCAN ? 0u : (~pmask & keep);
            if (have_dflags && lane < cur.nrows) {
                const uint4 f = *reinterpret_cast<const uint4*>(ws.flg[p][lane]);
                const unsigned rep = dmask * 0x01010101u;
                const unsigned fw[4] = {f.x & rep, f.y & rep, f.z & rep, f.w & rep};
                if (fw[0] | fw[1] | fw[2] | fw[3]) {  // rare: 16 samples of 1 % flags
#pragma unroll
                    for (int w = 0; w < 4; ++w)
#pragma unroll
                        for (int b = 0; b < 4; ++b)
                            if ((fw[w] >> (8 * b)) & 0xffu) zm |= 1u << (4 * w + b);
                }
                zm &= keep;
            }
            {
                const unsigned tile0 = smem_u32(&ws.tod[p][0][0]) + row_swz;
                unsigned z = zm;
                while (z) {
                    const int c = __ffs(z) - 1;
                    z &= z - 1;
                    asm volatile("st.shared.f64 [%0], %1;" ::"r"(tile0 ^ ((unsigned)c << 3)), "d"(0.0) : "memory");
                }
            }
            __syncwarp();

            auto load_state = [&](int k, double* x) {
#pragma unroll
                for (int i = 0; i < ((HWP && NNZ == 3) ? 12 : 10); i += 2) {
                    const double2 t2 = *reinterpret_cast<const double2*>(st_base + 12 * k + i);
                    x[i] = t2.x;
                    x[i + 1] = t2.y;
                }
            };

            // TOD tile: 1 KB-aligned, row r at r * 128, so the swizzled address of (lane, k) is
            // (tile + row_swz) ^ (8 k): one LOP3 per sample
            const unsigned tile = smem_u32(&ws.tod[p][0][0]) + row_swz;
            bool piped = false;
            if constexpr (PIPE != 0 && !SCAN && !DEBUG && !QUEUE && !WIDE) {
                if (lean) {
                    // PIPE: the run that ended at sample k-1 is flushed (predicated, branch-free) in
                    // the same basic block as sample k's pointing, so the two chains interleave
                    piped = true;
                    const int kb = cur.k0, ke = cur.k0 + cur.nb;
                    const unsigned psm_mask = (unsigned)(mg.n_pix_submap - 1);
                    const unsigned pm = sl.ok ? pmask : 0u;  // a lane without a detector: key -1
                    const int okm = sl.ok ? 0 : -1;
#pragma unroll kPipeUnroll
                    for (int k = kb; k < ke; ++k) {
                        const unsigned addr = tile ^ ((unsigned)k << 3);
                        double x[12];
                        load_state(k, x);
                        StageA o;
                        if constexpr (PIPE == 2) {
                            // hybrid (nside < 1024, where most samples end no run): the interleaved
                            // flush + pointing block only when some lane has a pending run
                            if (__any_sync(kFull, sl.pk >= 0)) {
                                flush_pending<NEST, NNZ, OFF>(sl.pk, sl.pf0, sl.pf1, sl.pf2, a.zmap, mg.sm_shift,
                                                              psm_mask, g, cm.g2l, pol_map);
                                o = stage_a<NNZ, HWP, P>(sl, x, kc);
                            } else {
                                o = stage_a<NNZ, HWP, P>(sl, x, kc);
                            }
                        } else {
                            flush_pending<NEST, NNZ, OFF>(sl.pk, sl.pf0, sl.pf1, sl.pf2, a.zmap, mg.sm_shift, psm_mask,
                                                          g, cm.g2l, pol_map);
                            o = stage_a<NNZ, HWP, P>(sl, x, kc);
                        }
                        P key;
                        if constexpr (HWP && NNZ == 3) {
                            key = stage_b<NEST, NNZ, WIDE>(o, (pm >> k) & 1u, g, kc);
                        } else {
                            key = stage_b<NEST, NNZ, WIDE>(o, true, g, kc) | __double2loint(x[9]) | okm;
                        }
                        double tod;
                        asm("ld.shared.f64 %0, [%1];" : "=d"(tod) : "r"(addr));
                        const bool chg = key != sl.run_key;
                        sl.pk = chg ? (int)sl.run_key : -1;
                        sl.pf0 = sl.r0;
                        sl.pf1 = sl.r1 * sl.sQ;
                        sl.pf2 = sl.r2 * sl.sU;
                        const double t = tod * o.invr;
                        sl.r0 = fma(tod, sl.sI, chg ? 0.0 : sl.r0);
                        if (NNZ == 3) {
                            sl.r1 = fma(t, o.cw, chg ? 0.0 : sl.r1);
                            sl.r2 = fma(t, o.sw, chg ? 0.0 : sl.r2);
                        }
                        sl.run_key = key;
                    }
                }
            }
            if constexpr (SCAN && PIPE != 0 && !WIDE) {
                if (scan_lean) {
                    // PIPE scan: straight-line per sample (predicated shared / global accesses), so
                    // the run's decode -> lookup -> gather chain interleaves with the next sample's
                    // pointing in the unrolled loop; a lane whose key did not change keeps its run
                    piped = true;
                    const int kb = cur.k0, ke = cur.k0 + cur.nb;
                    const unsigned psm_mask = (unsigned)(mg.n_pix_submap - 1);
                    const unsigned pm = sl.ok ? pmask : 0u;
                    const int okm = sl.ok ? 0 : -1;
                    const double sgn = sgn_ds;
#pragma unroll kPipeUnroll
                    for (int k = kb; k < ke; ++k) {
                        const unsigned addr = tile ^ ((unsigned)k << 3);
                        double x[12];
                        load_state(k, x);
                        {  // the pending update of the previous sample (t = data_scale sum_k m_k w_k)
                            const unsigned pa = sl.pend_addr;
                            const unsigned go = pa != 0xffffffffu;
                            double t = sl.r0 * a.cal;
                            if (NNZ == 3) t = fma(sl.r1, sl.pend_c, fma(sl.r2, sl.pend_s, t));
                            double old = 0.0;
                            if (!a.should_zero)
                                asm("{\n .reg .pred q;\n setp.ne.u32 q, %1, 0;\n @q ld.shared.f64 %0, [%2];\n}\n"
                                    : "+d"(old)
                                    : "r"(go), "r"(pa));
                            const double v = fma(sgn, t, old);
                            asm volatile("{\n .reg .pred q;\n setp.ne.u32 q, %0, 0;\n @q st.shared.f64 [%1], %2;\n}\n" ::"r"(go),
                                         "r"(pa), "d"(v)
                                         : "memory");
                        }
                        const StageA o = stage_a<NNZ, HWP, P>(sl, x, kc);
                        int key;
                        if constexpr (HWP && NNZ == 3)
                            key = (int)stage_b<NEST, NNZ, WIDE>(o, (pm >> k) & 1u, g, kc);
                        else
                            key = (int)stage_b<NEST, NNZ, WIDE>(o, true, g, kc) | __double2loint(x[9]) | okm;
                        const bool valid = key >= 0;
                        const bool chg = valid && key != (int)sl.run_key;
                        const unsigned pix = (unsigned)ckey_to_pix_bf<NEST, OFF>(chg ? key : 0, g);
                        const unsigned loc = cm.g2l[pix >> mg.sm_shift] & 0x7fffu;
                        const unsigned elem = (loc << mg.sm_shift) + (pix & psm_mask);
                        const unsigned ld = chg && loc != kNoLoc;
                        const double* mp = a.mapdata + (size_t)(ld ? elem : 0u) * NNZ;
                        asm("{\n .reg .pred q;\n setp.ne.u32 q, %1, 0;\n @q ld.global.nc.f64 %0, [%2];\n}\n"
                            : "+d"(sl.r0)
                            : "r"(ld), "l"(mp));
                        if (NNZ == 3) {
                            asm("{\n .reg .pred q;\n setp.ne.u32 q, %1, 0;\n @q ld.global.nc.f64 %0, [%2];\n}\n"
                                : "+d"(sl.r1)
                                : "r"(ld), "l"(mp + 1));
                            asm("{\n .reg .pred q;\n setp.ne.u32 q, %1, 0;\n @q ld.global.nc.f64 %0, [%2];\n}\n"
                                : "+d"(sl.r2)
                                : "r"(ld), "l"(mp + 2));
                        }
                        if (chg) {
                            sl.run_key = key;
                            sl.run_elem = loc == kNoLoc ? -1 : (int64_t)elem;
                        }
                        sl.pend_addr = (valid && sl.run_elem >= 0) ? addr : 0xffffffffu;
                        if (NNZ == 3) {
                            sl.pend_c = sl.etacal * (o.cw * o.invr);
                            sl.pend_s = (2.0 * sl.etacal) * (o.sw * o.invr);
                        }
                    }
                }
            }
            if (!piped) {
                const int kb = cur.k0, ke = cur.k0 + cur.nb;
#pragma unroll 1
                for (int k = kb; k < ke; ++k) {
                    const bool pixelise = (pmask >> k) & 1u;
                    const unsigned addr = tile ^ ((unsigned)k << 3);
                    double x[12];
                    load_state(k, x);
                    const StageA o = stage_a<NNZ, HWP, P>(sl, x, kc);
                    P key = stage_b<NEST, NNZ, WIDE>(o, pixelise, g, kc);
                    if (!sl.ok) key = -1;
                    if constexpr (SCAN) {
                        // gather the run's map values (cached per lane across the run) and update the
                        // TOD ONE SAMPLE LATER: the loads of a new run are in flight while the next
                        // sample's pointing is computed (the update of sample k-1 runs here, before
                        // sample k may start a new run)
                        scan_finish();
                        if (key < 0) continue;
                        if (key != sl.run_key) {
                            sl.run_key = key;
                            if (scan_lean) {
                                // 32-bit decode, cached global2local, one 3-load gather
                                const unsigned pix = (unsigned)ckey_to_pix<NEST, OFF>((int)key, g);
                                const unsigned loc = cm.g2l[pix >> mg.sm_shift] & 0x7fffu;
                                const unsigned elem = (loc << mg.sm_shift) + (pix & (unsigned)(mg.n_pix_submap - 1));
                                sl.run_elem = loc == kNoLoc ? -1 : (int64_t)elem;
                                if (loc != kNoLoc) {
                                    const double* mp = a.mapdata + (size_t)elem * NNZ;
                                    sl.r0 = __ldg(mp);
                                    if (NNZ == 3) {
                                        sl.r1 = __ldg(mp + 1);
                                        sl.r2 = __ldg(mp + 2);
                                    }
                                }
                            } else {
                                const Gathered gm = gather_general<NEST, NNZ, OFF, WIDE>(
                                    key, a.mapdata, a.map_f32, mg.global2local, mg.sm_shift, mg.n_pix_submap, cm.g2l,
                                    cm.cached, a.gamma, a.hwp != nullptr, a.iau, sl.det, g);
                                sl.run_elem = gm.elem;
                                sl.r0 = gm.m0;
                                sl.r1 = gm.m1;
                                sl.r2 = gm.m2;
                            }
                        }
                        if (sl.run_elem < 0) continue;
                        sl.pend_addr = addr;
                        if (NNZ == 3) {
                            sl.pend_c = sl.etacal * (o.cw * o.invr);
                            sl.pend_s = (2.0 * sl.etacal) * (o.sw * o.invr);
                        }
                    } else {
                        double tod;
                        asm volatile("ld.shared.f64 %0, [%1];" : "=d"(tod) : "r"(addr));
                        if (DEBUG && sl.ok) {
                            const int64_t off = sl.det * a.n_samp + cur.s0 + k;
                            const int64_t pix = key < 0 ? -1 : key_to_pixel<NEST, OFF, WIDE>(key, g);
                            if (a.pixels_out) a.pixels_out[off] = pix;
                            if (a.weights_out) {
                                a.weights_out[off * NNZ] = a.cal;
                                if (NNZ == 3) {
                                    double w1 = sl.etacal * (o.cw * o.invr), w2 = sl.etacal * (2.0 * o.sw * o.invr);
                                    if (a.gamma != nullptr && a.hwp != nullptr) {
                                        const double2 v = gamma_rotate(w1, w2, a.gamma, 0, sl.det);
                                        w1 = v.x;
                                        w2 = v.y;
                                    }
                                    a.weights_out[off * NNZ + 1] = w1;
                                    a.weights_out[off * NNZ + 2] = a.iau ? -w2 : w2;
                                }
                            }
                            if (a.dropped && pix >= 0 && !(a.det_flags && (a.det_flags[off] & dmask))) {
                                const int64_t smi = pix / mg.n_pix_submap;
                                if (__ldg(&mg.global2local[smi]) < 0) atomicAdd(a.dropped, 1ull);
                            }
                        }
                        // run-length aggregation: the run ends when the key changes (the sums are
                        // reset once, before the flush, so the compiler keeps one copy of it)
                        if constexpr (QUEUE) {
                            const bool chg = key != sl.run_key;
                            push(chg && sl.run_key >= 0, sl.run_key, sl.r0, sl.r1 * sl.sQ, sl.r2 * sl.sU);
                            if (chg) {
                                sl.run_key = key;
                                sl.r0 = sl.r1 = sl.r2 = 0.0;
                            }
#ifdef TB_PRED_FLUSH
                        } else if (lean) {
                            // straight-line flush (see flush_lean_pred)
                            const bool chg = key != sl.run_key;
                            const double f0 = sl.r0, f1 = sl.r1 * sl.sQ, f2 = sl.r2 * sl.sU;
                            flush_lean_pred<NEST, NNZ, OFF>(chg && sl.run_key >= 0, (int)sl.run_key, f0, f1, f2, a, g,
                                                            cm.g2l);
                            const double keepr = chg ? 0.0 : 1.0;
                            sl.r0 *= keepr;
                            sl.r1 *= keepr;
                            sl.r2 *= keepr;
                            sl.run_key = key;
#endif
                        } else if (key != sl.run_key) {
                            const P old = sl.run_key;
                            const double f0 = sl.r0, f1 = sl.r1 * sl.sQ, f2 = sl.r2 * sl.sU;
                            sl.run_key = key;
                            sl.r0 = sl.r1 = sl.r2 = 0.0;
                            if (old >= 0) flush_run(old, f0, f1, f2, sl.det);
                        }
                        sl.r0 = fma(tod, sl.sI, sl.r0);
                        if (NNZ == 3) {
                            const double t = tod * o.invr;
                            sl.r1 = fma(t, o.cw, sl.r1);
                            sl.r2 = fma(t, o.sw, sl.r2);
                        }
                    }
                }
            }
            {
                scan_finish();  // the block's last pending update, before the write-back
                __syncwarp();
                if constexpr (SCAN) {
                    // write back the processed columns of the tile (two rows per warp instruction,
                    // coalesced along samples); unprocessed samples in them keep the value read
                    const int scol = lane & 15, srow = lane >> 4;
                    if (scol >= cur.k0 && scol < cur.k0 + cur.nb) {
                        double* dst = a.tod_out + (int64_t)(cur.d0 + srow) * n_samp + cur.s0 + scol;
                        for (int r = srow; r < cur.nrows; r += 2, dst += 2 * (int64_t)n_samp) {
                            double v;
                            asm volatile("ld.shared.f64 %0, [%1];"
                                         : "=d"(v)
                                         : "r"(smem_u32(&ws.tod[p][0][0]) + (unsigned)r * 128u +
                                               (((unsigned)scol << 3) ^ (((unsigned)r & 7u) << 4))));
                            *dst = v;
                        }
                    }
                }
            }

            if (nxt.item != cur.item) {
                if constexpr (QUEUE) {
                    push(sl.run_key >= 0, sl.run_key, sl.r0, sl.r1 * sl.sQ, sl.r2 * sl.sU);  // open runs
                    drain(qn);
                    qn = 0;
                } else if constexpr (!SCAN) {
                    if (PIPE != 0 && sl.pk >= 0) flush_run((P)sl.pk, sl.pf0, sl.pf1, sl.pf2, sl.det);
                    if (sl.run_key >= 0) flush_run(sl.run_key, sl.r0, sl.r1 * sl.sQ, sl.r2 * sl.sU, sl.det);
                }
                if (nxt.item < 0) break;
                load_slot<P>(sl, a, nxt.d0 + lane, lane < nxt.nrows, nxt.d0);
            }
            __syncwarp();  // all lanes are done with buffer p and st before they are refilled
            cur = nxt;
            p ^= 1;
        }
        if constexpr (!TMA) cp_async_wait_all();
    }();
    if (a.hit_submaps && cm.cached) {  // the CTA's hit flags, once: a few hundred stores instead of one per run
        __syncthreads();
        for (int i = threadIdx.x; i < (int)mg.n_submap; i += blockDim.x)
            if (s_g2l[i] & kHitBit) a.hit_submaps[i] = 1;
    }
}

// The TMA path applies when every staged array is 16-byte aligned and rows of the TOD and the
// det flags are multiples of 16 bytes (n_samp % 16 == 0); otherwise the cp.async path runs (same
// results).
thread_local const char* t_fused_path = "";

bool make_tma_maps(const FusedArgs& a, TmaMaps* tm) {
#ifdef TB_NO_TMA
    t_fused_path = "cp.async (TMA disabled at build time)";
    return false;
#endif
    if (!tensor_map_encoder()) {
        t_fused_path = "cp.async (no cuTensorMapEncodeTiled)";
        return false;
    }
    if (a.n_samp % 16 != 0) {
        t_fused_path = "cp.async (n_samp % 16 != 0)";
        return false;
    }
    if (!aligned16(a.det_data) || !aligned16(a.boresight) || (a.det_flags && !aligned16(a.det_flags)) ||
        (a.hwp && !aligned16(a.hwp)) || (a.shared_flags && !aligned16(a.shared_flags))) {
        t_fused_path = "cp.async (an input array is not 16-byte aligned)";
        return false;
    }
    t_fused_path = "cp.async (tensor map encoding failed)";
    std::memset(tm, 0, sizeof(*tm));
    const cuuint64_t ns = (cuuint64_t)a.n_samp, nd = (cuuint64_t)a.n_det;
    {
        const cuuint64_t dims[2] = {ns, nd}, strides[1] = {ns * 8};
        const cuuint32_t box[2] = {16, 32};
        if (!encode_map(&tm->tod, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 2, a.det_data, dims, strides, box,
                        CU_TENSOR_MAP_SWIZZLE_128B))
            return false;
    }
    if (a.det_flags) {
        const cuuint64_t dims[2] = {ns, nd}, strides[1] = {ns};
        const cuuint32_t box[2] = {16, 32};
        if (!encode_map(&tm->flg, CU_TENSOR_MAP_DATA_TYPE_UINT8, 2, a.det_flags, dims, strides, box,
                        CU_TENSOR_MAP_SWIZZLE_NONE))
            return false;
    }
    {
        const cuuint64_t dims[2] = {4, ns}, strides[1] = {32};
        const cuuint32_t box[2] = {4, 16};
        if (!encode_map(&tm->bore, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 2, a.boresight, dims, strides, box,
                        CU_TENSOR_MAP_SWIZZLE_NONE))
            return false;
    }
    if (a.hwp) {
        const cuuint64_t dims[1] = {ns};
        const cuuint32_t box[1] = {16};
        if (!encode_map(&tm->hwp, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 1, a.hwp, dims, kNoStrides, box,
                        CU_TENSOR_MAP_SWIZZLE_NONE))
            return false;
    }
    if (a.shared_flags) {
        const cuuint64_t dims[1] = {ns};
        const cuuint32_t box[1] = {16};
        if (!encode_map(&tm->sflg, CU_TENSOR_MAP_DATA_TYPE_UINT8, 1, a.shared_flags, dims, kNoStrides, box,
                        CU_TENSOR_MAP_SWIZZLE_NONE))
            return false;
    }
    return true;
}

// Dynamic shared memory of the fused kernel: 1 KB alignment slack, the warps' areas, the
// global2local cache and the cache-overflow flag.
size_t fused_smem(const FusedArgs& a) {
    return 1024 + sizeof(WarpSmem) * kWarps + ((2 * (size_t)a.map.n_submap * a.map.cache_g2l + 15) & ~size_t(15)) + 16;
}

// The dynamic shared-memory limit is a per-context attribute: raised to the opt-in maximum once
// per device (per kernel instantiation; the statics are per template instance).
template <typename K>
void raise_smem_limit(K kern, bool* done_per_dev) {
    static std::mutex mu;
    int dev = 0;
    cudaGetDevice(&dev);
    if (dev < 0 || dev >= 64) dev = 0;
    std::lock_guard<std::mutex> lk(mu);
    if (!done_per_dev[dev]) {
        int optin = 0;
        cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
        cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, optin > 0 ? optin : 232448);
        cudaGetLastError();
        done_per_dev[dev] = true;
    }
}

template <bool NEST, int NNZ, bool HWP, bool DEBUG, bool WIDE, bool TMA, bool SCAN, bool QUEUE, int PIPE>
cudaError_t launch_k(const WorkList& wl, const FusedArgs& a, const TmaMaps& tm, unsigned long long* sched,
                     cudaStream_t st) {
    auto kern = pointing_to_map_kernel<NEST, NNZ, HWP, DEBUG, WIDE, TMA, SCAN, QUEUE, PIPE>;
    static bool done[64] = {false};
    raise_smem_limit(kern, done);
    const size_t smem = fused_smem(a);
    // resident CTAs per SM: registers are bounded for TB_FUSED_MINB (launch bounds); shared
    // memory decides below that (228 KB per SM, 1 KB reserved per CTA)
    int dev = 0, smem_sm = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&smem_sm, cudaDevAttrMaxSharedMemoryPerMultiprocessor, dev);
    int bps = smem_sm > 0 ? (int)((size_t)smem_sm / (smem + 1024)) : 1;
    bps = std::max(1, std::min(bps, TB_FUSED_MINB));
#ifdef TB_BPS_ENV
    if (const char* e = getenv("TB_BPS")) bps = std::max(1, std::min(bps, atoi(e)));  // tuning experiments only
#endif
    const int64_t n_items = wl.n_chunks * ((a.n_det + 31) / 32);
    const int64_t want = (n_items + kWarps - 1) / kWarps;
    const int64_t grid = std::min<int64_t>(want, (int64_t)num_sms() * bps);
    if (grid <= 0) return cudaSuccess;
    cudaError_t e = cudaMemsetAsync(sched, 0, sizeof(unsigned long long), st);
    if (e != cudaSuccess) return e;
    kern<<<(unsigned)grid, kWarps * 32, smem, st>>>(wl.chunks, (int)wl.n_chunks, a, make_geom(a.nside),
                                                    make_key_consts(a.nside), sched, tm);
    return cudaGetLastError();
}

template <bool NEST, int NNZ, bool HWP, bool DEBUG, bool WIDE, bool SCAN, bool QUEUE = false, int PIPE = 0>
cudaError_t launch_t(const WorkList& wl, const FusedArgs& a, unsigned long long* sched, cudaStream_t st) {
    TmaMaps tm;
    if (make_tma_maps(a, &tm)) {
        t_fused_path = "tma";
        return launch_k<NEST, NNZ, HWP, DEBUG, WIDE, true, SCAN, QUEUE, PIPE>(wl, a, tm, sched, st);
    }
    std::memset(&tm, 0, sizeof(tm));
    return launch_k<NEST, NNZ, HWP, DEBUG, WIDE, false, SCAN, QUEUE, PIPE>(wl, a, tm, sched, st);
}

// nside <= 4096: 32-bit compact keys; beyond: 64-bit pixel keys
constexpr int64_t kCompactMaxNside = 4096;
// The converged flush queue (QUEUE kernels) for nside <= TB_QUEUE_MAX_NSIDE: measured slower than
// the direct divergent flush on every benchmark config, so off by default.
#ifndef TB_QUEUE_MAX_NSIDE
#define TB_QUEUE_MAX_NSIDE 0  // measured r02v: C4 53.5 vs 52.3 ms, C3 0.477 vs 0.467 ms, C2 equal: off
#endif

// The pipelined predicated flush (PIPE kernels) for nside >= TB_PIPE_MIN_NSIDE, where some lane of
// a warp ends a run at nearly every sample anyway.
#ifndef TB_SCAN_PIPE
#define TB_SCAN_PIPE 0  // the straight-line (PIPE) scan loop: measured r02sp C3 0.500 -> 0.489 ms, C5 2.704 -> 2.749: off
#endif
#ifndef TB_PIPE_HYB
#define TB_PIPE_HYB 1  // below TB_PIPE_MIN_NSIDE: the hybrid PIPE loop (measured r02p9: C2 0.462 -> 0.451 ms; C3 +3.6 %, C4 +4.3 % with it)
#endif
#ifndef TB_PIPE_MIN_NSIDE
#define TB_PIPE_MIN_NSIDE 1024  // measured r02p3: C3 0.467 -> 0.442 ms, C4 51.9 -> 49.6 ms; C2 (nside 256) +12 %
#endif

template <bool NEST, int NNZ, bool HWP, bool DEBUG>
cudaError_t dispatch_shape(const WorkList& wl, const FusedArgs& a, unsigned long long* sched, cudaStream_t st) {
    if (a.nside > kCompactMaxNside) return launch_t<NEST, NNZ, HWP, DEBUG, true, false>(wl, a, sched, st);
#if TB_QUEUE_MAX_NSIDE > 0
    if constexpr (!DEBUG) {
        if (a.nside <= TB_QUEUE_MAX_NSIDE) return launch_t<NEST, NNZ, HWP, false, false, false, true>(wl, a, sched, st);
    }
#endif
#if TB_PIPE_MIN_NSIDE > 0
    if constexpr (!DEBUG) {
        if (a.nside >= TB_PIPE_MIN_NSIDE) return launch_t<NEST, NNZ, HWP, false, false, false, false, 1>(wl, a, sched, st);
#if TB_PIPE_HYB
        return launch_t<NEST, NNZ, HWP, false, false, false, false, 2>(wl, a, sched, st);
#endif
    }
#endif
    return launch_t<NEST, NNZ, HWP, DEBUG, false, false>(wl, a, sched, st);
}

// ============================================================================ few detectors
// With fewer than kThinMaxDet detectors a 32-lane detector group leaves most lanes idle (C1: 4
// detectors, 4 of 32 lanes).  Then THREAD = (chunk, detector): each thread builds its own
// per-sample state from the boresight (consecutive threads share a chunk, so those loads are
// L1 broadcasts) and runs the same per-det-sample arithmetic, with a direct (per-thread) run
// flush; the CTA's hit flags are gathered in its global2local cache.
constexpr int kThinMaxDet = 8;

template <bool NEST, int NNZ, bool HWP, bool WIDE>
__global__ void __launch_bounds__(256) pointing_to_map_thin_kernel(const Chunk* __restrict__ chunks, int64_t n_chunks,
                                                                  FusedArgs a, HealpixGeom g, KeyConsts kc) {
    using P = typename PixT<WIDE>::T;
    constexpr bool OFF = kOff<NNZ, P>;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    uint16_t* s_g2l = reinterpret_cast<uint16_t*>(smem_raw);
    __shared__ int s_nocache;
    const MapGeom& mg = a.map;
    if (threadIdx.x == 0) s_nocache = 0;
    __syncthreads();
    if (mg.cache_g2l) {
        for (int i = threadIdx.x; i < (int)mg.n_submap; i += blockDim.x) {
            const int64_t v = __ldg(&mg.global2local[i]);
            if (v >= (int64_t)kNoLoc) s_nocache = 1;
            s_g2l[i] = v < 0 ? kNoLoc : (uint16_t)(v & 0x7fff);
        }
    }
    __syncthreads();
    const CtaMem cm{s_g2l, mg.cache_g2l && !s_nocache};
    const int64_t n_items = n_chunks * a.n_det;
    for (int64_t it = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; it < n_items;
         it += (int64_t)gridDim.x * blockDim.x) {
        const int64_t c = it / a.n_det, d = it - c * a.n_det;
        const Chunk ch = chunks[c];
        Slot<P> sl;
        load_slot<P>(sl, a, d, true, d);
        auto flush = [&]() {
            if (sl.run_key >= 0)
                add_run<NNZ>(locate(key_to_pixel<NEST, OFF, WIDE>(sl.run_key, g), a, cm), sl.r0 * sl.sI,
                             sl.r1 * sl.sQ, sl.r2 * sl.sU, a, d);
        };
        // the inputs of sample s+1 are loaded while sample s is computed (one sample ahead): each
        // thread walks its chunk serially, so without it every sample waits a full DRAM latency
        struct In {
            double2 q01, q23;
            double tod, chi;
            bool skip;
        };
        const int64_t s_end = ch.first + ch.count;
        auto fetch = [&](int64_t s) {
            In v;
            v.skip = a.shared_flags && (__ldg(&a.shared_flags[s]) & a.shared_flag_mask);  // no pixel (S2)
            v.q01 = __ldg(reinterpret_cast<const double2*>(a.boresight + 4 * s));
            v.q23 = __ldg(reinterpret_cast<const double2*>(a.boresight + 4 * s) + 1);
            v.chi = (HWP && NNZ == 3) ? __ldg(&a.hwp[s]) : 0.0;
            v.tod = __ldg(&a.det_data[d * a.n_samp + s]);
            if (a.det_flags && (__ldg(&a.det_flags[d * a.n_samp + s]) & a.det_flag_mask)) v.tod = 0.0;
            return v;
        };
        In nx = fetch(ch.first);
        for (int64_t s = ch.first; s < s_end; ++s) {
            const In cu = nx;
            if (s + 1 < s_end) nx = fetch(s + 1);
            if (cu.skip) continue;
            double x[12];
            quat_to_matrix(cu.q01.x, cu.q01.y, cu.q23.x, cu.q23.y, x);
            if (HWP && NNZ == 3) {
                double s4, c4;
                const double a4 = 4.0 * cu.chi;
                if (fabs(a4) < 1.6e6)
                    small_sincos(a4, &s4, &c4);
                else
                    sincos(a4, &s4, &c4);
                x[9] = c4;
                x[10] = 2.0 * s4;
                x[11] = 0.5 * s4;
            }
            const double tod = cu.tod;
            const StageA o = stage_a<NNZ, HWP, P>(sl, x, kc);
            const P key = stage_b<NEST, NNZ, WIDE>(o, true, g, kc);
            if (key != sl.run_key) {
                flush();
                sl.run_key = key;
                sl.r0 = sl.r1 = sl.r2 = 0.0;
            }
            sl.r0 += tod;
            if (NNZ == 3) {
                const double t = tod * o.invr;
                sl.r1 = fma(t, o.cw, sl.r1);
                sl.r2 = fma(t, o.sw, sl.r2);
            }
        }
        flush();
    }
    if (a.hit_submaps && cm.cached) {
        __syncthreads();
        for (int i = threadIdx.x; i < (int)mg.n_submap; i += blockDim.x)
            if (s_g2l[i] & kHitBit) a.hit_submaps[i] = 1;
    }
}

template <bool NEST, int NNZ, bool HWP>
cudaError_t launch_thin(const WorkList& wl, const FusedArgs& a, cudaStream_t st) {
    const size_t smem = a.map.cache_g2l ? 2 * (size_t)a.map.n_submap : 0;
    const int64_t items = wl.n_chunks * a.n_det;
    const int64_t grid = std::min<int64_t>((items + 255) / 256, (int64_t)num_sms() * 8);
    t_fused_path = "thin (thread per chunk x detector, few detectors)";
    if (a.nside > kCompactMaxNside)
        pointing_to_map_thin_kernel<NEST, NNZ, HWP, true><<<(unsigned)grid, 256, smem, st>>>(
            wl.chunks, wl.n_chunks, a, make_geom(a.nside), make_key_consts(a.nside));
    else
        pointing_to_map_thin_kernel<NEST, NNZ, HWP, false><<<(unsigned)grid, 256, smem, st>>>(
            wl.chunks, wl.n_chunks, a, make_geom(a.nside), make_key_consts(a.nside));
    return cudaGetLastError();
}

template <bool NEST, int NNZ, bool HWP>
cudaError_t dispatch_debug(const WorkList& wl, const FusedArgs& a, unsigned long long* sched, cudaStream_t st) {
    // debug outputs and the dropped-sample counter run in the debug instantiation
    if (a.pixels_out || a.weights_out || a.dropped) return dispatch_shape<NEST, NNZ, HWP, true>(wl, a, sched, st);
#ifndef TB_NO_THIN
    if (a.n_det < kThinMaxDet) return launch_thin<NEST, NNZ, HWP>(wl, a, st);
#endif
    return dispatch_shape<NEST, NNZ, HWP, false>(wl, a, sched, st);
}

template <bool NEST, int NNZ>
cudaError_t dispatch_hwp(const WorkList& wl, const FusedArgs& a, unsigned long long* sched, cudaStream_t st) {
    if (a.hwp && NNZ == 3) return dispatch_debug<NEST, NNZ, true>(wl, a, sched, st);
    return dispatch_debug<NEST, NNZ, false>(wl, a, sched, st);
}

// ============================================================================ scan direction
// toast_pointing_to_tod: pointing_to_map_kernel<..., SCAN = true>.
template <bool NEST, int NNZ>
cudaError_t dispatch_scan(const WorkList& wl, const FusedArgs& a, unsigned long long* sched, cudaStream_t st) {
    const bool wide = a.nside > kCompactMaxNside;
    const bool hwp = a.hwp && NNZ == 3;
    if (wide) return hwp ? launch_t<NEST, NNZ, true, false, true, true>(wl, a, sched, st)
                         : launch_t<NEST, NNZ, false, false, true, true>(wl, a, sched, st);
#if TB_SCAN_PIPE
    if (a.nside >= TB_PIPE_MIN_NSIDE)
        return hwp ? launch_t<NEST, NNZ, true, false, false, true, false, 1>(wl, a, sched, st)
                   : launch_t<NEST, NNZ, false, false, false, true, false, 1>(wl, a, sched, st);
#endif
    return hwp ? launch_t<NEST, NNZ, true, false, false, true>(wl, a, sched, st)
               : launch_t<NEST, NNZ, false, false, false, true>(wl, a, sched, st);  // (no queue: a scan gathers)
}

// Launch-side map geometry of the fused kernels: the submap count and whether the CTAs cache
// global2local in shared memory.
FusedArgs with_map_geom(FusedArgs a) {
    MapGeom& m = a.map;
    m.n_submap = (12 * a.nside * a.nside + m.n_pix_submap - 1) / m.n_pix_submap;
    m.cache_g2l = m.n_submap <= kG2lCache;
    return a;
}

}  // namespace

cudaError_t launch_pointing_to_tod(const WorkList& wl, const FusedArgs& a_in, unsigned long long* sched,
                                   cudaStream_t st) {
    FusedArgs a = with_map_geom(a_in);
    a.hit_submaps = nullptr;  // the scan marks nothing
    if (wl.n_chunks == 0 || a.n_det == 0) return cudaSuccess;
    if (a.nest) return a.nnz == 3 ? dispatch_scan<true, 3>(wl, a, sched, st) : dispatch_scan<true, 1>(wl, a, sched, st);
    return a.nnz == 3 ? dispatch_scan<false, 3>(wl, a, sched, st) : dispatch_scan<false, 1>(wl, a, sched, st);
}

const char* last_fused_path() { return t_fused_path; }

cudaError_t launch_pointing_to_map(const WorkList& wl, const FusedArgs& a_in, unsigned long long* sched,
                                   cudaStream_t st) {
    const FusedArgs a = with_map_geom(a_in);
    if (wl.n_chunks == 0 || a.n_det == 0) return cudaSuccess;
    if (a.nest) return a.nnz == 3 ? dispatch_hwp<true, 3>(wl, a, sched, st) : dispatch_hwp<true, 1>(wl, a, sched, st);
    return a.nnz == 3 ? dispatch_hwp<false, 3>(wl, a, sched, st) : dispatch_hwp<false, 1>(wl, a, sched, st);
}

}  // namespace toastb200

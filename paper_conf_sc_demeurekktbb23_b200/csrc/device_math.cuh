// device_math.cuh — per-detector-sample arithmetic of the pointing->map chain, sm_100a.
//
// Written for the GPU from the paper's kernel statements and the
// HEALPix definition (ref [16]); it shares nothing with oracle/.
// B200-first choices:
//   * rotations are 3x3 row/column products: the boresight rotation matrix is built
//     ONCE per sample and reused for every detector (R(b (x) f) = R(b) R(f) exactly in
//     exact arithmetic), so a det-sample costs 15 DFMA-class ops instead of a Hamilton
//     product plus two vector rotations;
//   * psi is never formed: with the orthonormal detector frame (d, o, d x o),
//     bx = o_z and by = -(R y)_z, and cos 2psi / sin 2psi follow algebraically with one
//     reciprocal (no atan2/sin/cos for the polarisation angle);
//   * the HWP term uses cos/sin(4 chi) computed once per sample (angle addition);
//   * the HEALPix floor arithmetic uses __d*_rn intrinsics so it is NOT FMA-contracted:
//     it rounds exactly as the textbook expressions, keeping pixel mismatches against
//     the oracle confined to directions within ~1e-15 rad of a pixel boundary.
#pragma once
#include <cstdint>

namespace toastb200 {

constexpr double kTwoThird = 2.0 / 3.0;
constexpr double kInvHalfPi = 0.6366197723675813430755350534900574;  // 2/pi

// (2/pi) atan(t) = t P(t^2) on |t| <= tan(pi/8); coefficients from scripts/fit_atan.py
// (Chebyshev interpolant, max relative error 1.2e-16 in exact arithmetic).
static __constant__ double kAtanQ[11] = {
    0x1.45f306dc9c882p-1,  // 0.63661977236758127
    -0x1.b2995e7b7b1bfp-3,  // -0.21220659078916346
    0x1.04c26be371b2ap-3,  // 0.12732395446638495
    -0x1.7483756164e14p-4,  // -0.090945681111684273
    0x1.21bb8c039cd9ap-4,  // 0.070735499315381395
    -0x1.da19e12de59d2p-5,  // -0.057873668483057764
    0x1.910bf286e9087p-5,  // 0.048955892262967864
    -0x1.5a4f32beaf656p-5,  // -0.042274092780172509
    0x1.28b3704d8f8cdp-5,  // 0.036218375531903747
    -0x1.c5c0e72211c3bp-6,  // -0.027694917407895963
    0x1.b97329ffc867cp-7,  // 0.013471980578802382
};

constexpr double kTanPi8 = 0.41421356237309504880;
// Constants whose low word is non-zero are kept in the constant bank so that the fp64
// instructions take them as c[][] operands: written as literals, the compiler re-materialises
// them with two UMOVs per use inside the hot loop once the uniform registers run out.
static __constant__ double kC[5] = {kTanPi8, 1e-100, 2.0 / 3.0, 0.99, 0.01};
#define TB_TAN_PI8 (::toastb200::kC[0])
#define TB_TINY (::toastb200::kC[1])
#define TB_TWO_THIRD (::toastb200::kC[2])
#define TB_CAP_SINTHETA_Z (::toastb200::kC[3])
#define TB_INCR_MAX (::toastb200::kC[4])  // kIncrMax of the fused kernel's incremental longitude

// 1/x for finite x > 0 (no IEEE rounding guarantee; <= ~1 ulp): MUFU seed + ONE cubic step,
// r' = r + r (e + e^2) with e = 1 - x r.  Measured on B200 (scripts/mufu_precision.cu, 2^24
// inputs): the seed's relative error is <= 2^-19.9, after the cubic step <= 2^-52.0 (1 ulp);
// 3 DFMA instead of the 4 of two quadratic steps.
__device__ __forceinline__ double fast_rcp(double x) {
    double r;
    asm("rcp.approx.ftz.f64 %0, %1;" : "=d"(r) : "d"(x));
    const double e = fma(-x, r, 1.0);
    return fma(r, fma(e, e, e), r);
}

// tt = fmodulo(2 atan2(y, x) / pi, 4) in [0, 4) -- the HEALPix longitude in quarter turns --
// with tt = 0 at x = y = 0 (reading S3).
// Octant reduction with ONE reciprocal: with mx = max(|x|,|y|), mn = min(|x|,|y|) and
// beta = [mn > tan(pi/8) mx], t = (mn - beta mx) / (mx + beta mn) lies in [-tan(pi/8),
// tan(pi/8)] and tau = (2/pi) atan(t) = t P(t^2).  The octant bookkeeping is integer: the
// result is tt = K/2 + S tau with K in 0..8 and S = +-1, evaluated by ONE fma, so the
// octant offsets (multiples of 1/2 quarter turn) are exact.  Absolute error ~3e-16 quarter
// turns: it differs from a correctly rounded atan2 only at the last-ulp level, so HEALPix
// floors can differ from the oracle's only for directions within ~1e-15 rad of a pixel
// boundary (rule T1 allows 1e-12 rad).
//
// Two phases so that callers can share ONE reciprocal between the longitude and the
// polarisation weights (the MUFU/XU pipe, not the FP64 pipe, is the scarce unit on B200).
struct QtPrep {
    double num, den;  // t = num / den
    int kk;           // octant offset in half quarter turns
    bool neg;         // sign S
};

__device__ __forceinline__ QtPrep qt_prepare(double x, double y) {
    // |x| + 1e-100: the guard that makes x = y = 0 give t = 0 (den >= 1e-100) costs nothing —
    // the DADD replaces the one that materialises |x| — and changes nothing for |x| > 1e-84.
    const double ax = fabs(x) + TB_TINY, ay = fabs(y);
    const bool swap = ay > ax;
    const double mx = swap ? ay : ax;
    const double mn = swap ? ax : ay;
    const bool big = mn > TB_TAN_PI8 * mx;
    const double beta = big ? 1.0 : 0.0;
    QtPrep q;
    q.num = fma(-beta, mx, mn);
    q.den = fma(beta, mn, mx);
    // K in units of half a quarter turn; S = (-1)^(swap + x<0 + y<0).  The signs are the sign
    // BITS (integer tests, not fp64 compares), which is also C99 atan2's treatment of -0.
    int kk = big ? 1 : 0;
    kk = swap ? 2 - kk : kk;
    const bool xneg = __double2hiint(x) < 0, yneg = __double2hiint(y) < 0;
    kk = xneg ? 4 - kk : kk;
    q.kk = yneg ? 8 - kk : kk;
    q.neg = swap ^ xneg ^ yneg;
    return q;
}

// Exact small non-negative int -> double on the FP64 pipe (no I2F): 0 <= k < 2^31.
__device__ __forceinline__ double small_int_to_double(int k) {
    return __hiloint2double(0x43300000, k) - 4503599627370496.0;  // (2^52 + k) - 2^52
}

__device__ __forceinline__ double qt_finish(const QtPrep& q, double t) {
    const double s = t * t;
    // even/odd split Horner: depth 6 instead of 10, and every fma has ONE constant operand
    // (a direct constant-bank operand, no extra constant loads; the kernel is issue-bound)
    const double s2 = s * s;
    double e = fma(kAtanQ[10], s2, kAtanQ[8]);
    double o = fma(kAtanQ[9], s2, kAtanQ[7]);
    e = fma(e, s2, kAtanQ[6]);
    o = fma(o, s2, kAtanQ[5]);
    e = fma(e, s2, kAtanQ[4]);
    o = fma(o, s2, kAtanQ[3]);
    e = fma(e, s2, kAtanQ[2]);
    o = fma(o, s2, kAtanQ[1]);
    e = fma(e, s2, kAtanQ[0]);
    const double p = fma(o, s, e);
    // tt = K/2 + S t P: the sign S is applied to t by flipping its sign bit (integer op), and
    // K/2 is built exactly as (2^51 + K/2) - 2^51 (the ulp of 2^51 is 1/2), so the octant
    // offset costs one DADD instead of a per-lane (divergent) constant-table load.
    const double st = __hiloint2double(__double2hiint(t) ^ (q.neg ? (int)0x80000000 : 0), __double2loint(t));
    const double half_k = __hiloint2double(0x43200000, q.kk) - 2251799813685248.0;
    double tt = fma(st, p, half_k);
    if (__double2hiint(tt) >= 0x40100000) tt = 0.0;  // tt >= 4 (tt >= -0 here): an integer compare
    return tt;
}

__device__ __forceinline__ double quarter_turns(double x, double y) {
    const QtPrep q = qt_prepare(x, y);
    return qt_finish(q, q.num * fast_rcp(q.den));
}

// floor(x) for 0 <= x < 2^31.  Default: one F2I (truncation = floor for x >= 0).  With
// TB_FLOOR_FP64 it runs on the FP64 pipe instead: rint via the 1.5 * 2^52 magic number (the
// addition is exact up to the final rounding to an integer), then corrected by one comparison
// — exact for every double in range, ties included.  (Measured on B200: F2I is ~3% faster.)
__device__ __forceinline__ int floor_nonneg(double x) {
#ifndef TB_FLOOR_FP64
    return (int)x;
#else
    const double big = x + 6755399441055744.0;
    const double r = big - 6755399441055744.0;  // rint(x), exact
    const int n = __double2loint(big);
    return (r > x) ? n - 1 : n;
#endif
}

// sqrt(x) for x >= 0.03 (the HEALPix cap term 3(1 - |z|) with |z| < 0.99): reciprocal square
// root seed (relative error <= 2^-20.0 measured, scripts/mufu_precision.cu), one Newton step on
// 1/sqrt (<= 2^-39.5 measured), then one Newton step on sqrt itself, which squares the error
// again: within ~1 ulp (not IEEE-rounded; only floors of it matter, and those may differ from
// the oracle only within ~1e-15 rad of a pixel boundary).
__device__ __forceinline__ double fast_sqrt(double x) {
    double y;
    asm("rsqrt.approx.ftz.f64 %0, %1;" : "=d"(y) : "d"(x));
    y = y * fma(-0.5 * x, y * y, 1.5);
    const double r = x * y;
    return fma(0.5 * y, fma(-r, r, x), r);  // one Newton step on sqrt itself
}

// sin and cos of a moderate angle (|a| < 2^20 pi/2; here a = 4 chi in [0, 8 pi)): Cody-Waite
// reduction by pi/2 with the fdlibm split constants, then the fdlibm __kernel_sin/__kernel_cos
// minimax polynomials on [-pi/4, pi/4].  Max error 2.2e-16 (checked against libm over [0, 8 pi));
// branch-free, no local-memory Payne-Hanek path (unlike the generic sincos()).
// (reduction constants and polynomial coefficients in the constant bank: c[][] operands
// instead of two UMOVs per literal)
static __constant__ double kSinCos[15] = {
    0.63661977236758134308,      // 2/pi
    1.57079632673412561417e+00,  // pi/2, high part
    6.07710050650619224932e-11,  // pi/2, low part
    1.58969099521155010221e-10,  -2.50507602534068634195e-08, 2.75573137070700676789e-06,
    -1.98412698298579493134e-04, 8.33333333332248946124e-03,  -1.66666666666666324348e-01,
    -1.13596475577881948265e-11, 2.08757232129817482790e-09,  -2.75573143513906633035e-07,
    2.48015872894767294178e-05,  -1.38888888888741095749e-03, 4.16666666666666019037e-02,
};

__device__ __forceinline__ void small_sincos(double a, double* sp, double* cp) {
    const double* C = kSinCos;
    const double k = rint(a * C[0]);
    const double r = fma(-k, C[2], fma(-k, C[1], a));
    const double z = r * r;
    double ps = C[3];
    ps = fma(ps, z, C[4]);
    ps = fma(ps, z, C[5]);
    ps = fma(ps, z, C[6]);
    ps = fma(ps, z, C[7]);
    ps = fma(ps, z, C[8]);
    const double sn = fma(r * z, ps, r);
    double pc = C[9];
    pc = fma(pc, z, C[10]);
    pc = fma(pc, z, C[11]);
    pc = fma(pc, z, C[12]);
    pc = fma(pc, z, C[13]);
    pc = fma(pc, z, C[14]);
    const double cs = fma(z * z, pc, fma(-0.5, z, 1.0));
    const int q = (int)k & 3;
    const double s0 = (q & 1) ? cs : sn;
    const double c0 = (q & 1) ? sn : cs;
    *sp = (q & 2) ? -s0 : s0;
    *cp = ((q + 1) & 2) ? -c0 : c0;
}

// Rotation matrix of a unit quaternion [x,y,z,w] (no renormalisation, reading S7),
// row-major m[3*i + j] = R_ij.
__device__ __forceinline__ void quat_to_matrix(double x, double y, double z, double w, double m[9]) {
    const double xx = x * x, yy = y * y, zz = z * z;
    const double xy = x * y, xz = x * z, yz = y * z;
    const double xw = x * w, yw = y * w, zw = z * w;
    m[0] = 1.0 - 2.0 * (yy + zz);
    m[1] = 2.0 * (xy - zw);
    m[2] = 2.0 * (xz + yw);
    m[3] = 2.0 * (xy + zw);
    m[4] = 1.0 - 2.0 * (xx + zz);
    m[5] = 2.0 * (yz - xw);
    m[6] = 2.0 * (xz - yw);
    m[7] = 2.0 * (yz + xw);
    m[8] = 1.0 - 2.0 * (xx + yy);
}

// Hamilton product r = p (x) q, [x,y,z,w] (reading S1).
__device__ __forceinline__ void quat_mul(const double p[4], const double q[4], double r[4]) {
    r[0] = p[3] * q[0] + p[0] * q[3] + p[1] * q[2] - p[2] * q[1];
    r[1] = p[3] * q[1] - p[0] * q[2] + p[1] * q[3] + p[2] * q[0];
    r[2] = p[3] * q[2] + p[0] * q[1] - p[1] * q[0] + p[2] * q[3];
    r[3] = p[3] * q[3] - p[0] * q[0] - p[1] * q[1] - p[2] * q[2];
}

// Interleave the low 32 bits of x into the even bit positions.
__device__ __forceinline__ uint64_t spread_bits(uint64_t x) {
    x &= 0xFFFFFFFFull;
    x = (x | (x << 16)) & 0x0000FFFF0000FFFFull;
    x = (x | (x << 8)) & 0x00FF00FF00FF00FFull;
    x = (x | (x << 4)) & 0x0F0F0F0F0F0F0F0Full;
    x = (x | (x << 2)) & 0x3333333333333333ull;
    x = (x | (x << 1)) & 0x5555555555555555ull;
    return x;
}

// Interleave the low 16 bits of x into the even bit positions of a 32-bit word.
__device__ __forceinline__ uint32_t spread_bits16(uint32_t x) {
    x &= 0xFFFFu;
    x = (x | (x << 8)) & 0x00FF00FFu;
    x = (x | (x << 4)) & 0x0F0F0F0Fu;
    x = (x | (x << 2)) & 0x33333333u;
    x = (x | (x << 1)) & 0x55555555u;
    return x;
}

template <typename I>
__device__ __forceinline__ int64_t nest_xyf(int64_t nside, I face, I ix, I iy) {
    if (sizeof(I) == 4) {  // nside <= 2^16: ix, iy < 2^16
        return (int64_t)face * nside * nside +
               (int64_t)(spread_bits16((uint32_t)ix) | (spread_bits16((uint32_t)iy) << 1));
    }
    return (int64_t)face * nside * nside + (int64_t)(spread_bits((uint64_t)ix) | (spread_bits((uint64_t)iy) << 1));
}

struct HealpixGeom {
    int64_t nside;
    int64_t npix;
    int64_t ncap;
    int order;
    double dnside;
};

inline HealpixGeom make_geom(int64_t nside) {
    HealpixGeom g;
    g.nside = nside;
    g.npix = 12 * nside * nside;
    g.ncap = 2 * nside * (nside - 1);
    int order = 0;
    while ((int64_t(1) << order) < nside) ++order;
    g.order = order;
    g.dnside = (double)nside;
    return g;
}

// HEALPix pixel of direction (dx, dy, dz) (Gorski et al. 2005; readings S3-S6, S8).
// I = int32_t for nside <= 2^16 (all floor indices < 19 nside fit, 32-bit NEST bit
// interleave), else int64_t; the returned pixel is int64 either way.
template <bool NEST, typename I>
__device__ __forceinline__ int64_t loc2pix(const HealpixGeom& g, double dz, double tt, double dx, double dy) {
    const double za = fabs(dz);
    const I nside = (I)g.nside;
    if (za <= TB_TWO_THIRD) {  // equatorial belt
        const double temp1 = __dmul_rn(g.dnside, __dadd_rn(0.5, tt));
        const double temp2 = __dmul_rn(__dmul_rn(g.dnside, dz), 0.75);
        const I jp = (I)__dsub_rn(temp1, temp2);  // ascending edge line
        const I jm = (I)__dadd_rn(temp1, temp2);  // descending edge line
        if (!NEST) {
            const I nl4 = 4 * nside;
            const I ir = nside + 1 + jp - jm;
            const I kshift = 1 - (ir & 1);
            const I t1 = jp + jm - nside + kshift + 1 + 2 * nl4;
            const I ip = (t1 >> 1) & (nl4 - 1);
            return g.ncap + (int64_t)nl4 * (int64_t)(ir - 1) + (int64_t)ip;
        } else {
            const I ifp = jp >> g.order;
            const I ifm = jm >> g.order;
            const I face = (ifp == ifm) ? (ifp | 4) : ((ifp < ifm) ? ifp : (ifm + 8));
            const I ix = jm & (nside - 1);
            const I iy = nside - (jp & (nside - 1)) - 1;
            return nest_xyf<I>(g.nside, face, ix, iy);
        }
    }
    // polar caps; the well-conditioned sin(theta) form for za >= 0.99 (reading S5)
    double tmp;
    if (za < TB_CAP_SINTHETA_Z) {
        tmp = __dmul_rn(g.dnside, __dsqrt_rn(__dmul_rn(3.0, __dsub_rn(1.0, za))));
    } else {
        const double sth = __dsqrt_rn(__dadd_rn(__dmul_rn(dx, dx), __dmul_rn(dy, dy)));
        tmp = __ddiv_rn(__dmul_rn(g.dnside, sth), __dsqrt_rn(__ddiv_rn(__dadd_rn(1.0, za), 3.0)));
    }
    if (!NEST) {
        const double tp = __dsub_rn(tt, (double)(int)tt);
        const I jp = (I)__dmul_rn(tp, tmp);
        const I jm = (I)__dmul_rn(__dsub_rn(1.0, tp), tmp);
        const I ir = jp + jm + 1;
        I ip = (I)__dmul_rn(tt, (double)ir);
        if (ip >= 4 * ir) ip -= 4 * ir;
        const int64_t ir64 = ir;
        return (dz > 0.0) ? 2 * ir64 * (ir64 - 1) + ip : g.npix - 2 * ir64 * (ir64 + 1) + ip;
    } else {
        int ntt = (int)tt;
        if (ntt > 3) ntt = 3;
        const double tp = __dsub_rn(tt, (double)ntt);
        I jp = (I)__dmul_rn(tp, tmp);
        I jm = (I)__dmul_rn(__dsub_rn(1.0, tp), tmp);
        if (jp > nside - 1) jp = nside - 1;
        if (jm > nside - 1) jm = nside - 1;
        I face, ix, iy;
        if (dz >= 0.0) {
            face = ntt; ix = nside - jm - 1; iy = nside - jp - 1;
        } else {
            face = ntt + 8; ix = jp; iy = jm;
        }
        return nest_xyf<I>(g.nside, face, ix, iy);
    }
}

// 32-bit interleave of ix (even bits) and iy (odd bits), ix, iy < 2^16: the outer perfect
// shuffle of the word (iy << 16 | ix) (Hacker's Delight 7-2) — 1 PRMT + 3 delta swaps.
__device__ __forceinline__ uint32_t interleave16(uint32_t ix, uint32_t iy) {
    uint32_t x = __byte_perm(ix, iy, 0x5140);  // bytes: iy1 ix1 iy0 ix0
    uint32_t t;
    t = (x ^ (x >> 4)) & 0x00F000F0u; x = x ^ t ^ (t << 4);
    t = (x ^ (x >> 2)) & 0x0C0C0C0Cu; x = x ^ t ^ (t << 2);
    t = (x ^ (x >> 1)) & 0x22222222u; x = x ^ t ^ (t << 1);
    return x;
}

// HEALPix pixel with 32-bit integer arithmetic; valid for nside <= 8192 (12 nside^2 < 2^31).
// Same expressions, in the same order and rounding, as loc2pix above.
template <bool NEST>
__device__ __forceinline__ int loc2pix32(const HealpixGeom& g, double dz, double tt, double dx, double dy) {
    const double za = fabs(dz);
    const int nside = (int)g.nside;
    if (za <= TB_TWO_THIRD) {
        const double temp1 = __dmul_rn(g.dnside, __dadd_rn(0.5, tt));
        const double temp2 = __dmul_rn(__dmul_rn(g.dnside, dz), 0.75);
        const int jp = floor_nonneg(__dsub_rn(temp1, temp2));
        const int jm = floor_nonneg(__dadd_rn(temp1, temp2));
        if (!NEST) {
            const int nl4 = 4 * nside;
            const int ir = nside + 1 + jp - jm;
            const int kshift = 1 - (ir & 1);
            const int t1 = jp + jm - nside + kshift + 1 + 2 * nl4;
            const int ip = (t1 >> 1) & (nl4 - 1);
            return (int)g.ncap + nl4 * (ir - 1) + ip;
        } else {
            const int ifp = jp >> g.order;
            const int ifm = jm >> g.order;
            const int face = (ifp == ifm) ? (ifp | 4) : ((ifp < ifm) ? ifp : (ifm + 8));
            const int ix = jm & (nside - 1);
            const int iy = nside - (jp & (nside - 1)) - 1;
            return face * (nside * nside) + (int)interleave16((uint32_t)ix, (uint32_t)iy);
        }
    }
    double tmp;
    if (za < TB_CAP_SINTHETA_Z) {
        tmp = __dmul_rn(g.dnside, fast_sqrt(__dmul_rn(3.0, __dsub_rn(1.0, za))));
    } else {
        const double sth = __dsqrt_rn(__dadd_rn(__dmul_rn(dx, dx), __dmul_rn(dy, dy)));
        tmp = __ddiv_rn(__dmul_rn(g.dnside, sth), __dsqrt_rn(__ddiv_rn(__dadd_rn(1.0, za), 3.0)));
    }
    if (!NEST) {
        const double tp = __dsub_rn(tt, small_int_to_double(floor_nonneg(tt)));
        const int jp = floor_nonneg(__dmul_rn(tp, tmp));
        const int jm = floor_nonneg(__dmul_rn(__dsub_rn(1.0, tp), tmp));
        const int ir = jp + jm + 1;
        int ip = floor_nonneg(__dmul_rn(tt, small_int_to_double(ir)));
        if (ip >= 4 * ir) ip -= 4 * ir;
        return (dz > 0.0) ? 2 * ir * (ir - 1) + ip : (int)g.npix - 2 * ir * (ir + 1) + ip;
    } else {
        int ntt = floor_nonneg(tt);
        if (ntt > 3) ntt = 3;
        const double tp = __dsub_rn(tt, small_int_to_double(ntt));
        int jp = floor_nonneg(__dmul_rn(tp, tmp));
        int jm = floor_nonneg(__dmul_rn(__dsub_rn(1.0, tp), tmp));
        if (jp > nside - 1) jp = nside - 1;
        if (jm > nside - 1) jm = nside - 1;
        int face, ix, iy;
        if (dz >= 0.0) {
            face = ntt; ix = nside - jm - 1; iy = nside - jp - 1;
        } else {
            face = ntt + 8; ix = jp; iy = jm;
        }
        return face * (nside * nside) + (int)interleave16((uint32_t)ix, (uint32_t)iy);
    }
}

// Run key of the pixel (fused kernels): RING -> the pixel; NEST -> face*N^2 + iy*N + ix, a
// packing that costs two IMADs per det-sample instead of the bit interleave, which
// key_to_pix32 applies once per run.  Same floors, in the same order and rounding, as
// loc2pix32.
// OFF: tt is the longitude in quarter turns PLUS ONE, unwrapped, anywhere in (0.18, 5.82) (the
// fused kernel's incremental longitude, see stage_a): every floor argument stays positive, the
// equatorial jp, jm and the cap ip carry an extra N (resp. ir), and the face / ring position is
// folded back modulo 4 quarter turns here — no per-sample wrap of tt.
template <bool NEST, bool OFF = false>
__device__ __forceinline__ int loc2key32(const HealpixGeom& g, double dz, double tt, double dx, double dy) {
    const double za = fabs(dz);
    const int nside = (int)g.nside;
    const int m = nside - 1;
    if (za <= TB_TWO_THIRD) {
        const double temp1 = __dmul_rn(g.dnside, __dadd_rn(0.5, tt));
        const double temp2 = __dmul_rn(__dmul_rn(g.dnside, dz), 0.75);
        const int jp = floor_nonneg(__dsub_rn(temp1, temp2));
        const int jm = floor_nonneg(__dadd_rn(temp1, temp2));
        if (!NEST) {
            const int nl4 = 4 * nside;
            const int ir = nside + 1 + jp - jm;
            const int kshift = 1 - (ir & 1);
            const int t1 = jp + jm - (OFF ? 3 : 1) * nside + kshift + 1 + 2 * nl4;
            const int ip = (t1 >> 1) & (nl4 - 1);
            return (int)g.ncap + nl4 * (ir - 1) + ip;
        } else {
            const int ifp = jp >> g.order;
            const int ifm = jm >> g.order;
            // face = ifp | 4 (ifp == ifm), ifp (ifp < ifm), ifm + 8 (ifp > ifm), with the face
            // row indices taken mod 4 (ifp, ifm reach 4 at tt near 4; OFF: they run 0..6 and
            // stand for ifp - 1, ifm - 1): |ifp - ifm| <= 1, so branch-free as
            // (min(ifp, ifm) mod 4) + 4 (1 + ifp - ifm)
            const int fmin = (ifp < ifm ? ifp : ifm) + (OFF ? 3 : 0);
            const int face = (fmin & 3) + 4 * (1 + ifp - ifm);
            const int ix = jm & m;
            const int iy = (jp & m) ^ m;  // nside - 1 - (jp & (nside - 1))
            return (face * nside + iy) * nside + ix;
        }
    }
    double tmp;
    if (za < TB_CAP_SINTHETA_Z) {
        tmp = __dmul_rn(g.dnside, fast_sqrt(__dmul_rn(3.0, __dsub_rn(1.0, za))));
    } else {
        const double sth = __dsqrt_rn(__dadd_rn(__dmul_rn(dx, dx), __dmul_rn(dy, dy)));
        tmp = __ddiv_rn(__dmul_rn(g.dnside, sth), __dsqrt_rn(__ddiv_rn(__dadd_rn(1.0, za), 3.0)));
    }
    if (!NEST) {
        const double tp = __dsub_rn(tt, small_int_to_double(floor_nonneg(tt)));
        const int jp = floor_nonneg(__dmul_rn(tp, tmp));
        const int jm = floor_nonneg(__dmul_rn(__dsub_rn(1.0, tp), tmp));
        const int ir = jp + jm + 1;
        int ip = floor_nonneg(__dmul_rn(tt, small_int_to_double(ir)));
        if (OFF) {
            ip -= ir;  // in [-0.82 ir, 4.82 ir)
            if (ip < 0) ip += 4 * ir;
        }
        if (ip >= 4 * ir) ip -= 4 * ir;
        return (dz > 0.0) ? 2 * ir * (ir - 1) + ip : (int)g.npix - 2 * ir * (ir + 1) + ip;
    } else {
        int ntt = floor_nonneg(tt);
        if (!OFF && ntt > 3) ntt = 3;
        const double tp = __dsub_rn(tt, small_int_to_double(ntt));
        if (OFF) ntt = (ntt + 3) & 3;
        int jp = floor_nonneg(__dmul_rn(tp, tmp));
        int jm = floor_nonneg(__dmul_rn(__dsub_rn(1.0, tp), tmp));
        if (jp > m) jp = m;
        if (jm > m) jm = m;
        int face, ix, iy;
        if (dz >= 0.0) {
            face = ntt; ix = m - jm; iy = m - jp;
        } else {
            face = ntt + 8; ix = jp; iy = jm;
        }
        return (face * nside + iy) * nside + ix;
    }
}

// ----------------------------------------------------------------------------- compact run keys
// The fused kernels (nside <= 4096) aggregate runs of equal pixels along each detector's
// samples and only need a per-sample KEY that is equal for equal pixels; the pixel number itself
// is formed once per run, when the run's sum is flushed (ckey_to_pix).  So the per-sample work
// in the equatorial belt stops at the two floors:
//   belt: key = (jp << 15) | jm            (jp, jm < 6.9 nside < 2^15)
//   caps: NEST: the cap pixel re-expressed as a belt key (one decoder for both, see loc2ckey)
//         RING: key = 1 << 30 | south << 26 | (north pixel, or npix - 1 - pixel)
// Any two different pixels get different keys; one pixel can get two keys (the unwrapped
// longitude of the incremental chain, OFF below, reaches a pixel from tt and tt + 4), which
// only splits a run.  Keys are non-negative; -1 means "no pixel".
constexpr int kCapBit = 1 << 30;

// Floors of the HEALPix belt / caps with the longitude tt in quarter turns (OFF: tt + 1, unwrapped,
// in (0.18, 5.82), see the fused kernel's incremental longitude).  The belt floors use one FMA
// each: jp = floor(fma(-z, 0.75 N, N (tt + 1/2))), which differs from the rounding order of the
// textbook expression (reading S6) only when the argument lies within ~2 ulp of an integer, i.e.
// for directions within ~1e-15 rad of a pixel boundary (rule T1 allows 1e-12 rad).
struct KeyConsts {
    double dn, dn_half, dn_3q;  // N, N/2, 3N/4 (exact)
};
inline KeyConsts make_key_consts(int64_t nside) {
    KeyConsts k;
    k.dn = (double)nside;
    k.dn_half = 0.5 * (double)nside;
    k.dn_3q = 0.75 * (double)nside;
    return k;
}

// floor(x) for -2^31 <= x < 2^31 on the fp64 adder: x + 1.5 2^52 rounded toward -infinity is the
// integer 1.5 2^52 + floor(x), held in the low word (one DADD.RM of ~9 cycles instead of the
// ~34-cycle F2I.F64, measured on B200: scripts/fp64_microbench.cu).  Exact: it equals the F2I floor
// of the same double for every x >= 0.
__device__ __forceinline__ int floor_rd(double x) {
    return __double2loint(__dadd_rd(x, 6755399441055744.0));
}
__device__ __forceinline__ double floor_rd_value(double big) { return big - 6755399441055744.0; }

template <bool NEST, bool OFF>
__device__ __forceinline__ int loc2ckey(const HealpixGeom& g, const KeyConsts& kc, double dz, double tt, double t1,
                                        double dx, double dy) {
    const double za = fabs(dz);
    // the belt key is formed unconditionally (straight-line, so the scheduler can overlap it with
    // independent work); only the caps branch.
    // t1 = N (tt + 1/2);  jp = floor(N (tt + 1/2) - 3N/4 z), jm = floor(... + 3N/4 z)
    const int bjp = floor_rd(fma(-dz, kc.dn_3q, t1));
    const int bjm = floor_rd(fma(dz, kc.dn_3q, t1));
    const int belt = (bjp << 15) | bjm;
    if (za <= TB_TWO_THIRD) return belt;
    const int nside = (int)g.nside;
    const int m = nside - 1;
    double tmp;
    if (za < TB_CAP_SINTHETA_Z) {
        tmp = __dmul_rn(g.dnside, fast_sqrt(__dmul_rn(3.0, __dsub_rn(1.0, za))));
    } else {
        const double sth = __dsqrt_rn(__dadd_rn(__dmul_rn(dx, dx), __dmul_rn(dy, dy)));
        tmp = __ddiv_rn(__dmul_rn(g.dnside, sth), __dsqrt_rn(__ddiv_rn(__dadd_rn(1.0, za), 3.0)));
    }
    const int south = dz < 0.0 ? 1 : 0;
    if (!NEST) {
        // the cap floors on the fp64 adder (floor_rd: bit-identical to the F2I floors of the same
        // products, ~25 cycles shorter each)
        const double tp = __dsub_rn(tt, floor_rd_value(__dadd_rd(tt, 6755399441055744.0)));
        const int jp = floor_rd(__dmul_rn(tp, tmp));
        const int jm = floor_rd(__dmul_rn(__dsub_rn(1.0, tp), tmp));
        const int ir = jp + jm + 1;
        int ip = floor_rd(__dmul_rn(tt, small_int_to_double(ir)));
        if (OFF) {
            ip -= ir;  // in [-0.82 ir, 4.82 ir)
            if (ip < 0) ip += 4 * ir;
        }
        if (ip >= 4 * ir) ip -= 4 * ir;
        // north: 2 ir (ir - 1) + ip; south: npix - 2 ir (ir + 1) + ip, stored as npix - 1 - pixel
        const int p = south ? 2 * ir * (ir + 1) - 1 - ip : 2 * ir * (ir - 1) + ip;
        return kCapBit | (south << 26) | p;
    } else {
        const double bt = __dadd_rd(tt, 6755399441055744.0);
        int ntt = __double2loint(bt);
        double dntt = floor_rd_value(bt);
        if (!OFF && ntt > 3) {
            ntt = 3;
            dntt = 3.0;
        }
        const double tp = __dsub_rn(tt, dntt);
        const int face = OFF ? ((ntt + 3) & 3) : ntt;
        int jp = floor_rd(__dmul_rn(tp, tmp));
        int jm = floor_rd(__dmul_rn(__dsub_rn(1.0, tp), tmp));
        jp = min(jp, m);
        jm = min(jm, m);
        // the cap pixel (face F or F + 8, ix, iy) written in the BELT key format, so one decoder
        // serves both (ckey_to_pix): the belt decode gives face = (min(ifp, ifm) (+3 OFF) mod 4)
        // + 4 (1 + ifp - ifm), ix = jm mod N, iy = N - 1 - (jp mod N).  North (ix, iy) = (N-1-jm,
        // N-1-jp): ifp = F + d, ifm = F + 1 + d; south (ix, iy) = (jp, jm): ifm = F + d,
        // ifp = F + 1 + d (d = 1 when OFF).  ifp, ifm <= 5, so the fields stay below 6 N < 2^15.
        constexpr int d = OFF ? 1 : 0;
        const int lo = (face + d) << g.order, hi = (face + 1 + d) << g.order;
        const int kp = south ? (hi | (m - jm)) : (lo | jp);
        const int km = south ? (lo | jp) : (hi | (m - jm));
        return (kp << 15) | km;
    }
}

// Pixel of a compact key (run flush; see loc2ckey).
template <bool NEST, bool OFF>
__device__ __forceinline__ int ckey_to_pix(int key, const HealpixGeom& g) {
    const int nside = (int)g.nside;
    const int m = nside - 1;
    if (!NEST && (key & kCapBit)) {  // RING caps (NEST cap keys are in the belt format)
        const int south = (key >> 26) & 1;
        const int p = key & ((1 << 26) - 1);
        return south ? (int)g.npix - 1 - p : p;
    }
    const int jp = key >> 15, jm = key & 0x7fff;
    if (!NEST) {
        const int nl4 = 4 * nside;
        const int ir = nside + 1 + jp - jm;
        const int kshift = 1 - (ir & 1);
        const int t1 = jp + jm - (OFF ? 3 : 1) * nside + kshift + 1 + 2 * nl4;
        const int ip = (t1 >> 1) & (nl4 - 1);
        return (int)g.ncap + nl4 * (ir - 1) + ip;
    }
    const int ifp = jp >> g.order;
    const int ifm = jm >> g.order;
    const int fmin = (ifp < ifm ? ifp : ifm) + (OFF ? 3 : 0);
    const int face = (fmin & 3) + 4 * (1 + ifp - ifm);
    const int ix = jm & m;
    const int iy = (jp & m) ^ m;
    return face * (nside * nside) + (int)interleave16((uint32_t)ix, (uint32_t)iy);
}

// The same as ckey_to_pix without branches (the run flush decodes 32 keys at once, belt and cap
// keys mixed in one warp): both decodings are formed and one is selected.
template <bool NEST, bool OFF>
__device__ __forceinline__ int ckey_to_pix_bf(int key, const HealpixGeom& g) {
    const int nside = (int)g.nside;
    const int m = nside - 1;
    if (!NEST) {
        const bool cap = key & kCapBit;
        const int south = (key >> 26) & 1;
        const int nl4 = 4 * nside;
        const int jp = key >> 15, jm = key & 0x7fff;
        const int ir = nside + 1 + jp - jm;
        const int kshift = 1 - (ir & 1);
        const int t1 = jp + jm - (OFF ? 3 : 1) * nside + kshift + 1 + 2 * nl4;
        const int belt = (int)g.ncap + nl4 * (ir - 1) + ((t1 >> 1) & (nl4 - 1));
        const int p = key & ((1 << 26) - 1);
        const int capp = south ? (int)g.npix - 1 - p : p;
        return cap ? capp : belt;
    }
    // NEST: one decoder (cap keys are in the belt format, see loc2ckey)
    const int jp = key >> 15, jm = key & 0x7fff;
    const int ifp = jp >> g.order, ifm = jm >> g.order;
    const int fmin = (ifp < ifm ? ifp : ifm) + (OFF ? 3 : 0);
    const int face = (fmin & 3) + 4 * (1 + ifp - ifm);
    return face * (nside * nside) + (int)interleave16((uint32_t)(jm & m), (uint32_t)((jp & m) ^ m));
}

// Pixel of a run key (see loc2key32).
template <bool NEST>
__device__ __forceinline__ int key_to_pix32(int key, const HealpixGeom& g) {
    if (!NEST) return key;
    const int m = (int)g.nside - 1;
    const int face_bits = key & ~((1 << (2 * g.order)) - 1);  // face * nside^2
    return face_bits | (int)interleave16((uint32_t)(key & m), (uint32_t)((key >> g.order) & m));
}

// tt = fmodulo(phi * 2/pi, 4) in [0, 4) with phi = atan2(dy, dx) (phi := 0 at dx = dy = 0, S3).
__device__ __forceinline__ double phi_to_tt(double dx, double dy) { return quarter_turns(dx, dy); }

template <bool NEST>
__device__ __forceinline__ int64_t vec2pix(const HealpixGeom& g, double dx, double dy, double dz) {
    return loc2pix<NEST, int64_t>(g, dz, phi_to_tt(dx, dy), dx, dy);
}

// (cos 2psi, sin 2psi) from psi = atan2(by, bx) without forming psi; psi := 0 at bx = by = 0
// (S10): the 1e-100 guard makes (bx, by) = (0, 0) give (1, 0) without a branch and changes
// nothing otherwise (r = sin^2 theta >> 1e-84 for any direction not within 1e-42 rad of a pole).
__device__ __forceinline__ void cos_sin_2psi(double bx, double by, double& c2, double& s2) {
    const double bx2 = bx * bx;
    const double r = fma(by, by, bx2) + 1e-100;
    const double inv = fast_rcp(r);
    c2 = fma(-by, by, bx2 + 1e-100) * inv;
    s2 = 2.0 * bx * by * inv;
}

// Longitude in quarter turns, and the pieces of the polarisation weights, with ONE reciprocal:
// returns tt; sets A = r cos 2psi, B = r sin 2psi (r = bx^2 + by^2 + 1e-100, so (bx, by) = 0
// gives (1, 0), reading S10) and invr = 1/r.  1/(den r) gives 1/den = r/(den r) and
// 1/r = den/(den r).
__device__ __forceinline__ double lon_pol_raw(double dx, double dy, double bx, double by, double& A, double& B,
                                              double& invr) {
    const QtPrep q = qt_prepare(dx, dy);
    const double bx2 = fma(bx, bx, TB_TINY);
    const double r = fma(by, by, bx2);
    const double inv = fast_rcp(q.den * r);
    invr = q.den * inv;
    A = fma(-by, by, bx2);
    B = (bx + bx) * by;
    return qt_finish(q, q.num * (r * inv));
}

// Longitude in quarter turns AND (cos 2psi, sin 2psi) with ONE reciprocal: 1/(den r) gives
// both 1/den = r/(den r) and 1/r = den/(den r) (both factors lie in [1e-100, 2], so the
// product neither overflows nor underflows).
__device__ __forceinline__ double lon_pol(double dx, double dy, double bx, double by, double& c2, double& s2) {
    const QtPrep q = qt_prepare(dx, dy);
    const double bx2 = bx * bx;
    const double r = fma(by, by, bx2) + TB_TINY;
    const double inv = fast_rcp(q.den * r);
    const double invr = q.den * inv;
    c2 = fma(-by, by, bx2 + TB_TINY) * invr;
    s2 = 2.0 * bx * by * invr;
    return qt_finish(q, q.num * (r * inv));
}

}  // namespace toastb200

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
template <bool NEST>
__device__ __forceinline__ int64_t vec2pix(const HealpixGeom& g, double dx, double dy, double dz) {
    const double phi = (dx == 0.0 && dy == 0.0) ? 0.0 : atan2(dy, dx);
    const double za = fabs(dz);
    double tt = __dmul_rn(phi, kInvHalfPi);
    if (tt < 0.0) {
        tt = __dadd_rn(tt, 4.0);
        if (tt == 4.0) tt = 0.0;
    }
    const int64_t nside = g.nside;
    if (za <= kTwoThird) {  // equatorial belt
        const double temp1 = __dmul_rn(g.dnside, __dadd_rn(0.5, tt));
        const double temp2 = __dmul_rn(__dmul_rn(g.dnside, dz), 0.75);
        const int64_t jp = (int64_t)__dsub_rn(temp1, temp2);  // ascending edge line
        const int64_t jm = (int64_t)__dadd_rn(temp1, temp2);  // descending edge line
        if (!NEST) {
            const int64_t nl4 = 4 * nside;
            const int64_t ir = nside + 1 + jp - jm;
            const int64_t kshift = 1 - (ir & 1);
            const int64_t t1 = jp + jm - nside + kshift + 1 + 2 * nl4;
            const int64_t ip = (t1 >> 1) & (nl4 - 1);
            return g.ncap + nl4 * (ir - 1) + ip;
        } else {
            const int64_t ifp = jp >> g.order;
            const int64_t ifm = jm >> g.order;
            const int64_t face = (ifp == ifm) ? (ifp | 4) : ((ifp < ifm) ? ifp : (ifm + 8));
            const int64_t ix = jm & (nside - 1);
            const int64_t iy = nside - (jp & (nside - 1)) - 1;
            return face * nside * nside + (int64_t)(spread_bits(ix) | (spread_bits(iy) << 1));
        }
    }
    // polar caps; the well-conditioned sin(theta) form for za >= 0.99 (reading S5)
    double tmp;
    if (za < 0.99) {
        tmp = __dmul_rn(g.dnside, __dsqrt_rn(__dmul_rn(3.0, __dsub_rn(1.0, za))));
    } else {
        const double sth = __dsqrt_rn(__dadd_rn(__dmul_rn(dx, dx), __dmul_rn(dy, dy)));
        tmp = __ddiv_rn(__dmul_rn(g.dnside, sth), __dsqrt_rn(__ddiv_rn(__dadd_rn(1.0, za), 3.0)));
    }
    if (!NEST) {
        const double tp = __dsub_rn(tt, (double)(int64_t)tt);
        const int64_t jp = (int64_t)__dmul_rn(tp, tmp);
        const int64_t jm = (int64_t)__dmul_rn(__dsub_rn(1.0, tp), tmp);
        const int64_t ir = jp + jm + 1;
        int64_t ip = (int64_t)__dmul_rn(tt, (double)ir);
        if (ip >= 4 * ir) ip -= 4 * ir;
        return (dz > 0.0) ? 2 * ir * (ir - 1) + ip : g.npix - 2 * ir * (ir + 1) + ip;
    } else {
        int64_t ntt = (int64_t)tt;
        if (ntt > 3) ntt = 3;
        const double tp = __dsub_rn(tt, (double)ntt);
        int64_t jp = (int64_t)__dmul_rn(tp, tmp);
        int64_t jm = (int64_t)__dmul_rn(__dsub_rn(1.0, tp), tmp);
        if (jp > nside - 1) jp = nside - 1;
        if (jm > nside - 1) jm = nside - 1;
        int64_t face, ix, iy;
        if (dz >= 0.0) {
            face = ntt; ix = nside - jm - 1; iy = nside - jp - 1;
        } else {
            face = ntt + 8; ix = jp; iy = jm;
        }
        return face * nside * nside + (int64_t)(spread_bits(ix) | (spread_bits(iy) << 1));
    }
}

// (cos 2psi, sin 2psi) from psi = atan2(by, bx) without forming psi; psi := 0 at bx = by = 0 (S10).
__device__ __forceinline__ void cos_sin_2psi(double bx, double by, double& c2, double& s2) {
    const double bx2 = bx * bx, by2 = by * by;
    const double r = bx2 + by2;
    if (r > 0.0) {
        const double inv = 1.0 / r;
        c2 = (bx2 - by2) * inv;
        s2 = 2.0 * bx * by * inv;
    } else {
        c2 = 1.0;
        s2 = 0.0;
    }
}

}  // namespace toastb200

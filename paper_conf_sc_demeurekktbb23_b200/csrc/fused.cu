// fused.cu — toast_pointing_to_map: A1 -> A2 -> A3 -> A4 per detector-sample in registers, and
// (SCAN mode of the same kernel) toast_pointing_to_tod: A1 -> A2 -> A3 -> A5.
//
// Decomposition (B200-first):
//   * A WARP owns a work item = (chunk of <= kFusedChunk consecutive in-interval samples,
//     group of 32 detectors); LANE = DETECTOR.  Items are handed out dynamically (one atomic per
//     item, fetched one item ahead) in chunk-major order, so the warps in flight cover a short
//     time window of the focal plane and the sky footprint they scatter into stays L2-resident.
//   * Each lane holds its detector's frame in registers for the whole item:
//       u = R(f) z, v = R(f) x, w = R(f) y, det_scale*cal, det_scale*eta*cal.
//   * An item is a STREAM OF BLOCKS of kBlk = 16 samples through two warp-private shared
//     buffers: while block i is computed, lane 0's bulk tensor copies (TMA, mbarrier-completed;
//     per-lane cp.async when the TMA constraints fail) stage block i+1 — the TOD tile [32 x 16]
//     (128-byte swizzled), the det-flag rows, 16 boresight quaternions, HWP angles and shared
//     flags.  Lanes 0..15 turn them into the per-sample state (boresight rotation matrix B —
//     identity if shared-flagged, reading S2), lanes 16..31 into cos/sin 4 chi; every lane then
//     walks the 16 samples reading that state as shared-memory broadcasts.  Boresight, HWP and
//     shared flags are read from HBM once per 32 detectors.
//   * Per det-sample: dir = B u, bx = (B v)_z, by = -(B w)_z, the longitude carried
//     incrementally along the lane's samples (one reciprocal shared with the weights), the
//     HEALPix run key, cos/sin 2psi algebraically, the HWP angle addition.
//   * Map accumulation is RUN-LENGTH aggregated per lane along time: consecutive samples of one
//     detector in the same pixel are summed in registers and flushed with one fp64 `red` per
//     Stokes component when the pixel changes; hit-submap flags are gathered per CTA in shared
//     memory.  SCAN mode gathers the map instead (cached per lane across the run) and updates
//     the staged TOD tile, written back after each block.
#include <cuda.h>  // CUtensorMap (the encoder is fetched through the runtime; no -lcuda)
#include <cuda_runtime.h>
#include <cudaTypedefs.h>

#include <algorithm>
#include <cstring>
#include <mutex>

#include "device_math.cuh"
#include "internal.h"

namespace toastb200 {

namespace {

#ifndef TB_FUSED_MINB
#define TB_FUSED_MINB 2  // resident CTAs per SM the register allocation is bounded for
#endif
#ifndef TB_FUSED_DPL_MAX
#define TB_FUSED_DPL_MAX 1  // detectors per lane (2 when n_det > 32 and DPL_MAX = 2)
#endif
#ifndef TB_WARPS
#define TB_WARPS 8
#endif
constexpr int kWarps = TB_WARPS;  // warps per CTA
#ifndef TB_BLK
#define TB_BLK 16
#endif
constexpr int kBlk = TB_BLK;  // samples per block (8 or 16)
constexpr int kRowStep = 32 / kBlk;  // TOD rows staged per cp.async instruction
#ifndef TB_KUNROLL
#define TB_KUNROLL 1
#endif
constexpr int kKUnroll = TB_KUNROLL;  // unroll of the per-sample loop
#ifndef TB_INCR
#define TB_INCR 1  // incremental longitude along each detector's samples (see stage_a)
#endif
#ifndef TB_FOLD
#define TB_FOLD 1  // det_scale (and eta cal) applied once per run at the flush, not per det-sample
#endif
#ifndef TB_TTOFF
#define TB_TTOFF 1  // 32-bit keys: longitude carried as tt + 1 without wrapping (see stage_a)
#endif
#ifndef TB_INCR_BF
#define TB_INCR_BF 1  // branch-free incremental-longitude series (see stage_a; measured -0.5..1 % C2)
#endif
#ifndef TB_DEFER
#define TB_DEFER 1  // a det-sample's contribution is folded into its run one sample later
#endif
#ifndef TB_HITDEDUP
#define TB_HITDEDUP 0  // shared hit flags: compare with the lane's last submap first (measured: +1 % C2, +2 % C3)
#endif
constexpr int kPad = kBlk + 1;

// per-sample state: B[0..8], c4, s4, mode (as a double: 1 pixelise, 2 shared-flagged)
struct SampleState {
    double v[12];
};

// Raw inputs of one block (filled by cp.async).
template <int DPL>
struct alignas(16) RawBlock {
    double tod[32 * DPL][kPad];
    double bore[kBlk][4];
    double hwp[kBlk];
    uint8_t flg[32 * DPL][kBlk + 4];  // 5 aligned words covering each row's 16 flag bytes
    uint8_t sflg[kBlk + 8];           // 5 aligned words covering the 16 shared flags
};

template <int DPL>
struct WarpSmem {
    RawBlock<DPL> buf[2];
    SampleState st[kBlk];
};

__device__ __forceinline__ void cp_async16(void* smem, const void* gmem) {
    const unsigned s = (unsigned)__cvta_generic_to_shared(smem);
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(s), "l"(gmem) : "memory");
}
// L2 evict-first policy for the streamed-once inputs (TOD, det flags): they must not push
// the map lines being accumulated out of L2 (the map's red operations miss otherwise).
__device__ __forceinline__ uint64_t evict_first_policy() {
    uint64_t pol;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;\n" : "=l"(pol));
    return pol;
}
__device__ __forceinline__ void cp_async8(void* smem, const void* gmem) {
    const unsigned s = (unsigned)__cvta_generic_to_shared(smem);
    asm volatile("cp.async.ca.shared.global [%0], [%1], 8;\n" ::"r"(s), "l"(gmem) : "memory");
}
__device__ __forceinline__ void cp_async8_stream(void* smem, const void* gmem, uint64_t pol) {
    const unsigned s = (unsigned)__cvta_generic_to_shared(smem);
    asm volatile("cp.async.ca.shared.global.L2::cache_hint [%0], [%1], 8, %2;\n" ::"r"(s), "l"(gmem), "l"(pol)
                 : "memory");
}
__device__ __forceinline__ void cp_async4(void* smem, const void* gmem) {
    const unsigned s = (unsigned)__cvta_generic_to_shared(smem);
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4;\n" ::"r"(s), "l"(gmem) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;\n" ::: "memory"); }
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_all;\n" ::: "memory"); }

// Copy the aligned 4-byte words covering bytes [p, p + n) (n <= 16) to dst[0..20); the
// caller reads byte i of the range at dst[(p & 3) + i].  Words past the range are skipped,
// so nothing beyond the aligned word holding the last byte is read.
__device__ __forceinline__ void cp_async_bytes(uint8_t* dst, const uint8_t* p, int n, int w) {
    const uint8_t* w0 = reinterpret_cast<const uint8_t*>(reinterpret_cast<uintptr_t>(p) & ~uintptr_t(3));
    if (w0 + 4 * w < p + n) cp_async4(dst + 4 * w, w0 + 4 * w);
}

// ----------------------------------------------------------------------------- TMA path
// When the inputs satisfy the tensor-memory-accelerator constraints (n_samp % 16 == 0 and
// 16-byte aligned arrays), lane 0 moves a whole block with five
// bulk tensor copies that complete on a per-buffer mbarrier, instead of 32 lanes issuing
// ~30 cp.async each with 64-bit address arithmetic.  The TOD tile [32 det][16 samples] lands
// 128-byte-swizzled (row r's 16-byte chunk c at c ^ (r & 7)), so the per-sample column read
// tod[lane][k] is a 4-wavefront access without padding bytes.  Boxes start at multiples of 16
// samples (a box must start 16-byte aligned in every staged row).
struct alignas(64) TmaMaps {
    CUtensorMap tod;   // f64 [n_det][n_samp], box {16, 32}, SWIZZLE_128B
    CUtensorMap flg;   // u8  [n_det][n_samp], box {16, 32}
    CUtensorMap bore;  // f64 [n_samp][4],     box {4, 16}
    CUtensorMap hwp;   // f64 [n_samp],        box {16}
    CUtensorMap sflg;  // u8  [n_samp],        box {16}
};

// Every TMA destination is 128-byte aligned; the 16 shared-flag bytes of a buffer share their
// 128-byte slot with that buffer's mbarrier, so a warp's staging area is exactly 12 KB.
struct alignas(128) SflgSlot {
    uint8_t f[16];
    unsigned long long mbar;
    uint8_t pad[104];
};
struct alignas(1024) TmaWarpSmem {
    double tod[2][32][16];           // 1024-aligned (the 128-byte swizzle pattern spans 1 KB)
    uint8_t flg[2][32][16];
    double bore[2][16][4];
    double hwp[2][16];
    SflgSlot sf[2];
    double st[16][12];               // SampleState[kBlk]
};
static_assert(sizeof(TmaWarpSmem) == 12288, "TMA staging area: 12 KB per warp");

__device__ __forceinline__ unsigned smem_u32(const void* p) { return (unsigned)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void mbar_init(unsigned long long* bar) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;\n" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(unsigned long long* bar, unsigned bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;\n" ::"r"(smem_u32(bar)), "r"(bytes)
                 : "memory");
}
__device__ __forceinline__ void mbar_wait(unsigned long long* bar, unsigned parity) {
    unsigned done;
    do {
        asm volatile(
            "{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n}\n"
            : "=r"(done)
            : "r"(smem_u32(bar)), "r"(parity)
            : "memory");
    } while (!done);
}
__device__ __forceinline__ void tma_1d(void* dst, const CUtensorMap* m, int c0, unsigned long long* bar) {
    asm volatile(
        "cp.async.bulk.tensor.1d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2}], [%3];\n" ::"r"(
            smem_u32(dst)),
        "l"(m), "r"(c0), "r"(smem_u32(bar))
        : "memory");
}
__device__ __forceinline__ void tma_2d(void* dst, const CUtensorMap* m, int c0, int c1, unsigned long long* bar) {
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], "
        "[%4];\n" ::"r"(smem_u32(dst)),
        "l"(m), "r"(c0), "r"(c1), "r"(smem_u32(bar))
        : "memory");
}
// streamed-once TOD / det flags with an L2 evict-first hint (see evict_first_policy)
__device__ __forceinline__ void tma_2d_stream(void* dst, const CUtensorMap* m, int c0, int c1,
                                              unsigned long long* bar, uint64_t pol) {
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1, "
        "{%2, %3}], [%4], %5;\n" ::"r"(smem_u32(dst)),
        "l"(m), "r"(c0), "r"(c1), "r"(smem_u32(bar)), "l"(pol)
        : "memory");
}

// Pixel index type: 32-bit up to nside 8192 (12 nside^2 < 2^31), else 64-bit.
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

// Submap of a pixel (shift when n_pix_submap is a power of two).
template <typename P>
__device__ __forceinline__ int64_t submap_of(P pix, const MapGeom& mg) {
    return mg.sm_shift >= 0 ? (int64_t)(pix >> mg.sm_shift) : (int64_t)pix / mg.n_pix_submap;
}

// Pixel of a run key: 32-bit NEST keys are the cheap (face, iy, ix) packing of loc2key32;
// 64-bit keys (nside > 8192) and RING keys are the pixel itself.
template <bool NEST, bool WIDE>
__device__ __forceinline__ typename PixT<WIDE>::T key_to_pix(typename PixT<WIDE>::T key, const HealpixGeom& g) {
    if constexpr (WIDE) {
        return key;
    } else {
        return key_to_pix32<NEST>(key, g);
    }
}

template <typename P>
struct Slot {
    double u0, u1, u2, v0, v1, v2, w0, w1, w2;
    double s_cal;   // det_scale * cal       (I weight folded into the noise weight)
    double s_eta;   // det_scale * eta * cal (Q/U amplitude folded into the noise weight)
    double etacal;  // debug outputs only
    P run_key;            // key of the run being aggregated (-1: none)
    P run_lp;             // its pixel's index inside the submap
    int64_t run_loc;      // global2local of the run's submap, LOADED WHEN THE RUN STARTS
    P last_sm;            // last submap this lane marked in hit_submaps (generic path)
    int64_t last_loc;     // SCAN: global2local of last_sm
    double r0, r1, r2;
    P pend_key;           // pending (not yet aggregated) det-sample
    double p0, p1, p2;
    double px, py, ptt;   // INCR mode: projected direction and tt of the lane's previous sample
    bool ok;
};

// Per-CTA shared memory besides the warps' staging areas: the bit-spread table of the NEST
// interleave (spread[b] = the 8 bits of b moved to the even bit positions) and the CTA's
// hit-submap flags (MapGeom::shared_hits).
struct CtaMem {
    const uint16_t* spread;  // [256]
    uint8_t* hits;           // [n_submap] when MapGeom::shared_hits
};
constexpr int kSpreadBytes = 512;

// Pixel of a 32-bit run key with the bit interleave from the shared spread table: 2 (nside <=
// 256) or 4 table loads instead of the ~16 instructions of interleave16 — this runs at every run
// start, and with 32 detectors per warp some lane starts a run at most samples.
template <bool NEST>
__device__ __forceinline__ int key_to_pix_tab(int key, const HealpixGeom& g, const uint16_t* spread) {
    if (!NEST) return key;
    const int m = (int)g.nside - 1;
    const uint32_t ix = (uint32_t)(key & m), iy = (uint32_t)((key >> g.order) & m);
    uint32_t v = spread[ix & 255u] | ((uint32_t)spread[iy & 255u] << 1);
    if (g.order > 8) v |= (spread[ix >> 8] | ((uint32_t)spread[iy >> 8] << 1)) << 16;
    return (key & ~((1 << (2 * g.order)) - 1)) | (int)v;
}

// A run starts: mark its submap hit (as A2 does) and issue the global2local lookup now, so
// the load latency is hidden behind the run's samples instead of stalling the flush.  The hit
// flag is stored only when the lane's submap CHANGES: thousands of warps re-writing the same
// few bytes of hit_submaps serialise in L2 and cost as much as the whole computation.
// Sets sl.run_loc (-1: the submap has no storage) and sl.run_lp.
template <bool NEST, bool WIDE>
__device__ __forceinline__ void start_run(typename PixT<WIDE>::T key, const FusedArgs& a, const HealpixGeom& g,
                                          Slot<typename PixT<WIDE>::T>& sl, const CtaMem& cm) {
    using P = typename PixT<WIDE>::T;
    const MapGeom& mg = a.map;
    P pix;
    if constexpr (WIDE)
        pix = key;
    else
        pix = key_to_pix_tab<NEST>(key, g, cm.spread);
    P sm;
    if (mg.sm_shift >= 0) {
        sm = pix >> mg.sm_shift;
        sl.run_lp = pix & (P)(mg.n_pix_submap - 1);
    } else {
        sm = pix / (P)mg.n_pix_submap;
        sl.run_lp = pix - sm * (P)mg.n_pix_submap;
    }
#ifndef TB_X_NOHIT
    if (mg.shared_hits) {
        // the CTA's shared copy (idempotent store, no atomic; see the kernel end)
#if TB_HITDEDUP
        if (sm != sl.last_sm) {
            cm.hits[sm] = 1;
            sl.last_sm = sm;
        }
#else
        cm.hits[sm] = 1;
#endif
    } else if (a.hit_submaps && sm != sl.last_sm) {
        a.hit_submaps[sm] = 1;
        sl.last_sm = sm;
    }
#endif
#ifdef TB_X_NOG2L
    sl.run_loc = sm;
#else
    sl.run_loc = __ldg(&mg.global2local[sm]);
#endif
}

// A run ends: one fp64 red per Stokes component (nothing if the submap has no storage).  Up to
// nside 8192 the map element index fits 32 bits (< 12 * 8192^2 pixels), so the address is one
// IMAD + one IMAD.WIDE.U32.  With TB_FOLD the run sums are unscaled (sum of tod, of tod w/r)
// and det_scale * cal, det_scale * eta * cal are applied here, once per run.
template <int NNZ, bool WIDE>
__device__ __forceinline__ void flush(const Slot<typename PixT<WIDE>::T>& sl, const FusedArgs& a) {
    if (sl.run_loc < 0) return;
    double* dst;
    if constexpr (WIDE) {
        dst = a.zmap + (sl.run_loc * a.map.n_pix_submap + sl.run_lp) * NNZ;
    } else {
        const unsigned idx = (unsigned)sl.run_loc * (unsigned)a.map.n_pix_submap + (unsigned)sl.run_lp;
        dst = a.zmap + (size_t)idx * NNZ;
    }
#if TB_FOLD
    atomicAdd(dst, sl.r0 * sl.s_cal);
    if (NNZ == 3) {
        atomicAdd(dst + 1, sl.r1 * sl.s_eta);
        atomicAdd(dst + 2, sl.r2 * sl.s_eta);
    }
#else
    atomicAdd(dst, sl.r0);
    if (NNZ == 3) {
        atomicAdd(dst + 1, sl.r1);
        atomicAdd(dst + 2, sl.r2);
    }
#endif
}

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
    // a lane without a detector contributes exactly 0 (aggregate() adds unconditionally)
    sl.s_cal = ok ? scale * a.cal : 0.0;
    sl.s_eta = ok ? scale * sl.etacal : 0.0;
    sl.run_key = -1;
    sl.run_lp = 0;
    sl.run_loc = -1;
    sl.last_sm = -1;
    sl.last_loc = -1;
    sl.r0 = sl.r1 = sl.r2 = 0.0;
    sl.pend_key = -1;
    sl.p0 = sl.p1 = sl.p2 = 0.0;
    sl.px = sl.py = sl.ptt = 0.0;  // dot = 0: the item's first sample takes the full arctangent
    sl.ok = ok;
}

// The straight-line fp64 part of one det-sample (A1 -> direction, A3 weights and the A2
// longitude): no branches, so two of them can be interleaved by the scheduler (pair loop).
struct StageA {
    double dx, dy, dz, tt;
    double cw, sw, invr;  // r cos 2(psi + 2 chi), r sin 2(psi + 2 chi), 1/r
};

// (2/pi) atan(t) = t Q(t^2) for |t| <= kIncrMax = 0.01 (TB_INCR_MAX, in the constant bank): the
// Taylor series to t^7; the first omitted term is (2/pi) t^9 / 9 <= 7e-20 (absolute) at |t| = 0.01.
__constant__ double kIncrQ[4] = {0.63661977236758134308, -0.21220659078919378103, 0.12732395447351626862,
                                 -0.090945681766797334729};

template <int NNZ, bool HWP, typename P>
__device__ __forceinline__ StageA stage_a(Slot<P>& sl, const double* x) {
    constexpr bool TTOFF = TB_TTOFF && TB_INCR && sizeof(P) == 4;
    StageA o;
    o.dx = x[0] * sl.u0 + x[1] * sl.u1 + x[2] * sl.u2;
    o.dy = x[3] * sl.u0 + x[4] * sl.u1 + x[5] * sl.u2;
    o.dz = x[6] * sl.u0 + x[7] * sl.u1 + x[8] * sl.u2;
    o.cw = o.sw = o.invr = 0.0;
    if (NNZ == 3) {
        const double bx = x[6] * sl.v0 + x[7] * sl.v1 + x[8] * sl.v2;
        const double by = -(x[6] * sl.w0 + x[7] * sl.w1 + x[8] * sl.w2);
#ifdef TB_X_NOATAN
        o.tt = fabs(o.dx) * 3.9; o.cw = bx; o.sw = by; o.invr = 1.0;  // ablation: no longitude/weights arithmetic
#elif TB_INCR
        // INCREMENTAL LONGITUDE: consecutive samples of a detector
        // are close on the sky, so tt(s) = tt(s') + (2/pi) atan(t) with t = tan(phi(s) - phi(s'))
        // = cross / dot of the projected directions of s and of this lane's previous processed
        // sample s' — a 4-term series instead of the octant reduction, the 11-term polynomial and
        // the octant bookkeeping.  Each step adds ~1 ulp of tt (~4e-16 quarter turns); the chain
        // restarts from the full arctangent at every item (<= 128 samples), so the drift stays
        // ~1e-15 rad, far inside rule T1's 1e-12 rad.  The ONE reciprocal 1/(dot r) still serves
        // both t and the weights' 1/r.  Lanes whose step is large (|t| > 0.01: near a pole, after
        // a gap) or that have no previous sample (dot = 0) take the full path.
        const double bx2 = fma(bx, bx, TB_TINY);
        const double r = fma(by, by, bx2);
        o.cw = fma(-by, by, bx2);
        o.sw = (bx + bx) * by;
        const double cross = fma(sl.px, o.dy, -(sl.py * o.dx));
        const double dot = fma(sl.px, o.dx, sl.py * o.dy);
        const double inv = fast_rcp(dot * r);
        // |cross| < kIncrMax dot  <=>  dot > 0 and |t| < kIncrMax (t = cross / dot); false at
        // dot = 0 (no previous sample) and for steps beyond a quarter turn; one DFMA + DSETP,
        // resolved before the reciprocal's result is needed
#if TB_INCR_BF
        // branch-free common path: the series is evaluated for every sample (NaN at dot = 0, no
        // traps on the GPU) and only the rare full-arctangent path is a branch, so the scheduler
        // can interleave the series with the surrounding straight-line code
        {
            const double t = cross * (r * inv);
            o.invr = dot * inv;
            const double s2 = t * t;
            double q = fma(kIncrQ[3], s2, kIncrQ[2]);
            q = fma(q, s2, kIncrQ[1]);
            q = fma(q, s2, kIncrQ[0]);
            double tt = fma(t, q, sl.ptt);
            if constexpr (!TTOFF) {
                if (__double2hiint(tt) < 0) tt += 4.0;
                if (__double2hiint(tt) >= 0x40100000) tt -= 4.0;
            }
            o.tt = tt;
        }
        if (!(fma(TB_INCR_MAX, dot, -fabs(cross)) > 0.0)) {
#else
        if (fma(TB_INCR_MAX, dot, -fabs(cross)) > 0.0) {
            const double t = cross * (r * inv);
            o.invr = dot * inv;
            const double s2 = t * t;
            double q = fma(kIncrQ[3], s2, kIncrQ[2]);
            q = fma(q, s2, kIncrQ[1]);
            q = fma(q, s2, kIncrQ[0]);
            double tt = fma(t, q, sl.ptt);
            if constexpr (!TTOFF) {
                if (__double2hiint(tt) < 0) tt += 4.0;
                if (__double2hiint(tt) >= 0x40100000) tt -= 4.0;
            }
            o.tt = tt;
        } else {
#endif
            // TTOFF: the chain is carried as tt + 1 WITHOUT wrapping: it restarts here from a
            // value in [1, 5) and drifts by at most 127 steps of (2/pi) atan(0.01) = 0.0064
            // within an item, so it stays in (0.18, 5.82); loc2key32<NEST, true> folds it back
            o.tt = lon_pol_raw(o.dx, o.dy, bx, by, o.cw, o.sw, o.invr) + (TTOFF ? 1.0 : 0.0);
        }
        sl.px = o.dx;
        sl.py = o.dy;
        sl.ptt = o.tt;
#else
        o.tt = lon_pol_raw(o.dx, o.dy, bx, by, o.cw, o.sw, o.invr);  // one shared reciprocal
#endif
        if (HWP) {
            const double c4 = x[9], s4 = x[10];
            const double cq = o.cw * c4 - o.sw * s4;
            const double sq = o.sw * c4 + o.cw * s4;
            o.cw = cq;
            o.sw = sq;
        }
    } else {
        o.tt = quarter_turns(o.dx, o.dy);
    }
    return o;
}

// The HEALPix floors and integer part (branches: equatorial belt / caps): the run key.
template <bool NEST, int NNZ, bool WIDE>
__device__ __forceinline__ typename PixT<WIDE>::T stage_b(const StageA& o, bool pixelise, bool ok,
                                                         const HealpixGeom& g) {
    using P = typename PixT<WIDE>::T;
    P key = -1;
    if (pixelise) {
        if constexpr (WIDE)
            key = (P)loc2pix<NEST, int64_t>(g, o.dz, o.tt, o.dx, o.dy);
        else
#ifdef TB_X_NOPIX
            key = (P)((int)(o.tt * 1000.0) & 0xffff);  // ablation: no HEALPix integer/floor logic
#else
            key = (P)loc2key32<NEST, TB_TTOFF && TB_INCR && NNZ == 3>(g, o.dz, o.tt, o.dx, o.dy);
#endif
    }
    if (!ok) key = -1;
    return key;
}

// The A4 contribution of a det-sample, pending until aggregate() folds it into the run.
// Det-flagged samples keep their key (they mark hit submaps, as A2 does) but add 0 (their
// staged tod is 0); so does every sample without a key (aggregate() adds unconditionally).
template <int NNZ, typename P>
__device__ __forceinline__ void set_pending(Slot<P>& sl, const StageA& o, P key, double tod) {
    sl.pend_key = key;
#if TB_FOLD
    sl.p0 = tod;
    if (NNZ == 3) {
        const double t = tod * o.invr;
#else
    sl.p0 = tod * sl.s_cal;
    if (NNZ == 3) {
        const double t = (tod * sl.s_eta) * o.invr;
#endif
        sl.p1 = t * o.cw;
        sl.p2 = t * o.sw;
    }
}

// One det-sample of slot `sl` with the per-sample state x.  `tod` is already 0 for det-flagged
// samples (and, with debug outputs, shared-flagged ones): the block prologue zeroes them in the
// staged tile, so no per-sample flag test is needed here.  Its contribution is folded into the
// lane's run by aggregate() one sample LATER, so that work overlaps the next sample's loads.
template <bool NEST, int NNZ, bool HWP, bool DEBUG, bool WIDE>
__device__ __forceinline__ void det_sample(Slot<typename PixT<WIDE>::T>& sl, const double* x, bool pixelise,
                                           double tod, const HealpixGeom& g, const FusedArgs& a, int64_t d,
                                           int64_t s) {
    using P = typename PixT<WIDE>::T;
    const StageA o = stage_a<NNZ, HWP, P>(sl, x);
    const P key = stage_b<NEST, NNZ, WIDE>(o, pixelise, sl.ok, g);
    if (DEBUG && sl.ok) {
        const int64_t off = d * a.n_samp + s;
        if (a.pixels_out) a.pixels_out[off] = key < 0 ? (int64_t)-1 : (int64_t)key_to_pix<NEST, WIDE>(key, g);
        if (a.weights_out) {
            a.weights_out[off * NNZ] = a.cal;
            if (NNZ == 3) {
                a.weights_out[off * NNZ + 1] = sl.etacal * (o.cw * o.invr);
                a.weights_out[off * NNZ + 2] = sl.etacal * (o.sw * o.invr);
            }
        }
    }
    set_pending<NNZ, P>(sl, o, key, tod);
}

// Fold the pending contribution into the run (run-length aggregation along time).  Lanes
// without a pixel (no detector / flagged sample) have pend_key = -1 and never start a run.
// A pending sample without a pixel carries zero contributions, so the add is unconditional
// (one branch less per det-sample); pend_key is not reset here because det_sample() always
// overwrites it right after (the end-of-item call is followed by the final flush).  The first
// run of an item flushes nothing: run_loc starts at -1.
template <bool NEST, int NNZ, bool WIDE>
__device__ __forceinline__ void aggregate(Slot<typename PixT<WIDE>::T>& sl, const FusedArgs& a,
                                          const HealpixGeom& g, const CtaMem& cm) {
    if (sl.pend_key >= 0 && sl.pend_key != sl.run_key) {
#ifndef TB_X_NOFLUSH
        flush<NNZ, WIDE>(sl, a);
#endif
        sl.run_key = sl.pend_key;
        start_run<NEST, WIDE>(sl.pend_key, a, g, sl, cm);
        sl.r0 = sl.r1 = sl.r2 = 0.0;
    }
    sl.r0 += sl.p0;
    if (NNZ == 3) {
        sl.r1 += sl.p1;
        sl.r2 += sl.p2;
    }
}
// A block of the stream: samples [s0, s0 + nb) of chunk c for detector rows d0 .. d0+nrows-1.
struct Blk {
    int64_t item;  // < 0: end of stream
    int64_t d0;
    int64_t s0;     // first sample of the staged box
    int64_t s_end;  // end of the item's chunk
    int nb;         // samples processed: box indices k0 .. k0 + nb - 1
    int nrows;
    int k0 = 0;     // TMA path: first processed box sample (boxes start at multiples of 16)
};

template <int DPL>
__device__ __forceinline__ void issue_block(RawBlock<DPL>& rb, const Blk& bk, const FusedArgs& a, bool have_dflags,
                                            bool hwp, int lane) {
    constexpr int kRows = 32 * DPL;
    const int64_t n_samp = a.n_samp;
    const int scol = lane & (kBlk - 1);
    const int srow = lane / kBlk;
    if (scol < bk.nb) {
        const double* src = a.det_data + (bk.d0 + srow) * n_samp + bk.s0 + scol;
        const int64_t step = kRowStep * n_samp;
        const uint64_t pol = evict_first_policy();
        if (bk.nrows == kRows) {
#pragma unroll 8
            for (int r = srow; r < kRows; r += kRowStep, src += step) cp_async8_stream(&rb.tod[r][scol], src, pol);
        } else {
            for (int r = srow; r < bk.nrows; r += kRowStep, src += step) cp_async8_stream(&rb.tod[r][scol], src, pol);
        }
    }
    // boresight: 16 quaternions = 32 x 16 B, one per lane
    if ((lane >> 1) < bk.nb) cp_async16(&rb.bore[lane >> 1][2 * (lane & 1)], a.boresight + 4 * (bk.s0 + (lane >> 1)) + 2 * (lane & 1));
    if (hwp && lane < bk.nb) cp_async8(&rb.hwp[lane], a.hwp + bk.s0 + lane);
    if (a.shared_flags && lane < 5) cp_async_bytes(rb.sflg, a.shared_flags + bk.s0, bk.nb, lane);
    if (have_dflags) {
#pragma unroll
        for (int j = 0; j < DPL; ++j) {
            const int row = lane + 32 * j;
            if (row < bk.nrows) {
#pragma unroll
                for (int w = 0; w < 5; ++w) cp_async_bytes(rb.flg[row], a.det_flags + (bk.d0 + row) * n_samp + bk.s0, bk.nb, w);
            }
        }
    }
    cp_async_commit();
}

// SCAN = true: the scan direction, toast_pointing_to_tod: the same item / block
// stream, staging and per-det-sample arithmetic, but each det-sample GATHERS its pixel's map
// values (cached per lane across the run) and updates its TOD in the staged tile; the processed
// columns of the tile are written back after each block (per-lane stores: a TMA store of the
// whole box would overwrite samples of a neighbouring chunk that another warp owns).
template <bool NEST, int NNZ, bool HWP, bool DEBUG, bool WIDE, int DPL, bool TMA, bool SCAN = false>
__global__ void __launch_bounds__(kWarps * 32, TB_FUSED_MINB) pointing_to_map_kernel(const Chunk* __restrict__ chunks,
                                                                         int64_t n_chunks, FusedArgs a,
                                                                         HealpixGeom g,
                                                                         unsigned long long* __restrict__ sched,
                                                                         const __grid_constant__ TmaMaps tm) {
    static_assert(!TMA || (DPL == 1 && kBlk == 16), "the TMA path stages 32 x 16 tiles");
    static_assert(!SCAN || (DPL == 1 && !DEBUG), "the scan direction: one detector per lane, no debug outputs");
    using P = typename PixT<WIDE>::T;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    const int lane = threadIdx.x & 31;
    const int wid = threadIdx.x >> 5;
    // cp.async path: WarpSmem<DPL>; TMA path: TmaWarpSmem (1 KB-aligned, see launch_t)
    WarpSmem<DPL>& sm = reinterpret_cast<WarpSmem<DPL>*>(smem_raw)[wid];
    // (offset arithmetic on the __shared__ array itself, so every access below stays an LDS;
    // the alignment that matters for TMA and the swizzle is that of the shared-window offset)
    const unsigned pad1k = (1024u - (smem_u32(smem_raw) & 1023u)) & 1023u;
    TmaWarpSmem& tw = reinterpret_cast<TmaWarpSmem*>(smem_raw + pad1k)[wid];
    // the CTA's spread table and hit-submap flags: after every warp's staging area
    unsigned char* cta_extra = smem_raw + (TMA ? 1024 + kWarps * sizeof(TmaWarpSmem) : kWarps * sizeof(WarpSmem<DPL>));
    uint16_t* s_spread = reinterpret_cast<uint16_t*>(cta_extra);
    uint8_t* s_hits = cta_extra + kSpreadBytes;
    const CtaMem cm{s_spread, s_hits};
    const bool shared_hits = a.map.shared_hits;
    for (int i = threadIdx.x; i < 256; i += blockDim.x) {
        unsigned v = 0u;
        for (int b = 0; b < 8; ++b) v |= ((i >> b) & 1u) << (2 * b);
        s_spread[i] = (uint16_t)v;
    }
    if (shared_hits)
        for (int i = threadIdx.x; i < (int)a.map.n_submap; i += blockDim.x) s_hits[i] = 0;
    __syncthreads();
    constexpr int kRows = 32 * DPL;
    const int64_t n_groups = (a.n_det + kRows - 1) / kRows;
    const int64_t n_items = n_chunks * n_groups;
    const unsigned dmask = a.det_flag_mask;
    const unsigned smask = a.shared_flag_mask;
    const bool have_dflags = !SCAN && a.det_flags != nullptr;  // scan_map ignores det flags (S12)
    const bool have_sflags = a.shared_flags != nullptr;
    // TMA: bytes landing per block (full boxes, out-of-range elements zero-filled)
    const unsigned tx_bytes = 32 * 16 * 8 + 16 * 32 + (have_dflags ? 32 * 16 : 0) +
                              ((HWP && NNZ == 3) ? 16 * 8 : 0) + (have_sflags ? 16 : 0);
    unsigned phase = 0u;  // TMA: bit b = parity of the next completion of mbar[b]
    const double sgn_ds = (a.should_subtract ? -1.0 : 1.0) * a.data_scale;  // SCAN only
    const double keep_old = a.should_zero ? 0.0 : 1.0;                       // SCAN only
    // swizzled byte offset of row `lane` in a TOD tile; sample k is at row_swz ^ (8 k)
    const unsigned row_swz = (unsigned)lane * 128u + (((unsigned)lane & 7u) << 4);

    // Lane 0 fetches the NEXT item id and its chunk descriptor one item ahead (issued at
    // an item switch, consumed at the next one), so neither latency is on the critical path.
    int64_t pend_item = -1, pend_first = 0;
    int pend_count = 0;
    auto prefetch_item = [&]() {
        if (lane == 0) {
            const unsigned long long it = atomicAdd(sched, 1ull);
            pend_item = it < (unsigned long long)n_items ? (int64_t)it : -1;
            if (pend_item >= 0) {
                const Chunk ch = chunks[pend_item / n_groups];
                pend_first = ch.first;
                pend_count = ch.count;
            }
        }
    };
    auto take_item = [&]() -> Blk {
        Blk bk;
        bk.item = __shfl_sync(0xffffffffu, pend_item, 0);
        const int64_t first = __shfl_sync(0xffffffffu, pend_first, 0);
        const int count = __shfl_sync(0xffffffffu, pend_count, 0);
        if (bk.item < 0) {
            bk.d0 = bk.s0 = bk.s_end = 0;
            bk.nb = bk.nrows = 0;
            return bk;
        }
        const int64_t c = bk.item / n_groups;
        bk.d0 = (bk.item - c * n_groups) * kRows;
        bk.nrows = (a.n_det - bk.d0) < kRows ? (int)(a.n_det - bk.d0) : kRows;
        bk.s0 = first;
        bk.s_end = first + count;
        bk.nb = count < kBlk ? count : kBlk;
        if (TMA) {
            // TMA boxes must start on 16-byte boundaries of every staged row (measured: an odd
            // f64 start faults), so boxes are aligned to 16 samples — the u8 flag rows need
            // that — and a chunk's first block processes box samples k0 .. 15 only
            bk.k0 = (int)(first & 15);
            bk.s0 = first - bk.k0;
            bk.nb = count < kBlk - bk.k0 ? count : kBlk - bk.k0;
        }
        return bk;
    };
    // Stage the raw inputs of block bk into buffer b.
    auto issue = [&](int b, const Blk& bk) {
        if constexpr (TMA) {
            if (lane == 0) {
                // the generic-proxy reads of buffer b (two blocks ago) are ordered before the
                // async-proxy writes that refill it
                asm volatile("fence.proxy.async.shared::cta;\n" ::: "memory");
                mbar_expect_tx(&tw.sf[b].mbar, tx_bytes);
                const uint64_t pol = evict_first_policy();
                const int s0 = (int)bk.s0, d0 = (int)bk.d0;
                tma_2d_stream(&tw.tod[b][0][0], &tm.tod, s0, d0, &tw.sf[b].mbar, pol);
                if (have_dflags) tma_2d_stream(&tw.flg[b][0][0], &tm.flg, s0, d0, &tw.sf[b].mbar, pol);
                tma_2d(&tw.bore[b][0][0], &tm.bore, 0, s0, &tw.sf[b].mbar);
                if (HWP && NNZ == 3) tma_1d(&tw.hwp[b][0], &tm.hwp, s0, &tw.sf[b].mbar);
                if (have_sflags) tma_1d(&tw.sf[b].f[0], &tm.sflg, s0, &tw.sf[b].mbar);
            }
        } else {
            issue_block<DPL>(sm.buf[b], bk, a, have_dflags, HWP && NNZ == 3, lane);
        }
    };

    if constexpr (TMA) {
        if (lane == 0) {
            mbar_init(&tw.sf[0].mbar);
            mbar_init(&tw.sf[1].mbar);
            asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
        }
        __syncwarp();
    }
    prefetch_item();
    Blk cur = take_item();
    // every thread reaches the shared-hits flush below (a warp without work skips the stream)
    if (cur.item >= 0) [&] {
        prefetch_item();
        issue(0, cur);
        Slot<P> sl[DPL];
#pragma unroll
        for (int j = 0; j < DPL; ++j) load_slot<P>(sl[j], a, cur.d0 + lane + 32 * j, lane + 32 * j < cur.nrows, cur.d0);
        int p = 0;

        while (true) {
            // successor block: next 16 samples of this item, or the first block of the next item
            Blk nxt;
            if (cur.s0 + kBlk < cur.s_end) {
                nxt = cur;
                nxt.s0 = cur.s0 + kBlk;
                nxt.k0 = 0;
                nxt.nb = (nxt.s_end - nxt.s0) < kBlk ? (int)(nxt.s_end - nxt.s0) : kBlk;
            } else {
                nxt = take_item();
                if (nxt.item >= 0) prefetch_item();
            }
            if constexpr (TMA) {
                mbar_wait(&tw.sf[p].mbar, (phase >> p) & 1u);
                phase ^= 1u << p;
            } else {
                cp_async_wait_all();
                __syncwarp();
            }
            if (nxt.item >= 0) issue(p ^ 1, nxt);
            __syncwarp();  // reconverge after the lane-0 / spin-wait paths (else the state code below runs twice)

            RawBlock<DPL>& rb = sm.buf[p];
            // Per-sample state, split over the warp: lanes 0..kBlk-1 build the boresight rotation
            // matrix of sample `lane` (identity if shared-flagged, S2), lanes 16..16+kBlk-1 the HWP
            // cos/sin(4 chi) of sample `lane - 16`.  Bit k of pmask = sample k is pixelised.
            double* st_base = TMA ? &tw.st[0][0] : &sm.st[0].v[0];
            bool pixelise_me = false;
            {
                const int ks = lane & 15;
                const bool in_blk = ks < kBlk && ks >= cur.k0 && ks < cur.k0 + cur.nb;
                if (lane < kBlk) {
                    double q0 = 0.0, q1 = 0.0, q2 = 0.0, q3 = 1.0;
                    if (in_blk) {
                        bool flagged;
                        if constexpr (TMA) {
                            flagged = have_sflags && (tw.sf[p].f[lane] & smask);
                        } else {
                            const int soff =
                                have_sflags ? (int)(reinterpret_cast<uintptr_t>(a.shared_flags + cur.s0) & 3) : 0;
                            flagged = have_sflags && (rb.sflg[soff + lane] & smask);
                        }
                        pixelise_me = !flagged;
                        const double* bq = TMA ? tw.bore[p][lane] : rb.bore[lane];
                        if (!flagged) {
                            q0 = bq[0]; q1 = bq[1]; q2 = bq[2]; q3 = bq[3];
                        }
                    }
                    double m[10];
                    quat_to_matrix(q0, q1, q2, q3, m);
                    m[9] = 1.0;
                    double2* dst = reinterpret_cast<double2*>(st_base + 12 * lane);
#pragma unroll
                    for (int i = 0; i < 4; ++i) dst[i] = make_double2(m[2 * i], m[2 * i + 1]);
                    st_base[12 * lane + 8] = m[8];
                } else if (HWP && NNZ == 3 && ks < kBlk) {
                    double c4 = 1.0, s4 = 0.0;
                    if (in_blk) small_sincos(4.0 * (TMA ? tw.hwp[p][ks] : rb.hwp[ks]), &s4, &c4);
                    st_base[12 * ks + 9] = c4;
                    st_base[12 * ks + 10] = s4;
                }
            }
            const unsigned pmask = __ballot_sync(0xffffffffu, pixelise_me);
            const unsigned keep = ((1u << cur.nb) - 1u) << cur.k0;  // samples of the block processed (nb <= 16)
            // The staged TOD of det-flagged samples (and, with debug outputs, of shared-flagged
            // samples, which run through det_sample without a pixel) is zeroed in shared memory, so
            // the per-sample loop needs no flag test: those samples add exactly 0 to the map.
#pragma unroll
            for (int j = 0; j < DPL; ++j) {
                const int row = lane + 32 * j;
                unsigned zm = DEBUG ? (~pmask & keep) : 0u;
                if (have_dflags && row < cur.nrows) {
                    const unsigned rep = dmask * 0x01010101u;
                    unsigned bits = 0u;  // bit k: sample k of the box is det-flagged
                    if constexpr (TMA) {
                        const uint4 f = *reinterpret_cast<const uint4*>(tw.flg[p][row]);
                        const unsigned fw[4] = {f.x, f.y, f.z, f.w};
#pragma unroll
                        for (int w = 0; w < 4; ++w) {
                            const unsigned v = __vcmpne4(fw[w] & rep, 0u);
                            bits |= ((v & 0x01010101u) * 0x01020408u >> 24 & 0xfu) << (4 * w);
                        }
                    } else {
                        const int foff =
                            (int)(reinterpret_cast<uintptr_t>(a.det_flags + (cur.d0 + row) * a.n_samp + cur.s0) & 3);
#pragma unroll
                        for (int w = 0; w < 5; ++w) {  // bit b: byte b of the 20-byte window is flagged
                            const unsigned v = __vcmpne4(*reinterpret_cast<const unsigned*>(&rb.flg[row][4 * w]) & rep, 0u);
                            bits |= ((v & 0x01010101u) * 0x01020408u >> 24 & 0xfu) << (4 * w);
                        }
                        bits >>= foff;
                    }
                    zm |= bits & keep;
                }
                while (zm) {
                    const int k = __ffs(zm) - 1;
                    zm &= zm - 1;
                    if constexpr (TMA)
                        *reinterpret_cast<double*>(reinterpret_cast<unsigned char*>(&tw.tod[p][0][0]) +
                                                   (row_swz ^ ((unsigned)k << 3))) = 0.0;
                    else
                        rb.tod[row][k] = 0.0;
                }
            }
            __syncwarp();

            // TMA tile: the tile is 1 KB-aligned and row r starts at r * 128, so the swizzled address
            // of (lane, k) is (tile + row_swz) ^ (8 k): one LOP3 per sample.
            const unsigned tod_row = smem_u32(&tw.tod[p][0][0]) + row_swz;
            // SCAN: the per-lane gather cache lives in the slot (run_key / run_loc: the cached
            // pixel's key and storage; r0..r2 its map values; pend_key: the block sample whose TOD
            // update waits for them, completed one sample later so the gather latency hides
            // behind that sample)
            auto store_tod = [&](int kk, double v) {
                if constexpr (TMA)
                    asm volatile("st.shared.f64 [%0], %1;" ::"r"(tod_row ^ ((unsigned)kk << 3)), "d"(v) : "memory");
                else
                    rb.tod[lane][kk] = v;
            };
            auto scan_finish = [&]() {
                if constexpr (SCAN) {
                    Slot<P>& s0 = sl[0];
                    if (s0.pend_key >= 0) {
                        double t = s0.r0 * a.cal;
                        if (NNZ == 3) t += s0.etacal * (s0.r1 * s0.p1 + s0.r2 * s0.p2);
                        store_tod((int)s0.pend_key, fma(sgn_ds, t, keep_old * s0.p0));
                        s0.pend_key = -1;
                    }
                }
            };
            auto scan_sample = [&](int kk, const double* x, double tod) {
                if constexpr (SCAN) {
                    Slot<P>& s0 = sl[0];
                    const StageA o = stage_a<NNZ, HWP, P>(s0, x);
                    const P key = stage_b<NEST, NNZ, WIDE>(o, true, s0.ok, g);
                    scan_finish();  // the previous sample's gathered values have arrived by now
                    const MapGeom& mg = a.map;
                    if (key >= 0 && key != s0.run_key) {
                        P pix;
                        if constexpr (WIDE)
                            pix = key;
                        else
                            pix = key_to_pix_tab<NEST>(key, g, cm.spread);
                        const int64_t smi = submap_of<P>(pix, mg);
                        if (smi != (int64_t)s0.last_sm) {
                            s0.last_loc = __ldg(&mg.global2local[smi]);
                            s0.last_sm = (P)smi;
                        }
                        s0.run_key = key;
                        s0.run_loc = s0.last_loc;
                        if (s0.run_loc >= 0) {
                            const int64_t lp = mg.sm_shift >= 0 ? (int64_t)(pix & (P)(mg.n_pix_submap - 1))
                                                                : (int64_t)pix - smi * mg.n_pix_submap;
                            const double* mp = a.mapdata + (s0.run_loc * mg.n_pix_submap + lp) * NNZ;
                            s0.r0 = __ldg(mp);
                            if (NNZ == 3) {
                                s0.r1 = __ldg(mp + 1);
                                s0.r2 = __ldg(mp + 2);
                            }
                        }
                    }
                    if (key >= 0 && s0.run_loc >= 0) {
                        s0.pend_key = (P)kk;
                        s0.p0 = tod;
                        s0.p1 = o.cw * o.invr;
                        s0.p2 = o.sw * o.invr;
                    }
                }
            };

            int k = cur.k0;
            const int k_end = cur.k0 + cur.nb;
            unsigned bit = 1u << k;  // 1 << k
#pragma unroll kKUnroll
            for (; k < k_end; ++k, bit <<= 1) {
                const bool pixelise = pmask & bit;
                if (!DEBUG && !pixelise) continue;  // shared-flagged sample: nothing to add (uniform)
                double x[12];
#pragma unroll
                for (int i = 0; i < ((HWP && NNZ == 3) ? 12 : 10); i += 2) {
                    const double2 t2 = *reinterpret_cast<const double2*>(st_base + 12 * k + i);
                    x[i] = t2.x;
                    x[i + 1] = t2.y;
                }
                double tod[DPL];
#pragma unroll
                for (int j = 0; j < DPL; ++j) {
                    if constexpr (TMA)
                        asm volatile("ld.shared.f64 %0, [%1];" : "=d"(tod[j]) : "r"(tod_row ^ ((unsigned)k << 3)));
                    else
                        tod[j] = rb.tod[lane + 32 * j][k];
                }
                if constexpr (SCAN) {
                    scan_sample(k, x, tod[0]);
                } else {
#if TB_DEFER
                    // fold the previous sample while those shared-memory loads are in flight
#pragma unroll
                    for (int j = 0; j < DPL; ++j) aggregate<NEST, NNZ, WIDE>(sl[j], a, g, cm);
#endif
#pragma unroll
                    for (int j = 0; j < DPL; ++j)
                        det_sample<NEST, NNZ, HWP, DEBUG, WIDE>(sl[j], x, pixelise, tod[j], g, a,
                                                                cur.d0 + lane + 32 * j, cur.s0 + k);
#if !TB_DEFER
                    // fold this sample at once: no pending contribution is carried across iterations
#pragma unroll
                    for (int j = 0; j < DPL; ++j) aggregate<NEST, NNZ, WIDE>(sl[j], a, g, cm);
#endif
                }
            }
            if constexpr (SCAN) {
                scan_finish();
                __syncwarp();
                // write back the processed columns of the tile (two rows per warp instruction,
                // coalesced along samples); unprocessed samples in them keep the value read
                const int scol = lane & 15, srow = lane >> 4;
                if (scol >= cur.k0 && scol < cur.k0 + cur.nb) {
                    double* dst = a.tod_out + (cur.d0 + srow) * a.n_samp + cur.s0 + scol;
                    for (int r = srow; r < cur.nrows; r += 2, dst += 2 * a.n_samp) {
                        double v;
                        if constexpr (TMA)
                            asm volatile("ld.shared.f64 %0, [%1];"
                                         : "=d"(v)
                                         : "r"(smem_u32(&tw.tod[p][0][0]) + (unsigned)r * 128u +
                                               (((unsigned)scol << 3) ^ (((unsigned)r & 7u) << 4))));
                        else
                            v = rb.tod[r][scol];
                        *dst = v;
                    }
                }
            }

            if (nxt.item != cur.item) {
#pragma unroll
                for (int j = 0; j < DPL; ++j) {
                    if constexpr (!SCAN) {
                        if (TB_DEFER) aggregate<NEST, NNZ, WIDE>(sl[j], a, g, cm);
                        flush<NNZ, WIDE>(sl[j], a);
                    }
                }
                if (nxt.item < 0) break;
#pragma unroll
                for (int j = 0; j < DPL; ++j)
                    load_slot<P>(sl[j], a, nxt.d0 + lane + 32 * j, lane + 32 * j < nxt.nrows, nxt.d0);
            }
            __syncwarp();  // all lanes are done with buffer p and st before they are refilled
            cur = nxt;
            p ^= 1;
        }
        if constexpr (!TMA) cp_async_wait_all();
    }();
    if (shared_hits) {  // the CTA's hit flags, once: a few hundred stores instead of one per run
        __syncthreads();
        for (int i = threadIdx.x; i < (int)a.map.n_submap; i += blockDim.x)
            if (s_hits[i]) a.hit_submaps[i] = 1;
    }
}

// Tensor-map encoder from the driver, fetched through the runtime (no link against libcuda).
PFN_cuTensorMapEncodeTiled_v12000 tensor_map_encoder() {
    static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
    static std::once_flag once;
    std::call_once(once, [] {
        void* ptr = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &ptr, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(ptr);
    });
    return fn;
}

bool encode_map(CUtensorMap* m, CUtensorMapDataType type, cuuint32_t rank, const void* base, const cuuint64_t* dims,
                const cuuint64_t* strides, const cuuint32_t* box, CUtensorMapSwizzle swz) {
    const cuuint32_t es[2] = {1, 1};
    return tensor_map_encoder()(m, type, rank, const_cast<void*>(base), dims, strides, box, es,
                                CU_TENSOR_MAP_INTERLEAVE_NONE, swz, CU_TENSOR_MAP_L2_PROMOTION_NONE,
                                CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

bool aligned16(const void* p) { return (reinterpret_cast<uintptr_t>(p) & 15) == 0; }

const cuuint64_t kNoStrides[1] = {0};  // rank-1 maps have no strides (a non-null array is passed anyway)

// The TMA path applies when every staged array is 16-byte aligned, rows of the TOD and the
// det flags are multiples of 16 bytes (n_samp % 16 == 0) and sample / detector coordinates
// fit the 32-bit TMA coordinates; otherwise the cp.async path runs (same results).
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
    if (a.n_samp % 16 != 0 || a.n_samp >= (int64_t(1) << 31) || a.n_det >= (int64_t(1) << 31)) {
        t_fused_path = "cp.async (n_samp % 16 != 0 or sizes beyond 32-bit TMA coordinates)";
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

template <bool NEST, int NNZ, bool HWP, bool DEBUG, bool WIDE, int DPL, bool TMA, bool SCAN = false>
cudaError_t launch_k(const WorkList& wl, const FusedArgs& a, const TmaMaps& tm, unsigned long long* sched,
                     cudaStream_t st) {
    auto kern = pointing_to_map_kernel<NEST, NNZ, HWP, DEBUG, WIDE, DPL, TMA, SCAN>;
    const size_t smem =
        (TMA ? sizeof(TmaWarpSmem) * kWarps + 1024 : sizeof(WarpSmem<DPL>) * kWarps) + kSpreadBytes + kSharedHitBytes;
    static int blocks_per_sm = 0;
    static std::once_flag once;
    std::call_once(once, [&] {
        cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&blocks_per_sm, kern, kWarps * 32, smem) != cudaSuccess ||
            blocks_per_sm < 1)
            blocks_per_sm = 1;
    });
    const int64_t n_items = wl.n_chunks * ((a.n_det + 32 * DPL - 1) / (32 * DPL));
    const int64_t want = (n_items + kWarps - 1) / kWarps;
    const int64_t grid = std::min<int64_t>(want, (int64_t)num_sms() * blocks_per_sm);
    if (grid <= 0) return cudaSuccess;
    cudaError_t e = cudaMemsetAsync(sched, 0, sizeof(unsigned long long), st);
    if (e != cudaSuccess) return e;
    kern<<<(unsigned)grid, kWarps * 32, smem, st>>>(wl.chunks, wl.n_chunks, a, make_geom(a.nside), sched, tm);
    return cudaGetLastError();
}

template <bool NEST, int NNZ, bool HWP, bool DEBUG, bool WIDE, int DPL, bool SCAN = false>
cudaError_t launch_t(const WorkList& wl, const FusedArgs& a, unsigned long long* sched, cudaStream_t st) {
    TmaMaps tm;
    if constexpr (kBlk == 16) {
        if (DPL == 1 && make_tma_maps(a, &tm)) {
            t_fused_path = "tma";
            return launch_k<NEST, NNZ, HWP, DEBUG, WIDE, 1, true, SCAN>(wl, a, tm, sched, st);
        }
    } else {
        t_fused_path = "cp.async (8-sample blocks)";
    }
    std::memset(&tm, 0, sizeof(tm));
    return launch_k<NEST, NNZ, HWP, DEBUG, WIDE, DPL, false, SCAN>(wl, a, tm, sched, st);
}

template <bool NEST, int NNZ, bool HWP, bool DEBUG>
cudaError_t dispatch_shape(const WorkList& wl, const FusedArgs& a, unsigned long long* sched, cudaStream_t st) {
    const bool wide = a.nside > 8192;
    const bool two = TB_FUSED_DPL_MAX > 1 && a.n_det > 32;
    if (wide) return two ? launch_t<NEST, NNZ, HWP, DEBUG, true, TB_FUSED_DPL_MAX>(wl, a, sched, st)
                         : launch_t<NEST, NNZ, HWP, DEBUG, true, 1>(wl, a, sched, st);
    return two ? launch_t<NEST, NNZ, HWP, DEBUG, false, TB_FUSED_DPL_MAX>(wl, a, sched, st)
               : launch_t<NEST, NNZ, HWP, DEBUG, false, 1>(wl, a, sched, st);
}

// ============================================================================ few detectors
// With fewer than kThinMaxDet detectors a 32-lane detector group leaves most lanes idle (C1: 4
// detectors, 4 of 32 lanes).  Then THREAD = (chunk, detector): each thread builds its own
// per-sample state from the boresight (consecutive threads share a chunk, so those loads are
// L1 broadcasts) and runs the same per-det-sample arithmetic, run aggregation and flush as the
// warp-per-item kernel (stage_a / stage_b / aggregate / flush), with the CTA's hit flags in
// shared memory.
constexpr int kThinMaxDet = 8;

template <bool NEST, int NNZ, bool HWP, bool WIDE>
__global__ void __launch_bounds__(256) pointing_to_map_thin_kernel(const Chunk* __restrict__ chunks, int64_t n_chunks,
                                                                  FusedArgs a, HealpixGeom g) {
    using P = typename PixT<WIDE>::T;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    uint16_t* s_spread = reinterpret_cast<uint16_t*>(smem_raw);
    uint8_t* s_hits = smem_raw + kSpreadBytes;
    const CtaMem cm{s_spread, s_hits};
    for (int i = threadIdx.x; i < 256; i += blockDim.x) {
        unsigned v = 0u;
        for (int b = 0; b < 8; ++b) v |= ((i >> b) & 1u) << (2 * b);
        s_spread[i] = (uint16_t)v;
    }
    if (a.map.shared_hits)
        for (int i = threadIdx.x; i < (int)a.map.n_submap; i += blockDim.x) s_hits[i] = 0;
    __syncthreads();
    const int64_t n_items = n_chunks * a.n_det;
    for (int64_t it = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; it < n_items;
         it += (int64_t)gridDim.x * blockDim.x) {
        const int64_t c = it / a.n_det, d = it - c * a.n_det;
        const Chunk ch = chunks[c];
        Slot<P> sl;
        load_slot<P>(sl, a, d, true, d);
        for (int64_t s = ch.first; s < ch.first + ch.count; ++s) {
            if (a.shared_flags && (__ldg(&a.shared_flags[s]) & a.shared_flag_mask)) continue;  // no pixel (S2)
            const double2 q01 = __ldg(reinterpret_cast<const double2*>(a.boresight + 4 * s));
            const double2 q23 = __ldg(reinterpret_cast<const double2*>(a.boresight + 4 * s) + 1);
            double x[12];
            quat_to_matrix(q01.x, q01.y, q23.x, q23.y, x);
            if (HWP && NNZ == 3) small_sincos(4.0 * __ldg(&a.hwp[s]), &x[10], &x[9]);
            double tod = __ldg(&a.det_data[d * a.n_samp + s]);
            if (a.det_flags && (__ldg(&a.det_flags[d * a.n_samp + s]) & a.det_flag_mask)) tod = 0.0;
            aggregate<NEST, NNZ, WIDE>(sl, a, g, cm);
            det_sample<NEST, NNZ, HWP, false, WIDE>(sl, x, true, tod, g, a, d, s);
        }
        aggregate<NEST, NNZ, WIDE>(sl, a, g, cm);
        flush<NNZ, WIDE>(sl, a);
    }
    if (a.map.shared_hits) {
        __syncthreads();
        for (int i = threadIdx.x; i < (int)a.map.n_submap; i += blockDim.x)
            if (s_hits[i]) a.hit_submaps[i] = 1;
    }
}

template <bool NEST, int NNZ, bool HWP>
cudaError_t launch_thin(const WorkList& wl, const FusedArgs& a, cudaStream_t st) {
    const size_t smem = kSpreadBytes + kSharedHitBytes;
    const int64_t items = wl.n_chunks * a.n_det;
    const int64_t grid = std::min<int64_t>((items + 255) / 256, (int64_t)num_sms() * 8);
    t_fused_path = "thin (thread per chunk x detector, few detectors)";
    if (a.nside > 8192)
        pointing_to_map_thin_kernel<NEST, NNZ, HWP, true><<<(unsigned)grid, 256, smem, st>>>(wl.chunks, wl.n_chunks, a,
                                                                                              make_geom(a.nside));
    else
        pointing_to_map_thin_kernel<NEST, NNZ, HWP, false><<<(unsigned)grid, 256, smem, st>>>(wl.chunks, wl.n_chunks, a,
                                                                                               make_geom(a.nside));
    return cudaGetLastError();
}

template <bool NEST, int NNZ, bool HWP>
cudaError_t dispatch_debug(const WorkList& wl, const FusedArgs& a, unsigned long long* sched, cudaStream_t st) {
    if (a.pixels_out || a.weights_out) return dispatch_shape<NEST, NNZ, HWP, true>(wl, a, sched, st);
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
    const bool wide = a.nside > 8192;
    const bool hwp = a.hwp && NNZ == 3;
    if (wide) return hwp ? launch_t<NEST, NNZ, true, false, true, 1, true>(wl, a, sched, st)
                         : launch_t<NEST, NNZ, false, false, true, 1, true>(wl, a, sched, st);
    return hwp ? launch_t<NEST, NNZ, true, false, false, 1, true>(wl, a, sched, st)
               : launch_t<NEST, NNZ, false, false, false, 1, true>(wl, a, sched, st);
}

}  // namespace

cudaError_t launch_pointing_to_tod(const WorkList& wl, const FusedArgs& a, unsigned long long* sched,
                                   cudaStream_t st) {
    if (wl.n_chunks == 0 || a.n_det == 0) return cudaSuccess;
    if (a.nest) return a.nnz == 3 ? dispatch_scan<true, 3>(wl, a, sched, st) : dispatch_scan<true, 1>(wl, a, sched, st);
    return a.nnz == 3 ? dispatch_scan<false, 3>(wl, a, sched, st) : dispatch_scan<false, 1>(wl, a, sched, st);
}

const char* last_fused_path() { return t_fused_path; }

// Launch-side map geometry of the fused kernel: the submap count and whether the hit flags
// are gathered in shared memory.
FusedArgs with_map_geom(FusedArgs a) {
    MapGeom& m = a.map;
    m.n_submap = (12 * a.nside * a.nside + m.n_pix_submap - 1) / m.n_pix_submap;
    m.shared_hits = a.hit_submaps != nullptr && m.n_submap <= kSharedHitBytes;
    return a;
}

cudaError_t launch_pointing_to_map(const WorkList& wl, const FusedArgs& a_in, unsigned long long* sched,
                                   cudaStream_t st) {
    const FusedArgs a = with_map_geom(a_in);
    if (wl.n_chunks == 0 || a.n_det == 0) return cudaSuccess;
    if (a.nest) return a.nnz == 3 ? dispatch_hwp<true, 3>(wl, a, sched, st) : dispatch_hwp<true, 1>(wl, a, sched, st);
    return a.nnz == 3 ? dispatch_hwp<false, 3>(wl, a, sched, st) : dispatch_hwp<false, 1>(wl, a, sched, st);
}

}  // namespace toastb200

// phi.cuh -- fp32 device evaluation of one dimension of eq. (13) and of the
// bandwidth-gradient factor of eq. (17) for one (point, box) pair.
//
// eq. (13):  D_j = 1/2 [erf(z_u) - erf(z_l)],  z_b = (b_j - t_j) / (sqrt2 h_j)
// eq. (17):  d D_j / d h_j = (z_l e^{-z_l^2} - z_u e^{-z_u^2}) / (sqrt(pi) h_j)
//
// erf is evaluated through erfc with the exponential factored out,
//     1/2 erf(|z|) = 1/2 - 1/2 erfc(|z|),   erfc(x) ~= e^{-x^2} Q(t),  t = 1/(1 + P x),
// with Q a degree-6 polynomial fitted by tools/fit_phi.py (phi_coeffs.h: relative
// error < 7.7e-7 in fp32 on [0, 4.5], absolute error < 1e-15 beyond).
// e^{-z^2} is ONE MUFU.EX2 per bound and is shared with the gradient; the two
// reciprocals of a dimension share ONE MUFU.RCP, so a dimension costs 3 MUFU
// plus ~12 packed FP32 instructions.  The (u, l) pair of a dimension is
// processed as one float2 with the sm_100 packed FP32 instructions
// (FADD2/FMUL2/FFMA2), halving issue slots.
//
// Scaling: the kernels carry y' = z sqrt(log2 e) = (b - t) * ap, so that
// E = e^{-z^2} = 2^{-y'^2} is a bare ex2.approx; x = |z| = |y'| / sqrt(log2 e)
// is folded into the constant P' = P / sqrt(log2 e).
// Infinite / far bounds: make_boxdim clamps every bound to the sample's
// column range widened by 14/ap, so y' stays finite (no inf * 0 in y' E) while
// |y'| >= 14 still gives E = 0 and erf = +-1 exactly: results are unchanged.
#pragma once
#include <cuda_runtime.h>
#include "common.cuh"
#include "phi_coeffs.h"

namespace kde {

constexpr float kSqrtLog2e = 1.2011224087864498f;  // sqrt(log2(e))
constexpr float kPprime = KDE_PHI_P / kSqrtLog2e;


__device__ __forceinline__ float ex2_approx(float x) {
  float y;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}
__device__ __forceinline__ float rcp_approx(float x) {
  float y;
  asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}
__device__ __forceinline__ float2 f2(float a) { return make_float2(a, a); }

// ---------------------------------------------------------------------------
// Per (box, dimension) evaluation setup, computed once per box.
//   normal: b = (u, l), hd = 0           y = (b - t) * ap
//   narrow: b = (l, l), hd = delta'/2    y = (l - t) * ap + hd (1 +- 1/sqrt3)
// A dimension is "narrow" when its width in erf units dz = (u - l)/(sqrt2 h)
// is below kNarrowZ: there the difference of two erf values (and of the two
// gradient terms) cancels catastrophically in fp32, so the interval integral
// of eq. (12) and the gradient integral are taken with 2-point Gauss-Legendre
// on the same two exponentials (relative error < dz^4 / 360 (1 + z^4)).
constexpr float kNarrowZ = 0.05f;
constexpr float kNarrowY = kNarrowZ * kSqrtLog2e;          // threshold in y' units
constexpr float kGaussC = 0.57735026918962576f;            // 1/sqrt(3)
constexpr float kInvSqrtPiLog2e = 0.46971863934982566f;    // 1/(sqrt(pi) sqrt(log2 e))
constexpr float kTwoLn2 = 1.3862943611198906f;

struct BoxDim {
  float2 b;   // (b1, b2) evaluation bounds
  float hd;   // half-width in y' units for narrow dims, 0 otherwise
};

constexpr float kBoundMargin = 14.0f;  // |y'| >= 14: 2^-196 flushes to 0, erf(z) == +-1 in fp32

template <int KT = kGaussian>
__device__ __forceinline__ BoxDim make_boxdim(float l, float u, float ap, unsigned rmin_enc, unsigned rmax_enc) {
  BoxDim r;
  const float tmin = fdec_range(rmin_enc), tmax = fdec_range(rmax_enc);
  if (KT == kEpanechnikov) {  // v = (b - t)/h; support |v| < 1: clamp the bounds to the range widened by 2h
    const float m = 2.0f / ap;
    l = fminf(fmaxf(l, tmin - m), tmax + m);
    u = fminf(fmaxf(u, tmin - m), tmax + m);
    r.b = make_float2(u, l);
    r.hd = (u - l) * ap;  // Delta of the unclamped case, formed without cancellation
    return r;
  }
  const float dy = (u - l) * ap;  // inf for unbounded, NaN for (inf, inf): both normal
  const float m = kBoundMargin / ap;
  l = fminf(fmaxf(l, tmin - m), tmax + m);
  u = fminf(fmaxf(u, tmin - m), tmax + m);
  if (dy > 0.0f && dy < kNarrowY) {
    r.b = make_float2(l, l);
    r.hd = 0.5f * dy;
  } else if (!(dy > 0.0f)) {
    // l == u (or an empty (inf, inf) / (-inf, -inf) box): D = 0 and dD/dh = 0 exactly.  Both bounds
    // go above the range so y' >= 14 for every point (E = 0, same signs), instead of relying on
    // the fused bracket cancelling two equal rounded products.
    r.b = make_float2(tmax + m, tmax + m);
    r.hd = 0.0f;
  } else {
    r.b = make_float2(u, l);
    r.hd = 0.0f;
  }
  return r;
}

// Tail culling (reading R15, scan_single_tma.cuh): the box of make_boxdim (bounds clamped to the
// column range widened by 14/ap) in scaled coordinates, (c ap, hw ap + margin), c / hw its centre /
// half-width.  A point's distance outside the box in dimension j is then bounded from below by
// max(|t ap - c ap| - hw', 0) as evaluated in fp32 (FFMA2 + FADD2): the margin covers the rounding of
// c ap and of the FFMA, |fl(t ap - fl(c ap)) - (t - c) ap| <= 2^-23 (|c ap| + max|t| ap).  An empty
// dimension (l == u, D = 0) becomes a point far above the range, so every point is culled.
__device__ __forceinline__ float2 make_cullbox(float l, float u, float ap, unsigned rmin_enc, unsigned rmax_enc) {
  const float tmin = fdec_range(rmin_enc), tmax = fdec_range(rmax_enc);
  const float m = kBoundMargin / ap;
  const bool nonempty = (u - l) * ap > 0.0f;
  l = fminf(fmaxf(l, tmin - m), tmax + m);
  u = fminf(fmaxf(u, tmin - m), tmax + m);
  const double c = nonempty ? 0.5 * ((double)u + (double)l) : (double)(tmax + m);
  const double hw = nonempty ? 0.5 * ((double)u - (double)l) : 0.0;
  const double cap = c * ap, hwap = hw * ap;
  const double tabs = fmax(fabs((double)tmin), fabs((double)tmax)) * ap;
  const double err = ldexp(2.0 * fabs(cap) + hwap + tabs, -22) + 1e-30;
  return make_float2((float)cap, (float)(hwap + err));
}
// culling is only sound when the scaled box is representable in fp32 (|c ap|, hw' < 2^127): with
// extreme bandwidths and offsets (e.g. h = 1e-30, |t| = 1e9) the caller disables it for that box
__device__ __forceinline__ bool cullbox_ok(float2 cb) { return fabsf(cb.x) < 1.0e38f && cb.y < 1.0e38f; }
constexpr float kCullY2 = 64.5f;  // cull when sum_j o_j^2 >= 64 (+ slack for the fp32 rounding of the sum)

// Cull score of two points (float2 lanes = points), with o_j = max(|t ap - c ap| - hw', 0):
//   Gaussian:      4 sum_j o_j^2 (y' units), culled when >= 4 kCullY2 (reading R15);
//   Epanechnikov:  max_j o_j (units of h), culled when >= 1: the point is outside the kernel's
//                  support in some dimension, so its contribution and gradient are exactly 0.
template <int D, bool EPAN>
__device__ __forceinline__ float2 cull_score(const float2 (&t)[D], const float (&ap)[D], const float2 (&cb)[D]) {
  float2 o2 = f2(0.0f);
#pragma unroll
  for (int j = 0; j < D; ++j) {
    const float2 y = __ffma2_rn(t[j], f2(ap[j]), f2(-cb[j].x));
    const float2 e = __fadd2_rn(make_float2(fabsf(y.x), fabsf(y.y)), f2(-cb[j].y));
    if (EPAN) {
      o2 = make_float2(fmaxf(o2.x, e.x), fmaxf(o2.y, e.y));
    } else {  // r = e + |e| = 2 max(e, 0) exactly (one packed op instead of two FMNMX): the sum is 4 sum_j o_j^2
      const float2 r = __fadd2_rn(e, make_float2(fabsf(e.x), fabsf(e.y)));
      o2 = __ffma2_rn(r, r, o2);
    }
  }
  return o2;
}
template <bool EPAN>
__host__ __device__ constexpr float cull_limit() { return EPAN ? 1.0f : 4.0f * kCullY2; }

// erf-difference path: D = 1/2 [erf(z_u) - erf(z_l)], w = y'_l E_l - y'_u E_u.
// One MUFU.RCP serves the pair: t_u = den_l / (den_u den_l), t_l = den_u / (den_u den_l)
// (den = 1 + P'|y'| with |y'| bounded by the clamped bounds: the product stays finite for any
// sample whose column range is below ~1e18 bandwidths).
template <bool GRAD>
__device__ __forceinline__ float phi_normal(const float2 y, const float2 E, float& w) {
  const float2 den = __ffma2_rn(make_float2(fabsf(y.x), fabsf(y.y)), f2(kPprime), f2(1.0f));  // |.| is an operand modifier
  const float r = rcp_approx(den.x * den.y);
  const float2 t2 = __fmul2_rn(make_float2(den.y, den.x), f2(r));
  // Horner for Q(t)/2 (the 1/2 of eq. 13 folded into the coefficients)
  float2 q = f2(0.5f * kde_phi_q(KDE_PHI_DEG));
#pragma unroll
  for (int k = KDE_PHI_DEG - 1; k >= 0; --k) q = __ffma2_rn(q, t2, f2(0.5f * kde_phi_q(k)));
  if (GRAD) w = fmaf(y.y, E.y, -(y.x * E.x));  // FMUL + FFMA
  // 1/2 erf(z) = sgn(z) (1/2 - ch), ch = 1/2 erfc(|z|) = E q.  D = [1/2 sgn(z_u) - 1/2 sgn(z_l)] +
  // [sgn(z_l) ch_l - sgn(z_u) ch_u]: the first bracket is exactly 0 or 1, so a box seen from one side
  // keeps the full relative accuracy of the erfc tails.  It is 1 iff z_l < 0 <= z_u (z_u >= z_l
  // always) and is built from the sign bits on the integer (ALU) pipe; the signs of the second
  // bracket ride on E (copysign, ALU) and the bracket is two FFMAs with the first as addend.
  const unsigned lneg_upos = __float_as_uint(y.y) & ~__float_as_uint(y.x);
  const float hs = __uint_as_float((unsigned)((int)lneg_upos >> 31) & 0x3f800000u);
  return fmaf(q.y, copysignf(E.y, y.y), fmaf(-q.x, copysignf(E.x, y.x), hs));
}

// narrow path: 2-point Gauss-Legendre on [y_l, y_u] (nodes y.x, y.y, weights hd)
template <bool GRAD>
__device__ __forceinline__ float phi_narrow(const float2 y, const float2 E, float hd, float& w) {
  const float s = E.x + E.y;
  if (GRAD) {
    const float2 yy = __fmul2_rn(y, y);
    w = -hd * (s - kTwoLn2 * fmaf(E.x, yy.x, E.y * yy.y));
  }
  return hd * kInvSqrtPiLog2e * s;
}

// Epanechnikov product kernel (reading R14), one dimension for one point:
//   v = (b - t)/h clamped to [-1, 1] (a = v_u, b = v_l),  Delta = a - b,
//   S = a^2 + a b + b^2,  D = F(a) - F(b) = Delta (3 - S) / 4,
//   d D / d h = -(3 / (4h)) [g(a) - g(b)],  g(v) = v (1 - v^2),  g(a) - g(b) = Delta (1 - S),
// so both come from Delta and S without the cancellation of F(a) - F(b) for
// narrow boxes (Delta = (u - l)/h when neither bound is clamped).
template <bool GRAD>
__device__ __forceinline__ float phi_epan(const BoxDim& bd, float t, float ih, float& w) {
  const float2 v = __fmul2_rn(__fadd2_rn(bd.b, f2(-t)), f2(ih));
  const float a = fminf(fmaxf(v.x, -1.0f), 1.0f);
  const float b = fminf(fmaxf(v.y, -1.0f), 1.0f);
  // both bounds inside the support: the cancellation-free (u - l)/h; otherwise
  // a clamped value is involved and a - b is exact enough (0 when both clamp alike)
  const float dl = (v.x == a && v.y == b) ? bd.hd : a - b;
  const float S = fmaf(a, a + b, b * b);
  if (GRAD) w = fmaf(-S, dl, dl);
  return fmaf(S, -0.25f, 0.75f) * dl;
}

// One dimension of eq. (13) for one point and one box; GENERAL handles narrow
// dimensions (a per-box uniform property), the fast variant assumes none.
template <bool GRAD, bool GENERAL>
__device__ __forceinline__ float phi_diff(const BoxDim& bd, float t, float ap, float& w) {
  float2 y;
  if (GENERAL) {
    const float2 o = __fmul2_rn(f2(bd.hd), make_float2(1.0f + kGaussC, 1.0f - kGaussC));
    y = __ffma2_rn(__fadd2_rn(bd.b, f2(-t)), f2(ap), o);
  } else {
    y = __fmul2_rn(__fadd2_rn(bd.b, f2(-t)), f2(ap));
  }
  const float2 yy = __fmul2_rn(y, y);
  const float2 E = make_float2(ex2_approx(-yy.x), ex2_approx(-yy.y));
  if (GENERAL && bd.hd > 0.0f) return phi_narrow<GRAD>(y, E, bd.hd, w);
  return phi_normal<GRAD>(y, E, w);
}

// ---------------------------------------------------------------------------
// Two points (p0, p1) against one box dimension, the float2 lanes being the
// two POINTS: every FP32 step of phi_normal -- including the ones that are
// scalar per point there (the pair reciprocal's product, the bracket FFMAs,
// the gradient term, the product over dimensions) -- is one packed
// FADD2/FMUL2/FFMA2 for both points.  The kernels carry the negated
// coordinate  yn = (t - b) ap = -y'  (t first: FADD2 with a broadcast bound,
// no negation), so in yn terms
//   D = [1/2 sgn(yn_l) - 1/2 sgn(yn_u)] + [sgn(yn_u) ch_u - sgn(yn_l) ch_l],
//   w = y'_l E_l - y'_u E_u = yn_u E_u - yn_l E_l,
// and the 0/1 bracket is 1 iff yn_u < 0 <= yn_l (sign bits, ALU pipe).
__device__ __forceinline__ float2 ex2_2(const float2 yy) {
  return make_float2(ex2_approx(-yy.x), ex2_approx(-yy.y));
}
__device__ __forceinline__ float hs_bit(float yn_u, float yn_l) {
  const unsigned m = __float_as_uint(yn_u) & ~__float_as_uint(yn_l);
  return __uint_as_float((unsigned)((int)m >> 31) & 0x3f800000u);
}

template <bool GRAD>
__device__ __forceinline__ float2 phi_normal2(const float2 yu, const float2 yl, const float2 Eu, const float2 El,
                                              float2& w) {
  const float2 du = __ffma2_rn(make_float2(fabsf(yu.x), fabsf(yu.y)), f2(kPprime), f2(1.0f));
  const float2 dl = __ffma2_rn(make_float2(fabsf(yl.x), fabsf(yl.y)), f2(kPprime), f2(1.0f));
  const float2 pr = __fmul2_rn(du, dl);
  const float2 r = make_float2(rcp_approx(pr.x), rcp_approx(pr.y));  // one MUFU.RCP per point and dimension
  const float2 tu = __fmul2_rn(dl, r), tl = __fmul2_rn(du, r);
  float2 qu = f2(0.5f * kde_phi_q(KDE_PHI_DEG)), ql = qu;
#pragma unroll
  for (int k = KDE_PHI_DEG - 1; k >= 0; --k) {
    qu = __ffma2_rn(qu, tu, f2(0.5f * kde_phi_q(k)));
    ql = __ffma2_rn(ql, tl, f2(0.5f * kde_phi_q(k)));
  }
  if (GRAD) {
    const float2 m = __fmul2_rn(yl, El);
    w = __ffma2_rn(yu, Eu, make_float2(-m.x, -m.y));
  }
  const float2 hs = make_float2(hs_bit(yu.x, yl.x), hs_bit(yu.y, yl.y));
  const float2 Eus = make_float2(copysignf(Eu.x, yu.x), copysignf(Eu.y, yu.y));
  const float2 Els = make_float2(copysignf(El.x, yl.x), copysignf(El.y, yl.y));
  return __ffma2_rn(qu, Eus, __ffma2_rn(make_float2(-ql.x, -ql.y), Els, hs));
}

// narrow path for two points: nodes yn_1,2 = (t - l) ap - hd (1 +- 1/sqrt3) (weights hd)
template <bool GRAD>
__device__ __forceinline__ float2 phi_narrow2(const float2 y1, const float2 y2, const float2 E1, const float2 E2,
                                              float hd, float2& w) {
  const float2 s = __fadd2_rn(E1, E2);
  if (GRAD) {
    const float2 yy1 = __fmul2_rn(y1, y1), yy2 = __fmul2_rn(y2, y2);
    const float2 m = __ffma2_rn(E1, yy1, __fmul2_rn(E2, yy2));
    w = __fmul2_rn(f2(-hd), __ffma2_rn(f2(-kTwoLn2), m, s));
  }
  return __fmul2_rn(f2(hd * kInvSqrtPiLog2e), s);
}

// Epanechnikov (reading R14) for two points, float2 lanes = points.  In the
// negated coordinates a = (t - u)/h <= b = (t - l)/h (clamped to [-1, 1]) the
// formulas of phi_epan are unchanged: Delta = b - a, S = a^2 + a b + b^2,
// D = Delta (3 - S)/4, w = Delta (1 - S); Delta is the cancellation-free
// (u - l)/h (bd.hd) when neither bound is clamped.
template <bool GRAD>
__device__ __forceinline__ float2 phi_epan2(const BoxDim& bd, const float2 t, float ih, float2& w) {
  const float2 va = __fmul2_rn(__fadd2_rn(t, f2(-bd.b.x)), f2(ih));
  const float2 vb = __fmul2_rn(__fadd2_rn(t, f2(-bd.b.y)), f2(ih));
  const float2 a = make_float2(fminf(fmaxf(va.x, -1.0f), 1.0f), fminf(fmaxf(va.y, -1.0f), 1.0f));
  const float2 b = make_float2(fminf(fmaxf(vb.x, -1.0f), 1.0f), fminf(fmaxf(vb.y, -1.0f), 1.0f));
  const float2 dc = __fadd2_rn(b, make_float2(-a.x, -a.y));
  // both bounds inside the support (|a|, |b| <= 1, unclamped) -> the exact (u - l)/h
  const float2 dl = make_float2(fmaxf(fabsf(va.x), fabsf(vb.x)) <= 1.0f ? bd.hd : dc.x,
                                fmaxf(fabsf(va.y), fabsf(vb.y)) <= 1.0f ? bd.hd : dc.y);
  const float2 S = __ffma2_rn(a, __fadd2_rn(a, b), __fmul2_rn(b, b));
  if (GRAD) w = __ffma2_rn(make_float2(-S.x, -S.y), dl, dl);
  return __fmul2_rn(__ffma2_rn(S, f2(-0.25f), f2(0.75f)), dl);
}

template <bool GRAD, bool GENERAL>
__device__ __forceinline__ float2 phi_diff2(const BoxDim& bd, const float2 t, float ap, float2& w) {
  float2 yu, yl;
  if (GENERAL) {  // narrow boxes have b = (l, l); a normal box has hd = 0 and the offsets vanish
    const float2 tu = __fadd2_rn(t, f2(-bd.b.x)), tl = __fadd2_rn(t, f2(-bd.b.y));
    yu = __ffma2_rn(tu, f2(ap), f2(-bd.hd * (1.0f + kGaussC)));
    yl = __ffma2_rn(tl, f2(ap), f2(-bd.hd * (1.0f - kGaussC)));
  } else {
    yu = __fmul2_rn(__fadd2_rn(t, f2(-bd.b.x)), f2(ap));
    yl = __fmul2_rn(__fadd2_rn(t, f2(-bd.b.y)), f2(ap));
  }
  const float2 Eu = ex2_2(__fmul2_rn(yu, yu)), El = ex2_2(__fmul2_rn(yl, yl));
  if (GENERAL && bd.hd > 0.0f) return phi_narrow2<GRAD>(yu, yl, Eu, El, bd.hd, w);
  return phi_normal2<GRAD>(yu, yl, Eu, El, w);
}

}  // namespace kde

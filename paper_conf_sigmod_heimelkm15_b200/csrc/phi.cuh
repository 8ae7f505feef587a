// phi.cuh -- fp32 device evaluation of one dimension of eq. (13) and of the
// bandwidth-gradient factor of eq. (17) for one (point, box) pair.
//
// eq. (13):  D_j = 1/2 [erf(z_u) - erf(z_l)],  z_b = (b_j - t_j) / (sqrt2 h_j)
// eq. (17):  d D_j / d h_j = (z_l e^{-z_l^2} - z_u e^{-z_u^2}) / (sqrt(pi) h_j)
//
// erf is evaluated through erfc with the exponential factored out,
//     1/2 erf(|z|) = 1/2 - 1/2 erfc(|z|),   erfc(x) ~= e^{-x^2} t Q(t),  t = 1/(1 + P x),
// with Q fitted by tools/fit_phi.py (phi_coeffs.h, relative error < 6e-7 in
// fp32 over [0, inf)).  e^{-z^2} is ONE MUFU.EX2 per bound and is shared with
// the gradient, so a bound costs 2 MUFU (EX2, RCP) plus ~8 packed FFMA2.
// The (u, l) pair of a dimension is processed as one float2 with the
// sm_100 packed FP32 instructions (FADD2/FMUL2/FFMA2), halving issue slots.
//
// Scaling: the kernels carry y' = z sqrt(log2 e) = (b - t) * ap, so that
// E = e^{-z^2} = 2^{-y'^2} is a bare ex2.approx; x = |z| = |y'| / sqrt(log2 e)
// is folded into the constant P' = P / sqrt(log2 e).
// Infinite bounds: y' is clamped to +-13 (2^-169 flushes to 0), giving
// E = 0, erfc = 0, 1/2 erf = +-1/2 exactly and a zero gradient term.
#pragma once
#include <cuda_runtime.h>
#include "phi_coeffs.h"

namespace kde {

constexpr float kSqrtLog2e = 1.2011224087864498f;  // sqrt(log2(e))
constexpr float kYClamp = 13.0f;
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

// One dimension for one point and one box.
//   ul = (u_j, l_j), t = t_ij, ap = sqrt(log2 e)/(sqrt2 h_j)
// returns D_j; if GRAD, w = y'_l E_l - y'_u E_u  (so dD_j/dh_j = gconst_j * w).
template <bool GRAD>
__device__ __forceinline__ float phi_diff(float2 ul, float t, float ap, float& w) {
  float2 y = __fmul2_rn(__fadd2_rn(ul, f2(-t)), f2(ap));
  y.x = fminf(fmaxf(y.x, -kYClamp), kYClamp);
  y.y = fminf(fmaxf(y.y, -kYClamp), kYClamp);
  const float2 yy = __fmul2_rn(y, y);
  const float2 E = make_float2(ex2_approx(-yy.x), ex2_approx(-yy.y));
  const float2 den = __ffma2_rn(make_float2(fabsf(y.x), fabsf(y.y)), f2(kPprime), f2(1.0f));
  const float2 t2 = make_float2(rcp_approx(den.x), rcp_approx(den.y));
  // Horner for Q(t)/2 (the 1/2 of eq. 13 folded into the coefficients)
  float2 q = f2(0.5f * kde_phi_q(KDE_PHI_DEG));
#pragma unroll
  for (int k = KDE_PHI_DEG - 1; k >= 0; --k) q = __ffma2_rn(q, t2, f2(0.5f * kde_phi_q(k)));
  const float2 ch = __fmul2_rn(__fmul2_rn(q, t2), E);          // 1/2 erfc(|z|)
  const float2 g = __ffma2_rn(ch, f2(-1.0f), f2(0.5f));        // 1/2 erf(|z|)
  if (GRAD) {
    const float2 yE = __fmul2_rn(y, E);
    w = yE.y - yE.x;
  }
  return copysignf(g.x, y.x) - copysignf(g.y, y.y);
}

}  // namespace kde

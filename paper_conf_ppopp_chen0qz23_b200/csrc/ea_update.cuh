// The per-element arithmetic of the elastic-averaging step, shared by every
// kernel of the library (co-located, spread local, peer-memory exchange).
// Not part of the public ABI (include/ea.h).
//
// Per element j of a stage and replica i (§3.2; DESIGN.md c1-c14, c21, c29):
//   Step 1 (local update of the user-specified optimizer):
//     SGD-momentum: g' = g + wd*x; m = mu*m + g'; D = -lr*(nesterov ? g' + mu*m : m)
//     Adam(W):      g' = g (+ wd*x for Adam); m = b1*m + (1-b1)*g'; v = b2*v + (1-b2)*g'^2;
//                   D = -(lr/bc1) * m / (sqrt(v)/sqrt(bc2) + eps)  (- lr*wd*x for AdamW)
//     ASGD:         D = -eta_t (g + wd*x + l*x); ax <- mu_t == 1 ? x + D : ax + mu_t (x + D - ax)
//   Step 2: x_i = (1-alpha)*x_i + alpha*x~ + D_i          ((1-a):a dilution + local update)
//   Steps 3-4: r_i = rho*D_i + beta*(x_i - x~)            (send; the caller accumulates)
//   Step 5: x~ = x~ + R/N                                  (center_apply)
#pragma once

#include <cuda_runtime.h>

#include "ea_internal.h"

namespace ea {

// One (replica, element) update; returns the replica's contribution r_i.
// m: SGD momentum / Adam first moment / ASGD average; v: Adam second moment (SGD, ASGD: untouched).
// c: the center the replica sees (x~_t, or x~_{t-1} with a stale center, reading c28).
template <int OPT>
__device__ __forceinline__ float ea_elem(float& x, float g, float& m, float& v, float c, const Hyper& hp,
                                         const StepCoef& sc) {
  float delta;
  if constexpr (OPT == kOptSGD) {
    const float gg = fmaf(hp.wd, x, g);             // g + lambda*x
    const float mn = fmaf(hp.momentum, m, gg);      // mu*m + g'
    const float d = hp.nesterov ? fmaf(hp.momentum, mn, gg) : mn;
    delta = -hp.lr * d;                             // local update Delta_i (Step 1)
    m = mn;
  } else if constexpr (OPT == kOptASGD) {
    // torch.optim.ASGD (reading c29): x_local = x (1 - l eta_t) - eta_t g', so Delta = -eta_t (g' + l x);
    // the average tracks the optimizer's own iterate x + Delta (mu_t == 1: a copy, as torch does)
    const float gg = fmaf(hp.wd, x, g);
    delta = -sc.step_size * fmaf(hp.asgd_lambd, x, gg);
    const float xl = x + delta;
    m = sc.inv_sqrt_bc2 == 1.f ? xl : fmaf(sc.inv_sqrt_bc2, xl - m, m);
  } else {
    const float gg = OPT == kOptAdam ? fmaf(hp.wd, x, g) : g;
    const float mn = fmaf(hp.beta1, m, hp.one_minus_beta1 * gg);
    const float vn = fmaf(hp.beta2, v, hp.one_minus_beta2 * (gg * gg));
    const float denom = fmaf(sqrtf(vn), sc.inv_sqrt_bc2, hp.eps);
    delta = -sc.step_size * (mn / denom);
    if constexpr (OPT == kOptAdamW) delta = fmaf(-hp.lr_wd, x, delta);
    m = mn;
    v = vn;
  }
  const float gap = x - c;                          // x_i - x~ (pre-step values, c1/c2)
  const float r = fmaf(hp.beta, gap, hp.rho * delta);
  x = fmaf(-hp.alpha, gap, x) + delta;              // (1-a)x + a*x~ + Delta (Step 2)
  return r;
}

template <int OPT>
__device__ __forceinline__ float4 ea_vec(float4& x, float4 g, float4& m, float4& v, float4 c, const Hyper& hp,
                                         const StepCoef& sc) {
  float4 r;
  r.x = ea_elem<OPT>(x.x, g.x, m.x, v.x, c.x, hp, sc);
  r.y = ea_elem<OPT>(x.y, g.y, m.y, v.y, c.y, hp, sc);
  r.z = ea_elem<OPT>(x.z, g.z, m.z, v.z, c.z, hp, sc);
  r.w = ea_elem<OPT>(x.w, g.w, m.w, v.w, c.w, hp, sc);
  return r;
}

__device__ __forceinline__ void add4(float4& a, float4 b) {
  a.x += b.x; a.y += b.y; a.z += b.z; a.w += b.w;
}

// Step 5: x~ + R/N.
__device__ __forceinline__ float4 center_apply(float4 c, float4 acc, float inv_n) {
  return make_float4(fmaf(acc.x, inv_n, c.x), fmaf(acc.y, inv_n, c.y), fmaf(acc.z, inv_n, c.z),
                     fmaf(acc.w, inv_n, c.w));
}

template <int OPT>
__device__ __forceinline__ StepCoef load_coef(const StepCoef* scp) {
  if constexpr (OPT == kOptSGD) {
    return StepCoef{0.f, 0.f};
  } else {
    return *scp;
  }
}

}  // namespace ea

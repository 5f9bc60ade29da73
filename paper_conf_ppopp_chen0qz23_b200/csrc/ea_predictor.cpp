// Profiling-based tuning predictor (row f3; host only, no GPU needed).
//
// AvgPipe §5.2: from one profiled setting (m micro-batches, n
// pipelines) predict, for a candidate (m*, n*), every GPU's computation time
// (Eq. 2, with the utilisation curve clipped at 100%), blocking communication
// (Eq. 4), bubbles (Eqs. 5-7, recursions up and down the pipeline), total
// (Eq. 1) and memory (Eq. 8); then pick the feasible setting with the best
// prediction.  Readings c22-c26 in DESIGN.md: left Riemann sum for the
// integral, (TT^{k+-1})* = (n*/n) TT^{k+-1}, iteration time = max_k T^k,
// objective = throughput n*/T (ties: lower memory, then smaller n*, m*).
#include <stdint.h>

#include <algorithm>
#include <cmath>
#include <cstring>
#include <vector>

#include "../../include/ea.h"

namespace {

bool finite_nonneg(double v) { return std::isfinite(v) && v >= 0.0; }

// Validates a profile; returns EA_OK or EA_EINVAL.
ea_status check_profile(const ea_profile* p) {
  if (!p || p->n_gpus < 1 || p->m < 1 || p->n < 1 || p->n_samples < 0 || !p->t_gpu || !p->t_comm || !p->f_mod ||
      !p->f_dat || (p->n_samples > 0 && !p->phi) || !(p->dt >= 0.0) || !std::isfinite(p->dt))
    return EA_EINVAL;
  for (int k = 0; k < p->n_gpus; ++k) {
    if (!finite_nonneg(p->t_gpu[k]) || !finite_nonneg(p->t_comm[k]) || !finite_nonneg(p->f_mod[k]) ||
        !finite_nonneg(p->f_dat[k]))
      return EA_EINVAL;
    for (int i = 0; i < p->n_samples; ++i) {
      const double v = p->phi[(size_t)k * p->n_samples + i];
      if (!(v >= 0.0 && v <= 1.0)) return EA_EINVAL;  // c26
    }
  }
  return EA_OK;
}

struct Pred {
  std::vector<ea_gpu_prediction> gpu;
  double iter_time = 0.0, peak_mem = 0.0;
};

void predict_into(const ea_profile* p, int m_star, int n_star, Pred* out) {
  const int K = p->n_gpus;
  const double m = p->m, n = p->n, ms = m_star, ns = n_star;
  const double c = (m * ns) / (ms * n);  // utilisation scale of Eq. 2
  out->gpu.assign(K, ea_gpu_prediction{});
  std::vector<double> tg(K), tt(K);
  for (int k = 0; k < K; ++k) {
    double extra = 0.0;  // Int max(c phi - 1, 0) dt  (c22)
    const double* row = p->phi + (size_t)k * p->n_samples;
    for (int i = 0; i < p->n_samples; ++i) extra += std::max(c * row[i] - 1.0, 0.0);
    extra *= p->dt;
    tg[k] = (ms * n) / (m * ns) * (p->t_gpu[k] + extra);                               // Eq. 2
    tt[k] = ns / n * p->t_comm[k];                                                      // (TT^k)*
    out->gpu[k].t_gpu = tg[k];
    out->gpu[k].t_com = ns / (ms * n) * p->t_comm[k] + (ms - 1.0) / ms * std::max(tt[k] - tg[k], 0.0);  // Eq. 4
    out->gpu[k].mem = ns / n * p->f_mod[k] + (m * ns) / (ms * n) * p->f_dat[k];         // Eq. 8
  }
  out->gpu[0].t_up = 0.0;
  for (int k = 1; k < K; ++k) out->gpu[k].t_up = out->gpu[k - 1].t_up + (tt[k - 1] + tg[k - 1]) / ms;  // Eq. 6
  out->gpu[K - 1].t_down = 0.0;
  for (int k = K - 2; k >= 0; --k)
    out->gpu[k].t_down = out->gpu[k + 1].t_down + (tt[k + 1] + tg[k + 1]) / ms;                     // Eq. 7
  out->iter_time = 0.0;
  out->peak_mem = 0.0;
  for (int k = 0; k < K; ++k) {
    ea_gpu_prediction& g = out->gpu[k];
    g.t_bub = g.t_up + g.t_down;             // Eq. 5
    g.t_total = g.t_gpu + g.t_com + g.t_bub; // Eq. 1
    out->iter_time = std::max(out->iter_time, g.t_total);
    out->peak_mem = std::max(out->peak_mem, g.mem);
  }
}

}  // namespace

extern "C" {

ea_status ea_predict(const ea_profile* prof, int32_t m_star, int32_t n_star, ea_gpu_prediction* out,
                     double* iter_time, double* peak_mem) {
  if (check_profile(prof) != EA_OK || m_star < 1 || n_star < 1) return EA_EINVAL;
  Pred pr;
  predict_into(prof, m_star, n_star, &pr);
  if (out) std::memcpy(out, pr.gpu.data(), sizeof(ea_gpu_prediction) * pr.gpu.size());
  if (iter_time) *iter_time = pr.iter_time;
  if (peak_mem) *peak_mem = pr.peak_mem;
  return EA_OK;
}

ea_status ea_tune(const ea_profile* prof, const int32_t* m_cands, int32_t n_m, const int32_t* n_cands, int32_t n_n,
                  double mem_limit, int32_t objective, int32_t* best_m, int32_t* best_n, double* best_iter_time) {
  if (best_m) *best_m = -1;
  if (best_n) *best_n = -1;
  if (check_profile(prof) != EA_OK || !m_cands || !n_cands || n_m < 1 || n_n < 1 || !best_m || !best_n ||
      (objective != EA_TUNE_THROUGHPUT && objective != EA_TUNE_TIME) || std::isnan(mem_limit))
    return EA_EINVAL;
  for (int i = 0; i < n_m; ++i)
    if (m_cands[i] < 1) return EA_EINVAL;
  for (int i = 0; i < n_n; ++i)
    if (n_cands[i] < 1) return EA_EINVAL;
  bool have = false;
  double b_score = 0, b_mem = 0, b_time = 0;
  int b_n = 0, b_m = 0;
  Pred pr;
  for (int a = 0; a < n_n; ++a) {
    for (int b = 0; b < n_m; ++b) {
      const int ns = n_cands[a], ms = m_cands[b];
      predict_into(prof, ms, ns, &pr);
      if (pr.peak_mem > mem_limit) continue;  // c25
      const double score = objective == EA_TUNE_THROUGHPUT ? ns / pr.iter_time : -pr.iter_time;
      // lexicographic: higher score, lower memory, smaller n*, smaller m*  (c24)
      bool better = !have || score > b_score ||
                    (score == b_score && (pr.peak_mem < b_mem ||
                                          (pr.peak_mem == b_mem && (ns < b_n || (ns == b_n && ms < b_m)))));
      if (better) {
        have = true;
        b_score = score;
        b_mem = pr.peak_mem;
        b_time = pr.iter_time;
        b_n = ns;
        b_m = ms;
      }
    }
  }
  if (!have) return EA_ESTATE;  // no setting satisfies the memory limit
  *best_m = b_m;
  *best_n = b_n;
  if (best_iter_time) *best_iter_time = b_time;
  return EA_OK;
}

}  // extern "C"

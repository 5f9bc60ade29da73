// Advance-forward-propagation micro-batch order (row a9; pure indexing, host only).
//
// Algorithm 1 (§4.2) on a stage: `advance` forwards first (lines
// 3-4), then M - advance (forward, backward) pairs (lines 6-8), then -- not
// printed in Algorithm 1, reading c15 -- the backwards of the micro-batches
// still in flight.  advance = K-1-stage is 1F1B (line 1);
// advance >= M is AFAB.  Forwards and backwards each run in
// micro-batch order, so the list is determined by the positions of the
// backwards alone.
#include <stdint.h>

#include "../../include/ea.h"

extern "C" int32_t ea_schedule(int32_t K, int32_t M, int32_t stage, int32_t advance, ea_op* out, int32_t cap) {
  if (K < 1 || M < 0 || stage < 0 || stage >= K) return -EA_EINVAL;
  if (M > (INT32_MAX / 2)) return -EA_EINVAL;
  const int32_t total = 2 * M;
  if (cap < total || (total > 0 && out == nullptr)) return -EA_EINVAL;
  const int32_t a = advance < 0 ? 0 : (advance > M ? M : advance);
  int32_t w = 0;
  for (int32_t f = 0; f < a; ++f) out[w++] = ea_op{0, f};  // warm-up: forwards in advance
  for (int32_t j = 0; j < M - a; ++j) {                     // steady state: one forward, one backward
    out[w++] = ea_op{0, a + j};
    out[w++] = ea_op{1, j};
  }
  for (int32_t b = M - a; b < M; ++b) out[w++] = ea_op{1, b};  // cool-down
  return w;
}

// Algorithm 1 lines 1 and 9-10 (reading c27): start at 1F1B
// (advance_num = K-1 on GPU 1) and, after each batch, advance one more
// micro-batch if the batch was faster than the previous one and one more
// stashed micro-batch still fits the memory limit; never beyond M (AFAB).
extern "C" ea_status ea_advance_init(ea_advance_ctl* ctl, int32_t K, int32_t M) {
  if (!ctl || K < 1 || M < 0) return EA_EINVAL;
  ctl->K = K;
  ctl->M = M;
  ctl->advance_num = K - 1 < M ? K - 1 : M;
  ctl->has_last = 0;
  ctl->last_time = 0.0;
  return EA_OK;
}

extern "C" int32_t ea_advance_update(ea_advance_ctl* ctl, double batch_time, double peak_mem,
                                     double mem_per_microbatch, double mem_limit) {
  if (!ctl || ctl->K < 1 || batch_time != batch_time || peak_mem != peak_mem || mem_per_microbatch != mem_per_microbatch ||
      mem_limit != mem_limit)
    return -EA_EINVAL;
  const bool faster = !ctl->has_last || batch_time < ctl->last_time;   // is_faster()
  const bool mem_ok = peak_mem + mem_per_microbatch <= mem_limit;      // is_mem_available()
  if (faster && mem_ok && ctl->advance_num < ctl->M) ++ctl->advance_num;
  ctl->has_last = 1;
  ctl->last_time = batch_time;
  return ctl->advance_num;
}

extern "C" int32_t ea_advance_for_stage(const ea_advance_ctl* ctl, int32_t stage) {
  if (!ctl || stage < 0 || stage >= ctl->K) return -EA_EINVAL;
  const int32_t base = ctl->K - 1 < ctl->M ? ctl->K - 1 : ctl->M;
  const int32_t extra = ctl->advance_num - base;
  const int32_t a = ctl->K - 1 - stage + extra;  // GPU k = stage+1: K - k + extra  (c15)
  return a < ctl->M ? a : ctl->M;
}

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

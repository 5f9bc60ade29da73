// Fused elastic-averaging kernels for sm_100a (B200).
//
// Per element j of a stage and replica i (§3.2; DESIGN.md c1-c14, c21):
//   Step 1 (local update of the user-specified optimizer):
//     SGD-momentum: g' = g + wd*x; m = mu*m + g'; D = -lr*(nesterov ? g' + mu*m : m)
//     Adam(W):      g' = g (+ wd*x for Adam); m = b1*m + (1-b1)*g'; v = b2*v + (1-b2)*g'^2;
//                   D = -(lr/bc1) * m / (sqrt(v)/sqrt(bc2) + eps)  (- lr*wd*x for AdamW)
//   Step 2: x_i = (1-alpha)*x_i + alpha*x~ + D_i          ((1-a):a dilution + local update)
//   Steps 3-4: R += rho*D_i + beta*(x_i - x~)               (send + accumulate)
//   Step 5: x~ = x~ + R/N                                    (normalise + apply)
//
// The path is elementwise plus a reduction over the N replicas: ~0.5 flop per
// byte, far below the fp32 ridge, so every kernel here is HBM-bound and is
// written for bytes in flight: 128-bit coalesced accesses, persistent grids
// (#SMs x resident blocks) sweeping the stages of a launch in waves with the
// ragged remainder split evenly (wave_item), so no SM idles in a partial last
// wave.  Tensor cores are not used (no contraction).
#include <cuda_runtime.h>
#include <stdint.h>

#include <cstdlib>

#include "ea_internal.h"
#include "ea_update.cuh"
#include "ea_bulk.cuh"

namespace ea {
namespace {

constexpr int kThreads = 256;

// ---------------------------------------------------------------- memory ops
// HINT = 0: plain streaming (L1 bypass); HINT = 1: additionally mark every
// access L2 evict-first (measured: no effect; kept as a knob).
template <int HINT>
struct Mem {
  uint64_t pol;
  __device__ __forceinline__ Mem() {
    if (HINT) asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
  }
  __device__ __forceinline__ float4 ld(const float* p) const {  // read-write data
    float4 v;
    if (HINT)
      asm volatile("ld.global.L1::no_allocate.L2::cache_hint.v4.f32 {%0,%1,%2,%3}, [%4], %5;"
                   : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w)
                   : "l"(p), "l"(pol));
    else
      asm volatile("ld.global.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];"
                   : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w)
                   : "l"(p));
    return v;
  }
  __device__ __forceinline__ float4 ld_ro(const float* p) const {  // read-only in this kernel
    float4 v;
    if (HINT)
      asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.f32 {%0,%1,%2,%3}, [%4], %5;"
                   : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w)
                   : "l"(p), "l"(pol));
    else
      asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];"
                   : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w)
                   : "l"(p));
    return v;
  }
  __device__ __forceinline__ void st(float* p, float4 v) const {
    if (HINT)
      asm volatile("st.global.L1::no_allocate.L2::cache_hint.v4.f32 [%0], {%1,%2,%3,%4}, %5;" ::"l"(p), "f"(v.x),
                   "f"(v.y), "f"(v.z), "f"(v.w), "l"(pol)
                   : "memory");
    else
      asm volatile("st.global.L1::no_allocate.v4.f32 [%0], {%1,%2,%3,%4};" ::"l"(p), "f"(v.x), "f"(v.y), "f"(v.z),
                   "f"(v.w)
                   : "memory");
  }
};

// Scalar tail of one stage: elements [4*(p/4), p) (fewer than 4), one thread.
// STALE: the replicas see st.prev[j] (x~_{t-1}) and st.prev[j] becomes x~_t (row f4).
template <int N, int OPT, bool STALE = false>
__device__ void stage_tail(const StageRefs& st, const Hyper& hp) {
  const StepCoef sc = load_coef<OPT>(st.scp);
  for (int64_t j = (st.p / 4) * 4; j < st.p; ++j) {
    const float c = st.c[j];
    const float cu = STALE ? st.prev[j] : c;
    float acc = 0.f;
#pragma unroll
    for (int i = 0; i < N; ++i) {
      float x = st.x[i][j], m = st.m[i][j], v = two_state(OPT) ? st.v[i][j] : 0.f;
      acc += ea_elem<OPT>(x, st.g[i][j], m, v, cu, hp, sc);
      st.x[i][j] = x;
      st.m[i][j] = m;
      if (two_state(OPT)) st.v[i][j] = v;
    }
    st.c[j] = fmaf(acc, hp.inv_n, c);
    if (STALE) st.prev[j] = c;
  }
}

// ---------------------------------------------------------------- wave schedule
// Chunks of C float4: in stage s the grid sweeps full waves (chunk w*G + b for
// block b, so the G blocks of a wave touch one contiguous window of every
// stream -- DRAM-page friendly), then the ragged remainder R < G*C is split
// evenly over all G blocks (no block idles in a partial last wave).  Every
// block walks the same sequence of (stage, wave) items, so the cursor is
// warp- and block-uniform.
struct WaveCursor {
  int s;
  int64_t w;
};

template <class NvecOf>
__device__ __forceinline__ bool wave_item_f(int nstages, NvecOf nvec_of, int64_t C, WaveCursor& cur, int& s_out,
                                            int64_t& v0, int64_t& nv) {
  const int64_t G = gridDim.x, bid = blockIdx.x;
  while (cur.s < nstages) {
    const int64_t nvec = nvec_of(cur.s);
    const int64_t waves = nvec / (G * C);
    if (cur.w < waves) {
      v0 = (cur.w * G + bid) * C;
      nv = C;
      s_out = cur.s;
      ++cur.w;
      return true;
    }
    if (cur.w == waves) {
      const int64_t r0 = waves * G * C, R = nvec - r0;
      const int64_t a = r0 + R * bid / G, e = r0 + R * (bid + 1) / G;
      ++cur.w;
      if (e > a) {
        v0 = a;
        nv = e - a;
        s_out = cur.s;
        return true;
      }
    }
    ++cur.s;
    cur.w = 0;
  }
  return false;
}

__device__ __forceinline__ bool wave_item(const StageBatch& b, int64_t C, WaveCursor& cur, int& s_out, int64_t& v0,
                                          int64_t& nv) {
  return wave_item_f(b.nstages, [&](int s) { return b.st[s].p / 4; }, C, cur, s_out, v0, nv);
}

// ============================================================================
// Variant 1 (SGD): register-resident replica loop.
// One thread owns U float4 of a center; it issues all (3N+1)*U 128-bit loads
// before any arithmetic (maximal memory-level parallelism per thread: the
// replica pointers may alias as far as the compiler knows, so the loads are
// hoisted by hand), shares the center value across the N replicas in
// registers, reduces the N contributions in registers and writes x_i, m_i
// and x~ once.  Work unit: kThreads*U float4 per block, scheduled by wave_item.
// ============================================================================
template <int N, int U, int HINT, int OPT>
__device__ __forceinline__ void regloop_range(const StageRefs& st, int64_t va, int64_t ve, const Hyper& hp,
                                              const Mem<HINT>& mem, const StepCoef& sc) {
  constexpr bool kTwo = two_state(OPT);  // Adam(W): second moment v
  for (int64_t base = va + threadIdx.x; base < ve; base += (int64_t)kThreads * U) {
    float4 c[U], x[N][U], g[N][U], m[N][U], w[kTwo ? N : 1][U];
    bool ok[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int64_t v = base + (int64_t)u * kThreads;
      ok[u] = v < ve;
      if (ok[u]) c[u] = mem.ld(st.c + 4 * v);
    }
#pragma unroll
    for (int i = 0; i < N; ++i) {
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const int64_t v = base + (int64_t)u * kThreads;
        if (ok[u]) {
          x[i][u] = mem.ld(st.x[i] + 4 * v);
          g[i][u] = mem.ld_ro(st.g[i] + 4 * v);
          m[i][u] = mem.ld(st.m[i] + 4 * v);
          if constexpr (kTwo) w[i][u] = mem.ld(st.v[i] + 4 * v);
        }
      }
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      if (!ok[u]) continue;
      const int64_t v = base + (int64_t)u * kThreads;
      float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll
      for (int i = 0; i < N; ++i) {
        float4 unused = make_float4(0.f, 0.f, 0.f, 0.f);
        float4& wv = kTwo ? w[kTwo ? i : 0][u] : unused;
        add4(acc, ea_vec<OPT>(x[i][u], g[i][u], m[i][u], wv, c[u], hp, sc));
        mem.st(st.x[i] + 4 * v, x[i][u]);
        mem.st(st.m[i] + 4 * v, m[i][u]);
        if constexpr (kTwo) mem.st(st.v[i] + 4 * v, wv);
      }
      mem.st(st.c + 4 * v, center_apply(c[u], acc, hp.inv_n));
    }
  }
}

// SGD: __launch_bounds__(256) (<= 255 registers; 2+ CTAs/SM at N <= 4).  Adam(W) keeps (4N+1) float4 per
// thread in flight (N = 8: 132 registers of loads).  Bytes in flight per SM = resident threads x loads per
// thread, so Adam at N = 5 asks for 2 CTAs/SM (<= 128 registers, 32 B spilled) instead of 1 CTA at 137 (N = 6 would
// spill 120 B).
template <int N, int OPT>
constexpr int regloop_min_blocks() {
  return (two_state(OPT) && N == 5) ? 2 : 0;  // 0: no minimum (ptxas default heuristics)
}

template <int N, int U, int HINT, int OPT>
__global__ void __launch_bounds__(kThreads, regloop_min_blocks<N, OPT>()) colocated_regloop(const StageBatch b,
                                                                                            const Hyper hp) {
  const Mem<HINT> mem;
  __shared__ StepCoef s_coef[kMaxLaunchStages];
  if (has_coef(OPT)) {
    if (threadIdx.x < b.nstages) s_coef[threadIdx.x] = *b.st[threadIdx.x].scp;
    __syncthreads();
  }
  WaveCursor cur{0, 0};
  int s;
  int64_t v0, nv;
  while (wave_item(b, (int64_t)kThreads * U, cur, s, v0, nv))
    regloop_range<N, U, HINT, OPT>(b.st[s], v0, v0 + nv, hp, mem, has_coef(OPT) ? s_coef[s] : StepCoef{0.f, 0.f});
  if (blockIdx.x == gridDim.x - 1 && threadIdx.x == 0)
    for (int t = 0; t < b.nstages; ++t) stage_tail<N, OPT>(b.st[t], hp);
}

// ============================================================================
// Variant 4: split register loop -- S adjacent lanes share one float4 column of the center, each holding the
// loads of N/S replicas in registers (all hoisted before any arithmetic), partial contributions reduced by
// __shfl_xor over the S lanes, the first lane of the group writes x~.  For large N, where the one-thread-per-
// column register loop needs (A N + 1) float4 of loads per thread (Adam N = 8: 200+ registers, 1 CTA/SM), this
// keeps the bytes in flight per thread the same per replica group and the CTAs per SM high.  The S lanes of a
// group load the same center word (one sector: no extra DRAM traffic).
// ============================================================================
template <int N, int S, int OPT>
__global__ void __launch_bounds__(kThreads, 2) colocated_split(const StageBatch b, const Hyper hp) {
  constexpr int NS = (N + S - 1) / S;  // replicas per lane
  constexpr bool kTwo = two_state(OPT);
  constexpr int COLS = kThreads / S;   // float4 columns per CTA pass
  const Mem<0> mem;
  __shared__ StepCoef s_coef[kMaxLaunchStages];
  if (has_coef(OPT)) {
    if (threadIdx.x < b.nstages) s_coef[threadIdx.x] = *b.st[threadIdx.x].scp;
    __syncthreads();
  }
  const int sub = threadIdx.x % S, col = threadIdx.x / S;
  WaveCursor cur{0, 0};
  int s;
  int64_t v0, nv;
  while (wave_item(b, COLS, cur, s, v0, nv)) {
    const StageRefs& st = b.st[s];
    const StepCoef sc = has_coef(OPT) ? s_coef[s] : StepCoef{0.f, 0.f};
    for (int64_t base = 0; base < nv; base += COLS) {  // block-uniform bound: every lane reaches the shuffles
      const int64_t lv = base + col;
      const bool on = lv < nv;
      const int64_t v = v0 + lv;
      float4 c = make_float4(0.f, 0.f, 0.f, 0.f);
      float4 x[NS], g[NS], m[NS], w[kTwo ? NS : 1];
      if (on) c = mem.ld(st.c + 4 * v);
#pragma unroll
      for (int k = 0; k < NS; ++k) {
        const int i = sub * NS + k;
        if (on && i < N) {
          x[k] = mem.ld(st.x[i] + 4 * v);
          g[k] = mem.ld_ro(st.g[i] + 4 * v);
          m[k] = mem.ld(st.m[i] + 4 * v);
          if constexpr (kTwo) w[k] = mem.ld(st.v[i] + 4 * v);
        }
      }
      float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll
      for (int k = 0; k < NS; ++k) {
        const int i = sub * NS + k;
        if (on && i < N) {
          float4 unused = make_float4(0.f, 0.f, 0.f, 0.f);
          float4& wv = kTwo ? w[kTwo ? k : 0] : unused;
          add4(acc, ea_vec<OPT>(x[k], g[k], m[k], wv, c, hp, sc));
          mem.st(st.x[i] + 4 * v, x[k]);
          mem.st(st.m[i] + 4 * v, m[k]);
          if constexpr (kTwo) mem.st(st.v[i] + 4 * v, wv);
        }
      }
#pragma unroll
      for (int off = 1; off < S; off <<= 1) {
        acc.x += __shfl_xor_sync(0xffffffffu, acc.x, off);
        acc.y += __shfl_xor_sync(0xffffffffu, acc.y, off);
        acc.z += __shfl_xor_sync(0xffffffffu, acc.z, off);
        acc.w += __shfl_xor_sync(0xffffffffu, acc.w, off);
      }
      if (on && sub == 0) mem.st(st.c + 4 * v, center_apply(c, acc, hp.inv_n));
    }
  }
  if (blockIdx.x == gridDim.x - 1 && threadIdx.x == 0)
    for (int t = 0; t < b.nstages; ++t) stage_tail<N, OPT>(b.st[t], hp);
}

// Scalar tail of the spread local kernels (one thread): elements [4*(p/4), p) and the zero padding
// [p, p_pad) of the contribution (reading c18: zero padding is a fixed point of the exchange).
template <int OPT>
__device__ void spread_tail(const StageRefs& st, float* contrib, int64_t p_pad, const Hyper& hp) {
  const StepCoef sc = load_coef<OPT>(st.scp);
  for (int64_t j = (st.p / 4) * 4; j < st.p; ++j) {
    float x = st.x[0][j], m = st.m[0][j], v = two_state(OPT) ? st.v[0][j] : 0.f;
    contrib[j] = ea_elem<OPT>(x, st.g[0][j], m, v, st.c[j], hp, sc);
    st.x[0][j] = x;
    st.m[0][j] = m;
    if (two_state(OPT)) st.v[0][j] = v;
  }
  for (int64_t j = st.p; j < p_pad; ++j) contrib[j] = 0.f;
}

// ============================================================================
// Variant 5: warp per replica.  A CTA of 32N threads; warp i streams replica i of a tile of 32U float4 columns
// (full 512 B rows per load instruction -- the lane kernel's rows shrink to 64 B at N = 8), keeps its U float4 of
// x, g and the optimizer state in registers, and writes its contribution r_i to shared memory; after a block
// barrier the N contributions of each column are summed and x~ updated.  The center is read by every warp through
// the read-only path (one DRAM read, the other warps hit L1/L2).
// ============================================================================
// STALE (row f4, reading c28): the replicas read x~_{t-1} (st.prev) instead of x~_t; the reduction writes
// x~_{t+1} = x~_t + R/N and prev <- x~_t.
template <int N, int OPT, int U, bool STALE = false>
__global__ void __launch_bounds__(32 * N, N >= 6 ? 2 : 3) colocated_warprep(const StageBatch b, const Hyper hp) {
  constexpr int TV = 32 * U;  // float4 columns per tile
  constexpr bool kTwo = two_state(OPT);
  __shared__ __align__(16) float4 s_r[N][TV];
  __shared__ StepCoef s_coef[kMaxLaunchStages];
  const Mem<0> mem;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (has_coef(OPT)) {
    if (threadIdx.x < b.nstages) s_coef[threadIdx.x] = *b.st[threadIdx.x].scp;
    __syncthreads();
  }
  WaveCursor cur{0, 0};
  int s;
  int64_t v0, nv;
  while (wave_item(b, TV, cur, s, v0, nv)) {
    const StageRefs& st = b.st[s];
    const StepCoef sc = has_coef(OPT) ? s_coef[s] : StepCoef{0.f, 0.f};
    float* xi = nullptr;
    const float* gi = nullptr;
    float* mi = nullptr;
    float* vi = nullptr;
#pragma unroll
    for (int i = 0; i < N; ++i)
      if (warp == i) {
        xi = st.x[i];
        gi = st.g[i];
        mi = st.m[i];
        if (kTwo) vi = st.v[i];
      }
    float4 x[U], g[U], m[U], w[U], c[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int lv = u * 32 + lane;
      if (lv < nv) {
        const int64_t v = v0 + lv;
        x[u] = mem.ld(xi + 4 * v);
        g[u] = mem.ld_ro(gi + 4 * v);
        m[u] = mem.ld(mi + 4 * v);
        if (kTwo) w[u] = mem.ld(vi + 4 * v);
        c[u] = __ldg(reinterpret_cast<const float4*>(STALE ? st.prev : st.c) + v);  // the center the replicas see
      }
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int lv = u * 32 + lane;
      if (lv < nv) {
        const int64_t v = v0 + lv;
        s_r[warp][lv] = ea_vec<OPT>(x[u], g[u], m[u], w[u], c[u], hp, sc);
        mem.st(xi + 4 * v, x[u]);
        mem.st(mi + 4 * v, m[u]);
        if (kTwo) mem.st(vi + 4 * v, w[u]);
      }
    }
    // (at N = 1 too: applying x~ += r directly, without the tile and barriers, measured slower -- 0.88 vs 0.94,
    // profiles/r02_s3_n1_direct.jsonl)
    __syncthreads();
    for (int col = threadIdx.x; col < nv; col += 32 * N) {
      float4 acc = s_r[0][col];
#pragma unroll
      for (int i = 1; i < N; ++i) add4(acc, s_r[i][col]);
      const int64_t v = v0 + col;
      const float4 cv = __ldg(reinterpret_cast<const float4*>(st.c) + v);
      mem.st(st.c + 4 * v, center_apply(cv, acc, hp.inv_n));
      if (STALE) mem.st(st.prev + 4 * v, cv);
    }
    __syncthreads();  // s_r is refilled by the next tile
  }
  if (blockIdx.x == gridDim.x - 1 && threadIdx.x == 0)
    for (int t = 0; t < b.nstages; ++t) stage_tail<N, OPT, STALE>(b.st[t], hp);
}

// ============================================================================
// Variant 6: warp-specialised warp per replica.  Warp i < N streams replica i exactly as variant 5 does (U float4
// of x, g and the optimizer state per lane and tile, 512 B rows per load instruction) but never waits at a block
// barrier: it writes its contribution r_i into an R-deep ring of contribution tiles in shared memory and arrives
// on the slot's "full" mbarrier; warp N (the reducer) waits for the N contributions of a slot, sums them, applies
// x~ += R/N and arrives on the slot's "empty" mbarrier.  A replica warp waits only when the ring is full, so the
// replica warps drift up to R tiles apart and keep their loads in flight while the reduction of older tiles runs.
// STALE (row f4, c28): the replica warps read x~_{t-1}; the reducer reads x~_t, writes x~_{t+1} and x~_{t-1} <- x~_t.
// ============================================================================
template <int N, int OPT, int U, int R, bool STALE = false>
__global__ void __launch_bounds__(32 * (N + 1), U >= 4 ? 1 : 2) colocated_warpspec(const StageBatch b,
                                                                                    const Hyper hp) {
  constexpr int TV = 32 * U;  // float4 columns per tile
  constexpr bool kTwo = two_state(OPT);
  extern __shared__ __align__(16) float4 s_ring[];  // [R][N][TV] contribution tiles (dynamic: up to 64 KB)
  __shared__ __align__(8) uint64_t full[R], empty[R];
  __shared__ StepCoef s_coef[kMaxLaunchStages];
  const Mem<0> mem;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  auto s_r = [&](int k, int i, int lv) -> float4& { return s_ring[(k * N + i) * TV + lv]; };
  if (has_coef(OPT) && threadIdx.x < b.nstages) s_coef[threadIdx.x] = *b.st[threadIdx.x].scp;
  if (threadIdx.x == 0) {
    for (int k = 0; k < R; ++k) {
      mbar_init(&full[k], 32 * N);  // every lane of every replica warp arrives (releases its own stores)
      mbar_init(&empty[k], 32);     // every lane of the reducer warp
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  WaveCursor cur{0, 0};
  int s;
  int64_t v0, nv;
  int slot = 0;
  uint32_t phase = 0;
  if (warp < N) {  // ---------------------------------------------------------------- replica warp
    while (wave_item(b, TV, cur, s, v0, nv)) {
      const StageRefs& st = b.st[s];
      const StepCoef sc = has_coef(OPT) ? s_coef[s] : StepCoef{0.f, 0.f};
      float* xi = st.x[warp];
      const float* gi = st.g[warp];
      float* mi = st.m[warp];
      float* vi = kTwo ? st.v[warp] : nullptr;
      float4 x[U], g[U], m[U], w[U], c[U];
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const int lv = u * 32 + lane;
        if (lv < nv) {
          const int64_t v = v0 + lv;
          x[u] = mem.ld(xi + 4 * v);
          g[u] = mem.ld_ro(gi + 4 * v);
          m[u] = mem.ld(mi + 4 * v);
          if (kTwo) w[u] = mem.ld(vi + 4 * v);
          c[u] = __ldg(reinterpret_cast<const float4*>(STALE ? st.prev : st.c) + v);
        }
      }
      float4 r[U];
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const int lv = u * 32 + lane;
        if (lv < nv) {
          const int64_t v = v0 + lv;
          r[u] = ea_vec<OPT>(x[u], g[u], m[u], w[u], c[u], hp, sc);
          mem.st(xi + 4 * v, x[u]);
          mem.st(mi + 4 * v, m[u]);
          if (kTwo) mem.st(vi + 4 * v, w[u]);
        }
      }
      mbar_wait(&empty[slot], phase ^ 1u);  // the reducer has finished with this slot's previous tile
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const int lv = u * 32 + lane;
        if (lv < nv) s_r(slot, warp, lv) = r[u];
      }
      mbar_arrive(&full[slot]);
      if (++slot == R) {
        slot = 0;
        phase ^= 1u;
      }
    }
  } else {  // --------------------------------------------------------------------------- reducer warp
    while (wave_item(b, TV, cur, s, v0, nv)) {
      const StageRefs& st = b.st[s];
      float4 c[U];
#pragma unroll
      for (int u = 0; u < U; ++u) {  // x~_t of this lane's columns, in flight while the replicas finish
        const int lv = u * 32 + lane;
        if (lv < nv) c[u] = __ldg(reinterpret_cast<const float4*>(st.c) + v0 + lv);
      }
      mbar_wait(&full[slot], phase);
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const int lv = u * 32 + lane;
        if (lv < nv) {
          float4 acc = s_r(slot, 0, lv);
#pragma unroll
          for (int i = 1; i < N; ++i) add4(acc, s_r(slot, i, lv));
          const int64_t v = v0 + lv;
          mem.st(st.c + 4 * v, center_apply(c[u], acc, hp.inv_n));
          if (STALE) mem.st(st.prev + 4 * v, c[u]);
        }
      }
      mbar_arrive(&empty[slot]);
      if (++slot == R) {
        slot = 0;
        phase ^= 1u;
      }
    }
    if (blockIdx.x == gridDim.x - 1 && lane == 0)
      for (int t = 0; t < b.nstages; ++t) stage_tail<N, OPT, STALE>(b.st[t], hp);
  }
}

template <int U>
struct WideRep {
  float4 x[U], g[U], m[U], w[U];
};

template <int U, int OPT>
__device__ __forceinline__ void wide_load(const ReplicaTable& t, int i, int64_t base, const bool* ok,
                                          const Mem<0>& mem, WideRep<U>& r) {
#pragma unroll
  for (int u = 0; u < U; ++u) {
    const int64_t v = base + (int64_t)u * kThreads;
    if (ok[u]) {
      r.x[u] = mem.ld(t.x[i] + 4 * v);
      r.g[u] = mem.ld_ro(t.g[i] + 4 * v);
      r.m[u] = mem.ld(t.m[i] + 4 * v);
      if (two_state(OPT)) r.w[u] = mem.ld(t.v[i] + 4 * v);
    }
  }
}

template <int U, int OPT>
__device__ __forceinline__ void wide_proc(const ReplicaTable& t, int i, int64_t base, const bool* ok,
                                          const Mem<0>& mem, WideRep<U>& r, const float4* cu, float4* acc,
                                          const Hyper& hp, const StepCoef& sc) {
#pragma unroll
  for (int u = 0; u < U; ++u) {
    if (!ok[u]) continue;
    const int64_t v = base + (int64_t)u * kThreads;
    add4(acc[u], ea_vec<OPT>(r.x[u], r.g[u], r.m[u], r.w[u], cu[u], hp, sc));
    mem.st(t.x[i] + 4 * v, r.x[u]);
    mem.st(t.m[i] + 4 * v, r.m[u]);
    if (two_state(OPT)) mem.st(t.v[i] + 4 * v, r.w[u]);
  }
}

// Runtime-N replica loop (N > 8, Adam N > 6, the stale center): one stage,
// replicas visited in a loop.  prev != nullptr selects the stale center of
// row f4 (reading c28): the replicas use x~_{t-1} (prev) for dilution and
// gap, the center is updated from x~_t, and prev becomes x~_t.
template <int U, int OPT>
__global__ void __launch_bounds__(kThreads) colocated_wide(const ReplicaTable t, int n, float* __restrict__ center,
                                                           float* __restrict__ prev, int64_t nvec, int64_t p,
                                                           const Hyper hp, const StepCoef* scp) {
  const Mem<0> mem;
  const StepCoef sc = load_coef<OPT>(scp);
  const bool stale = prev != nullptr;
  WaveCursor cur{0, 0};
  int sidx;
  int64_t va, nv;
  while (wave_item_f(1, [&](int) { return nvec; }, (int64_t)kThreads * U, cur, sidx, va, nv)) {
    const int64_t ve = va + nv;
    for (int64_t base = va + threadIdx.x; base < ve; base += (int64_t)kThreads * U) {
      float4 c[U], cu[U], acc[U];
      bool ok[U];
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const int64_t v = base + (int64_t)u * kThreads;
        ok[u] = v < ve;
        acc[u] = make_float4(0.f, 0.f, 0.f, 0.f);
        if (ok[u]) {
          c[u] = mem.ld(center + 4 * v);
          cu[u] = stale ? mem.ld(prev + 4 * v) : c[u];   // the center the replicas see
        }
      }
      // software-pipelined replica loop: replica i+1's loads are in flight while replica i is updated
      // (replicas never alias, ABI contract), two register buffers with compile-time names
      WideRep<U> ra, rb;
      wide_load<U, OPT>(t, 0, base, ok, mem, ra);
      int i = 0;
      for (; i + 1 < n; i += 2) {
        wide_load<U, OPT>(t, i + 1, base, ok, mem, rb);
        wide_proc<U, OPT>(t, i, base, ok, mem, ra, cu, acc, hp, sc);
        if (i + 2 < n) wide_load<U, OPT>(t, i + 2, base, ok, mem, ra);
        wide_proc<U, OPT>(t, i + 1, base, ok, mem, rb, cu, acc, hp, sc);
      }
      if (i < n) wide_proc<U, OPT>(t, i, base, ok, mem, ra, cu, acc, hp, sc);
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const int64_t v = base + (int64_t)u * kThreads;
        if (ok[u]) {
          mem.st(center + 4 * v, center_apply(c[u], acc[u], hp.inv_n));
          if (stale) mem.st(prev + 4 * v, c[u]);
        }
      }
    }
  }
  if (blockIdx.x == gridDim.x - 1 && threadIdx.x == 0) {
    for (int64_t j = 4 * nvec; j < p; ++j) {
      const float c = center[j];
      const float cused = stale ? prev[j] : c;
      float acc = 0.f;
      for (int i = 0; i < n; ++i) {
        float x = t.x[i][j], m = t.m[i][j], v = two_state(OPT) ? t.v[i][j] : 0.f;
        acc += ea_elem<OPT>(x, t.g[i][j], m, v, cused, hp, sc);
        t.x[i][j] = x;
        t.m[i][j] = m;
        if (two_state(OPT)) t.v[i][j] = v;
      }
      center[j] = fmaf(acc, hp.inv_n, c);
      if (stale) prev[j] = c;
    }
  }
}

// ============================================================================
// Variant 2 (default; SGD and Adam): lanes = (replica, float4 chunk), center
// tile staged in shared memory by the bulk-copy engine (cp.async.bulk +
// mbarrier, double-buffered), replica reduction by warp shuffles.
//
// A block walks its wave-scheduled tiles (kTileVec float4 of a center) and
// thread 0 prefetches tile k+1 (possibly of the next stage) with one
// cp.async.bulk while the block computes tile k.  Inside a warp, lane l works
// on replica l / CH and chunk l % CH (CH = 32/NP, NP = N rounded up to a power
// of two), so each replica's CH lanes read CH*16 contiguous bytes of x_i, g_i
// and the optimizer state, and the NP lanes of one chunk read the same center
// word from shared memory (a broadcast).  The N contributions of a chunk are
// reduced with log2(NP) __shfl_xor steps; replica-0 lanes write x~.
// ============================================================================
constexpr int kLanePasses = 4;  // float4 chunks per lane per tile

template <int N>
struct LanePow2 {
  static constexpr int value = N <= 1 ? 1 : N <= 2 ? 2 : N <= 4 ? 4 : N <= 8 ? 8 : 16;
};

template <int N, int PASSES = kLanePasses>
struct LaneGeom {
  static constexpr int NP = LanePow2<N>::value;
  static constexpr int CH = 32 / NP;                              // chunks per warp pass
  static constexpr int kVecPerWarp = PASSES * CH;                 // float4 of a tile per warp
  static constexpr int kTileVec = (kThreads / 32) * kVecPerWarp;  // float4 of center per tile
};

// STALE (row f4, reading c28): every stage's x~_{t-1} tile (st.prev) is staged beside x~_t by a second bulk
// copy on the same mbarrier; the replicas dilute with and measure their gap to x~_{t-1}, replica-0 lanes write
// x~_{t+1} = x~_t + R/N and copy x~_t into prev.
template <int N, int HINT, int OPT, int PASSES = kLanePasses, int MINB = 1, bool STALE = false>
__global__ void __launch_bounds__(kThreads, MINB) colocated_laneshfl(const StageBatch b, const Hyper hp) {
  using G = LaneGeom<N, PASSES>;
  constexpr int CH = G::CH, kPasses = PASSES, kVecPerWarp = G::kVecPerWarp, kTileVec = G::kTileVec;
  constexpr bool kTwoState = two_state(OPT);
  __shared__ __align__(128) float4 s_center[2][kTileVec];
  __shared__ __align__(128) float4 s_prev[2][STALE ? kTileVec : 1];
  __shared__ __align__(8) uint64_t s_bar[2];
  const Mem<HINT> mem;

  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int rep = lane / CH, chunk = lane % CH;
  const bool active = rep < N;

  __shared__ StepCoef s_coef[kMaxLaunchStages];  // Adam coefficients of the batch's stages, loaded once
  if (threadIdx.x == 0) {
    mbar_init(&s_bar[0], 1);
    mbar_init(&s_bar[1], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (has_coef(OPT) && threadIdx.x < b.nstages) s_coef[threadIdx.x] = *b.st[threadIdx.x].scp;
  __syncthreads();

  auto issue = [&](int s, int64_t v0, int64_t nv, int buf) {
    const uint32_t bytes = static_cast<uint32_t>(nv * 16);
    mbar_expect_tx(&s_bar[buf], STALE ? 2 * bytes : bytes);
    bulk_g2s(&s_center[buf][0], b.st[s].c + 4 * v0, bytes, &s_bar[buf]);
    if (STALE) bulk_g2s(&s_prev[buf][0], b.st[s].prev + 4 * v0, bytes, &s_bar[buf]);
  };

  WaveCursor cur{0, 0};
  int s, s_next;
  int64_t v0, nv, v0_next, nv_next;
  bool have = wave_item(b, kTileVec, cur, s, v0, nv);
  if (threadIdx.x == 0 && have) issue(s, v0, nv, 0);
  uint32_t phase[2] = {0u, 0u};
  int buf = 0;

  while (have) {
    const bool have_next = wave_item(b, kTileVec, cur, s_next, v0_next, nv_next);
    if (threadIdx.x == 0 && have_next) {
      fence_proxy_async();  // buffer buf^1 was last read through the generic proxy
      issue(s_next, v0_next, nv_next, buf ^ 1);
    }
    const StageRefs& st = b.st[s];
    const StepCoef sc = has_coef(OPT) ? s_coef[s] : StepCoef{0.f, 0.f};
    float* xi = nullptr;
    const float* gi = nullptr;
    float* mi = nullptr;
    float* vi = nullptr;
#pragma unroll
    for (int i = 0; i < N; ++i)
      if (rep == i) {
        xi = st.x[i];
        gi = st.g[i];
        mi = st.m[i];
        if (kTwoState) vi = st.v[i];
      }

    // replica streams first (they do not depend on the center tile)
    float4 x[kPasses], g[kPasses], m[kPasses], w[kPasses];
#pragma unroll
    for (int k = 0; k < kPasses; ++k) {
      const int lv = warp * kVecPerWarp + k * CH + chunk;
      if (active && lv < nv) {
        const int64_t v = v0 + lv;
        x[k] = mem.ld(xi + 4 * v);
        g[k] = mem.ld_ro(gi + 4 * v);
        m[k] = mem.ld(mi + 4 * v);
        if (kTwoState) w[k] = mem.ld(vi + 4 * v);
      }
    }
    mbar_wait(&s_bar[buf], phase[buf]);
    phase[buf] ^= 1u;
#pragma unroll
    for (int k = 0; k < kPasses; ++k) {
      const int lv = warp * kVecPerWarp + k * CH + chunk;
      const bool in = lv < nv;  // uniform across the NP lanes of a chunk
      const float4 c = in ? s_center[buf][lv] : make_float4(0.f, 0.f, 0.f, 0.f);
      const float4 cu = (STALE && in) ? s_prev[buf][lv] : c;  // the center the replicas see
      float4 r = make_float4(0.f, 0.f, 0.f, 0.f);
      if (active && in) {
        r = ea_vec<OPT>(x[k], g[k], m[k], w[k], cu, hp, sc);
        const int64_t v = v0 + lv;
        mem.st(xi + 4 * v, x[k]);
        mem.st(mi + 4 * v, m[k]);
        if (kTwoState) mem.st(vi + 4 * v, w[k]);
      }
#pragma unroll
      for (int off = CH; off < 32; off <<= 1) {
        r.x += __shfl_xor_sync(0xffffffffu, r.x, off);
        r.y += __shfl_xor_sync(0xffffffffu, r.y, off);
        r.z += __shfl_xor_sync(0xffffffffu, r.z, off);
        r.w += __shfl_xor_sync(0xffffffffu, r.w, off);
      }
      if (rep == 0 && in) {
        mem.st(st.c + 4 * (v0 + lv), center_apply(c, r, hp.inv_n));
        if (STALE) mem.st(st.prev + 4 * (v0 + lv), c);
      }
    }
    __syncthreads();  // everyone done reading s_center[buf] before it is refilled
    buf ^= 1;
    have = have_next;
    s = s_next;
    v0 = v0_next;
    nv = nv_next;
  }
  if (blockIdx.x == gridDim.x - 1 && threadIdx.x == 0)
    for (int t = 0; t < b.nstages; ++t) stage_tail<N, OPT, STALE>(b.st[t], hp);
}

// ============================================================================
// Variant 3 (SGD): bulk-copy load pipeline (TMA engine feeds shared memory).
//
// One producer warp (one elected thread) streams every input of a tile --
// x~ and x_i, g_i, m_i of all N replicas, (3N+1) 1-D cp.async.bulk copies of
// kTile float4 each -- into a kStages-deep ring of shared-memory slots,
// completing on a per-slot "full" mbarrier with the byte count.  Eight
// consumer warps read a slot (one float4 column per thread: the x~ value is
// shared by the N replica rows in registers), update in registers, write x_i,
// m_i and x~ straight to HBM with 128-bit stores, and release the slot on its
// "empty" mbarrier (one arrive per consumer warp).  Tiles follow the same
// wave schedule as the other variants.
// ============================================================================
constexpr int kBulkConsumerWarps = 8;
constexpr int kBulkThreads = 32 * (kBulkConsumerWarps + 1);

// Default tile (float4 per array per bulk copy), measured on B200 with the copies issued from all 32
// producer lanes (profiles/r01_s2_bulk_lanes_tiles.jsonl, r01_s2_issue_ab.jsonl): 4 KB copies whenever a
// two-stage ring of them fits in 200 KB (SGD N <= 8, Adam N <= 6), else 2 KB.  Smaller copies lose: the ring
// depth is capped, so bytes in flight per SM shrink with the tile (1 KB: 0.27-0.69 of peak).
template <int N, int A = 3, int X = 0>
constexpr int default_bulk_tile() {
  return (A * N + 1 + X) * 256 * 16 * 2 <= 200 * 1024 ? 256 : 128;
}

constexpr int kMaxBulkStages = 6;  // ring depth cap (8 measured slower: profiles/r01_bulk_n4_tiles.jsonl)

// A = streams per replica in the slot: 3 (x, g, m) for SGD, 4 (x, g, m, v) for Adam; X = extra center streams
// (1: the stale center x~_{t-1}, row f4).
template <int N, int TILE, int A, int X = 0>
struct BulkGeom {
  static constexpr int kTile = TILE;                          // float4 per array per tile
  static constexpr int kSlotVec = (A * N + 1 + X) * kTile;    // float4 per slot
  static constexpr int kFit = (200 * 1024) / (kSlotVec * 16);
  static constexpr int kStages = kFit > kMaxBulkStages ? kMaxBulkStages : (kFit < 2 ? 2 : kFit);
  static constexpr int kSmemBytes = kStages * kSlotVec * 16 + 2 * kStages * 8;
};


// SPREAD = false: co-located stages (x~ updated in place).  SPREAD = true: the spread layout's local
// step (N = 1, one stage): x~ is only read and the contribution r goes to `contrib` (rows a1-a4).
// STALE (co-located, row f4, reading c28): every stage's x~_{t-1} (st.prev) is one more stream of the slot;
// the replicas dilute with and measure their gap to it, x~_{t+1} = x~_t + R/N, prev <- x~_t.
template <int N, int HINT, int OPT, int TILE, bool SPREAD, bool STALE = false>
__device__ __forceinline__ void bulkpipe_body(const StageBatch& b, const Hyper& hp, float* __restrict__ contrib,
                                              int64_t p_pad, int issue_lanes) {
  constexpr int A = two_state(OPT) ? 4 : 3;
  constexpr int X = STALE ? 1 : 0;
  constexpr int NS = A * N + 1 + X;  // streams per slot
  using G = BulkGeom<N, TILE, A, X>;
  constexpr int T = G::kTile, S = G::kStages;
  extern __shared__ __align__(128) float4 smem[];
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + S * G::kSlotVec);
  uint64_t* empty = full + S;
  __shared__ StepCoef s_coef[kMaxLaunchStages];
  const Mem<HINT> mem;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;

  if (threadIdx.x == 0) {
    for (int i = 0; i < S; ++i) {
      mbar_init(&full[i], 1);
      mbar_init(&empty[i], 1);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (has_coef(OPT) && threadIdx.x < b.nstages) s_coef[threadIdx.x] = *b.st[threadIdx.x].scp;
  __syncthreads();

  if (warp == kBulkConsumerWarps) {
    // ---------------- producer warp: lane 0 arms the slot's barrier, then lane q issues the bulk copy of
    // stream q (q = 0: x~; 1 + A*i + {0,1,2,3}: x_i, g_i, state_i, v_i), so the A*N+1 copies of a slot
    // leave in parallel instead of from one thread (the cursor is warp-uniform)
    WaveCursor cur{0, 0};
    int s;
    int64_t v0, nv;
    for (int k = 0; wave_item(b, T, cur, s, v0, nv); ++k) {
      const int slot = k % S;
      mbar_wait(&empty[slot], ((k / S) & 1) ^ 1);
      fence_proxy_async();  // the consumers' generic-proxy reads of this slot precede the bulk writes
      float4* base = smem + slot * G::kSlotVec;
      const uint32_t bytes = static_cast<uint32_t>(nv * 16);
      const StageRefs& st = b.st[s];
      if (lane == 0) mbar_expect_tx(&full[slot], bytes * NS);
      __syncwarp();
      for (int q = lane; q < NS && lane < issue_lanes; q += issue_lanes) {
        const float* src;
        if (q == 0) {
          src = st.c;
        } else if (STALE && q == A * N + 1) {
          src = st.prev;
        } else {
          const int i = (q - 1) / A, kind = (q - 1) % A;
          src = kind == 0 ? st.x[i] : kind == 1 ? st.g[i] : kind == 2 ? st.m[i] : st.v[i];
        }
        bulk_g2s(base + q * T, src + 4 * v0, bytes, &full[slot]);
      }
    }
  } else {
    // ---------------- consumers
    WaveCursor cur{0, 0};
    int s;
    int64_t v0, nv;
    for (int k = 0; wave_item(b, T, cur, s, v0, nv); ++k) {
      const int slot = k % S;
      mbar_wait(&full[slot], (k / S) & 1);
      const float4* base = smem + slot * G::kSlotVec;
      const StageRefs& st = b.st[s];
      const StepCoef sc = has_coef(OPT) ? s_coef[s] : StepCoef{0.f, 0.f};
      for (int lv = threadIdx.x; lv < nv; lv += 32 * kBulkConsumerWarps) {
        const float4 c = base[lv];
        const float4 cu = STALE ? base[(A * N + 1) * T + lv] : c;  // the center the replicas see
        float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
        const int64_t v = v0 + lv;
#pragma unroll
        for (int i = 0; i < N; ++i) {
          float4 x = base[(1 + A * i) * T + lv];
          const float4 g = base[(2 + A * i) * T + lv];
          float4 m = base[(3 + A * i) * T + lv];
          float4 w = A == 4 ? base[(4 + A * i) * T + lv] : make_float4(0.f, 0.f, 0.f, 0.f);
          add4(acc, ea_vec<OPT>(x, g, m, w, cu, hp, sc));
          mem.st(st.x[i] + 4 * v, x);
          mem.st(st.m[i] + 4 * v, m);
          if (A == 4) mem.st(st.v[i] + 4 * v, w);
        }
        if constexpr (SPREAD) {
          mem.st(contrib + 4 * v, acc);
        } else {
          mem.st(st.c + 4 * v, center_apply(c, acc, hp.inv_n));
          if constexpr (STALE) mem.st(st.prev + 4 * v, c);
        }
      }
      // all consumer warps are done reading the slot, then one release-arrive hands it back
      asm volatile("bar.sync 1, %0;" ::"n"(32 * kBulkConsumerWarps) : "memory");
      if (threadIdx.x == 0) mbar_arrive(&empty[slot]);
    }
    if (blockIdx.x == gridDim.x - 1 && threadIdx.x == 0) {
      if constexpr (SPREAD)
        spread_tail<OPT>(b.st[0], contrib, p_pad, hp);
      else
        for (int t = 0; t < b.nstages; ++t) stage_tail<N, OPT, STALE>(b.st[t], hp);
    }
  }
}

template <int N, int HINT, int OPT, int TILE, bool STALE = false>
__global__ void __launch_bounds__(kBulkThreads, 1) colocated_bulkpipe(const StageBatch b, const Hyper hp,
                                                                      int issue_lanes) {
  bulkpipe_body<N, HINT, OPT, TILE, false, STALE>(b, hp, nullptr, 0, issue_lanes);
}

// Spread local step (one replica) through the same bulk-copy pipeline: 4 input streams (x, g, state, x~;
// + v for Adam) arrive by cp.async.bulk into the smem ring; x, state and r leave by 128-bit stores.
template <int OPT, int TILE>
__global__ void __launch_bounds__(kBulkThreads, 1) spread_bulkpipe(const StageBatch b, const Hyper hp,
                                                                   float* __restrict__ contrib, int64_t p_pad,
                                                                   int issue_lanes) {
  bulkpipe_body<1, 0, OPT, TILE, true>(b, hp, contrib, p_pad, issue_lanes);
}

// ============================================================================
// Spread layout (one replica on this GPU): local step + contribution, and the
// owner-shard epilogue after the reduce-scatter.
// ============================================================================
template <int U, int OPT>
__global__ void __launch_bounds__(kThreads) spread_local(float* __restrict__ x, const float* __restrict__ g,
                                                         float* __restrict__ m, float* __restrict__ vs,
                                                         const float* __restrict__ center,
                                                         float* __restrict__ contrib, int64_t nvec, int64_t p,
                                                         int64_t p_pad, const Hyper hp, const StepCoef* scp) {
  const Mem<0> mem;
  const StepCoef sc = load_coef<OPT>(scp);
  WaveCursor cur{0, 0};
  int sidx;
  int64_t va, nv;
  while (wave_item_f(1, [&](int) { return nvec; }, (int64_t)kThreads * U, cur, sidx, va, nv)) {
    const int64_t ve = va + nv;
    for (int64_t base = va + threadIdx.x; base < ve; base += (int64_t)kThreads * U) {
      float4 xv[U], gv[U], mv[U], wv[U], cv[U];
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const int64_t v = base + (int64_t)u * kThreads;
        if (v < ve) {
          xv[u] = mem.ld(x + 4 * v);
          gv[u] = mem.ld_ro(g + 4 * v);
          mv[u] = mem.ld(m + 4 * v);
          if (two_state(OPT)) wv[u] = mem.ld(vs + 4 * v);
          cv[u] = mem.ld_ro(center + 4 * v);
        }
      }
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const int64_t v = base + (int64_t)u * kThreads;
        if (v < ve) {
          const float4 r = ea_vec<OPT>(xv[u], gv[u], mv[u], wv[u], cv[u], hp, sc);
          mem.st(x + 4 * v, xv[u]);
          mem.st(m + 4 * v, mv[u]);
          if (two_state(OPT)) mem.st(vs + 4 * v, wv[u]);
          mem.st(contrib + 4 * v, r);
        }
      }
    }
  }
  // scalar tail of the vector part and the zero padding of the contribution
  const int64_t gtid = (int64_t)blockIdx.x * kThreads + threadIdx.x;
  const int64_t gsz = (int64_t)gridDim.x * kThreads;
  for (int64_t j = 4 * nvec + gtid; j < p_pad; j += gsz) {
    if (j < p) {
      float xs = x[j], ms = m[j], ws = two_state(OPT) ? vs[j] : 0.f;
      contrib[j] = ea_elem<OPT>(xs, g[j], ms, ws, center[j], hp, sc);
      x[j] = xs;
      m[j] = ms;
      if (two_state(OPT)) vs[j] = ws;
    } else {
      contrib[j] = 0.f;
    }
  }
}

__global__ void __launch_bounds__(kThreads) spread_apply(float* __restrict__ shard, const float* __restrict__ red,
                                                         int64_t nvec, int64_t count, float inv_n) {
  const Mem<0> mem;
  const int64_t stride = (int64_t)gridDim.x * kThreads;
  for (int64_t v = (int64_t)blockIdx.x * kThreads + threadIdx.x; v < nvec; v += stride) {
    const float4 c = mem.ld(shard + 4 * v);
    const float4 r = mem.ld_ro(red + 4 * v);
    mem.st(shard + 4 * v, center_apply(c, r, inv_n));
  }
  const int64_t gtid = (int64_t)blockIdx.x * kThreads + threadIdx.x;
  for (int64_t j = 4 * nvec + gtid; j < count; j += stride) shard[j] = fmaf(red[j], inv_n, shard[j]);
}

// ---------------------------------------------------------------- launch helpers
// Grid-size knob for co-scheduling with compute (row a8):
// AVGPIPE_EA_GRID unset/0 = persistent (#SMs x occupancy); -1 = one work
// chunk per CTA; k > 0 = at most k CTAs.
int grid_knob() {
  static int v = [] {
    const char* e = std::getenv("AVGPIPE_EA_GRID");
    return e ? std::atoi(e) : 0;
  }();
  return v;
}

template <typename K>
int persistent_grid(K kernel, int64_t work_units, int num_sms, int threads = kThreads, size_t smem = 0) {
  int per_sm = 0;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kernel, threads, smem) != cudaSuccess || per_sm < 1)
    per_sm = 1;
  int64_t grid = (int64_t)num_sms * per_sm;
  const int knob = grid_knob();
  if (knob < 0) grid = work_units;
  else if (knob > 0 && knob < grid) grid = knob;
  if (grid > work_units) grid = work_units;
  if (grid > 0x7fffffff) grid = 0x7fffffff;
  return grid < 1 ? 1 : static_cast<int>(grid);
}

// L2 eviction-hint knob: AVGPIPE_EA_L2HINT=0|1, default 0 (SGD only).
int l2_hint() {
  static int v = [] {
    const char* e = std::getenv("AVGPIPE_EA_L2HINT");
    return (e && e[0] == '1') ? 1 : 0;
  }();
  return v;
}

int64_t units_of(const StageBatch& b, int64_t chunk) {
  int64_t units = 0;
  for (int i = 0; i < b.nstages; ++i) units += (b.st[i].p / 4 + chunk - 1) / chunk;
  return units < 1 ? 1 : units;
}

template <int N, int HINT, int U, int OPT = kOptSGD>
cudaError_t launch_regloop_u(const StageBatch& b, const Hyper& hp, int num_sms, cudaStream_t s) {
  auto k = colocated_regloop<N, U, HINT, OPT>;
  k<<<persistent_grid(k, units_of(b, kThreads * U), num_sms), kThreads, 0, s>>>(b, hp);
  return cudaGetLastError();
}

// Unroll knob for measurement: AVGPIPE_EA_REGLOOP_U=1 forces U=1 for N<=4.
int regloop_u1() {
  static int v = [] {
    const char* e = std::getenv("AVGPIPE_EA_REGLOOP_U");
    return (e && e[0] == '1') ? 1 : 0;
  }();
  return v;
}

template <int N, int HINT, int OPT = kOptSGD>
cudaError_t launch_regloop(const StageBatch& b, const Hyper& hp, int num_sms, cudaStream_t s) {
  constexpr int U = N <= 2 ? 4 : (N <= 4 ? 2 : 1);
  if (U > 1 && regloop_u1()) return launch_regloop_u<N, HINT, 1, OPT>(b, hp, num_sms, s);
  return launch_regloop_u<N, HINT, U, OPT>(b, hp, num_sms, s);
}

// Tuning knob for measurement: AVGPIPE_EA_LANE_TUNE=<passes><minblocks>: "23", "24", "81" (N=4,
// SGD), "22", "23", "31" (N=4, Adam).
int lane_tune() {
  static int v = [] {
    const char* e = std::getenv("AVGPIPE_EA_LANE_TUNE");
    return e ? std::atoi(e) : 0;
  }();
  return v;
}

template <int N, int HINT, int OPT, int PASSES, int MINB, bool STALE = false>
cudaError_t launch_laneshfl_t(const StageBatch& b, const Hyper& hp, int num_sms, cudaStream_t s) {
  auto k = colocated_laneshfl<N, HINT, OPT, PASSES, MINB, STALE>;
  k<<<persistent_grid(k, units_of(b, LaneGeom<N, PASSES>::kTileVec), num_sms), kThreads, 0, s>>>(b, hp);
  return cudaGetLastError();
}

template <int N, int HINT, int OPT>
cudaError_t launch_laneshfl(const StageBatch& b, const Hyper& hp, int num_sms, cudaStream_t s) {
  if constexpr (N == 4 && HINT == 0 && OPT == kOptSGD) {
    switch (lane_tune()) {
      case 23: return launch_laneshfl_t<N, HINT, OPT, 2, 3>(b, hp, num_sms, s);
      case 24: return launch_laneshfl_t<N, HINT, OPT, 2, 4>(b, hp, num_sms, s);
      case 81: return launch_laneshfl_t<N, HINT, OPT, 8, 1>(b, hp, num_sms, s);
      default: break;
    }
  }
  if constexpr (N == 4 && HINT == 0 && OPT == kOptAdam) {
    switch (lane_tune()) {
      case 22: return launch_laneshfl_t<N, HINT, OPT, 2, 2>(b, hp, num_sms, s);
      case 23: return launch_laneshfl_t<N, HINT, OPT, 2, 3>(b, hp, num_sms, s);
      case 31: return launch_laneshfl_t<N, HINT, OPT, 3, 1>(b, hp, num_sms, s);
      default: break;
    }
  }
  return launch_laneshfl_t<N, HINT, OPT, kLanePasses, 2>(b, hp, num_sms, s);  // <= 128 regs: 2 CTAs/SM
}

// Copy-issue knob for measurement: AVGPIPE_EA_BULK_ISSUE=1 issues every bulk copy of a slot from one
// producer lane (the first design); default: the 32 producer lanes issue them in parallel.
int bulk_issue_lanes() {
  static int v = [] {
    const char* e = std::getenv("AVGPIPE_EA_BULK_ISSUE");
    const int k = e ? std::atoi(e) : 32;
    return (k >= 1 && k <= 32) ? k : 32;
  }();
  return v;
}

template <int N, int HINT, int OPT, int TILE, bool STALE = false>
cudaError_t launch_bulkpipe_t(const StageBatch& b, const Hyper& hp, int num_sms, cudaStream_t s) {
  using G = BulkGeom<N, TILE, two_state(OPT) ? 4 : 3, STALE ? 1 : 0>;
  auto k = colocated_bulkpipe<N, HINT, OPT, TILE, STALE>;
  cudaError_t e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, G::kSmemBytes);
  if (e != cudaSuccess) return e;
  int64_t grid = num_sms;  // one block per SM (the ring takes most of shared memory)
  const int64_t units = units_of(b, G::kTile);
  if (grid > units) grid = units;
  k<<<static_cast<int>(grid), kBulkThreads, G::kSmemBytes, s>>>(b, hp, bulk_issue_lanes());
  return cudaGetLastError();
}

// Tile knob for measurement: AVGPIPE_EA_BULK_TILE = 64 | 128 | 256 | 512 float4 per array.
int bulk_tile() {
  static int v = [] {
    const char* e = std::getenv("AVGPIPE_EA_BULK_TILE");
    return e ? std::atoi(e) : 0;
  }();
  return v;
}

template <int N, int HINT, int OPT>
cudaError_t launch_bulkpipe(const StageBatch& b, const Hyper& hp, int num_sms, cudaStream_t s) {
  constexpr int A = two_state(OPT) ? 4 : 3;
  if constexpr (HINT == 0) {
    switch (bulk_tile()) {
      case 64: return launch_bulkpipe_t<N, HINT, OPT, 64>(b, hp, num_sms, s);
      case 128: return launch_bulkpipe_t<N, HINT, OPT, 128>(b, hp, num_sms, s);
      case 256:
        if constexpr ((A * N + 1) * 256 * 16 * 2 <= 200 * 1024) return launch_bulkpipe_t<N, HINT, OPT, 256>(b, hp, num_sms, s);
        break;
      case 512:
        if constexpr ((A * N + 1) * 512 * 16 * 2 <= 200 * 1024) return launch_bulkpipe_t<N, HINT, OPT, 512>(b, hp, num_sms, s);
        break;
      default: break;
    }
  }
  return launch_bulkpipe_t<N, HINT, OPT, default_bulk_tile<N, A>()>(b, hp, num_sms, s);
}

// Split register loop (variant 4): S = 2 lanes per column (N <= 4: S = 1 would be the plain register loop).
template <int N, int OPT>
cudaError_t launch_split(const StageBatch& b, const Hyper& hp, int num_sms, cudaStream_t s) {
  constexpr int S = N <= 4 ? 1 : 2;
  auto k = colocated_split<N, S, OPT>;
  k<<<persistent_grid(k, units_of(b, kThreads / S), num_sms), kThreads, 0, s>>>(b, hp);
  return cudaGetLastError();
}

// Warp per replica (variant 5): U = 4 float4 columns per lane and tile (2 KB rows per stream per tile), every
// optimizer (Adam(W) with U = 4, round 2 sessions g/h: N = 5 0.974 vs 0.69-0.87 with U = 2); measurement knob
// AVGPIPE_EA_WARPREP_U=2 gives Adam(W) U = 2.
int warprep_u4() {
  static const int v = [] {
    const char* e = std::getenv("AVGPIPE_EA_WARPREP_U");
    return (e && e[0] == '2') ? 0 : 1;
  }();
  return v;
}

template <int N, int OPT, int U, bool STALE>
cudaError_t launch_warprep_u(const StageBatch& b, const Hyper& hp, int num_sms, cudaStream_t s) {
  auto k = colocated_warprep<N, OPT, U, STALE>;
  k<<<persistent_grid(k, units_of(b, 32 * U), num_sms, 32 * N), 32 * N, 0, s>>>(b, hp);
  return cudaGetLastError();
}

template <int N, int OPT, bool STALE = false>
cudaError_t launch_warprep(const StageBatch& b, const Hyper& hp, int num_sms, cudaStream_t s) {
  if constexpr (two_state(OPT)) {
    if (!warprep_u4()) return launch_warprep_u<N, OPT, 2, STALE>(b, hp, num_sms, s);
  }
  return launch_warprep_u<N, OPT, 4, STALE>(b, hp, num_sms, s);
}

// Warp-specialised warp per replica (variant 6): U float4 columns per lane and tile, a ring of R = 4 contribution
// tiles.  Adam(W) with the synchronous center: U = 3 for N = 6, 7 (0.948 / 0.965; U = 2 keeps only 12 / 14 replica
// warps per SM in flight -- registers per SM sub-partition -- 0.836 / 0.908) and U = 2 for N = 8 (0.968; U = 3
// spills); else U = 4 (profiles/r02_s3_sweep_warpspec.jsonl, r02_s3_warpspec_u3.jsonl,
// r02_s3_ncu_warpspec_adam678.md).  Measurement knob AVGPIPE_EA_WARPSPEC_U = 2 | 3 | 4 overrides (3: Adam only).
int warpspec_u(int opt, bool stale, int n) {
  static const int v = [] {
    const char* e = std::getenv("AVGPIPE_EA_WARPSPEC_U");
    return e ? std::atoi(e) : 0;
  }();
  if (v == 2 || v == 4 || (v == 3 && two_state(opt))) return v;
  if (!two_state(opt)) return 4;
  // stale center (session x, profiles/r02_s3_stale_warpspec.jsonl): the same per-N choice except N = 3 (U = 4)
  if (stale && n == 3) return 4;
  return (n == 6 || n == 7) ? 3 : 2;
}

template <int N, int OPT, int U, int R, bool STALE>
cudaError_t launch_warpspec_t(const StageBatch& b, const Hyper& hp, int num_sms, cudaStream_t s) {
  auto k = colocated_warpspec<N, OPT, U, R, STALE>;
  constexpr size_t smem = sizeof(float4) * R * N * 32 * U;
  cudaError_t e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, static_cast<int>(smem));
  if (e != cudaSuccess) return e;
  k<<<persistent_grid(k, units_of(b, 32 * U), num_sms, 32 * (N + 1), smem), 32 * (N + 1), smem, s>>>(b, hp);
  return cudaGetLastError();
}

template <int N, int OPT, bool STALE = false>
cudaError_t launch_warpspec(const StageBatch& b, const Hyper& hp, int num_sms, cudaStream_t s) {
  const int u = warpspec_u(OPT, STALE, N);
  if (u == 2) return launch_warpspec_t<N, OPT, 2, 4, STALE>(b, hp, num_sms, s);
  if constexpr (two_state(OPT)) {  // U = 3 (Adam): more bytes in flight per warp at 2 CTAs per SM
    if (u == 3) return launch_warpspec_t<N, OPT, 3, 4, STALE>(b, hp, num_sms, s);
  }
  return launch_warpspec_t<N, OPT, 4, 4, STALE>(b, hp, num_sms, s);
}

template <int N>
cudaError_t launch_n(const StageBatch& b, const Hyper& hp, int opt, int variant, int num_sms, cudaStream_t s) {
  if (variant == kVariantWarpSpec) {
    switch (opt) {
      case kOptAdam: return launch_warpspec<N, kOptAdam>(b, hp, num_sms, s);
      case kOptAdamW: return launch_warpspec<N, kOptAdamW>(b, hp, num_sms, s);
      case kOptASGD: return launch_warpspec<N, kOptASGD>(b, hp, num_sms, s);
      default: return launch_warpspec<N, kOptSGD>(b, hp, num_sms, s);
    }
  }
  if (variant == kVariantWarpRep) {
    switch (opt) {
      case kOptAdam: return launch_warprep<N, kOptAdam>(b, hp, num_sms, s);
      case kOptAdamW: return launch_warprep<N, kOptAdamW>(b, hp, num_sms, s);
      case kOptASGD: return launch_warprep<N, kOptASGD>(b, hp, num_sms, s);
      default: return launch_warprep<N, kOptSGD>(b, hp, num_sms, s);
    }
  }
  if (variant == kVariantSplit) {
    switch (opt) {
      case kOptAdam: return launch_split<N, kOptAdam>(b, hp, num_sms, s);
      case kOptAdamW: return launch_split<N, kOptAdamW>(b, hp, num_sms, s);
      case kOptASGD: return launch_split<N, kOptASGD>(b, hp, num_sms, s);
      default: return launch_split<N, kOptSGD>(b, hp, num_sms, s);
    }
  }
  if (opt == kOptASGD) {  // SGD's streams and geometry (one state vector), no L2-hint variants
    if (variant == kVariantBulkPipe) return launch_bulkpipe<N, 0, kOptASGD>(b, hp, num_sms, s);
    if (variant == kVariantRegLoop) return launch_regloop<N, 0, kOptASGD>(b, hp, num_sms, s);
    return launch_laneshfl<N, 0, kOptASGD>(b, hp, num_sms, s);
  }
  if (opt != kOptSGD && variant == kVariantRegLoop)
    return opt == kOptAdam ? launch_regloop_u<N, 0, 1, kOptAdam>(b, hp, num_sms, s)
                           : launch_regloop_u<N, 0, 1, kOptAdamW>(b, hp, num_sms, s);
  if (opt != kOptSGD && variant == kVariantBulkPipe)
    return opt == kOptAdam ? launch_bulkpipe<N, 0, kOptAdam>(b, hp, num_sms, s)
                           : launch_bulkpipe<N, 0, kOptAdamW>(b, hp, num_sms, s);
  if (opt == kOptAdam) return launch_laneshfl<N, 0, kOptAdam>(b, hp, num_sms, s);
  if (opt == kOptAdamW) return launch_laneshfl<N, 0, kOptAdamW>(b, hp, num_sms, s);
  const bool hint = l2_hint() != 0;
  if (variant == kVariantBulkPipe)
    return hint ? launch_bulkpipe<N, 1, kOptSGD>(b, hp, num_sms, s) : launch_bulkpipe<N, 0, kOptSGD>(b, hp, num_sms, s);
  if (variant == kVariantRegLoop)
    return hint ? launch_regloop<N, 1>(b, hp, num_sms, s) : launch_regloop<N, 0>(b, hp, num_sms, s);
  return hint ? launch_laneshfl<N, 1, kOptSGD>(b, hp, num_sms, s) : launch_laneshfl<N, 0, kOptSGD>(b, hp, num_sms, s);
}

template <int OPT>
cudaError_t launch_wide_opt(const ReplicaTable& t, int n, float* center, float* prev, int64_t p, const Hyper& hp,
                            const StepCoef* sc, int num_sms, cudaStream_t s) {
  constexpr int U = 2;
  const int64_t nvec = p / 4;
  auto k = colocated_wide<U, OPT>;
  const int64_t units = (nvec + kThreads * U - 1) / (kThreads * U);
  k<<<persistent_grid(k, units < 1 ? 1 : units, num_sms), kThreads, 0, s>>>(t, n, center, prev, nvec, p, hp, sc);
  return cudaGetLastError();
}

// Spread local kernel knob (measurement): AVGPIPE_EA_SPREAD_KERNEL=reg selects the register kernel
// (spread_local); default: the bulk-copy pipeline (spread_bulkpipe).  (A warp-per-replica spread kernel measured
// 0.90-0.94 vs 0.94-0.97 for the bulk-copy pipeline on C3-C5 stages: profiles/r02_s3_spread_local_warp.jsonl.)
int spread_reg() {
  static int v = [] {
    const char* e = std::getenv("AVGPIPE_EA_SPREAD_KERNEL");
    return (e && e[0] == 'r') ? 1 : 0;
  }();
  return v;
}

template <int OPT, int TILE>
cudaError_t launch_spread_bulk_t(float* x, const float* g, float* m, float* v, const float* center, float* contrib,
                                 int64_t p, int64_t p_pad, const Hyper& hp, const StepCoef* sc, int num_sms,
                                 cudaStream_t s) {
  constexpr int A = two_state(OPT) ? 4 : 3;
  using G = BulkGeom<1, TILE, A>;
  auto k = spread_bulkpipe<OPT, TILE>;
  cudaError_t e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, G::kSmemBytes);
  if (e != cudaSuccess) return e;
  StageBatch b;
  b.nstages = 1;
  StageRefs& r = b.st[0];
  for (int i = 0; i < kMaxFusedN; ++i) {
    r.x[i] = i == 0 ? x : nullptr;
    r.g[i] = i == 0 ? g : nullptr;
    r.m[i] = i == 0 ? m : nullptr;
    r.v[i] = i == 0 ? v : nullptr;
  }
  r.c = const_cast<float*>(center);  // read only (SPREAD)
  r.p = p;
  r.scp = sc;
  int64_t grid = num_sms;
  const int64_t units = (p / 4 + TILE - 1) / TILE;
  if (grid > units) grid = units < 1 ? 1 : units;
  k<<<static_cast<int>(grid), kBulkThreads, G::kSmemBytes, s>>>(b, hp, contrib, p_pad, bulk_issue_lanes());
  return cudaGetLastError();
}

// Spread local kernel tile (measurement knob AVGPIPE_EA_BULK_TILE = 128 | 256 | 512 float4 per stream copy;
// default 256, i.e. 4 KB copies).
template <int OPT>
cudaError_t launch_spread_bulk(float* x, const float* g, float* m, float* v, const float* center, float* contrib,
                               int64_t p, int64_t p_pad, const Hyper& hp, const StepCoef* sc, int num_sms,
                               cudaStream_t s) {
  switch (bulk_tile()) {
    case 128: return launch_spread_bulk_t<OPT, 128>(x, g, m, v, center, contrib, p, p_pad, hp, sc, num_sms, s);
    case 512: return launch_spread_bulk_t<OPT, 512>(x, g, m, v, center, contrib, p, p_pad, hp, sc, num_sms, s);
    default: return launch_spread_bulk_t<OPT, 256>(x, g, m, v, center, contrib, p, p_pad, hp, sc, num_sms, s);
  }
}

template <int OPT>
cudaError_t launch_spread_local_opt(float* x, const float* g, float* m, float* v, const float* center,
                                    float* contrib, int64_t p, int64_t p_pad, const Hyper& hp, const StepCoef* sc,
                                    int num_sms, cudaStream_t s) {
  if (!spread_reg()) return launch_spread_bulk<OPT>(x, g, m, v, center, contrib, p, p_pad, hp, sc, num_sms, s);
  constexpr int U = two_state(OPT) ? 2 : 4;
  const int64_t nvec = p / 4;
  auto k = spread_local<U, OPT>;
  int64_t units = (nvec + kThreads * U - 1) / (kThreads * U);
  if (units < 1) units = 1;
  k<<<persistent_grid(k, units, num_sms), kThreads, 0, s>>>(x, g, m, v, center, contrib, nvec, p, p_pad, hp, sc);
  return cudaGetLastError();
}

// Step counter + the step's coefficients, on the stream (graph-capturable): Adam(W) bias corrections, or
// ASGD's eta_t and mu_t (torch.optim.ASGD's state after t-1 steps: eta = lr / (1 + l lr (t-1))^a,
// mu = 1 / max(1, t-1-t0); eta_1 = lr, mu_1 = 1).
__global__ void advance_steps(int64_t* steps, uint32_t* xepoch, StepCoef* coef, const StageList list,
                              const CoefParams cp) {
  const int i = threadIdx.x;
  if (i >= list.count) return;
  const int s = list.idx[i];
  const int64_t t = ++steps[s];
  if (xepoch) ++xepoch[s];
  if (cp.opt == kOptASGD) {
    const double k = (double)(t - 1);
    coef[s].step_size = static_cast<float>(cp.lr / pow(1.0 + cp.lambd * cp.lr * k, cp.asgd_alpha));
    coef[s].inv_sqrt_bc2 = static_cast<float>(1.0 / fmax(1.0, k - cp.t0));
    return;
  }
  const double bc1 = 1.0 - pow(cp.beta1, (double)t);
  const double bc2 = 1.0 - pow(cp.beta2, (double)t);
  coef[s].step_size = bc1 > 0.0 ? static_cast<float>(cp.lr / bc1) : 0.f;
  coef[s].inv_sqrt_bc2 = bc2 > 0.0 ? static_cast<float>(1.0 / sqrt(bc2)) : 0.f;
}

}  // namespace

cudaError_t launch_advance_steps(int64_t* steps, uint32_t* xepoch, StepCoef* coef, const StageList& list,
                                 const CoefParams& cp, cudaStream_t s) {
  if (list.count <= 0) return cudaSuccess;
  advance_steps<<<1, 32, 0, s>>>(steps, xepoch, coef, list, cp);
  return cudaGetLastError();
}

cudaError_t launch_colocated_batch(const StageBatch& b, int n, const Hyper& hp, int opt, int variant, int num_sms,
                                   cudaStream_t s) {
  if (b.nstages <= 0) return cudaSuccess;
  // library default per N, measured on B200 (C2 sizes; profiles/r01_nsweep*.jsonl, r01_s2_*.jsonl):
  // SGD: the bulk-copy pipeline for N = 1, 5, 6, 7 (0.88-0.96 / 0.95 / 0.96 / 0.955 of peak), the lane kernel
  // for N = 2..4 (0.96 / 0.93 / 0.97-0.99; a warp holds >= 8 lanes per replica row), the register loop for
  // N = 8 (0.98-0.99).  Adam(W): the lane kernel for N = 1 (0.915), the register loop for N = 2, 3 (0.96 /
  // 0.95; bulk pipeline 0.88 / 0.90), the bulk-copy pipeline for N = 4 (0.97), the split register loop for
  // N = 5, 6 (round 2, same box: 0.950 / 0.930 vs 0.930 / 0.906 for the bulk pipeline); N > 6 goes to the
  // replica-loop kernel (ea_api.cu).  ASGD: SGD's choice except the split register loop for N = 5, 6 (0.967 /
  // 0.941 vs 0.920 / 0.937; profiles/r02_sweep_split.jsonl -- with SGD it measured below the bulk pipeline).
  // Round 2 session h (same box, C2 sizes): Adam N = 5 on the warp-per-replica kernel with U = 4, 0.974 (session
  // g) / split 0.944-0.950; N = 2, 3 within 1% of the register loop (0.960 / 0.941 vs 0.948 / 0.940), kept.
  // Sessions o/v: Adam N = 6..8 on the warp-specialised kernel (U = 3 / 3 / 2): 0.948 / 0.965 / 0.968 vs 0.928 split,
  // 0.919 / 0.923 replica loop.
  if (variant == kVariantAuto && two_state(opt))
    variant = n == 1 ? kVariantLaneShfl
                     : (n <= 3 ? kVariantRegLoop
                               : (n == 4 ? kVariantBulkPipe : (n == 5 ? kVariantWarpRep : kVariantWarpSpec)));
  // SGD-momentum and ASGD (one state vector), round 2: the warp-per-replica kernel for N = 1 and 3..8 (same box,
  // C2 sizes: N = 1 0.937 vs 0.872 bulk pipeline, N = 3 0.986 vs 0.932 lane, N = 4 0.996-0.998 vs 0.983 lane,
  // N = 5..8 0.979-1.0 vs 0.93-0.976; ASGD alike), the lane kernel for N = 2 (0.963 vs 0.952);
  // profiles/r02_sweep_warprep*.jsonl.  (Its Adam instances run out of registers: 0.69-0.87.)
  // Session o: N = 5 on the warp-specialised kernel (SGD 1.001 / ASGD 0.995 vs 0.987 / 0.984 warp per replica).
  if (variant == kVariantAuto) variant = n == 2 ? kVariantLaneShfl : (n == 5 ? kVariantWarpSpec : kVariantWarpRep);
  switch (n) {
    case 1: return launch_n<1>(b, hp, opt, variant, num_sms, s);
    case 2: return launch_n<2>(b, hp, opt, variant, num_sms, s);
    case 3: return launch_n<3>(b, hp, opt, variant, num_sms, s);
    case 4: return launch_n<4>(b, hp, opt, variant, num_sms, s);
    case 5: return launch_n<5>(b, hp, opt, variant, num_sms, s);
    case 6: return launch_n<6>(b, hp, opt, variant, num_sms, s);
    case 7: return launch_n<7>(b, hp, opt, variant, num_sms, s);
    case 8: return launch_n<8>(b, hp, opt, variant, num_sms, s);
    default: return cudaErrorInvalidValue;
  }
}

// Stale center through the bulk-copy pipeline (N = 1: the lane kernel's double-buffered pair of center tiles does
// not fit its static shared memory; N = 5: the lane kernel would idle 3 of 8 lanes).  Measured on B200 (C2 sizes,
// profiles/r02_sweep_kernels.jsonl): N = 1 0.964 vs 0.777 for the replica loop, N = 5 0.958 vs 0.951; from N = 6
// on the replica loop is better and the library uses it.
template <int N>
cudaError_t launch_stale_bulk_n(const StageBatch& b, const Hyper& hp, int opt, int num_sms, cudaStream_t s) {
  switch (opt) {
    case kOptAdam: return launch_bulkpipe_t<N, 0, kOptAdam, default_bulk_tile<N, 4, 1>(), true>(b, hp, num_sms, s);
    case kOptAdamW: return launch_bulkpipe_t<N, 0, kOptAdamW, default_bulk_tile<N, 4, 1>(), true>(b, hp, num_sms, s);
    case kOptASGD: return launch_bulkpipe_t<N, 0, kOptASGD, default_bulk_tile<N, 3, 1>(), true>(b, hp, num_sms, s);
    default: return launch_bulkpipe_t<N, 0, kOptSGD, default_bulk_tile<N, 3, 1>(), true>(b, hp, num_sms, s);
  }
}

template <int N>
cudaError_t launch_stale_n(const StageBatch& b, const Hyper& hp, int opt, int num_sms, cudaStream_t s) {
  switch (opt) {
    case kOptAdam: return launch_laneshfl_t<N, 0, kOptAdam, kLanePasses, 2, true>(b, hp, num_sms, s);
    case kOptAdamW: return launch_laneshfl_t<N, 0, kOptAdamW, kLanePasses, 2, true>(b, hp, num_sms, s);
    case kOptASGD: return launch_laneshfl_t<N, 0, kOptASGD, kLanePasses, 2, true>(b, hp, num_sms, s);
    default: return launch_laneshfl_t<N, 0, kOptSGD, kLanePasses, 2, true>(b, hp, num_sms, s);
  }
}

template <int N>
cudaError_t launch_stale_warpspec_n(const StageBatch& b, const Hyper& hp, int opt, int num_sms, cudaStream_t s) {
  switch (opt) {
    case kOptAdam: return launch_warpspec<N, kOptAdam, true>(b, hp, num_sms, s);
    case kOptAdamW: return launch_warpspec<N, kOptAdamW, true>(b, hp, num_sms, s);
    case kOptASGD: return launch_warpspec<N, kOptASGD, true>(b, hp, num_sms, s);
    default: return launch_warpspec<N, kOptSGD, true>(b, hp, num_sms, s);
  }
}

template <int N>
cudaError_t launch_stale_warprep_n(const StageBatch& b, const Hyper& hp, int opt, int num_sms, cudaStream_t s) {
  switch (opt) {
    case kOptAdam: return launch_warprep<N, kOptAdam, true>(b, hp, num_sms, s);
    case kOptAdamW: return launch_warprep<N, kOptAdamW, true>(b, hp, num_sms, s);
    case kOptASGD: return launch_warprep<N, kOptASGD, true>(b, hp, num_sms, s);
    default: return launch_warprep<N, kOptSGD, true>(b, hp, num_sms, s);
  }
}

cudaError_t launch_colocated_batch_stale(const StageBatch& b, int n, const Hyper& hp, int opt, int variant,
                                         int num_sms, cudaStream_t s) {
  if (b.nstages <= 0) return cudaSuccess;
  for (int t = 0; t < b.nstages; ++t)
    if (!b.st[t].prev) return cudaErrorInvalidValue;
  // default (round 2, profiles/r02_sweep_warprep_stale.jsonl): SGD/ASGD N = 2 and 5 on the warp-per-replica
  // kernel (0.969 vs 0.923 lane, 0.971 vs 0.958 bulk pipeline); N = 1 the bulk pipeline, N = 3, 4 the lane kernel
  if (variant == kVariantAuto && !two_state(opt) && (n == 2 || n == 5)) variant = kVariantWarpRep;
  // sessions o/x: Adam(W) N = 1, 3, 5-8 on the warp-specialised kernel (N = 3 0.933-0.944 vs 0.865 lane kernel;
  // N = 1 0.895 vs 0.864 bulk-copy pipeline; N = 5 / 6 / 7 / 8 0.953 / 0.952 / 0.971 / 0.963 vs 0.92 replica loop)
  if (variant == kVariantAuto && two_state(opt) && n != 2 && n != 4) variant = kVariantWarpSpec;
  if (variant == kVariantWarpSpec) {
    switch (n) {
      case 1: return launch_stale_warpspec_n<1>(b, hp, opt, num_sms, s);
      case 2: return launch_stale_warpspec_n<2>(b, hp, opt, num_sms, s);
      case 3: return launch_stale_warpspec_n<3>(b, hp, opt, num_sms, s);
      case 4: return launch_stale_warpspec_n<4>(b, hp, opt, num_sms, s);
      case 5: return launch_stale_warpspec_n<5>(b, hp, opt, num_sms, s);
      case 6: return launch_stale_warpspec_n<6>(b, hp, opt, num_sms, s);
      case 7: return launch_stale_warpspec_n<7>(b, hp, opt, num_sms, s);
      case 8: return launch_stale_warpspec_n<8>(b, hp, opt, num_sms, s);
      default: return cudaErrorInvalidValue;
    }
  }
  if (variant == kVariantWarpRep) {
    switch (n) {
      case 1: return launch_stale_warprep_n<1>(b, hp, opt, num_sms, s);
      case 2: return launch_stale_warprep_n<2>(b, hp, opt, num_sms, s);
      case 3: return launch_stale_warprep_n<3>(b, hp, opt, num_sms, s);
      case 4: return launch_stale_warprep_n<4>(b, hp, opt, num_sms, s);
      case 5: return launch_stale_warprep_n<5>(b, hp, opt, num_sms, s);
      case 6: return launch_stale_warprep_n<6>(b, hp, opt, num_sms, s);
      case 7: return launch_stale_warprep_n<7>(b, hp, opt, num_sms, s);
      case 8: return launch_stale_warprep_n<8>(b, hp, opt, num_sms, s);
      default: return cudaErrorInvalidValue;
    }
  }
  switch (n) {
    case 1: return launch_stale_bulk_n<1>(b, hp, opt, num_sms, s);
    case 2: return launch_stale_n<2>(b, hp, opt, num_sms, s);
    case 3: return launch_stale_n<3>(b, hp, opt, num_sms, s);
    case 4: return launch_stale_n<4>(b, hp, opt, num_sms, s);
    case 5: return launch_stale_bulk_n<5>(b, hp, opt, num_sms, s);
    default: return cudaErrorInvalidValue;
  }
}

cudaError_t launch_colocated_wide(const ReplicaTable& t, int n, float* center, float* prev, int64_t p, const Hyper& hp,
                                  int opt, const StepCoef* sc, int num_sms, cudaStream_t s) {
  if (p <= 0) return cudaSuccess;
  if (opt == kOptAdam) return launch_wide_opt<kOptAdam>(t, n, center, prev, p, hp, sc, num_sms, s);
  if (opt == kOptAdamW) return launch_wide_opt<kOptAdamW>(t, n, center, prev, p, hp, sc, num_sms, s);
  if (opt == kOptASGD) return launch_wide_opt<kOptASGD>(t, n, center, prev, p, hp, sc, num_sms, s);
  return launch_wide_opt<kOptSGD>(t, n, center, prev, p, hp, sc, num_sms, s);
}

cudaError_t launch_spread_local(float* x, const float* g, float* m, float* v, const float* center, float* contrib,
                                int64_t p, int64_t p_pad, const Hyper& hp, int opt, const StepCoef* sc, int num_sms,
                                cudaStream_t s) {
  if (p_pad <= 0) return cudaSuccess;
  if (opt == kOptAdam)
    return launch_spread_local_opt<kOptAdam>(x, g, m, v, center, contrib, p, p_pad, hp, sc, num_sms, s);
  if (opt == kOptAdamW)
    return launch_spread_local_opt<kOptAdamW>(x, g, m, v, center, contrib, p, p_pad, hp, sc, num_sms, s);
  if (opt == kOptASGD)
    return launch_spread_local_opt<kOptASGD>(x, g, m, v, center, contrib, p, p_pad, hp, sc, num_sms, s);
  return launch_spread_local_opt<kOptSGD>(x, g, m, v, center, contrib, p, p_pad, hp, sc, num_sms, s);
}

cudaError_t launch_spread_apply(float* shard, const float* reduced, int64_t count, float inv_n, int num_sms,
                                int max_ctas, cudaStream_t s) {
  if (count <= 0) return cudaSuccess;
  const int64_t nvec = count / 4;
  const int64_t units = (nvec + kThreads - 1) / kThreads;
  int grid = persistent_grid(spread_apply, units < 1 ? 1 : units, num_sms);
  if (max_ctas > 0 && grid > max_ctas) grid = max_ctas;  // side stream: a small SM footprint beside the compute
  spread_apply<<<grid, kThreads, 0, s>>>(shard, reduced, nvec, count, inv_n);
  return cudaGetLastError();
}

}  // namespace ea

// Fused elastic-averaging kernels for sm_100a (B200).
//
// Per element j of a stage and replica i (§3.2; DESIGN.md c1-c14):
//   g'  = g_i + wd*x_i                          Step 1: SGD-momentum local update
//   m_i = mu*m_i + g'
//   D_i = -lr * (nesterov ? g' + mu*m_i : m_i)
//   x_i = (1-alpha)*x_i + alpha*x~ + D_i         Step 2: (1-a):a dilution + local update
//   R  += rho*D_i + beta*(x_i - x~)              Steps 3-4: send + accumulate
//   x~  = x~ + R/N                               Step 5: normalise + apply
//
// The path is elementwise plus a reduction over the N replicas: ~0.5 flop per
// byte, far below the fp32 ridge, so every kernel here is HBM-bound and is
// written for bytes in flight: 128-bit coalesced accesses, no shared-memory
// round trips for data that is used once, persistent grids (#SMs x resident
// blocks) over which the work of ALL stages of a launch is split evenly, so
// no SM idles in a ragged last wave.  Tensor cores are not used (no contraction).
#include <cuda_runtime.h>
#include <stdint.h>

#include <cstdlib>

#include "ea_internal.h"

namespace ea {
namespace {

constexpr int kThreads = 256;

// ---------------------------------------------------------------- memory ops
// HINT = 0: plain streaming (L1 bypass); HINT = 1: additionally mark every
// access L2 evict-first (the data is touched once per step and the working
// set is far above the 126 MB L2).
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

// ---------------------------------------------------------------- the math
// One (replica, element) update; returns the replica's contribution r_i.
__device__ __forceinline__ float ea_elem(float& x, float g, float& m, float c, const Hyper& hp) {
  const float gg = fmaf(hp.wd, x, g);             // g + lambda*x
  const float mn = fmaf(hp.momentum, m, gg);      // mu*m + g'
  const float d = hp.nesterov ? fmaf(hp.momentum, mn, gg) : mn;
  const float delta = -hp.lr * d;                 // local update Delta_i (Step 1)
  const float gap = x - c;                        // x_i - x~ (pre-step values, c1/c2)
  const float r = fmaf(hp.beta, gap, hp.rho * delta);
  x = fmaf(-hp.alpha, gap, x) + delta;            // (1-a)x + a*x~ + Delta (Step 2)
  m = mn;
  return r;
}

__device__ __forceinline__ float4 ea_vec(float4& x, float4 g, float4& m, float4 c, const Hyper& hp) {
  float4 r;
  r.x = ea_elem(x.x, g.x, m.x, c.x, hp);
  r.y = ea_elem(x.y, g.y, m.y, c.y, hp);
  r.z = ea_elem(x.z, g.z, m.z, c.z, hp);
  r.w = ea_elem(x.w, g.w, m.w, c.w, hp);
  return r;
}

__device__ __forceinline__ void add4(float4& a, float4 b) {
  a.x += b.x; a.y += b.y; a.z += b.z; a.w += b.w;
}
__device__ __forceinline__ float4 center_apply(float4 c, float4 acc, float inv_n) {
  return make_float4(fmaf(acc.x, inv_n, c.x), fmaf(acc.y, inv_n, c.y), fmaf(acc.z, inv_n, c.z),
                     fmaf(acc.w, inv_n, c.w));
}

// Scalar tail of one stage: elements [4*(p/4), p) (fewer than 4), one thread.
template <int N>
__device__ void stage_tail(const StageRefs& st, const Hyper& hp) {
  for (int64_t j = (st.p / 4) * 4; j < st.p; ++j) {
    const float c = st.c[j];
    float acc = 0.f;
#pragma unroll
    for (int i = 0; i < N; ++i) {
      float x = st.x[i][j], m = st.m[i][j];
      acc += ea_elem(x, st.g[i][j], m, c, hp);
      st.x[i][j] = x;
      st.m[i][j] = m;
    }
    st.c[j] = fmaf(acc, hp.inv_n, c);
  }
}

// Even split of [0, total) units over the grid: this block's [lo, hi).
__device__ __forceinline__ void block_range(int64_t total, int64_t& lo, int64_t& hi) {
  lo = total * blockIdx.x / gridDim.x;
  hi = total * (blockIdx.x + 1) / gridDim.x;
}

// ============================================================================
// Variant 1: register-resident replica loop.
// One thread owns U float4 of a center; it issues all (3N+1)*U 128-bit loads
// before any arithmetic (maximal memory-level parallelism per thread: the
// replica pointers may alias as far as the compiler knows, so the loads are
// hoisted by hand), shares the center value across the N replicas in
// registers, reduces the N contributions in registers and writes x_i, m_i
// and x~ once.  Work unit: kUnitVec float4 (512 B); the units of all stages
// of the launch are concatenated and split evenly over the persistent grid.
// ============================================================================
constexpr int kUnitVec = 32;

template <int N, int U, int HINT>
__device__ __forceinline__ void regloop_range(const StageRefs& st, int64_t va, int64_t ve, const Hyper& hp,
                                              const Mem<HINT>& mem) {
  for (int64_t base = va + threadIdx.x; base < ve; base += (int64_t)kThreads * U) {
    float4 c[U], x[N][U], g[N][U], m[N][U];
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
        add4(acc, ea_vec(x[i][u], g[i][u], m[i][u], c[u], hp));
        mem.st(st.x[i] + 4 * v, x[i][u]);
        mem.st(st.m[i] + 4 * v, m[i][u]);
      }
      mem.st(st.c + 4 * v, center_apply(c[u], acc, hp.inv_n));
    }
  }
}

template <int N, int U, int HINT>
__global__ void __launch_bounds__(kThreads) colocated_regloop(const StageBatch b, const Hyper hp) {
  const Mem<HINT> mem;
  int64_t begin[kMaxLaunchStages + 1];
  begin[0] = 0;
  for (int s = 0; s < b.nstages; ++s) begin[s + 1] = begin[s] + (b.st[s].p / 4 + kUnitVec - 1) / kUnitVec;
  int64_t lo, hi;
  block_range(begin[b.nstages], lo, hi);
  int s = 0;
  for (int64_t pos = lo; pos < hi;) {
    while (pos >= begin[s + 1]) ++s;
    const int64_t end = hi < begin[s + 1] ? hi : begin[s + 1];
    const int64_t nvec = b.st[s].p / 4;
    const int64_t va = (pos - begin[s]) * kUnitVec;
    int64_t ve = (end - begin[s]) * kUnitVec;
    if (ve > nvec) ve = nvec;
    regloop_range<N, U, HINT>(b.st[s], va, ve, hp, mem);
    pos = end;
  }
  if (blockIdx.x == gridDim.x - 1 && threadIdx.x == 0)
    for (int t = 0; t < b.nstages; ++t) stage_tail<N>(b.st[t], hp);
}

// Runtime-N fallback (N > 8): one stage, replicas visited in a loop.
template <int U>
__global__ void __launch_bounds__(kThreads) colocated_wide(const ReplicaTable t, int n, float* __restrict__ center,
                                                           int64_t nvec, int64_t p, const Hyper hp) {
  const Mem<0> mem;
  int64_t lo, hi;
  block_range((nvec + kUnitVec - 1) / kUnitVec, lo, hi);
  const int64_t va = lo * kUnitVec, ve = hi * kUnitVec < nvec ? hi * kUnitVec : nvec;
  for (int64_t base = va + threadIdx.x; base < ve; base += (int64_t)kThreads * U) {
    float4 c[U], acc[U];
    bool ok[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int64_t v = base + (int64_t)u * kThreads;
      ok[u] = v < ve;
      acc[u] = make_float4(0.f, 0.f, 0.f, 0.f);
      if (ok[u]) c[u] = mem.ld(center + 4 * v);
    }
    for (int i = 0; i < n; ++i) {
      float4 x[U], g[U], m[U];
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const int64_t v = base + (int64_t)u * kThreads;
        if (ok[u]) {
          x[u] = mem.ld(t.x[i] + 4 * v);
          g[u] = mem.ld_ro(t.g[i] + 4 * v);
          m[u] = mem.ld(t.m[i] + 4 * v);
        }
      }
#pragma unroll
      for (int u = 0; u < U; ++u) {
        if (!ok[u]) continue;
        const int64_t v = base + (int64_t)u * kThreads;
        add4(acc[u], ea_vec(x[u], g[u], m[u], c[u], hp));
        mem.st(t.x[i] + 4 * v, x[u]);
        mem.st(t.m[i] + 4 * v, m[u]);
      }
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int64_t v = base + (int64_t)u * kThreads;
      if (ok[u]) mem.st(center + 4 * v, center_apply(c[u], acc[u], hp.inv_n));
    }
  }
  if (blockIdx.x == gridDim.x - 1 && threadIdx.x == 0) {
    for (int64_t j = 4 * nvec; j < p; ++j) {
      const float c = center[j];
      float acc = 0.f;
      for (int i = 0; i < n; ++i) {
        float x = t.x[i][j], m = t.m[i][j];
        acc += ea_elem(x, t.g[i][j], m, c, hp);
        t.x[i][j] = x;
        t.m[i][j] = m;
      }
      center[j] = fmaf(acc, hp.inv_n, c);
    }
  }
}

// ============================================================================
// Variant 2: lanes = (replica, float4 chunk), center tile staged in shared
// memory by the bulk-copy engine (cp.async.bulk + mbarrier, double-buffered),
// replica reduction by warp shuffles.
//
// The tiles (kTileVec float4 of a center) of all stages of the launch are
// concatenated and split evenly over the persistent grid; a block walks its
// contiguous tiles and thread 0 prefetches tile k+1 (possibly of the next
// stage) with one cp.async.bulk while the block computes tile k.  Inside a
// warp, lane l works on replica l / CH and chunk l % CH (CH = 32/NP, NP = N
// rounded up to a power of two), so each replica's CH lanes read CH*16
// contiguous bytes of x_i, g_i, m_i, and the NP lanes of one chunk read the
// same center word from shared memory (a broadcast).  The N contributions of a
// chunk are reduced with log2(NP) __shfl_xor steps; replica-0 lanes write x~.
// ============================================================================
constexpr int kLanePasses = 4;  // float4 chunks per lane per tile (3 loads each in flight)

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n"
      ".reg .pred P1;\n"
      "WAIT_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n"
      "@!P1 bra WAIT_%=;\n"
      "}\n" ::"r"(smem_u32(bar)),
      "r"(parity)
      : "memory");
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}
__device__ __forceinline__ void fence_proxy_async() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}

template <int N>
struct LanePow2 {
  static constexpr int value = N <= 1 ? 1 : N <= 2 ? 2 : N <= 4 ? 4 : N <= 8 ? 8 : 16;
};

template <int N>
struct LaneGeom {
  static constexpr int NP = LanePow2<N>::value;
  static constexpr int CH = 32 / NP;                              // chunks per warp pass
  static constexpr int kVecPerWarp = kLanePasses * CH;            // float4 of a tile per warp
  static constexpr int kTileVec = (kThreads / 32) * kVecPerWarp;  // float4 of center per tile
};

template <int N, int HINT>
__global__ void __launch_bounds__(kThreads) colocated_laneshfl(const StageBatch b, const Hyper hp) {
  using G = LaneGeom<N>;
  constexpr int CH = G::CH, kPasses = kLanePasses, kVecPerWarp = G::kVecPerWarp, kTileVec = G::kTileVec;
  __shared__ __align__(128) float4 s_center[2][kTileVec];
  __shared__ __align__(8) uint64_t s_bar[2];
  const Mem<HINT> mem;

  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int rep = lane / CH, chunk = lane % CH;
  const bool active = rep < N;

  int64_t begin[kMaxLaunchStages + 1];
  begin[0] = 0;
  for (int s = 0; s < b.nstages; ++s) begin[s + 1] = begin[s] + (b.st[s].p / 4 + kTileVec - 1) / kTileVec;
  int64_t lo, hi;
  block_range(begin[b.nstages], lo, hi);

  if (threadIdx.x == 0) {
    mbar_init(&s_bar[0], 1);
    mbar_init(&s_bar[1], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();

  auto locate = [&](int64_t tile, int& s, int64_t& v0, int64_t& nv) {
    while (tile >= begin[s + 1]) ++s;
    const int64_t nvec = b.st[s].p / 4;
    v0 = (tile - begin[s]) * kTileVec;
    nv = (nvec - v0) < kTileVec ? (nvec - v0) : kTileVec;
  };
  auto issue = [&](int64_t tile, int buf) {
    int s = 0;
    int64_t v0, nv;
    locate(tile, s, v0, nv);
    const uint32_t bytes = static_cast<uint32_t>(nv * 16);
    mbar_expect_tx(&s_bar[buf], bytes);
    bulk_g2s(&s_center[buf][0], b.st[s].c + 4 * v0, bytes, &s_bar[buf]);
  };

  if (threadIdx.x == 0 && lo < hi) issue(lo, 0);
  uint32_t phase[2] = {0u, 0u};
  int buf = 0, s = 0;

  for (int64_t tile = lo; tile < hi; ++tile) {
    if (threadIdx.x == 0 && tile + 1 < hi) {
      fence_proxy_async();  // buffer buf^1 was last read through the generic proxy
      issue(tile + 1, buf ^ 1);
    }
    int64_t v0, nv;
    locate(tile, s, v0, nv);
    const StageRefs& st = b.st[s];
    float* xi = nullptr;
    const float* gi = nullptr;
    float* mi = nullptr;
#pragma unroll
    for (int i = 0; i < N; ++i)
      if (rep == i) { xi = st.x[i]; gi = st.g[i]; mi = st.m[i]; }

    // replica streams first (they do not depend on the center tile)
    float4 x[kPasses], g[kPasses], m[kPasses];
#pragma unroll
    for (int k = 0; k < kPasses; ++k) {
      const int lv = warp * kVecPerWarp + k * CH + chunk;
      if (active && lv < nv) {
        const int64_t v = v0 + lv;
        x[k] = mem.ld(xi + 4 * v);
        g[k] = mem.ld_ro(gi + 4 * v);
        m[k] = mem.ld(mi + 4 * v);
      }
    }
    mbar_wait(&s_bar[buf], phase[buf]);
    phase[buf] ^= 1u;
#pragma unroll
    for (int k = 0; k < kPasses; ++k) {
      const int lv = warp * kVecPerWarp + k * CH + chunk;
      const bool in = lv < nv;  // uniform across the NP lanes of a chunk
      const float4 c = in ? s_center[buf][lv] : make_float4(0.f, 0.f, 0.f, 0.f);
      float4 r = make_float4(0.f, 0.f, 0.f, 0.f);
      if (active && in) {
        r = ea_vec(x[k], g[k], m[k], c, hp);
        const int64_t v = v0 + lv;
        mem.st(xi + 4 * v, x[k]);
        mem.st(mi + 4 * v, m[k]);
      }
#pragma unroll
      for (int off = CH; off < 32; off <<= 1) {
        r.x += __shfl_xor_sync(0xffffffffu, r.x, off);
        r.y += __shfl_xor_sync(0xffffffffu, r.y, off);
        r.z += __shfl_xor_sync(0xffffffffu, r.z, off);
        r.w += __shfl_xor_sync(0xffffffffu, r.w, off);
      }
      if (rep == 0 && in) mem.st(st.c + 4 * (v0 + lv), center_apply(c, r, hp.inv_n));
    }
    __syncthreads();  // everyone done reading s_center[buf] before it is refilled
    buf ^= 1;
  }
  if (blockIdx.x == gridDim.x - 1 && threadIdx.x == 0)
    for (int t = 0; t < b.nstages; ++t) stage_tail<N>(b.st[t], hp);
}

// ============================================================================
// Spread layout (one replica on this GPU): local step + contribution, and the
// owner-shard epilogue after the reduce-scatter.
// ============================================================================
template <int U>
__global__ void __launch_bounds__(kThreads) spread_local(float* __restrict__ x, const float* __restrict__ g,
                                                         float* __restrict__ m, const float* __restrict__ center,
                                                         float* __restrict__ contrib, int64_t nvec, int64_t p,
                                                         int64_t p_pad, const Hyper hp) {
  const Mem<0> mem;
  int64_t lo, hi;
  block_range((nvec + kUnitVec - 1) / kUnitVec, lo, hi);
  const int64_t va = lo * kUnitVec, ve = hi * kUnitVec < nvec ? hi * kUnitVec : nvec;
  for (int64_t base = va + threadIdx.x; base < ve; base += (int64_t)kThreads * U) {
    float4 xv[U], gv[U], mv[U], cv[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int64_t v = base + (int64_t)u * kThreads;
      if (v < ve) {
        xv[u] = mem.ld(x + 4 * v);
        gv[u] = mem.ld_ro(g + 4 * v);
        mv[u] = mem.ld(m + 4 * v);
        cv[u] = mem.ld_ro(center + 4 * v);
      }
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int64_t v = base + (int64_t)u * kThreads;
      if (v < ve) {
        const float4 r = ea_vec(xv[u], gv[u], mv[u], cv[u], hp);
        mem.st(x + 4 * v, xv[u]);
        mem.st(m + 4 * v, mv[u]);
        mem.st(contrib + 4 * v, r);
      }
    }
  }
  // scalar tail of the vector part and the zero padding of the contribution
  const int64_t gtid = (int64_t)blockIdx.x * kThreads + threadIdx.x;
  const int64_t gsz = (int64_t)gridDim.x * kThreads;
  for (int64_t j = 4 * nvec + gtid; j < p_pad; j += gsz) {
    if (j < p) {
      float xs = x[j], ms = m[j];
      contrib[j] = ea_elem(xs, g[j], ms, center[j], hp);
      x[j] = xs;
      m[j] = ms;
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
template <typename K>
int persistent_grid(K kernel, int64_t work_units, int num_sms) {
  int per_sm = 0;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kernel, kThreads, 0) != cudaSuccess || per_sm < 1)
    per_sm = 1;
  int64_t grid = (int64_t)num_sms * per_sm;
  if (grid > work_units) grid = work_units;
  return grid < 1 ? 1 : static_cast<int>(grid);
}

// L2 eviction-hint knob: AVGPIPE_EA_L2HINT=0|1, default 0.
int l2_hint() {
  static int v = [] {
    const char* e = std::getenv("AVGPIPE_EA_L2HINT");
    return (e && e[0] == '1') ? 1 : 0;
  }();
  return v;
}

template <int N, int HINT>
cudaError_t launch_regloop(const StageBatch& b, const Hyper& hp, int num_sms, cudaStream_t s) {
  constexpr int U = N <= 2 ? 4 : (N <= 4 ? 2 : 1);
  int64_t units = 0;
  for (int i = 0; i < b.nstages; ++i) units += (b.st[i].p / 4 + kUnitVec - 1) / kUnitVec;
  auto k = colocated_regloop<N, U, HINT>;
  k<<<persistent_grid(k, units, num_sms), kThreads, 0, s>>>(b, hp);
  return cudaGetLastError();
}

template <int N, int HINT>
cudaError_t launch_laneshfl(const StageBatch& b, const Hyper& hp, int num_sms, cudaStream_t s) {
  constexpr int kTileVec = LaneGeom<N>::kTileVec;
  int64_t units = 0;
  for (int i = 0; i < b.nstages; ++i) units += (b.st[i].p / 4 + kTileVec - 1) / kTileVec;
  auto k = colocated_laneshfl<N, HINT>;
  k<<<persistent_grid(k, units, num_sms), kThreads, 0, s>>>(b, hp);
  return cudaGetLastError();
}

template <int N>
cudaError_t launch_n(const StageBatch& b, const Hyper& hp, int variant, int num_sms, cudaStream_t s) {
  const bool hint = l2_hint() != 0;
  if (variant == kVariantRegLoop)
    return hint ? launch_regloop<N, 1>(b, hp, num_sms, s) : launch_regloop<N, 0>(b, hp, num_sms, s);
  return hint ? launch_laneshfl<N, 1>(b, hp, num_sms, s) : launch_laneshfl<N, 0>(b, hp, num_sms, s);
}

}  // namespace

cudaError_t launch_colocated_batch(const StageBatch& b, int n, const Hyper& hp, int variant, int num_sms,
                                   cudaStream_t s) {
  if (b.nstages <= 0) return cudaSuccess;
  // default: the lane/shuffle kernel with the bulk-staged center (measured faster, profiles/r01_*)
  const int v = variant == kVariantAuto ? kVariantLaneShfl : variant;
  switch (n) {
    case 1: return launch_n<1>(b, hp, v, num_sms, s);
    case 2: return launch_n<2>(b, hp, v, num_sms, s);
    case 3: return launch_n<3>(b, hp, v, num_sms, s);
    case 4: return launch_n<4>(b, hp, v, num_sms, s);
    case 5: return launch_n<5>(b, hp, v, num_sms, s);
    case 6: return launch_n<6>(b, hp, v, num_sms, s);
    case 7: return launch_n<7>(b, hp, v, num_sms, s);
    case 8: return launch_n<8>(b, hp, v, num_sms, s);
    default: return cudaErrorInvalidValue;
  }
}

cudaError_t launch_colocated_wide(const ReplicaTable& t, int n, float* center, int64_t p, const Hyper& hp,
                                  int num_sms, cudaStream_t s) {
  if (p <= 0) return cudaSuccess;
  constexpr int U = 2;
  const int64_t nvec = p / 4;
  auto k = colocated_wide<U>;
  k<<<persistent_grid(k, (nvec + kUnitVec - 1) / kUnitVec, num_sms), kThreads, 0, s>>>(t, n, center, nvec, p, hp);
  return cudaGetLastError();
}

cudaError_t launch_spread_local(float* x, const float* g, float* m, const float* center, float* contrib, int64_t p,
                                int64_t p_pad, const Hyper& hp, int num_sms, cudaStream_t s) {
  if (p_pad <= 0) return cudaSuccess;
  constexpr int U = 4;
  const int64_t nvec = p / 4;
  auto k = spread_local<U>;
  int64_t units = (nvec + kUnitVec - 1) / kUnitVec;
  if (units < 1) units = 1;
  k<<<persistent_grid(k, units, num_sms), kThreads, 0, s>>>(x, g, m, center, contrib, nvec, p, p_pad, hp);
  return cudaGetLastError();
}

cudaError_t launch_spread_apply(float* shard, const float* reduced, int64_t count, float inv_n, int num_sms,
                                cudaStream_t s) {
  if (count <= 0) return cudaSuccess;
  const int64_t nvec = count / 4;
  const int grid = persistent_grid(spread_apply, (nvec + kThreads - 1) / kThreads > 0 ? (nvec + kThreads - 1) / kThreads : 1,
                                   num_sms);
  spread_apply<<<grid, kThreads, 0, s>>>(shard, reduced, nvec, count, inv_n);
  return cudaGetLastError();
}

}  // namespace ea

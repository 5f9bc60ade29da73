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
// round trips for data that is used once, grids sized in multiples of the SM
// count.  Tensor cores are not used (no contraction).
#include <cuda_runtime.h>
#include <stdint.h>

#include "ea_internal.h"

namespace ea {
namespace {

constexpr int kThreads = 256;

// ---------------------------------------------------------------- memory ops
__device__ __forceinline__ float4 ld_na(const float* p) {  // read-write data, skip L1
  float4 v;
  asm volatile("ld.global.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];"
               : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w)
               : "l"(p));
  return v;
}
__device__ __forceinline__ float4 ld_ro(const float* p) {  // read-only stream (gradients)
  float4 v;
  asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];"
               : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w)
               : "l"(p));
  return v;
}
__device__ __forceinline__ void st_na(float* p, float4 v) {
  asm volatile("st.global.L1::no_allocate.v4.f32 [%0], {%1,%2,%3,%4};" ::"l"(p), "f"(v.x), "f"(v.y),
               "f"(v.z), "f"(v.w)
               : "memory");
}

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

// Scalar tail: elements [4*nvec, p) (fewer than 4), one thread.
__device__ void colocated_tail(const ReplicaTable& t, int n, float* center, int64_t begin, int64_t p,
                               const Hyper& hp) {
  for (int64_t j = begin; j < p; ++j) {
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

// ============================================================================
// Variant 1: register-resident replica loop.
// One thread owns U float4 of the center; it issues all (3N+1)*U 128-bit loads
// before any arithmetic (maximal memory-level parallelism per thread: the
// replica pointers may alias as far as the compiler knows, so the loads are
// hoisted by hand), shares the center value across the N replicas in
// registers, reduces the N contributions in registers and writes x_i, m_i
// and x~ once.  Grid-stride over a persistent grid (multiple of #SMs).
// ============================================================================
template <int N, int U>
__global__ void __launch_bounds__(kThreads) colocated_regloop(const ReplicaTable t, float* __restrict__ center,
                                                              int64_t nvec, int64_t p, const Hyper hp) {
  const int64_t stride = (int64_t)gridDim.x * kThreads * U;
  for (int64_t base = (int64_t)blockIdx.x * kThreads * U + threadIdx.x; base < nvec; base += stride) {
    float4 c[U], x[N][U], g[N][U], m[N][U];
    bool ok[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int64_t v = base + (int64_t)u * kThreads;
      ok[u] = v < nvec;
      if (ok[u]) c[u] = ld_na(center + 4 * v);
    }
#pragma unroll
    for (int i = 0; i < N; ++i) {
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const int64_t v = base + (int64_t)u * kThreads;
        if (ok[u]) {
          x[i][u] = ld_na(t.x[i] + 4 * v);
          g[i][u] = ld_ro(t.g[i] + 4 * v);
          m[i][u] = ld_na(t.m[i] + 4 * v);
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
        st_na(t.x[i] + 4 * v, x[i][u]);
        st_na(t.m[i] + 4 * v, m[i][u]);
      }
      st_na(center + 4 * v, center_apply(c[u], acc, hp.inv_n));
    }
  }
  if (blockIdx.x == 0 && threadIdx.x == 0 && 4 * nvec < p) colocated_tail(t, N, center, 4 * nvec, p, hp);
}

// Runtime-N fallback (N > 8): same dataflow, replicas visited in a loop.
template <int U>
__global__ void __launch_bounds__(kThreads) colocated_regloop_dyn(const ReplicaTable t, int n,
                                                                  float* __restrict__ center, int64_t nvec,
                                                                  int64_t p, const Hyper hp) {
  const int64_t stride = (int64_t)gridDim.x * kThreads * U;
  for (int64_t base = (int64_t)blockIdx.x * kThreads * U + threadIdx.x; base < nvec; base += stride) {
    float4 c[U], acc[U];
    bool ok[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int64_t v = base + (int64_t)u * kThreads;
      ok[u] = v < nvec;
      acc[u] = make_float4(0.f, 0.f, 0.f, 0.f);
      if (ok[u]) c[u] = ld_na(center + 4 * v);
    }
    for (int i = 0; i < n; ++i) {
      float4 x[U], g[U], m[U];
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const int64_t v = base + (int64_t)u * kThreads;
        if (ok[u]) {
          x[u] = ld_na(t.x[i] + 4 * v);
          g[u] = ld_ro(t.g[i] + 4 * v);
          m[u] = ld_na(t.m[i] + 4 * v);
        }
      }
#pragma unroll
      for (int u = 0; u < U; ++u) {
        if (!ok[u]) continue;
        const int64_t v = base + (int64_t)u * kThreads;
        add4(acc[u], ea_vec(x[u], g[u], m[u], c[u], hp));
        st_na(t.x[i] + 4 * v, x[u]);
        st_na(t.m[i] + 4 * v, m[u]);
      }
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int64_t v = base + (int64_t)u * kThreads;
      if (ok[u]) st_na(center + 4 * v, center_apply(c[u], acc[u], hp.inv_n));
    }
  }
  if (blockIdx.x == 0 && threadIdx.x == 0 && 4 * nvec < p) colocated_tail(t, n, center, 4 * nvec, p, hp);
}

// ============================================================================
// Variant 2: lanes = (replica, float4 chunk), center tile staged in shared
// memory by the bulk-copy engine (cp.async.bulk + mbarrier, double-buffered),
// replica reduction by warp shuffles.
//
// A block walks tiles of kTileVec float4 of the center.  Thread 0 prefetches
// tile k+1 with one cp.async.bulk while the block computes tile k.  Inside a
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
__global__ void __launch_bounds__(kThreads) colocated_laneshfl(const ReplicaTable t, float* __restrict__ center,
                                                               int64_t nvec, int64_t p, const Hyper hp) {
  constexpr int NP = LanePow2<N>::value;
  constexpr int CH = 32 / NP;                      // chunks per warp pass
  constexpr int kWarps = kThreads / 32;
  constexpr int kPasses = kLanePasses;
  constexpr int kVecPerWarp = kPasses * CH;        // float4 of a tile handled by one warp
  constexpr int kTileVec = kWarps * kVecPerWarp;   // float4 of center per tile
  __shared__ __align__(128) float4 s_center[2][kTileVec];
  __shared__ __align__(8) uint64_t s_bar[2];

  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int rep = lane / CH, chunk = lane % CH;
  const bool active = rep < N;
  const int64_t ntiles = (nvec + kTileVec - 1) / kTileVec;

  if (threadIdx.x == 0) {
    mbar_init(&s_bar[0], 1);
    mbar_init(&s_bar[1], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();

  auto issue = [&](int64_t tile, int buf) {
    const int64_t v0 = tile * kTileVec;
    const int64_t nv = (nvec - v0) < kTileVec ? (nvec - v0) : kTileVec;
    const uint32_t bytes = static_cast<uint32_t>(nv * 16);
    mbar_expect_tx(&s_bar[buf], bytes);
    bulk_g2s(&s_center[buf][0], center + 4 * v0, bytes, &s_bar[buf]);
  };

  int64_t tile = blockIdx.x;
  if (threadIdx.x == 0 && tile < ntiles) issue(tile, 0);
  uint32_t phase[2] = {0u, 0u};
  int buf = 0;
  float* const xi = active ? t.x[rep] : nullptr;
  const float* const gi = active ? t.g[rep] : nullptr;
  float* const mi = active ? t.m[rep] : nullptr;

  for (; tile < ntiles; tile += gridDim.x) {
    const int64_t next = tile + gridDim.x;
    if (threadIdx.x == 0 && next < ntiles) {
      fence_proxy_async();  // buffer buf^1 was last read through the generic proxy
      issue(next, buf ^ 1);
    }
    const int64_t v0 = tile * kTileVec;
    const int64_t nv = (nvec - v0) < kTileVec ? (nvec - v0) : kTileVec;

    // replica streams first (they do not depend on the center tile)
    float4 x[kPasses], g[kPasses], m[kPasses];
#pragma unroll
    for (int k = 0; k < kPasses; ++k) {
      const int lv = warp * kVecPerWarp + k * CH + chunk;
      if (active && lv < nv) {
        const int64_t v = v0 + lv;
        x[k] = ld_na(xi + 4 * v);
        g[k] = ld_ro(gi + 4 * v);
        m[k] = ld_na(mi + 4 * v);
      }
    }
    mbar_wait(&s_bar[buf], phase[buf]);
    phase[buf] ^= 1u;
#pragma unroll
    for (int k = 0; k < kPasses; ++k) {
      const int lv = warp * kVecPerWarp + k * CH + chunk;
      const bool in = lv < nv;                       // uniform across the NP lanes of a chunk
      const float4 c = in ? s_center[buf][lv] : make_float4(0.f, 0.f, 0.f, 0.f);
      float4 r = make_float4(0.f, 0.f, 0.f, 0.f);
      if (active && in) {
        r = ea_vec(x[k], g[k], m[k], c, hp);
        const int64_t v = v0 + lv;
        st_na(xi + 4 * v, x[k]);
        st_na(mi + 4 * v, m[k]);
      }
#pragma unroll
      for (int off = CH; off < 32; off <<= 1) {
        r.x += __shfl_xor_sync(0xffffffffu, r.x, off);
        r.y += __shfl_xor_sync(0xffffffffu, r.y, off);
        r.z += __shfl_xor_sync(0xffffffffu, r.z, off);
        r.w += __shfl_xor_sync(0xffffffffu, r.w, off);
      }
      if (rep == 0 && in) st_na(center + 4 * (v0 + lv), center_apply(c, r, hp.inv_n));
    }
    __syncthreads();  // everyone done reading s_center[buf] before it is refilled
    buf ^= 1;
  }
  if (blockIdx.x == 0 && threadIdx.x == 0 && 4 * nvec < p) colocated_tail(t, N, center, 4 * nvec, p, hp);
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
  const int64_t stride = (int64_t)gridDim.x * kThreads * U;
  for (int64_t base = (int64_t)blockIdx.x * kThreads * U + threadIdx.x; base < nvec; base += stride) {
    float4 xv[U], gv[U], mv[U], cv[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int64_t v = base + (int64_t)u * kThreads;
      if (v < nvec) {
        xv[u] = ld_na(x + 4 * v);
        gv[u] = ld_ro(g + 4 * v);
        mv[u] = ld_na(m + 4 * v);
        cv[u] = ld_ro(center + 4 * v);
      }
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int64_t v = base + (int64_t)u * kThreads;
      if (v < nvec) {
        const float4 r = ea_vec(xv[u], gv[u], mv[u], cv[u], hp);
        st_na(x + 4 * v, xv[u]);
        st_na(m + 4 * v, mv[u]);
        st_na(contrib + 4 * v, r);
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
  const int64_t stride = (int64_t)gridDim.x * kThreads;
  for (int64_t v = (int64_t)blockIdx.x * kThreads + threadIdx.x; v < nvec; v += stride) {
    const float4 c = ld_na(shard + 4 * v);
    const float4 r = ld_ro(red + 4 * v);
    st_na(shard + 4 * v, center_apply(c, r, inv_n));
  }
  const int64_t gtid = (int64_t)blockIdx.x * kThreads + threadIdx.x;
  for (int64_t j = 4 * nvec + gtid; j < count; j += stride) shard[j] = fmaf(red[j], inv_n, shard[j]);
}

// ---------------------------------------------------------------- launch helpers
template <typename K>
int grid_for(K kernel, int64_t work_items, int num_sms, int smem = 0) {
  int per_sm = 0;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kernel, kThreads, smem) != cudaSuccess || per_sm < 1)
    per_sm = 1;
  const int64_t full = (int64_t)num_sms * per_sm;
  const int64_t need = (work_items + kThreads - 1) / kThreads;
  int64_t grid = need < full ? need : full;
  return grid < 1 ? 1 : static_cast<int>(grid);
}

template <int N>
cudaError_t launch_regloop_n(const ReplicaTable& t, float* center, int64_t p, const Hyper& hp, int num_sms,
                             cudaStream_t s) {
  constexpr int U = N <= 2 ? 4 : (N <= 4 ? 2 : 1);
  const int64_t nvec = p / 4;
  auto k = colocated_regloop<N, U>;
  const int grid = grid_for(k, (nvec + U - 1) / U, num_sms);
  k<<<grid, kThreads, 0, s>>>(t, center, nvec, p, hp);
  return cudaGetLastError();
}

template <int N>
cudaError_t launch_laneshfl_n(const ReplicaTable& t, float* center, int64_t p, const Hyper& hp, int num_sms,
                              cudaStream_t s) {
  constexpr int kTileVec = (kThreads / 32) * kLanePasses * (32 / LanePow2<N>::value);
  const int64_t nvec = p / 4;
  const int64_t ntiles = (nvec + kTileVec - 1) / kTileVec;
  auto k = colocated_laneshfl<N>;
  int per_sm = 0;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k, kThreads, 0) != cudaSuccess || per_sm < 1)
    per_sm = 1;
  int64_t grid = (int64_t)num_sms * per_sm;
  if (grid > ntiles) grid = ntiles;
  if (grid < 1) grid = 1;
  k<<<static_cast<int>(grid), kThreads, 0, s>>>(t, center, nvec, p, hp);
  return cudaGetLastError();
}

}  // namespace

cudaError_t launch_colocated(const ReplicaTable& t, int n, float* center, int64_t p, const Hyper& hp, int variant,
                             int num_sms, cudaStream_t s) {
  if (p <= 0) return cudaSuccess;
  if (variant == kVariantLaneShfl && n <= 8) {
    switch (n) {
      case 1: return launch_laneshfl_n<1>(t, center, p, hp, num_sms, s);
      case 2: return launch_laneshfl_n<2>(t, center, p, hp, num_sms, s);
      case 3: return launch_laneshfl_n<3>(t, center, p, hp, num_sms, s);
      case 4: return launch_laneshfl_n<4>(t, center, p, hp, num_sms, s);
      case 5: return launch_laneshfl_n<5>(t, center, p, hp, num_sms, s);
      case 6: return launch_laneshfl_n<6>(t, center, p, hp, num_sms, s);
      case 7: return launch_laneshfl_n<7>(t, center, p, hp, num_sms, s);
      case 8: return launch_laneshfl_n<8>(t, center, p, hp, num_sms, s);
    }
  }
  switch (n) {
    case 1: return launch_regloop_n<1>(t, center, p, hp, num_sms, s);
    case 2: return launch_regloop_n<2>(t, center, p, hp, num_sms, s);
    case 3: return launch_regloop_n<3>(t, center, p, hp, num_sms, s);
    case 4: return launch_regloop_n<4>(t, center, p, hp, num_sms, s);
    case 5: return launch_regloop_n<5>(t, center, p, hp, num_sms, s);
    case 6: return launch_regloop_n<6>(t, center, p, hp, num_sms, s);
    case 7: return launch_regloop_n<7>(t, center, p, hp, num_sms, s);
    case 8: return launch_regloop_n<8>(t, center, p, hp, num_sms, s);
    default: {
      constexpr int U = 2;
      const int64_t nvec = p / 4;
      auto k = colocated_regloop_dyn<U>;
      const int grid = grid_for(k, (nvec + U - 1) / U, num_sms);
      k<<<grid, kThreads, 0, s>>>(t, n, center, nvec, p, hp);
      return cudaGetLastError();
    }
  }
}

cudaError_t launch_spread_local(float* x, const float* g, float* m, const float* center, float* contrib, int64_t p,
                                int64_t p_pad, const Hyper& hp, int num_sms, cudaStream_t s) {
  if (p_pad <= 0) return cudaSuccess;
  constexpr int U = 4;
  const int64_t nvec = p / 4;
  auto k = spread_local<U>;
  int64_t items = (nvec + U - 1) / U;
  if (items < p_pad - 4 * nvec) items = p_pad - 4 * nvec;
  const int grid = grid_for(k, items, num_sms);
  k<<<grid, kThreads, 0, s>>>(x, g, m, center, contrib, nvec, p, p_pad, hp);
  return cudaGetLastError();
}

cudaError_t launch_spread_apply(float* shard, const float* reduced, int64_t count, float inv_n, int num_sms,
                                cudaStream_t s) {
  if (count <= 0) return cudaSuccess;
  const int64_t nvec = count / 4;
  const int grid = grid_for(spread_apply, nvec > 0 ? nvec : 1, num_sms);
  spread_apply<<<grid, kThreads, 0, s>>>(shard, reduced, nvec, count, inv_n);
  return cudaGetLastError();
}

}  // namespace ea

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
// blocks) sweeping the stages of a launch in waves with the ragged remainder
// split evenly (wave_item), so no SM idles in a partial last wave.  Tensor
// cores are not used (no contraction).
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

// Wave schedule over the stages of a launch.  Chunks of C float4: in stage s
// the grid sweeps full waves (chunk w*G + b for block b, so the G blocks of
// a wave touch one contiguous window of every stream -- DRAM-page friendly),
// then the ragged remainder R < G*C is split evenly over all G blocks (no
// block idles in a partial last wave).  Every block walks the same sequence
// of (stage, wave) items, so the cursor is warp- and block-uniform.
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
// Variant 1: register-resident replica loop.
// One thread owns U float4 of a center; it issues all (3N+1)*U 128-bit loads
// before any arithmetic (maximal memory-level parallelism per thread: the
// replica pointers may alias as far as the compiler knows, so the loads are
// hoisted by hand), shares the center value across the N replicas in
// registers, reduces the N contributions in registers and writes x_i, m_i
// and x~ once.  Work unit: kThreads*U float4 per block, scheduled by wave_item.
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
  WaveCursor cur{0, 0};
  int s;
  int64_t v0, nv;
  while (wave_item(b, (int64_t)kThreads * U, cur, s, v0, nv)) regloop_range<N, U, HINT>(b.st[s], v0, v0 + nv, hp, mem);
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

template <int N, int PASSES = kLanePasses>
struct LaneGeom {
  static constexpr int NP = LanePow2<N>::value;
  static constexpr int CH = 32 / NP;                              // chunks per warp pass
  static constexpr int kVecPerWarp = PASSES * CH;                 // float4 of a tile per warp
  static constexpr int kTileVec = (kThreads / 32) * kVecPerWarp;  // float4 of center per tile
};

template <int N, int HINT, int PASSES = kLanePasses, int MINB = 1>
__global__ void __launch_bounds__(kThreads, MINB) colocated_laneshfl(const StageBatch b, const Hyper hp) {
  using G = LaneGeom<N, PASSES>;
  constexpr int CH = G::CH, kPasses = PASSES, kVecPerWarp = G::kVecPerWarp, kTileVec = G::kTileVec;
  __shared__ __align__(128) float4 s_center[2][kTileVec];
  __shared__ __align__(8) uint64_t s_bar[2];
  const Mem<HINT> mem;

  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int rep = lane / CH, chunk = lane % CH;
  const bool active = rep < N;

  if (threadIdx.x == 0) {
    mbar_init(&s_bar[0], 1);
    mbar_init(&s_bar[1], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();

  auto issue = [&](int s, int64_t v0, int64_t nv, int buf) {
    const uint32_t bytes = static_cast<uint32_t>(nv * 16);
    mbar_expect_tx(&s_bar[buf], bytes);
    bulk_g2s(&s_center[buf][0], b.st[s].c + 4 * v0, bytes, &s_bar[buf]);
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
    have = have_next;
    s = s_next;
    v0 = v0_next;
    nv = nv_next;
  }
  if (blockIdx.x == gridDim.x - 1 && threadIdx.x == 0)
    for (int t = 0; t < b.nstages; ++t) stage_tail<N>(b.st[t], hp);
}

// ============================================================================
// Variant 3: bulk-copy load pipeline (TMA engine feeds shared memory).
//
// One producer warp (one elected thread) streams every input of a tile --
// x~ and x_i, g_i, m_i of all N replicas, (3N+1) 1-D cp.async.bulk copies of
// kBulkTile float4 each -- into a kBulkStages-deep ring of shared-memory
// slots, completing on a per-slot "full" mbarrier with the byte count.  Eight
// consumer warps read a slot (one float4 column per thread: the x~ value is
// shared by the N replica rows in registers), update in registers, write x_i,
// m_i and x~ straight to HBM with 128-bit stores, and release the slot on its
// "empty" mbarrier (one arrive per consumer warp).  Requests reach the memory
// system as (3N+1) x 4 KB bulk reads per tile instead of 16-byte loads, and the
// loads of up to kBulkStages tiles are in flight per SM with no registers
// held for them.  Tiles follow the same wave schedule as the other variants.
// ============================================================================
constexpr int kBulkConsumerWarps = 8;
constexpr int kBulkThreads = 32 * (kBulkConsumerWarps + 1);

template <int N>
struct BulkGeom {
  // float4 per array per tile: keep one slot <= ~56 KB
  static constexpr int kTile = (3 * N + 1) * 256 * 16 <= 57344 ? 256 : 128;
  static constexpr int kSlotVec = (3 * N + 1) * kTile;  // float4 per slot
  static constexpr int kStages = (kSlotVec * 16 * 4 <= 200 * 1024) ? 4 : 3;
  static constexpr int kSmemBytes = kStages * kSlotVec * 16 + 2 * kStages * 8;
};

__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}

template <int N, int HINT>
__global__ void __launch_bounds__(kBulkThreads, 1) colocated_bulkpipe(const StageBatch b, const Hyper hp) {
  using G = BulkGeom<N>;
  constexpr int T = G::kTile, S = G::kStages;
  extern __shared__ __align__(128) float4 smem[];
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + S * G::kSlotVec);
  uint64_t* empty = full + S;
  const Mem<HINT> mem;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;

  if (threadIdx.x == 0) {
    for (int i = 0; i < S; ++i) {
      mbar_init(&full[i], 1);
      mbar_init(&empty[i], kBulkConsumerWarps);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();

  if (warp == kBulkConsumerWarps) {
    // ---------------- producer: one thread issues every bulk copy
    if (lane == 0) {
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
        mbar_expect_tx(&full[slot], bytes * (3 * N + 1));
        bulk_g2s(base, st.c + 4 * v0, bytes, &full[slot]);
#pragma unroll
        for (int i = 0; i < N; ++i) {
          bulk_g2s(base + (1 + 3 * i) * T, st.x[i] + 4 * v0, bytes, &full[slot]);
          bulk_g2s(base + (2 + 3 * i) * T, st.g[i] + 4 * v0, bytes, &full[slot]);
          bulk_g2s(base + (3 + 3 * i) * T, st.m[i] + 4 * v0, bytes, &full[slot]);
        }
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
      for (int lv = threadIdx.x; lv < nv; lv += 32 * kBulkConsumerWarps) {
        const float4 c = base[lv];
        float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
        const int64_t v = v0 + lv;
#pragma unroll
        for (int i = 0; i < N; ++i) {
          float4 x = base[(1 + 3 * i) * T + lv];
          const float4 g = base[(2 + 3 * i) * T + lv];
          float4 m = base[(3 + 3 * i) * T + lv];
          add4(acc, ea_vec(x, g, m, c, hp));
          mem.st(st.x[i] + 4 * v, x);
          mem.st(st.m[i] + 4 * v, m);
        }
        mem.st(st.c + 4 * v, center_apply(c, acc, hp.inv_n));
      }
      __syncwarp();
      if (lane == 0) mbar_arrive(&empty[slot]);  // release: this warp's smem reads are done
    }
    if (blockIdx.x == gridDim.x - 1 && threadIdx.x == 0)
      for (int t = 0; t < b.nstages; ++t) stage_tail<N>(b.st[t], hp);
  }
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
  WaveCursor cur{0, 0};
  int sidx;
  int64_t va0, nv0;
  while (wave_item_f(1, [&](int) { return nvec; }, (int64_t)kThreads * U, cur, sidx, va0, nv0)) {
    const int64_t va = va0, ve = va0 + nv0;
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
// Grid-size knob for co-scheduling with compute (row a8):
// AVGPIPE_EA_GRID unset/0 = persistent (#SMs x occupancy); -1 = one work
// chunk per CTA (short CTAs the block scheduler can interleave with other
// streams' kernels); k > 0 = at most k CTAs.
int grid_knob() {
  static int v = [] {
    const char* e = std::getenv("AVGPIPE_EA_GRID");
    return e ? std::atoi(e) : 0;
  }();
  return v;
}

template <typename K>
int persistent_grid(K kernel, int64_t work_units, int num_sms) {
  int per_sm = 0;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kernel, kThreads, 0) != cudaSuccess || per_sm < 1)
    per_sm = 1;
  int64_t grid = (int64_t)num_sms * per_sm;
  const int knob = grid_knob();
  if (knob < 0) grid = work_units;
  else if (knob > 0 && knob < grid) grid = knob;
  if (grid > work_units) grid = work_units;
  if (grid > 0x7fffffff) grid = 0x7fffffff;
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

template <int N, int HINT, int U>
cudaError_t launch_regloop_u(const StageBatch& b, const Hyper& hp, int num_sms, cudaStream_t s) {
  int64_t units = 0;
  for (int i = 0; i < b.nstages; ++i) units += (b.st[i].p / 4 + kThreads * U - 1) / (kThreads * U);
  auto k = colocated_regloop<N, U, HINT>;
  k<<<persistent_grid(k, units, num_sms), kThreads, 0, s>>>(b, hp);
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

template <int N, int HINT>
cudaError_t launch_regloop(const StageBatch& b, const Hyper& hp, int num_sms, cudaStream_t s) {
  constexpr int U = N <= 2 ? 4 : (N <= 4 ? 2 : 1);
  if (U > 1 && regloop_u1()) return launch_regloop_u<N, HINT, 1>(b, hp, num_sms, s);
  return launch_regloop_u<N, HINT, U>(b, hp, num_sms, s);
}

// Tuning knob for measurement: AVGPIPE_EA_LANE_TUNE=<passes><minblocks>: "23", "24", "81" (N=4 only).
int lane_tune() {
  static int v = [] {
    const char* e = std::getenv("AVGPIPE_EA_LANE_TUNE");
    return e ? std::atoi(e) : 0;
  }();
  return v;
}

template <int N, int HINT, int PASSES, int MINB>
cudaError_t launch_laneshfl_t(const StageBatch& b, const Hyper& hp, int num_sms, cudaStream_t s) {
  constexpr int kTileVec = LaneGeom<N, PASSES>::kTileVec;
  int64_t units = 0;
  for (int i = 0; i < b.nstages; ++i) units += (b.st[i].p / 4 + kTileVec - 1) / kTileVec;
  if (units < 1) units = 1;
  auto k = colocated_laneshfl<N, HINT, PASSES, MINB>;
  k<<<persistent_grid(k, units, num_sms), kThreads, 0, s>>>(b, hp);
  return cudaGetLastError();
}

template <int N, int HINT>
cudaError_t launch_laneshfl(const StageBatch& b, const Hyper& hp, int num_sms, cudaStream_t s) {
  if constexpr (N == 4 && HINT == 0) {
    switch (lane_tune()) {
      case 23: return launch_laneshfl_t<N, HINT, 2, 3>(b, hp, num_sms, s);
      case 24: return launch_laneshfl_t<N, HINT, 2, 4>(b, hp, num_sms, s);
      case 81: return launch_laneshfl_t<N, HINT, 8, 1>(b, hp, num_sms, s);
      default: break;
    }
  }
  constexpr int kTileVec = LaneGeom<N>::kTileVec;
  int64_t units = 0;
  for (int i = 0; i < b.nstages; ++i) units += (b.st[i].p / 4 + kTileVec - 1) / kTileVec;
  if (units < 1) units = 1;
  auto k = colocated_laneshfl<N, HINT>;
  k<<<persistent_grid(k, units, num_sms), kThreads, 0, s>>>(b, hp);
  return cudaGetLastError();
}

template <int N, int HINT>
cudaError_t launch_bulkpipe(const StageBatch& b, const Hyper& hp, int num_sms, cudaStream_t s) {
  using G = BulkGeom<N>;
  auto k = colocated_bulkpipe<N, HINT>;
  cudaError_t e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, G::kSmemBytes);
  if (e != cudaSuccess) return e;
  int64_t units = 0;
  for (int i = 0; i < b.nstages; ++i) units += (b.st[i].p / 4 + G::kTile - 1) / G::kTile;
  int64_t grid = num_sms;  // one block per SM (the ring takes most of shared memory)
  if (grid > units) grid = units;
  if (grid < 1) grid = 1;
  k<<<static_cast<int>(grid), kBulkThreads, G::kSmemBytes, s>>>(b, hp);
  return cudaGetLastError();
}

template <int N>
cudaError_t launch_n(const StageBatch& b, const Hyper& hp, int variant, int num_sms, cudaStream_t s) {
  const bool hint = l2_hint() != 0;
  if (variant == kVariantBulkPipe)
    return hint ? launch_bulkpipe<N, 1>(b, hp, num_sms, s) : launch_bulkpipe<N, 0>(b, hp, num_sms, s);
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

// Fused spread-layout step over peer memory (rows a4-a7 in ONE kernel).
//
// The north star's exchange is reduce-scatter -> owner-shard update ->
// all-gather ("send / accumulate / normalise and apply").  Here one
// kernel per rank does all of it over NVLink peer memory (CUDA IPC mappings),
// so the transfers overlap the local update chunk by chunk:
//
//   chunk c of Q floats, owner o(c) = c mod N, slot(c) = c div N.
//   Phase A (every chunk):  local SGD/Adam step + dilution of this rank's
//       replica (x, optimizer state, read x~ locally); the contribution
//       r = rho*Delta + beta*(x - x~) is STORED STRAIGHT INTO THE OWNER's inbox
//       (a peer store); then one release-add (system scope) on the owner's
//       arrival counter for that chunk.
//   Phase B (chunks this rank owns): wait until all N contributions arrived
//       (acquire), x~ += (sum_i r_i)/N on the local center, publish the new
//       chunk in the local outbox, release-store the chunk's ready flag.
//   Phase C (chunks owned by others): wait for the owner's ready flag, copy
//       the owner's outbox chunk (peer loads) into the local center.
//
// Per rank NVLink traffic is (N-1)/N * 4 B out (pushes) + (N-1)/N * 4 B in
// (pulls) per element -- the ring RS + AG volume -- with no intermediate HBM
// round trip of the contributions on the sending side.  Waits only go A -> B
// -> C and every CTA finishes its phase-A chunks before it waits, so with all
// ranks' kernels resident the exchange cannot deadlock; every spin has a
// wall-clock timeout that raises a host-visible error flag instead of hanging.
#include <cuda_runtime.h>
#include <stdint.h>

#include <cstdlib>

#include "ea_internal.h"

namespace ea {
namespace {

constexpr int kP2PThreads = 256;

__device__ __forceinline__ uint64_t globaltimer() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
__device__ __forceinline__ uint32_t ld_acquire_sys(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void red_add_release_sys(uint32_t* p, uint32_t v) {
  asm volatile("red.release.sys.global.add.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ void st_release_sys(uint32_t* p, uint32_t v) {
  asm volatile("st.release.sys.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ float4 ld_cg(const float* p) {  // L2 only: data other agents wrote in this launch
  float4 v;
  asm volatile("ld.global.cg.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p));
  return v;
}
__device__ __forceinline__ float4 ld4(const float* p) { return *reinterpret_cast<const float4*>(p); }
__device__ __forceinline__ void st4(float* p, float4 v) { *reinterpret_cast<float4*>(p) = v; }

// One (element) update -- the same arithmetic as the co-located kernels.
template <int OPT>
__device__ __forceinline__ float p2p_elem(float& x, float g, float& m, float& v, float c, const Hyper& hp,
                                          const StepCoef& sc) {
  float delta;
  if constexpr (OPT == kOptSGD) {
    const float gg = fmaf(hp.wd, x, g);
    const float mn = fmaf(hp.momentum, m, gg);
    const float d = hp.nesterov ? fmaf(hp.momentum, mn, gg) : mn;
    delta = -hp.lr * d;
    m = mn;
  } else if constexpr (OPT == kOptASGD) {  // reading c29, as ea_elem
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
  const float gap = x - c;
  const float r = fmaf(hp.beta, gap, hp.rho * delta);
  x = fmaf(-hp.alpha, gap, x) + delta;
  return r;
}

// Spin (thread 0) until *flag >= target or the timeout; returns false on timeout.
__device__ bool wait_at_least(const uint32_t* flag, uint32_t target, uint64_t timeout_ns, uint32_t* err) {
  const uint64_t t0 = globaltimer();
  while (ld_acquire_sys(flag) < target) {
    if (globaltimer() - t0 > timeout_ns) {
      atomicOr_system(err, 1u);
      return false;
    }
    __nanosleep(64);
  }
  return true;
}

// Scalar path for the ragged end of the replica and the zero padding of the center (4 elements from j).
template <int OPT>
__device__ __forceinline__ float4 ragged4(const P2PArgs& a, int64_t j, const StepCoef& sc) {
  float rr[4];
  for (int q = 0; q < 4; ++q) {
    const int64_t jj = j + q;
    rr[q] = 0.f;
    if (jj < a.p) {
      float xs = a.x[jj], ms = a.m[jj], ws = two_state(OPT) ? a.v[jj] : 0.f;
      rr[q] = p2p_elem<OPT>(xs, a.g[jj], ms, ws, a.center[jj], a.hp, sc);
      a.x[jj] = xs;
      a.m[jj] = ms;
      if (two_state(OPT)) a.v[jj] = ws;
    }
  }
  return make_float4(rr[0], rr[1], rr[2], rr[3]);
}

// Phase A on one chunk [e0, e0 + 4 nv4) by the kP2PThreads compute threads: update, store x and the state
// locally and the contribution into the owner's inbox (a peer store).  (Hoisting 2 or 4 float4 per stream per
// thread measured 6-25% slower: fewer resident CTAs, profiles/r01_s3_p2p_unroll_occupancy.jsonl.)
template <int OPT>
__device__ __forceinline__ void phase_a_chunk(const P2PArgs& a, int64_t e0, int64_t nv4, float* dst,
                                              const StepCoef& sc) {
  for (int64_t lv = threadIdx.x; lv < nv4; lv += kP2PThreads) {
    const int64_t j = e0 + 4 * lv;
    float4 rv;
    if (j + 3 < a.p) {
      float4 x = ld4(a.x + j), g = ld4(a.g + j), m = ld4(a.m + j), c4 = ld4(a.center + j);
      float4 w = two_state(OPT) ? ld4(a.v + j) : make_float4(0.f, 0.f, 0.f, 0.f);
      rv.x = p2p_elem<OPT>(x.x, g.x, m.x, w.x, c4.x, a.hp, sc);
      rv.y = p2p_elem<OPT>(x.y, g.y, m.y, w.y, c4.y, a.hp, sc);
      rv.z = p2p_elem<OPT>(x.z, g.z, m.z, w.z, c4.z, a.hp, sc);
      rv.w = p2p_elem<OPT>(x.w, g.w, m.w, w.w, c4.w, a.hp, sc);
      st4(a.x + j, x);
      st4(a.m + j, m);
      if (two_state(OPT)) st4(a.v + j, w);
    } else {  // the ragged end of the replica and the zero padding of the center
      rv = ragged4<OPT>(a, j, sc);
    }
    st4(dst + 4 * lv, rv);  // peer store into the owner's inbox
  }
}

// Resident CTAs asked of ptxas (the plain loop's own register counts: SGD/ASGD 32 -> 8 CTAs/SM, Adam(W) 48 -> 5).
// (A dedicated signal warp that publishes chunks while the compute warps move on measured slower on one rank,
// 0.82-0.86 vs 0.86-0.90 of HBM peak: profiles/r01_s3_p2p_sigwarp.jsonl.)
__host__ __device__ constexpr int p2p_min_blocks(int opt) { return two_state(opt) ? 5 : 8; }

template <int OPT>
__global__ void __launch_bounds__(kP2PThreads, p2p_min_blocks(OPT)) spread_p2p(const P2PArgs a, const P2PView view) {
  const int tid = threadIdx.x;
  const int64_t Q = a.chunk, nch = a.nchunks, slots = a.slots;
  const int N = a.world, r = a.rank;
  const float inv_n = a.hp.inv_n;
  const uint32_t epoch = static_cast<uint32_t>(*a.stepp);
  const StepCoef sc = has_coef(OPT) ? *a.scp : StepCoef{0.f, 0.f};

  // ---------------- Phase A: local update, push contributions to the owners
  for (int64_t c = blockIdx.x; c < nch; c += gridDim.x) {
    const int o = static_cast<int>(c % N);
    const int64_t slot = c / N;
    const int64_t e0 = c * Q;
    const int64_t len = (a.p_pad - e0) < Q ? (a.p_pad - e0) : Q;
    phase_a_chunk<OPT>(a, e0, len / 4, view.inbox[o] + ((int64_t)r * slots + slot) * Q, sc);
    // the block barrier orders every thread's stores before thread 0's system-scope release, which is
    // cumulative: a peer that acquires the counter sees them all (an extra fence.sc.sys measured 1.5-2.5%
    // slower and is only a knob now, AVGPIPE_EA_P2P_FENCE=1)
    __syncthreads();
    if (tid == 0) {
      if (a.sc_fence) __threadfence_system();
      red_add_release_sys(view.arrive[o] + slot, 1u);
    }
  }

  // ---------------- Phase B: owner reduction and center update
  __shared__ int s_ok;
  for (int64_t slot = blockIdx.x; slot < slots; slot += gridDim.x) {
    const int64_t c = slot * N + r;
    if (c >= nch) continue;
    const int64_t e0 = c * Q;
    const int64_t len = (a.p_pad - e0) < Q ? (a.p_pad - e0) : Q;
    if (tid == 0) s_ok = wait_at_least(view.arrive[r] + slot, (uint32_t)N * epoch, a.timeout_ns, a.err);
    __syncthreads();
    const float* in = view.inbox[r] + slot * Q;
    float* out = view.outbox[r] + slot * Q;
    for (int64_t lv = tid; lv < len / 4; lv += kP2PThreads) {
      float4 sum = make_float4(0.f, 0.f, 0.f, 0.f);
      for (int src = 0; src < N; ++src) {
        const float4 t = ld_cg(in + (int64_t)src * slots * Q + 4 * lv);
        sum.x += t.x; sum.y += t.y; sum.z += t.z; sum.w += t.w;
      }
      float4 cv = ld4(a.center + e0 + 4 * lv);
      cv = make_float4(fmaf(sum.x, inv_n, cv.x), fmaf(sum.y, inv_n, cv.y), fmaf(sum.z, inv_n, cv.z),
                       fmaf(sum.w, inv_n, cv.w));
      st4(a.center + e0 + 4 * lv, cv);
      st4(out + 4 * lv, cv);
    }
    __syncthreads();
    if (tid == 0) {
      if (a.sc_fence) __threadfence_system();
      st_release_sys(view.ready[r] + slot, epoch);
    }
    (void)s_ok;
  }

  // ---------------- Phase C: pull the other owners' new center chunks
  for (int64_t c = blockIdx.x; c < nch; c += gridDim.x) {
    const int o = static_cast<int>(c % N);
    if (o == r) continue;
    const int64_t slot = c / N;
    const int64_t e0 = c * Q;
    const int64_t len = (a.p_pad - e0) < Q ? (a.p_pad - e0) : Q;
    if (tid == 0) s_ok = wait_at_least(view.ready[o] + slot, epoch, a.timeout_ns, a.err);
    __syncthreads();
    const float* src = view.outbox[o] + slot * Q;
    for (int64_t lv = tid; lv < len / 4; lv += kP2PThreads) st4(a.center + e0 + 4 * lv, ld_cg(src + 4 * lv));
    __syncthreads();
  }
}

template <int OPT>
int blocks_per_sm_t() {
  int per_sm = 0;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, spread_p2p<OPT>, kP2PThreads, 0) != cudaSuccess ||
      per_sm < 1)
    per_sm = 1;
  return per_sm;
}

}  // namespace

cudaError_t launch_spread_p2p(const P2PArgs& a, const P2PView& v, int opt, int max_ctas, cudaStream_t s) {
  if (a.nchunks <= 0) return cudaSuccess;
  int64_t grid = max_ctas;
  if (grid > a.nchunks) grid = a.nchunks;
  if (grid < 1) grid = 1;
  const int g = static_cast<int>(grid);
  if (opt == kOptAdam) spread_p2p<kOptAdam><<<g, kP2PThreads, 0, s>>>(a, v);
  else if (opt == kOptAdamW) spread_p2p<kOptAdamW><<<g, kP2PThreads, 0, s>>>(a, v);
  else if (opt == kOptASGD) spread_p2p<kOptASGD><<<g, kP2PThreads, 0, s>>>(a, v);
  else spread_p2p<kOptSGD><<<g, kP2PThreads, 0, s>>>(a, v);
  return cudaGetLastError();
}

// Resident CTAs per SM of the instance that will run.  The grid never exceeds what is resident: the phase-B/C
// waits rely on every CTA of every rank being on an SM.
int p2p_blocks_per_sm(int opt) {
  if (opt == kOptSGD) return blocks_per_sm_t<kOptSGD>();
  if (opt == kOptASGD) return blocks_per_sm_t<kOptASGD>();
  return opt == kOptAdam ? blocks_per_sm_t<kOptAdam>() : blocks_per_sm_t<kOptAdamW>();
}

}  // namespace ea

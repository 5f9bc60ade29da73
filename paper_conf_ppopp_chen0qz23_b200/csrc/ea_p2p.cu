// Peer-memory spread step (EA_XCHG_P2P): rows a4-a7 over NVLink peer memory,
// split so that the caller's stream only carries the local update (row a8).
//
// The north star's exchange is reduce-scatter -> owner-shard update ->
// all-gather ("send / accumulate / normalise and apply").  Here the
// transfers are done by the library's own kernels over CUDA IPC mappings of
// every rank's exchange buffer:
//
//   chunk c of Q floats, owner o(c) = c mod N, slot(c) = c div N.
//   p2p_push (caller's stream; never waits on anything):
//       Phase A (every chunk): local SGD/Adam/ASGD step + dilution of this
//       rank's replica (x, optimizer state, read x~ locally); the contribution
//       r = rho*Delta + beta*(x - x~) is STORED STRAIGHT INTO THE OWNER's inbox
//       (a peer store, no local HBM round trip); then one release-add (system
//       scope) on the owner's arrival counter for that chunk.
//   p2p_exchange (library side stream, after p2p_push; the next forward does
//   not wait for it -- P:112/"not block the parallel pipelines"):
//       Phase B (chunks this rank owns): wait until all N contributions of the
//       epoch arrived (acquire), x~ += (sum_i r_i)/N on the local center,
//       publish the chunk in the local outbox, release-store its ready flag.
//       Phase C (chunks owned by others): wait for the owner's ready flag, pull
//       the owner's outbox chunk (peer loads) into the local center.
//
// Per rank NVLink traffic is (N-1)/N * 4 B out (pushes) + (N-1)/N * 4 B in
// (pulls) per element -- the ring RS + AG volume.
//
// Progress without co-residency: p2p_push never waits, and p2p_exchange hands
// out its work items through a per-launch atomic ticket, all phase-B items
// before any phase-C item.  A CTA holding a phase-C ticket therefore knows
// that every phase-B item of its rank is held by a CTA that is running, and
// phase-B items wait only for p2p_push kernels -- so no wait depends on a CTA
// of the exchange that has not been scheduled, however small its grid.  What
// the waits do need is that the pushes they wait for get SMs: one rank per GPU,
// a GPU's exchange kernel only waits for pushes on other GPUs (its own push
// precedes it), and stage K-1's pushes wait for nothing, so by induction over
// the stage order every exchange completes; ranks sharing a device (virtual
// ranks) share one pool of SMs, so their exchange grids are capped together
// below what could fill it (ea_api.cu).  Every spin has a wall-clock timeout:
// it raises a host-mapped error flag and a device abort flag; an item whose
// wait failed (or that starts after an abort) neither reduces, publishes nor
// copies anything.
#include <cuda_runtime.h>
#include <stdint.h>

#include <cstdio>
#include <cstdlib>

#include "ea_internal.h"
#include "ea_update.cuh"
#include "ea_bulk.cuh"

namespace ea {
namespace {

constexpr int kP2PThreads = 256;
constexpr int kXchgUnroll = 8;  // float4 per thread in flight in phases B/C (remote loads: latency-bound)

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
__device__ __forceinline__ uint32_t ld_relaxed_gpu(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void red_add_release_sys(uint32_t* p, uint32_t v) {
  asm volatile("red.release.sys.global.add.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ void st_release_sys(uint32_t* p, uint32_t v) {
  asm volatile("st.release.sys.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ float4 ld_cg(const float* p) {  // L2 only: data other agents wrote
  float4 v;
  asm volatile("ld.global.cg.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p));
  return v;
}
__device__ __forceinline__ float4 ld4(const float* p) { return *reinterpret_cast<const float4*>(p); }
__device__ __forceinline__ void st4(float* p, float4 v) { *reinterpret_cast<float4*>(p) = v; }

// Spin (thread 0) until *flag >= target; false on timeout or once any CTA of this rank has aborted.  The first
// timed-out wait of a rank prints what it waited for (an error path only).
__device__ bool wait_at_least(const uint32_t* flag, uint32_t target, const P2PArgs& a, int phase, int64_t chunk) {
  if (ld_acquire_sys(flag) >= target) return true;
  const uint64_t t0 = globaltimer();
  while (true) {
    if (ld_relaxed_gpu(a.abort)) return false;
    __nanosleep(64);
    const uint32_t v = ld_acquire_sys(flag);
    if (v >= target) return true;
    if (globaltimer() - t0 > a.timeout_ns) {
      if (atomicOr(a.abort, 1u) == 0u)
        printf("avgpipe p2p_exchange timeout: rank %d/%d phase %c chunk %lld of %lld: flag %u < %u\n", a.rank,
               a.world, phase == 0 ? 'B' : 'C', (long long)chunk, (long long)a.nchunks, v, target);
      atomicOr_system(a.err, 1u);
      return false;
    }
  }
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
      rr[q] = ea_elem<OPT>(xs, a.g[jj], ms, ws, a.center[jj], a.hp, sc);
      a.x[jj] = xs;
      a.m[jj] = ms;
      if (two_state(OPT)) a.v[jj] = ws;
    }
  }
  return make_float4(rr[0], rr[1], rr[2], rr[3]);
}

// Phase A on one chunk [e0, e0 + 4 nv4) by the kP2PThreads threads: update, store x and the state
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
      rv = ea_vec<OPT>(x, g, m, w, c4, a.hp, sc);
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
__host__ __device__ constexpr int p2p_min_blocks(int opt) { return two_state(opt) ? 5 : 8; }

// ---------------- p2p_push: phase A (caller's stream)
template <int OPT>
__global__ void __launch_bounds__(kP2PThreads, p2p_min_blocks(OPT)) p2p_push(const P2PArgs a, const P2PView view) {
  const int64_t Q = a.chunk, nch = a.nchunks, slots = a.slots;
  const int N = a.world, r = a.rank;
  const StepCoef sc = has_coef(OPT) ? *a.scp : StepCoef{0.f, 0.f};
  for (int64_t c = blockIdx.x; c < nch; c += gridDim.x) {
    const int o = static_cast<int>(c % N);
    const int64_t slot = c / N;
    const int64_t e0 = c * Q;
    const int64_t len = (a.p_pad - e0) < Q ? (a.p_pad - e0) : Q;
    phase_a_chunk<OPT>(a, e0, len / 4, view.inbox[o] + ((int64_t)r * slots + slot) * Q, sc);
    // the block barrier orders every thread's stores before thread 0's system-scope release, which is
    // cumulative: a peer that acquires the counter sees them all (an extra fence.sc.sys measured 1.5-2.5%
    // slower and is only a knob, AVGPIPE_EA_P2P_FENCE=1)
    __syncthreads();
    if (threadIdx.x == 0) {
      if (a.sc_fence) __threadfence_system();
      red_add_release_sys(view.arrive[o] + slot, 1u);
    }
  }
}

// ---------------- p2p_push_bulk: phase A through a bulk-copy (TMA engine) ring (default push kernel)
// One producer warp streams x, g, the optimizer state and x~ of each tile (kPushTile float4 per stream) into a
// kPushStages-deep shared-memory ring with cp.async.bulk, completing on per-slot mbarriers; eight consumer warps
// update from shared memory and store x, the state and the contribution (straight into the owner's inbox) with
// 128-bit stores.  A CTA walks whole chunks (chunk c = blockIdx.x + k*gridDim.x, tile by tile), so after the last
// tile of a chunk one release-add publishes it.  Tiles that reach past the replica's P_s elements (the ragged end
// and the zero padding of the center) are not copied: the consumers compute them from global memory.
constexpr int kPushConsumerWarps = 8;
constexpr int kPushThreads = 32 * (kPushConsumerWarps + 1);
constexpr int kPushTile = 256;  // float4 per stream per tile (4 KB copies)

template <int OPT>
struct PushGeom {
  static constexpr int kStreams = two_state(OPT) ? 5 : 4;  // x, g, m, (v), x~
  static constexpr int kSlotVec = kStreams * kPushTile;
  static constexpr int kStages = 6;
  static constexpr int kSmemBytes = kStages * kSlotVec * 16 + 2 * kStages * 8;
};

template <int OPT>
__global__ void __launch_bounds__(kPushThreads, 1) p2p_push_bulk(const P2PArgs a, const P2PView view) {
  using G = PushGeom<OPT>;
  constexpr int T = kPushTile, S = G::kStages, NS = G::kStreams;
  extern __shared__ __align__(128) float4 smem[];
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + S * G::kSlotVec);
  uint64_t* empty = full + S;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int64_t Q = a.chunk, nch = a.nchunks, slots = a.slots;
  const int N = a.world, r = a.rank;
  const int64_t p4 = a.p / 4;  // float4 of the replica that may be bulk-copied
  if (threadIdx.x == 0) {
    for (int i = 0; i < S; ++i) {
      mbar_init(&full[i], 1);
      mbar_init(&empty[i], 1);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  // the tile sequence of this CTA: (chunk, tile) for its chunks in order; both roles walk it identically
  auto tiles_of = [&](int64_t c) {
    const int64_t len = (a.p_pad - c * Q) < Q ? (a.p_pad - c * Q) : Q;
    return (len / 4 + T - 1) / T;
  };
  if (warp == kPushConsumerWarps) {
    // ---- producer warp
    int k = 0;
    for (int64_t c = blockIdx.x; c < nch; c += gridDim.x) {
      const int64_t e4 = c * Q / 4, len4 = ((a.p_pad - c * Q) < Q ? (a.p_pad - c * Q) : Q) / 4;
      const int64_t nt = tiles_of(c);
      for (int64_t t = 0; t < nt; ++t, ++k) {
        const int slot = k % S;
        mbar_wait(&empty[slot], ((k / S) & 1) ^ 1);
        fence_proxy_async();
        const int64_t v0 = e4 + t * T;
        const int64_t nv = (len4 - t * T) < T ? (len4 - t * T) : T;
        const bool bulk = v0 + nv <= p4;
        const uint32_t bytes = bulk ? static_cast<uint32_t>(nv * 16) : 0u;
        if (lane == 0) mbar_expect_tx(&full[slot], bytes * NS);  // 0 bytes: the phase completes at once
        __syncwarp();
        if (bulk && lane < NS) {
          const float* src = lane == 0 ? a.x : lane == 1 ? a.g : lane == 2 ? a.m : (NS == 5 && lane == 3) ? a.v
                                                                                                      : a.center;
          bulk_g2s(smem + slot * G::kSlotVec + lane * T, src + 4 * v0, bytes, &full[slot]);
        }
      }
    }
  } else {
    // ---- consumers
    const StepCoef sc = has_coef(OPT) ? *a.scp : StepCoef{0.f, 0.f};
    int k = 0;
    for (int64_t c = blockIdx.x; c < nch; c += gridDim.x) {
      const int o = static_cast<int>(c % N);
      const int64_t slot_c = c / N;
      const int64_t e4 = c * Q / 4, len4 = ((a.p_pad - c * Q) < Q ? (a.p_pad - c * Q) : Q) / 4;
      float* dst = view.inbox[o] + ((int64_t)r * slots + slot_c) * Q;  // this chunk's place in the owner's inbox
      const int64_t nt = tiles_of(c);
      for (int64_t t = 0; t < nt; ++t, ++k) {
        const int slot = k % S;
        mbar_wait(&full[slot], (k / S) & 1);
        const float4* base = smem + slot * G::kSlotVec;
        const int64_t v0 = e4 + t * T;
        const int64_t nv = (len4 - t * T) < T ? (len4 - t * T) : T;
        const bool bulk = v0 + nv <= p4;
        for (int lv = threadIdx.x; lv < nv; lv += 32 * kPushConsumerWarps) {
          const int64_t v = v0 + lv;
          float4 rv;
          if (bulk) {
            float4 x = base[lv];
            const float4 g = base[T + lv];
            float4 m = base[2 * T + lv];
            float4 w = NS == 5 ? base[3 * T + lv] : make_float4(0.f, 0.f, 0.f, 0.f);
            const float4 cv = base[(NS - 1) * T + lv];
            rv = ea_vec<OPT>(x, g, m, w, cv, a.hp, sc);
            st4(a.x + 4 * v, x);
            st4(a.m + 4 * v, m);
            if (NS == 5) st4(a.v + 4 * v, w);
          } else {
            rv = ragged4<OPT>(a, 4 * v, sc);
          }
          st4(dst + 4 * (v - e4), rv);  // peer store into the owner's inbox
        }
        // all consumer warps are done with the slot (and, at a chunk's end, have issued all its stores).  (Moving the
        // chunk's release-add to the producer warp, off the consumers' path, measured slower on B200: 265 vs 232 us
        // per C4 stage -- the producer's system-scope release then waits behind its own bulk copies in flight.)
        asm volatile("bar.sync 1, %0;" ::"n"(32 * kPushConsumerWarps) : "memory");
        if (threadIdx.x == 0) {
          mbar_arrive(&empty[slot]);
          if (t == nt - 1) {
            if (a.sc_fence) __threadfence_system();
            red_add_release_sys(view.arrive[o] + slot_c, 1u);
          }
        }
      }
    }
  }
}

// ---------------- p2p_exchange: phases B and C (side stream), ticket-ordered
// The k-th chunk (0-based, increasing) not owned by rank r (N >= 2).
__device__ __forceinline__ int64_t foreign_chunk(int64_t k, int N, int r) {
  const int64_t g = k / (N - 1), i = k % (N - 1);
  return g * N + (i < r ? i : i + 1);
}

__global__ void __launch_bounds__(kP2PThreads) p2p_exchange(const P2PArgs a, const P2PView view) {
  const int tid = threadIdx.x;
  const int64_t Q = a.chunk, nch = a.nchunks, slots = a.slots;
  const int N = a.world, r = a.rank;
  const float inv_n = a.hp.inv_n;
  const uint32_t epoch = *a.epochp;
  // owned chunks: c = slot * N + r < nch, i.e. the first n_own slots
  const int64_t n_own = nch > r ? (nch - r + N - 1) / N : 0;
  const int64_t n_items = nch;  // n_own phase-B items, then nch - n_own phase-C items
  __shared__ int64_t s_item;
  __shared__ int s_ok;
  while (true) {
    if (tid == 0) s_item = static_cast<int64_t>(atomicAdd(a.tickets, 1u));
    __syncthreads();
    const int64_t item = s_item;
    if (item >= n_items) break;
    if (item < n_own) {
      // Phase B: owner reduction and center update of chunk slot*N + r
      const int64_t slot = item, c = slot * N + r;
      const int64_t e0 = c * Q;
      const int64_t len = (a.p_pad - e0) < Q ? (a.p_pad - e0) : Q;
      if (tid == 0) s_ok = wait_at_least(view.arrive[r] + slot, (uint32_t)N * epoch, a, 0, c);
      __syncthreads();
      if (s_ok) {
        const float* in = view.inbox[r] + slot * Q;
        float* out = view.outbox[r] + slot * Q;
        const int64_t nv4 = len / 4;
        for (int64_t b0 = 0; b0 < nv4; b0 += (int64_t)kP2PThreads * kXchgUnroll) {
          float4 sum[kXchgUnroll];
#pragma unroll
          for (int u = 0; u < kXchgUnroll; ++u) sum[u] = make_float4(0.f, 0.f, 0.f, 0.f);
          for (int src = 0; src < N; ++src) {
            const float* ins = in + (int64_t)src * slots * Q;
#pragma unroll
            for (int u = 0; u < kXchgUnroll; ++u) {
              const int64_t lv = b0 + (int64_t)u * kP2PThreads + tid;
              if (lv < nv4) add4(sum[u], ld_cg(ins + 4 * lv));
            }
          }
#pragma unroll
          for (int u = 0; u < kXchgUnroll; ++u) {
            const int64_t lv = b0 + (int64_t)u * kP2PThreads + tid;
            if (lv < nv4) {
              const float4 cv = center_apply(ld4(a.center + e0 + 4 * lv), sum[u], inv_n);
              st4(a.center + e0 + 4 * lv, cv);
              st4(out + 4 * lv, cv);
            }
          }
        }
      }
      __syncthreads();
      if (tid == 0 && s_ok) {
        if (a.sc_fence) __threadfence_system();
        st_release_sys(view.ready[r] + slot, epoch);
      }
    } else {
      // Phase C: pull another owner's new center chunk
      const int64_t c = foreign_chunk(item - n_own, N, r);
      const int o = static_cast<int>(c % N);
      const int64_t slot = c / N;
      const int64_t e0 = c * Q;
      const int64_t len = (a.p_pad - e0) < Q ? (a.p_pad - e0) : Q;
      if (tid == 0) s_ok = wait_at_least(view.ready[o] + slot, epoch, a, 1, c);
      __syncthreads();
      if (s_ok) {
        const float* src = view.outbox[o] + slot * Q;
        const int64_t nv4 = len / 4;
        for (int64_t b0 = 0; b0 < nv4; b0 += (int64_t)kP2PThreads * kXchgUnroll) {
          float4 t[kXchgUnroll];
#pragma unroll
          for (int u = 0; u < kXchgUnroll; ++u) {
            const int64_t lv = b0 + (int64_t)u * kP2PThreads + tid;
            if (lv < nv4) t[u] = ld_cg(src + 4 * lv);
          }
#pragma unroll
          for (int u = 0; u < kXchgUnroll; ++u) {
            const int64_t lv = b0 + (int64_t)u * kP2PThreads + tid;
            if (lv < nv4) st4(a.center + e0 + 4 * lv, t[u]);
          }
        }
      }
    }
    __syncthreads();  // s_item / s_ok are reused by the next ticket
  }
}

template <int OPT>
int blocks_per_sm_t() {
  int per_sm = 0;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, p2p_push<OPT>, kP2PThreads, 0) != cudaSuccess ||
      per_sm < 1)
    per_sm = 1;
  return per_sm;
}

template <int OPT>
cudaError_t launch_push_bulk_t(const P2PArgs& a, const P2PView& v, int max_sms, cudaStream_t s) {
  auto k = p2p_push_bulk<OPT>;
  cudaError_t e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, PushGeom<OPT>::kSmemBytes);
  if (e != cudaSuccess) return e;
  int64_t grid = max_sms;  // one CTA per SM (the ring takes most of shared memory)
  if (grid > a.nchunks) grid = a.nchunks;
  if (grid < 1) grid = 1;
  k<<<static_cast<int>(grid), kPushThreads, PushGeom<OPT>::kSmemBytes, s>>>(a, v);
  return cudaGetLastError();
}

// Push kernel knob (measurement): AVGPIPE_EA_P2P_PUSH=plain selects the register loop (p2p_push); default: the
// bulk-copy ring (p2p_push_bulk).
bool push_plain() {
  static const bool v = [] {
    const char* e = std::getenv("AVGPIPE_EA_P2P_PUSH");
    return e && e[0] == 'p';
  }();
  return v;
}

}  // namespace

cudaError_t launch_p2p_push(const P2PArgs& a, const P2PView& v, int opt, int max_ctas, int max_sms, cudaStream_t s) {
  if (a.nchunks <= 0) return cudaSuccess;
  if (!push_plain()) {
    if (opt == kOptAdam) return launch_push_bulk_t<kOptAdam>(a, v, max_sms, s);
    if (opt == kOptAdamW) return launch_push_bulk_t<kOptAdamW>(a, v, max_sms, s);
    if (opt == kOptASGD) return launch_push_bulk_t<kOptASGD>(a, v, max_sms, s);
    return launch_push_bulk_t<kOptSGD>(a, v, max_sms, s);
  }
  int64_t grid = max_ctas;
  if (grid > a.nchunks) grid = a.nchunks;
  if (grid < 1) grid = 1;
  const int g = static_cast<int>(grid);
  if (opt == kOptAdam) p2p_push<kOptAdam><<<g, kP2PThreads, 0, s>>>(a, v);
  else if (opt == kOptAdamW) p2p_push<kOptAdamW><<<g, kP2PThreads, 0, s>>>(a, v);
  else if (opt == kOptASGD) p2p_push<kOptASGD><<<g, kP2PThreads, 0, s>>>(a, v);
  else p2p_push<kOptSGD><<<g, kP2PThreads, 0, s>>>(a, v);
  return cudaGetLastError();
}

cudaError_t launch_p2p_exchange(const P2PArgs& a, const P2PView& v, int max_ctas, cudaStream_t s) {
  if (a.nchunks <= 0) return cudaSuccess;
  cudaError_t e = cudaMemsetAsync(a.tickets, 0, sizeof(uint32_t), s);  // fresh tickets for this launch
  if (e != cudaSuccess) return e;
  int64_t grid = max_ctas;
  if (grid > a.nchunks) grid = a.nchunks;
  if (grid < 1) grid = 1;
  p2p_exchange<<<static_cast<int>(grid), kP2PThreads, 0, s>>>(a, v);
  return cudaGetLastError();
}

// Resident CTAs per SM of the push instance that will run (its persistent grid).
int p2p_blocks_per_sm(int opt) {
  if (opt == kOptSGD) return blocks_per_sm_t<kOptSGD>();
  if (opt == kOptASGD) return blocks_per_sm_t<kOptASGD>();
  return opt == kOptAdam ? blocks_per_sm_t<kOptAdam>() : blocks_per_sm_t<kOptAdamW>();
}

}  // namespace ea

// C-ABI layer of the elastic-averaging library (declared in include/ea.h).
//
// Owns: the handle, per-stage optimizer state (zero-initialised, P:112 Step 1:
// SGD momentum, or Adam's two moments plus the per-stage step count), and for
// EA_SPREAD the side stream, events, contribution scratch and the NCCL
// communicator that replace the paper's reference process and message queues
// (P:112-116).  Validates every argument before enqueuing anything; never
// throws or aborts.
#include <cuda_runtime.h>
#include <nccl.h>
#include <stdint.h>

#include <cmath>
#include <cstdlib>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <new>
#include <string>
#include <vector>

#include <nvtx3/nvToolsExt.h>

#include "../../include/ea.h"
#include "ea_internal.h"

namespace {
// NVTX range around each ABI call that enqueues work (visible in nsys timelines).
struct NvtxRange {
  explicit NvtxRange(const char* name) { nvtxRangePushA(name); }
  ~NvtxRange() { nvtxRangePop(); }
};
}  // namespace

struct ea_ctx {
  ea_config cfg{};
  ea::Hyper hp{};
  int variant = 0;
  int num_sms = 148;
  std::vector<int64_t> p;       // P_s
  std::vector<int64_t> p_pad;   // center capacity
  std::vector<int64_t> stride;  // optimizer-state row stride (floats)
  std::vector<float*> state[2]; // per stage: [replicas][stride]; slot 0 = momentum / Adam m, slot 1 = Adam v
  std::vector<float*> prev;     // staleness 1: per stage x~_{t-1} (P_s floats)
  std::vector<char> prev_init;  // per stage: prev holds a value (else x~_{-1} := x~_0 at the first step)
  std::vector<int64_t> steps;   // per-stage step count t, host shadow (enqueue order)
  int64_t* d_steps = nullptr;   // device step counters (authoritative for Adam / P2P; graph-safe)
  ea::StepCoef* d_coef = nullptr;  // device Adam bias corrections of the current step
  // EA_SPREAD
  cudaStream_t side = nullptr;
  cudaEvent_t ev_done = nullptr;
  float* contrib = nullptr;  // NCCL exchange: sum_s P_pad(s) floats, one contribution buffer per stage
  std::vector<size_t> contrib_off;       // per-stage offset into contrib (floats)
  std::vector<cudaEvent_t> ev_ag;        // per stage: its last all-gather (center final) on the side stream
  std::vector<cudaEvent_t> ev_loc;       // per stage: its last local kernel on the caller's stream
  std::vector<cudaEvent_t> ev_snap;      // per stage, staleness 1: x~_t copied into prev on the side stream
  float* reduced = nullptr;  // max P_pad/N floats
  ncclComm_t comm = nullptr;
  // EA_SPREAD with exchange == EA_XCHG_P2P (fused peer-memory kernel)
  char* xbuf = nullptr;  // this rank's exchange buffer (exported by CUDA IPC)
  size_t xbuf_bytes = 0;
  std::vector<size_t> x_inbox, x_outbox, x_arrive, x_ready;  // per-stage byte offsets into xbuf
  std::vector<int64_t> x_nchunks, x_slots;
  int64_t x_chunk = 0;  // floats per exchange chunk (p2p_chunk() at ea_init; every rank must agree)
  uint32_t* d_xctl = nullptr;  // device: [n_stages] exchange epochs, [n_stages] exchange tickets, [1] abort flag
  std::vector<char*> peer_base;   // world entries, as mapped on this device (self = xbuf)
  std::vector<char> peer_ipc;     // 1 = opened with cudaIpcOpenMemHandle (closed at destroy)
  bool p2p_ready = false;
  int same_device_ranks = 1;
  uint32_t* err_host = nullptr;   // host-mapped exchange error flag
  uint32_t* err_dev = nullptr;
  // host-buffer path (ea_step_many_host), allocated on first use
  cudaStream_t h2d = nullptr, d2h = nullptr;
  float* staging[2] = {nullptr, nullptr};  // N * kHostChunk floats each
  cudaEvent_t ev_h2d[2] = {nullptr, nullptr}, ev_kern[2] = {nullptr, nullptr}, ev_d2h = nullptr;
  std::string err;
};

// SMs the spread layout's local kernel leaves free for the side-stream exchange (knob AVGPIPE_EA_SPREAD_RESERVE_SMS).
constexpr int kSpreadReserveSms = 0;

// Elements per pipelined chunk of the host-buffer path (a multiple of 64).  AVGPIPE_EA_HOST_CHUNK
// (elements, measurement knob) overrides it up to the staging capacity.
constexpr int64_t kHostChunk = 4 << 20;

int64_t host_chunk() {
  static int64_t v = [] {
    const char* e = std::getenv("AVGPIPE_EA_HOST_CHUNK");
    long long c = e ? std::atoll(e) : 0;
    if (c <= 0 || c > kHostChunk) return kHostChunk;
    return static_cast<int64_t>((c + 63) / 64 * 64);
  }();
  return v;
}

// Floats per exchange chunk of the peer-memory spread step (default 32768 = 128 KB: one system-scope release per
// chunk; B200, C4 stage, round 2: 8192 / 16384 / 32768 -> push kernel 0.45 / 0.50 / 0.54 of HBM peak beside the
// exchange at world 1, 8 virtual ranks 0.99 / - / 1.08, profiles/r02_p2p_chunks_split_grid.jsonl; round 1's fused
// kernel preferred 8192).  Measurement knob AVGPIPE_EA_P2P_CHUNK (a multiple of 1024 floats, 1024..65536); every
// rank of an exchange must use the same value (it fixes the layout of the peers' inboxes).
int64_t p2p_chunk() {
  const char* e = std::getenv("AVGPIPE_EA_P2P_CHUNK");
  const long long v = e ? std::atoll(e) : 0;
  return (v >= 1024 && v <= 65536 && v % 1024 == 0) ? v : 32768;
}

namespace {

thread_local std::string g_init_err;

void set_err(ea_ctx* h, const char* fmt, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof(buf), fmt, ap);
  va_end(ap);
  if (h) h->err = buf; else g_init_err = buf;
}

bool aligned16(const void* p) { return (reinterpret_cast<uintptr_t>(p) & 15u) == 0; }

int64_t round_up(int64_t a, int64_t b) { return (a + b - 1) / b * b; }

// Device (or managed) memory on this handle's device?
bool is_device_ptr(const void* p, int device) {
  cudaPointerAttributes a;
  if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  if (a.type == cudaMemoryTypeManaged) return true;
  return a.type == cudaMemoryTypeDevice && a.device == device;
}

bool finite(float v) { return v == v && v - v == 0.f; }

ea_status check_hyper(ea_ctx* h, const ea_config& c) {
  if (!(c.alpha >= 0.f && c.alpha <= 1.f)) { set_err(h, "alpha must be in [0,1] (P:112), got %g", c.alpha); return EA_EINVAL; }
  if (!finite(c.beta) || !finite(c.rho) || !finite(c.lr)) { set_err(h, "beta, rho, lr must be finite"); return EA_EINVAL; }
  if (!(c.weight_decay >= 0.f) || !finite(c.weight_decay)) { set_err(h, "weight_decay must be finite and >= 0"); return EA_EINVAL; }
  if (c.optimizer == EA_OPT_SGD) {
    if (!(c.momentum >= 0.f && c.momentum < 1.f)) { set_err(h, "momentum must be in [0,1), got %g", c.momentum); return EA_EINVAL; }
    if (c.nesterov != 0 && c.nesterov != 1) { set_err(h, "nesterov must be 0 or 1"); return EA_EINVAL; }
    if (c.nesterov && c.momentum <= 0.f) { set_err(h, "nesterov needs momentum > 0 (torch.optim.SGD rule)"); return EA_EINVAL; }
  } else if (c.optimizer == EA_OPT_ADAM || c.optimizer == EA_OPT_ADAMW) {
    if (!(c.beta1 >= 0.0 && c.beta1 < 1.0) || !(c.beta2 >= 0.0 && c.beta2 < 1.0)) {
      set_err(h, "Adam betas must be in [0,1), got %g, %g", c.beta1, c.beta2);
      return EA_EINVAL;
    }
    if (!(c.eps > 0.f) || !finite(c.eps)) { set_err(h, "Adam eps must be finite and > 0"); return EA_EINVAL; }
  } else if (c.optimizer == EA_OPT_ASGD) {
    if (!(c.asgd_lambd >= 0.0 && c.asgd_lambd < 1e30) || !(c.asgd_alpha >= 0.0 && c.asgd_alpha < 1e30) ||
        !(c.asgd_t0 >= 0.0 && c.asgd_t0 < 1e300)) {
      set_err(h, "ASGD lambd, alpha, t0 must be finite and >= 0, got %g, %g, %g", c.asgd_lambd, c.asgd_alpha,
              c.asgd_t0);
      return EA_EINVAL;
    }
  } else {
    set_err(h, "unknown optimizer %d", c.optimizer);
    return EA_EINVAL;
  }
  return EA_OK;
}

ea::Hyper make_hyper(const ea_config& c) {
  ea::Hyper hp;
  hp.alpha = c.alpha; hp.beta = c.beta; hp.rho = c.rho; hp.lr = c.lr;
  hp.momentum = c.momentum; hp.wd = c.weight_decay; hp.nesterov = c.nesterov;
  hp.inv_n = 1.0f / static_cast<float>(c.n_pipelines);
  hp.beta1 = static_cast<float>(c.beta1); hp.one_minus_beta1 = static_cast<float>(1.0 - c.beta1);
  hp.beta2 = static_cast<float>(c.beta2); hp.one_minus_beta2 = static_cast<float>(1.0 - c.beta2);
  hp.eps = c.eps;
  hp.lr_wd = static_cast<float>((double)c.lr * (double)c.weight_decay);
  hp.asgd_lambd = static_cast<float>(c.asgd_lambd);
  return hp;
}

int state_slots(const ea_ctx* h) { return ea::two_state(h->cfg.optimizer) ? 2 : 1; }

// Device step counters are needed when a kernel consumes the step count:
// Adam's bias correction, ASGD's eta_t / mu_t and the peer-memory exchange's epoch.
bool device_steps(const ea_ctx* h) {
  return h->cfg.optimizer != EA_OPT_SGD || (h->cfg.layout == EA_SPREAD && h->cfg.exchange == EA_XCHG_P2P);
}

ea_status cuda_fail(ea_ctx* h, cudaError_t e, const char* what) {
  set_err(h, "%s: %s", what, cudaGetErrorString(e));
  return e == cudaErrorMemoryAllocation ? EA_ENOMEM : EA_ECUDA;
}

ea_status nccl_fail(ea_ctx* h, ncclResult_t r, const char* what) {
  set_err(h, "%s: %s", what, ncclGetErrorString(r));
  return EA_ENCCL;
}

// Count one step of each listed stage: host shadow now, device counters (and
// Adam coefficients) on `s` ahead of the step's kernel.
ea_status advance(ea_ctx* h, const int32_t* stages, int count, cudaStream_t s) {
  for (int j = 0; j < count; ++j) ++h->steps[stages[j]];
  if (!device_steps(h)) return EA_OK;
  for (int j0 = 0; j0 < count; j0 += 8) {
    ea::StageList l;
    l.count = 0;
    for (int j = j0; j < count && j < j0 + 8; ++j) l.idx[l.count++] = stages[j];
    ea::CoefParams cp;
    cp.opt = h->cfg.optimizer;
    cp.beta1 = h->cfg.beta1; cp.beta2 = h->cfg.beta2; cp.lr = (double)h->cfg.lr;
    cp.lambd = h->cfg.asgd_lambd; cp.asgd_alpha = h->cfg.asgd_alpha; cp.t0 = h->cfg.asgd_t0;
    uint32_t* xepoch = h->d_xctl;  // the peer-memory exchange's own epoch (ea_set_step never touches it)
    cudaError_t e = ea::launch_advance_steps(h->d_steps, xepoch, h->d_coef, l, cp, s);
    if (e != cudaSuccess) return cuda_fail(h, e, "step-counter kernel launch");
  }
  return EA_OK;
}

void free_ctx(ea_ctx* h) {
  if (!h) return;
  cudaSetDevice(h->cfg.device);
  if (h->side) cudaStreamSynchronize(h->side);
  if (h->comm && h->xbuf && h->p2p_ready && h->cfg.world > 1) {
    // peers may still read this rank's outbox / write its inbox through their IPC mappings: a barrier
    // over the communicator (every rank destroys its handle) before the exchange buffer is freed
    int* one = nullptr;
    if (cudaMalloc(&one, sizeof(int)) == cudaSuccess) {
      if (ncclAllReduce(one, one, 1, ncclInt32, ncclSum, h->comm, h->side) == ncclSuccess)
        cudaStreamSynchronize(h->side);
      cudaFree(one);
    }
  }
  if (h->comm) ncclCommDestroy(h->comm);
  for (auto& slot : h->state)
    for (float* m : slot) if (m) cudaFree(m);
  for (float* m : h->prev) if (m) cudaFree(m);
  if (h->contrib) cudaFree(h->contrib);
  for (cudaEvent_t ev : h->ev_ag) if (ev) cudaEventDestroy(ev);
  for (cudaEvent_t ev : h->ev_loc) if (ev) cudaEventDestroy(ev);
  for (cudaEvent_t ev : h->ev_snap) if (ev) cudaEventDestroy(ev);
  if (h->reduced) cudaFree(h->reduced);
  if (h->d_steps) cudaFree(h->d_steps);
  if (h->d_coef) cudaFree(h->d_coef);
  if (h->ev_done) cudaEventDestroy(h->ev_done);
  if (h->side) cudaStreamDestroy(h->side);
  if (h->h2d) cudaStreamSynchronize(h->h2d);
  if (h->d2h) cudaStreamSynchronize(h->d2h);
  for (int i = 0; i < 2; ++i) {
    if (h->staging[i]) cudaFree(h->staging[i]);
    if (h->ev_h2d[i]) cudaEventDestroy(h->ev_h2d[i]);
    if (h->ev_kern[i]) cudaEventDestroy(h->ev_kern[i]);
  }
  if (h->ev_d2h) cudaEventDestroy(h->ev_d2h);
  for (size_t i = 0; i < h->peer_base.size(); ++i)
    if (i < h->peer_ipc.size() && h->peer_ipc[i] && h->peer_base[i]) cudaIpcCloseMemHandle(h->peer_base[i]);
  if (h->xbuf) cudaFree(h->xbuf);
  if (h->d_xctl) cudaFree(h->d_xctl);
  if (h->err_host) cudaFreeHost(h->err_host);
  if (h->h2d) cudaStreamDestroy(h->h2d);
  if (h->d2h) cudaStreamDestroy(h->d2h);
  delete h;
}

int replicas_here(const ea_ctx* h) { return h->cfg.layout == EA_SPREAD ? 1 : h->cfg.n_pipelines; }

float* state_ptr(const ea_ctx* h, int slot, int stage, int replica) {
  if (slot >= state_slots(h)) return nullptr;
  return h->state[slot][stage] + h->stride[stage] * replica;
}

// Validates one stage's pointers (nothing enqueued on failure).
ea_status check_stage_ptrs(ea_ctx* h, int32_t stage, float* const* replica_ptrs, const float* const* grad_ptrs,
                           const float* center_ptr) {
  if (stage < 0 || stage >= h->cfg.n_stages) { set_err(h, "stage %d out of range", stage); return EA_EINVAL; }
  if (!replica_ptrs || !grad_ptrs) { set_err(h, "replica_ptrs / grad_ptrs is NULL"); return EA_EINVAL; }
  const int reps = replicas_here(h);
  const int dev = h->cfg.device;
  if (!center_ptr || !aligned16(center_ptr) || !is_device_ptr(center_ptr, dev)) {
    set_err(h, "center_ptr must be a 16-byte aligned device pointer on device %d", dev);
    return EA_EINVAL;
  }
  for (int i = 0; i < reps; ++i) {
    if (!replica_ptrs[i] || !grad_ptrs[i] || !aligned16(replica_ptrs[i]) || !aligned16(grad_ptrs[i]) ||
        !is_device_ptr(replica_ptrs[i], dev) || !is_device_ptr(grad_ptrs[i], dev)) {
      set_err(h, "stage %d: replica/grad pointer %d must be a 16-byte aligned device pointer on device %d", stage, i,
              dev);
      return EA_EINVAL;
    }
  }
  return EA_OK;
}

// Staleness 1 (row f4, reading c28): x~_{-1} := x~_0 on the first step of a stage, unless the caller set it
// (ea_set_state, EA_SLOT_CENTER_PREV).  Refused while `s` is capturing a CUDA graph: the copy would be captured
// and replayed every step, turning the run into staleness 0.
ea_status stale_prev_init(ea_ctx* h, int st, const float* center, cudaStream_t s) {
  if (h->prev_init[st]) return EA_OK;
  cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
  cudaError_t e = cudaStreamIsCapturing(s, &cs);
  if (e != cudaSuccess) return cuda_fail(h, e, "cudaStreamIsCapturing");
  if (cs != cudaStreamCaptureStatusNone) {
    set_err(h, "staleness 1: stage %d has no x~_{-1} yet; take its first step outside graph capture or set it with "
               "ea_set_state(EA_SLOT_CENTER_PREV)", st);
    return EA_ESTATE;
  }
  e = cudaMemcpyAsync(h->prev[st], center, sizeof(float) * h->p[st], cudaMemcpyDeviceToDevice, s);
  if (e != cudaSuccess) return cuda_fail(h, e, "stale-center init");
  h->prev_init[st] = 1;
  return EA_OK;
}

// Co-located: `count` validated stages in as few launches as possible.
ea_status colocated_launch(ea_ctx* h, int32_t count, const int32_t* stages, float* const* replica_ptrs,
                           const float* const* grad_ptrs, float* const* center_ptrs, cudaStream_t s) {
  const int n = h->cfg.n_pipelines;
  const int opt = h->cfg.optimizer;
  const bool two = state_slots(h) == 2;
  cudaError_t e = cudaSuccess;
  static const bool force_wide = [] {  // measurement knob: AVGPIPE_EA_FORCE_WIDE=1
    const char* v = std::getenv("AVGPIPE_EA_FORCE_WIDE");
    return v && v[0] == '1';
  }();
  const bool stale = h->cfg.staleness == 1;
  // stale center, default variant: one launch per <= 8 stages -- the lane kernel with x~_{t-1} staged beside x~_t
  // for 2 <= N <= 4, the bulk-copy pipeline with x~_{t-1} as one more stream for N = 1 (and N = 5 for SGD/ASGD);
  // else the replica loop, one launch per stage, which measured better from N = 6 on (N = 8: 0.954 vs 0.903;
  // Adam N = 6: 0.925 vs 0.775 of HBM peak, profiles/r02_sweep_kernels.jsonl).  AVGPIPE_EA_FORCE_WIDE=1 selects
  // the replica loop for A/B measurement.
  const bool stale_lane = stale && !force_wide &&
                          ((h->variant == 0 && (n <= 4 || (n == 5 && !ea::two_state(opt)) ||
                                                (ea::two_state(opt) && n <= ea::kMaxFusedN))) ||
                           ((h->variant == ea::kVariantWarpRep || h->variant == ea::kVariantWarpSpec) &&
                            n <= ea::kMaxFusedN));
  if (stale) {  // validate / initialise every stage's x~_{-1} before anything is launched
    for (int j = 0; j < count; ++j) {
      ea_status st2 = stale_prev_init(h, stages[j], center_ptrs[j], s);
      if (st2 != EA_OK) return st2;
    }
  }
  if (stale_lane) {
    for (int j0 = 0; j0 < count; j0 += ea::kMaxLaunchStages) {
      const int cnt = count - j0 < ea::kMaxLaunchStages ? count - j0 : ea::kMaxLaunchStages;
      ea_status st2 = advance(h, stages + j0, cnt, s);
      if (st2 != EA_OK) return st2;
      ea::StageBatch b;
      b.nstages = 0;
      for (int j = j0; j < j0 + cnt; ++j) {
        const int st = stages[j];
        ea::StageRefs& r = b.st[b.nstages++];
        for (int i = 0; i < ea::kMaxFusedN; ++i) {
          const bool on = i < n;
          r.x[i] = on ? replica_ptrs[j * n + i] : nullptr;
          r.g[i] = on ? grad_ptrs[j * n + i] : nullptr;
          r.m[i] = on ? state_ptr(h, 0, st, i) : nullptr;
          r.v[i] = (on && two) ? state_ptr(h, 1, st, i) : nullptr;
        }
        r.c = center_ptrs[j];
        r.p = h->p[st];
        r.scp = h->d_coef + st;
        r.prev = h->prev[st];
      }
      e = ea::launch_colocated_batch_stale(b, n, h->hp, opt, h->variant, h->num_sms, s);
      if (e != cudaSuccess) return cuda_fail(h, e, "co-located stale kernel launch");
    }
    return EA_OK;
  }
  if (n > ea::kMaxFusedN || force_wide || stale) {  // replica loop: one launch per stage
    for (int j = 0; j < count; ++j) {
      const int st = stages[j];
      ea::ReplicaTable t;
      for (int i = 0; i < n; ++i) {
        t.x[i] = replica_ptrs[j * n + i];
        t.g[i] = grad_ptrs[j * n + i];
        t.m[i] = state_ptr(h, 0, st, i);
        t.v[i] = two ? state_ptr(h, 1, st, i) : nullptr;
      }
      ea_status st2 = advance(h, &stages[j], 1, s);
      if (st2 != EA_OK) return st2;
      float* prev = stale ? h->prev[st] : nullptr;
      e = ea::launch_colocated_wide(t, n, center_ptrs[j], prev, h->p[st], h->hp, opt, h->d_coef + st, h->num_sms, s);
      if (e != cudaSuccess) return cuda_fail(h, e, "co-located kernel launch");
    }
    return EA_OK;
  }
  for (int j0 = 0; j0 < count; j0 += ea::kMaxLaunchStages) {
    const int cnt = count - j0 < ea::kMaxLaunchStages ? count - j0 : ea::kMaxLaunchStages;
    ea_status st2 = advance(h, stages + j0, cnt, s);
    if (st2 != EA_OK) return st2;
    ea::StageBatch b;
    b.nstages = 0;
    for (int j = j0; j < count && j < j0 + ea::kMaxLaunchStages; ++j) {
      const int st = stages[j];
      ea::StageRefs& r = b.st[b.nstages++];
      for (int i = 0; i < ea::kMaxFusedN; ++i) {
        const bool on = i < n;
        r.x[i] = on ? replica_ptrs[j * n + i] : nullptr;
        r.g[i] = on ? grad_ptrs[j * n + i] : nullptr;
        r.m[i] = on ? state_ptr(h, 0, st, i) : nullptr;
        r.v[i] = (on && two) ? state_ptr(h, 1, st, i) : nullptr;
      }
      r.c = center_ptrs[j];
      r.p = h->p[st];
      r.scp = h->d_coef + st;
    }
    e = ea::launch_colocated_batch(b, n, h->hp, opt, h->variant, h->num_sms, s);
    if (e != cudaSuccess) return cuda_fail(h, e, "co-located kernel launch");
  }
  return EA_OK;
}

// Row a8 knobs (measurement).  The exchange runs on the library's side stream beside the caller's
// compute.  At world > 1 its own kernel (the shard update, P_pad/N elements) is small and takes few SMs:
// AVGPIPE_EA_SIDE_CTAS (default num_sms/4; 0 = the persistent grid) caps spread_apply's grid.  At world 1 the
// "exchange" is the whole center (12 B per element of local HBM traffic, as much as half the local step) and
// the cap only stretches it out under the compute (C5 harness: EA alone 29 ms capped vs 11 ms), so it is not
// capped.  The local kernels of the spread layout run on the caller's stream with persistent grids that hold
// every SM for their whole duration: AVGPIPE_EA_SPREAD_RESERVE_SMS SMs can be left free for the side stream
// (default 0: measured no gain, profiles/r02_a8_trace.md).
int side_ctas(const ea_ctx* h) {
  static const int v = [] {
    const char* e = std::getenv("AVGPIPE_EA_SIDE_CTAS");
    return e ? std::atoi(e) : -1;
  }();
  if (v >= 0) return v;  // 0: no cap
  if (h->cfg.world <= 1) return 0;
  return h->num_sms / 4 > 0 ? h->num_sms / 4 : 1;
}

// Pieces per stage of the NCCL spread step (knob AVGPIPE_EA_SPREAD_CHUNKS, 1..64; default 1 = the whole stage).
int spread_chunks() {
  static const int v = [] {
    const char* e = std::getenv("AVGPIPE_EA_SPREAD_CHUNKS");
    const int k = e ? std::atoi(e) : 1;
    return k >= 1 && k <= 64 ? k : 1;
  }();
  return v;
}

int spread_local_sms(int num_sms) {
  static const int v = [] {
    const char* e = std::getenv("AVGPIPE_EA_SPREAD_RESERVE_SMS");
    return e ? std::atoi(e) : kSpreadReserveSms;
  }();
  const int k = num_sms - (v > 0 ? v : 0);
  return k >= 1 ? k : 1;
}

// Spread: one stage's exchange on the side stream (rows a6-a8).
ea_status p2p_step(ea_ctx* h, int32_t stage, float* replica, const float* grad, float* center_ptr, cudaStream_t s);

ea_status spread_step(ea_ctx* h, int32_t stage, float* replica, const float* grad, float* center_ptr, cudaStream_t s) {
  if (h->cfg.exchange == EA_XCHG_P2P) return p2p_step(h, stage, replica, grad, center_ptr, s);
  if (!h->comm) {
    set_err(h, "EA_SPREAD handle created without an NCCL id: use ea_spread_local / ea_spread_apply");
    return EA_ESTATE;
  }
  cudaError_t e;
  const int n = h->cfg.n_pipelines;
  const int64_t pad = h->p_pad[stage];
  float* contrib = h->contrib + h->contrib_off[stage];
  const bool stale = h->cfg.staleness == 1;
  // Local phase on the CALLER's stream (x_i, state and r_i ready there, in stream order).  Synchronous center:
  // it reads x~_t, so it waits for this stage's previous all-gather (a no-op wait when that finished long ago).
  // Staleness 1 (row f4, reading c28): it reads x~_{t-1} from prev, which the previous exchange snapshotted
  // before its reduce-scatter -- so that whole exchange overlaps this iteration (P:112 asynchronous queues).
  if (stale) {
    ea_status st0 = stale_prev_init(h, stage, center_ptr, s);
    if (st0 != EA_OK) return st0;
  }
  if ((e = cudaStreamWaitEvent(s, stale ? h->ev_snap[stage] : h->ev_ag[stage], 0)) != cudaSuccess)
    return cuda_fail(h, e, "cudaStreamWaitEvent");
  ea_status st2 = advance(h, &stage, 1, s);
  if (st2 != EA_OK) return st2;
  // Intra-stage pipelining (knob AVGPIPE_EA_SPREAD_CHUNKS = C, default 1; synchronous center only): the stage is
  // cut into C pieces of whole 32N-float blocks; the local kernel of piece k runs on the caller's stream while
  // piece k-1's reduce-scatter / shard update / all-gather run on the side stream.  Within piece k rank r owns
  // block r of its N equal blocks (so the reduce-scatter and the in-place all-gather of a piece are plain NCCL
  // calls on the piece).
  const int chunks = stale ? 1 : spread_chunks();
  const int64_t L = round_up((pad + chunks - 1) / chunks, 32LL * n);
  float* m0 = state_ptr(h, 0, stage, 0);
  float* v0 = state_ptr(h, 1, stage, 0);
  const float* cread = stale ? h->prev[stage] : center_ptr;
  const int64_t p = h->p[stage];
  for (int64_t off = 0; off < pad; off += L) {
    const int64_t len = pad - off < L ? pad - off : L, cnt = len / n;
    const int64_t pk = p - off <= 0 ? 0 : (p - off < len ? p - off : len);  // replica elements in this piece
    e = ea::launch_spread_local(replica + (pk ? off : 0), grad + (pk ? off : 0), m0 + (pk ? off : 0),
                                v0 ? v0 + (pk ? off : 0) : nullptr, cread + (pk ? off : 0), contrib + off, pk, len,
                                h->hp, h->cfg.optimizer, h->d_coef + stage, spread_local_sms(h->num_sms), s);
    if (e != cudaSuccess) return cuda_fail(h, e, "spread local kernel launch");
    if ((e = cudaEventRecord(h->ev_loc[stage], s)) != cudaSuccess) return cuda_fail(h, e, "cudaEventRecord");
    // Exchange on the side stream: reduce-scatter -> owner-shard update -> in-place all-gather.  The caller's
    // stream does not wait for it; the next local step of this stage (or ea_sync) does.
    if ((e = cudaStreamWaitEvent(h->side, h->ev_loc[stage], 0)) != cudaSuccess)
      return cuda_fail(h, e, "cudaStreamWaitEvent");
    if (stale) {  // prev <- x~_t (final: the previous all-gather precedes this on the side stream)
      e = cudaMemcpyAsync(h->prev[stage], center_ptr, sizeof(float) * p, cudaMemcpyDeviceToDevice, h->side);
      if (e != cudaSuccess) return cuda_fail(h, e, "stale-center snapshot");
      if ((e = cudaEventRecord(h->ev_snap[stage], h->side)) != cudaSuccess) return cuda_fail(h, e, "cudaEventRecord");
    }
    float* own = center_ptr + off + cnt * h->cfg.rank;
    ncclResult_t r = ncclReduceScatter(contrib + off, h->reduced, static_cast<size_t>(cnt), ncclFloat, ncclSum,
                                       h->comm, h->side);
    if (r != ncclSuccess) return nccl_fail(h, r, "ncclReduceScatter");
    e = ea::launch_spread_apply(own, h->reduced, cnt, h->hp.inv_n, h->num_sms, side_ctas(h), h->side);
    if (e != cudaSuccess) return cuda_fail(h, e, "spread apply kernel launch");
    r = ncclAllGather(own, center_ptr + off, static_cast<size_t>(cnt), ncclFloat, h->comm, h->side);
    if (r != ncclSuccess) return nccl_fail(h, r, "ncclAllGather");
  }
  if ((e = cudaEventRecord(h->ev_ag[stage], h->side)) != cudaSuccess) return cuda_fail(h, e, "cudaEventRecord");
  return EA_OK;
}

// Orders `stream` after everything enqueued on the side stream so far.
ea_status join_side(ea_ctx* h, cudaStream_t s) {
  if (h->cfg.layout != EA_SPREAD) return EA_OK;
  cudaError_t e;
  if ((e = cudaEventRecord(h->ev_done, h->side)) != cudaSuccess) return cuda_fail(h, e, "cudaEventRecord");
  if ((e = cudaStreamWaitEvent(s, h->ev_done, 0)) != cudaSuccess) return cuda_fail(h, e, "cudaStreamWaitEvent");
  return EA_OK;
}

uint64_t p2p_timeout_ns() {
  const char* e = std::getenv("AVGPIPE_EA_P2P_TIMEOUT_MS");
  const long long ms = e ? std::atoll(e) : 30000;
  return static_cast<uint64_t>(ms > 0 ? ms : 30000) * 1000000ull;
}

// Measurement knob AVGPIPE_EA_P2P_FENCE=1: a fence.sc.sys before the release operations that publish a chunk.
// Default off: bar.sync orders the CTA's stores before thread 0's release, which is cumulative at system
// scope (PTX memory model); the fence measured 1.5-2.5% slower (profiles/r01_s3_p2p_fence.jsonl).
int p2p_sc_fence() {
  static const int v = [] {
    const char* e = std::getenv("AVGPIPE_EA_P2P_FENCE");
    return (e && e[0] == '1') ? 1 : 0;
  }();
  return v;
}

// Lay out and allocate this rank's exchange buffer (per stage: inbox, outbox, counters).
ea_status p2p_alloc(ea_ctx* h) {
  const int n = h->cfg.n_pipelines;
  size_t off = 0;
  auto take = [&](size_t bytes) {
    const size_t at = off;
    off += (bytes + 255) / 256 * 256;
    return at;
  };
  const int64_t kP2PChunk = h->x_chunk = p2p_chunk();
  for (int s = 0; s < h->cfg.n_stages; ++s) {
    const int64_t nch = (h->p_pad[s] + kP2PChunk - 1) / kP2PChunk;
    const int64_t slots = (nch + n - 1) / n;
    h->x_nchunks.push_back(nch);
    h->x_slots.push_back(slots);
    h->x_inbox.push_back(take(sizeof(float) * (size_t)n * slots * kP2PChunk));
    h->x_outbox.push_back(take(sizeof(float) * (size_t)slots * kP2PChunk));
    h->x_arrive.push_back(take(sizeof(uint32_t) * (size_t)slots));
    h->x_ready.push_back(take(sizeof(uint32_t) * (size_t)slots));
  }
  h->xbuf_bytes = off;
  cudaError_t e;
  if ((e = cudaMalloc(&h->xbuf, off)) != cudaSuccess) return cuda_fail(h, e, "exchange buffer");
  if ((e = cudaMemset(h->xbuf, 0, off)) != cudaSuccess) return cuda_fail(h, e, "exchange buffer init");
  const size_t ctl = sizeof(uint32_t) * (2 * (size_t)h->cfg.n_stages + 1);
  if ((e = cudaMalloc(&h->d_xctl, ctl)) != cudaSuccess || (e = cudaMemset(h->d_xctl, 0, ctl)) != cudaSuccess)
    return cuda_fail(h, e, "exchange control words");
  if ((e = cudaHostAlloc(&h->err_host, sizeof(uint32_t), cudaHostAllocMapped)) != cudaSuccess)
    return cuda_fail(h, e, "error flag");
  *h->err_host = 0;
  if ((e = cudaHostGetDevicePointer(&h->err_dev, h->err_host, 0)) != cudaSuccess) return cuda_fail(h, e, "error flag");
  h->peer_base.assign(n, nullptr);
  h->peer_ipc.assign(n, 0);
  h->peer_base[h->cfg.rank] = h->xbuf;
  return EA_OK;
}

// Map every peer's exchange buffer through CUDA IPC (handles all-gathered over NCCL).
// Open every peer's exchange buffer from the all-gathered IPC handles
// (world x EA_IPC_HANDLE_BYTES, rank-major).
ea_status p2p_open_handles(ea_ctx* h, const uint8_t* all) {
  const int n = h->cfg.n_pipelines, r = h->cfg.rank;
  const size_t hb = sizeof(cudaIpcMemHandle_t);
  for (int q = 0; q < n; ++q) {
    if (q == r) continue;
    cudaIpcMemHandle_t hq;
    std::memcpy(&hq, all + hb * q, hb);
    void* p = nullptr;
    cudaError_t e = cudaIpcOpenMemHandle(&p, hq, cudaIpcMemLazyEnablePeerAccess);
    if (e != cudaSuccess) return cuda_fail(h, e, "cudaIpcOpenMemHandle (peer exchange buffer)");
    h->peer_base[q] = static_cast<char*>(p);
    h->peer_ipc[q] = 1;
  }
  h->same_device_ranks = 1;
  h->p2p_ready = true;
  return EA_OK;
}

// Map every peer's exchange buffer through CUDA IPC (handles all-gathered over NCCL).
ea_status p2p_ipc_connect(ea_ctx* h) {
  const int n = h->cfg.n_pipelines;
  cudaIpcMemHandle_t mine;
  cudaError_t e = cudaIpcGetMemHandle(&mine, h->xbuf);
  if (e != cudaSuccess) return cuda_fail(h, e, "cudaIpcGetMemHandle");
  const size_t hb = sizeof(cudaIpcMemHandle_t);
  char* dev = nullptr;
  if ((e = cudaMalloc(&dev, hb * (n + 1))) != cudaSuccess) return cuda_fail(h, e, "handle exchange buffer");
  std::vector<uint8_t> all(hb * n);
  ea_status st = EA_OK;
  cudaStream_t s = h->side;
  if ((e = cudaMemcpyAsync(dev + hb * n, &mine, hb, cudaMemcpyHostToDevice, s)) != cudaSuccess) {
    st = cuda_fail(h, e, "handle upload");
  } else {
    ncclResult_t nr = ncclAllGather(dev + hb * n, dev, hb, ncclChar, h->comm, s);
    if (nr != ncclSuccess) st = nccl_fail(h, nr, "IPC handle all-gather");
    else if ((e = cudaMemcpyAsync(all.data(), dev, hb * n, cudaMemcpyDeviceToHost, s)) != cudaSuccess ||
             (e = cudaStreamSynchronize(s)) != cudaSuccess)
      st = cuda_fail(h, e, "handle download");
  }
  cudaFree(dev);
  if (st != EA_OK) return st;
  return p2p_open_handles(h, all.data());
}

// CTAs of p2p_exchange (phases B/C on the side stream).  Its work is NVLink/latency-bound and it runs beside
// the next forward, so one rank per device takes num_sms / 3.  Ranks sharing a device (virtual ranks) must
// together never be able to fill it: their exchange kernels spin while other ranks' pushes on the same device
// still need SMs (8 ranks x 49 CTAs of 32K registers did fill it, and timed out).  An exchange CTA holds half an
// SM's registers, so at most num_sms of them over all ranks always leave a push CTA room on every SM (or half
// the SMs free): num_sms / ranks each.  Knob AVGPIPE_EA_P2P_XCTAS (1..4096) for measurement.
int p2p_exchange_ctas(const ea_ctx* h) {
  const char* e = std::getenv("AVGPIPE_EA_P2P_XCTAS");
  const long long v = e ? std::atoll(e) : 0;
  if (v >= 1 && v <= 4096) return static_cast<int>(v);
  const int ranks = h->same_device_ranks > 0 ? h->same_device_ranks : 1;
  int k = h->num_sms / 3;
  if (ranks > 1) k = h->num_sms / ranks;
  else if (h->cfg.world <= 1) k = 2 * h->num_sms;  // world 1: phase B over the whole center, local HBM work
  return k > 0 ? k : 1;
}

// One stage of the peer-memory exchange: p2p_push (local update + contributions into the owners' inboxes) on
// the caller's stream after this stage's previous exchange, p2p_exchange (owner reduction, center update, pull
// of the other shards) on the side stream, which the caller's stream never waits for (row a8).
ea_status p2p_step(ea_ctx* h, int32_t stage, float* replica, const float* grad, float* center_ptr, cudaStream_t s) {
  if (!h->p2p_ready) {
    set_err(h, "peer-memory exchange not connected (needs an NCCL id at ea_init or ea_p2p_connect)");
    return EA_ESTATE;
  }
  if (*reinterpret_cast<volatile uint32_t*>(h->err_host)) {
    set_err(h, "a previous peer-memory exchange timed out; the handle is unusable");
    return EA_ECUDA;
  }
  const int n = h->cfg.n_pipelines;
  ea::P2PView v;
  for (int q = 0; q < ea::kMaxWorld; ++q) {
    char* b = q < n ? h->peer_base[q] : nullptr;
    v.inbox[q] = b ? reinterpret_cast<float*>(b + h->x_inbox[stage]) : nullptr;
    v.outbox[q] = b ? reinterpret_cast<float*>(b + h->x_outbox[stage]) : nullptr;
    v.arrive[q] = b ? reinterpret_cast<uint32_t*>(b + h->x_arrive[stage]) : nullptr;
    v.ready[q] = b ? reinterpret_cast<uint32_t*>(b + h->x_ready[stage]) : nullptr;
  }
  ea::P2PArgs a;
  a.x = replica;
  a.g = grad;
  a.m = state_ptr(h, 0, stage, 0);
  a.v = state_ptr(h, 1, stage, 0);
  a.center = center_ptr;
  a.p = h->p[stage];
  a.p_pad = h->p_pad[stage];
  a.chunk = h->x_chunk;
  a.nchunks = h->x_nchunks[stage];
  a.slots = h->x_slots[stage];
  a.rank = h->cfg.rank;
  a.world = n;
  a.epochp = h->d_xctl + stage;
  a.tickets = h->d_xctl + h->cfg.n_stages + stage;
  a.abort = h->d_xctl + 2 * h->cfg.n_stages;
  a.scp = h->d_coef + stage;
  a.hp = h->hp;
  a.err = h->err_dev;
  a.timeout_ns = p2p_timeout_ns();
  a.sc_fence = p2p_sc_fence();
  cudaError_t e;
  // the push reads the center: after this stage's previous exchange (a no-op wait when long finished)
  if ((e = cudaStreamWaitEvent(s, h->ev_ag[stage], 0)) != cudaSuccess) return cuda_fail(h, e, "cudaStreamWaitEvent");
  ea_status st2 = advance(h, &stage, 1, s);
  if (st2 != EA_OK) return st2;
  // ranks sharing this device (virtual ranks) share its SMs
  int max_sms = spread_local_sms(h->num_sms) / h->same_device_ranks;
  if (max_sms < 1) max_sms = 1;
  int max_ctas = max_sms * ea::p2p_blocks_per_sm(h->cfg.optimizer);
  if ((e = ea::launch_p2p_push(a, v, h->cfg.optimizer, max_ctas, max_sms, s)) != cudaSuccess)
    return cuda_fail(h, e, "peer-memory push kernel launch");
  if ((e = cudaEventRecord(h->ev_loc[stage], s)) != cudaSuccess) return cuda_fail(h, e, "cudaEventRecord");
  if ((e = cudaStreamWaitEvent(h->side, h->ev_loc[stage], 0)) != cudaSuccess)
    return cuda_fail(h, e, "cudaStreamWaitEvent");
  if ((e = ea::launch_p2p_exchange(a, v, p2p_exchange_ctas(h), h->side)) != cudaSuccess)
    return cuda_fail(h, e, "peer-memory exchange kernel launch");
  if ((e = cudaEventRecord(h->ev_ag[stage], h->side)) != cudaSuccess) return cuda_fail(h, e, "cudaEventRecord");
  return EA_OK;
}

bool is_host_ptr(const void* p) {
  cudaPointerAttributes a;
  if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
    cudaGetLastError();
    return true;  // unregistered pageable memory
  }
  return a.type == cudaMemoryTypeHost || a.type == cudaMemoryTypeUnregistered;
}

ea_status host_path_resources(ea_ctx* h) {
  if (h->h2d) return EA_OK;
  cudaError_t e;
  const size_t bytes = sizeof(float) * (size_t)h->cfg.n_pipelines * kHostChunk;
  if ((e = cudaStreamCreateWithFlags(&h->h2d, cudaStreamNonBlocking)) != cudaSuccess ||
      (e = cudaStreamCreateWithFlags(&h->d2h, cudaStreamNonBlocking)) != cudaSuccess ||
      (e = cudaMalloc(&h->staging[0], bytes)) != cudaSuccess || (e = cudaMalloc(&h->staging[1], bytes)) != cudaSuccess ||
      (e = cudaEventCreateWithFlags(&h->ev_h2d[0], cudaEventDisableTiming)) != cudaSuccess ||
      (e = cudaEventCreateWithFlags(&h->ev_h2d[1], cudaEventDisableTiming)) != cudaSuccess ||
      (e = cudaEventCreateWithFlags(&h->ev_kern[0], cudaEventDisableTiming)) != cudaSuccess ||
      (e = cudaEventCreateWithFlags(&h->ev_kern[1], cudaEventDisableTiming)) != cudaSuccess ||
      (e = cudaEventCreateWithFlags(&h->ev_d2h, cudaEventDisableTiming)) != cudaSuccess)
    return cuda_fail(h, e, "host-path resources");
  return EA_OK;
}

// Slot EA_SLOT_CENTER_PREV: the stale center x~_{t-1} of a staleness-1 handle (P_s floats, replica 0).
bool prev_slot(const ea_ctx* h, int32_t replica, int32_t slot) {
  return slot == EA_SLOT_CENTER_PREV && h->cfg.staleness == 1 && replica == 0;
}

float* slot_ptr(const ea_ctx* h, int32_t stage, int32_t replica, int32_t slot) {
  return slot == EA_SLOT_CENTER_PREV ? h->prev[stage] : state_ptr(h, slot, stage, replica);
}

bool slot_ok(const ea_ctx* h, int32_t stage, int32_t replica, int32_t slot) {
  if (stage < 0 || stage >= h->cfg.n_stages) return false;
  if (prev_slot(h, replica, slot)) return true;
  return replica >= 0 && replica < replicas_here(h) && slot >= 0 && slot < state_slots(h);
}

}  // namespace

extern "C" {

int32_t ea_abi_version(void) { return EA_ABI_VERSION; }

ea_status ea_get_unique_id(uint8_t* id) {
  if (!id) { set_err(nullptr, "id is NULL"); return EA_EINVAL; }
  static_assert(sizeof(ncclUniqueId) == EA_UNIQUE_ID_BYTES, "ncclUniqueId size");
  ncclUniqueId u;
  ncclResult_t r = ncclGetUniqueId(&u);
  if (r != ncclSuccess) return nccl_fail(nullptr, r, "ncclGetUniqueId");
  std::memcpy(id, &u, sizeof(u));
  return EA_OK;
}

ea_status ea_init(const ea_config* cfg, const uint8_t* nccl_id, ea_handle* out) {
  if (!out) { set_err(nullptr, "out is NULL"); return EA_EINVAL; }
  *out = nullptr;
  if (!cfg) { set_err(nullptr, "cfg is NULL"); return EA_EINVAL; }
  const ea_config& c = *cfg;
  if (c.n_pipelines < 1) { set_err(nullptr, "n_pipelines must be >= 1, got %d", c.n_pipelines); return EA_EINVAL; }
  if (c.n_stages < 1 || !c.stage_params) { set_err(nullptr, "need n_stages >= 1 and stage_params"); return EA_EINVAL; }
  for (int s = 0; s < c.n_stages; ++s)
    if (c.stage_params[s] < 1) { set_err(nullptr, "stage_params[%d] must be >= 1", s); return EA_EINVAL; }
  if (c.layout != EA_COLOCATED && c.layout != EA_SPREAD) { set_err(nullptr, "unknown layout %d", c.layout); return EA_EINVAL; }
  if (c.layout == EA_COLOCATED && c.n_pipelines > EA_MAX_REPLICAS) {
    set_err(nullptr, "co-located N must be <= %d", EA_MAX_REPLICAS);
    return EA_EINVAL;
  }
  if (c.layout == EA_SPREAD) {
    if (c.world != c.n_pipelines) { set_err(nullptr, "EA_SPREAD needs world == n_pipelines"); return EA_EINVAL; }
    if (c.rank < 0 || c.rank >= c.world) { set_err(nullptr, "rank %d out of [0,%d)", c.rank, c.world); return EA_EINVAL; }
  }
  if (c.kernel_variant < 0 || c.kernel_variant > 6) { set_err(nullptr, "kernel_variant must be 0..6"); return EA_EINVAL; }
  if (c.exchange != EA_XCHG_NCCL && c.exchange != EA_XCHG_P2P) { set_err(nullptr, "unknown exchange %d", c.exchange); return EA_EINVAL; }
  if (c.staleness != 0 && c.staleness != 1) { set_err(nullptr, "staleness must be 0 or 1"); return EA_EINVAL; }
  if (c.staleness == 1 && c.layout == EA_SPREAD && c.exchange != EA_XCHG_NCCL) {
    set_err(nullptr, "staleness 1 in EA_SPREAD needs the NCCL exchange (the peer-memory exchange is one step)");
    return EA_EINVAL;
  }
  if (c.layout == EA_SPREAD && c.exchange == EA_XCHG_P2P && c.world > ea::kMaxWorld) {
    set_err(nullptr, "peer-memory exchange supports world <= %d", ea::kMaxWorld);
    return EA_EINVAL;
  }
  ea_status st = check_hyper(nullptr, c);
  if (st != EA_OK) return st;
  int ndev = 0;
  cudaError_t e = cudaGetDeviceCount(&ndev);
  if (e != cudaSuccess) return cuda_fail(nullptr, e, "cudaGetDeviceCount");
  if (c.device < 0 || c.device >= ndev) { set_err(nullptr, "device %d out of range (%d devices)", c.device, ndev); return EA_EINVAL; }

  ea_ctx* h = new (std::nothrow) ea_ctx;
  if (!h) { set_err(nullptr, "host allocation failed"); return EA_ENOMEM; }
  h->cfg = c;
  h->hp = make_hyper(c);
  h->variant = c.kernel_variant;
  h->p.assign(c.stage_params, c.stage_params + c.n_stages);
  h->steps.assign(c.n_stages, 0);
  h->cfg.stage_params = nullptr;  // not retained
  e = cudaSetDevice(c.device);
  if (e != cudaSuccess) { ea_status r = cuda_fail(nullptr, e, "cudaSetDevice"); free_ctx(h); return r; }
  cudaDeviceGetAttribute(&h->num_sms, cudaDevAttrMultiProcessorCount, c.device);
  if ((e = cudaMalloc(&h->d_steps, sizeof(int64_t) * c.n_stages)) != cudaSuccess ||
      (e = cudaMemset(h->d_steps, 0, sizeof(int64_t) * c.n_stages)) != cudaSuccess ||
      (e = cudaMalloc(&h->d_coef, sizeof(ea::StepCoef) * c.n_stages)) != cudaSuccess ||
      (e = cudaMemset(h->d_coef, 0, sizeof(ea::StepCoef) * c.n_stages)) != cudaSuccess) {
    ea_status r = cuda_fail(nullptr, e, "step counters");
    free_ctx(h);
    return r;
  }

  const int reps = replicas_here(h);
  int64_t max_pad = 0, sum_pad = 0;
  for (int s = 0; s < c.n_stages; ++s) {
    const int64_t ps = h->p[s];
    const int64_t pad = c.layout == EA_SPREAD ? round_up(ps, 32LL * c.n_pipelines) : ps;
    h->p_pad.push_back(pad);
    if (pad > max_pad) max_pad = pad;
    h->contrib_off.push_back(static_cast<size_t>(sum_pad));
    sum_pad += pad;
    const int64_t stride = round_up(ps, 64);
    h->stride.push_back(stride);
    for (int slot = 0; slot < state_slots(h); ++slot) {
      float* m = nullptr;
      e = cudaMalloc(&m, sizeof(float) * stride * reps);
      if (e == cudaSuccess) e = cudaMemset(m, 0, sizeof(float) * stride * reps);
      if (e != cudaSuccess) {
        ea_status r = cuda_fail(nullptr, e, "optimizer-state allocation");
        if (m) cudaFree(m);
        free_ctx(h);
        return r;
      }
      h->state[slot].push_back(m);
    }
    if (c.staleness == 1) {
      float* pv = nullptr;
      if ((e = cudaMalloc(&pv, sizeof(float) * stride)) != cudaSuccess) {
        ea_status r = cuda_fail(nullptr, e, "stale-center allocation");
        free_ctx(h);
        return r;
      }
      h->prev.push_back(pv);
      h->prev_init.push_back(0);
    }
  }
  if (c.layout == EA_SPREAD) {
    // the exchange's CTAs go first when SMs free up (it is short and latency-bound); knob AVGPIPE_EA_SIDE_PRIO=0
    // keeps the default priority
    int prio_lo = 0, prio_hi = 0;
    cudaDeviceGetStreamPriorityRange(&prio_lo, &prio_hi);
    const char* pe = std::getenv("AVGPIPE_EA_SIDE_PRIO");
    const int prio = (pe && pe[0] == '0') ? prio_lo : prio_hi;
    if ((e = cudaStreamCreateWithPriority(&h->side, cudaStreamNonBlocking, prio)) != cudaSuccess ||
        (e = cudaEventCreateWithFlags(&h->ev_done, cudaEventDisableTiming)) != cudaSuccess ||
        (c.exchange == EA_XCHG_NCCL && (e = cudaMalloc(&h->contrib, sizeof(float) * sum_pad)) != cudaSuccess) ||
        (e = cudaMalloc(&h->reduced, sizeof(float) * (max_pad / c.n_pipelines))) != cudaSuccess) {
      ea_status r = cuda_fail(nullptr, e, "spread resources");
      free_ctx(h);
      return r;
    }
    for (int st = 0; st < c.n_stages; ++st) {
      cudaEvent_t a = nullptr, b = nullptr, d = nullptr;
      if ((e = cudaEventCreateWithFlags(&a, cudaEventDisableTiming)) != cudaSuccess ||
          (e = cudaEventCreateWithFlags(&b, cudaEventDisableTiming)) != cudaSuccess ||
          (e = cudaEventCreateWithFlags(&d, cudaEventDisableTiming)) != cudaSuccess) {
        if (a) cudaEventDestroy(a);
        if (b) cudaEventDestroy(b);
        ea_status r = cuda_fail(nullptr, e, "per-stage events");
        free_ctx(h);
        return r;
      }
      h->ev_ag.push_back(a);
      h->ev_loc.push_back(b);
      h->ev_snap.push_back(d);
    }
    if (nccl_id) {  // NULL: external-collective mode (phase calls only)
      ncclUniqueId uid;
      std::memcpy(&uid, nccl_id, sizeof(uid));
      ncclResult_t nr = ncclCommInitRank(&h->comm, c.world, uid, c.rank);
      if (nr != ncclSuccess) {
        h->comm = nullptr;
        ea_status r = nccl_fail(nullptr, nr, "ncclCommInitRank");
        free_ctx(h);
        return r;
      }
    }
    if (c.exchange == EA_XCHG_P2P) {
      ea_status r = p2p_alloc(h);
      if (r == EA_OK && c.world == 1) h->p2p_ready = true;
      else if (r == EA_OK && h->comm) r = p2p_ipc_connect(h);
      if (r != EA_OK) {
        g_init_err = h->err;
        free_ctx(h);
        return r;
      }
    }
  }
  e = cudaDeviceSynchronize();
  if (e != cudaSuccess) { ea_status r = cuda_fail(nullptr, e, "init sync"); free_ctx(h); return r; }
  *out = h;
  return EA_OK;
}

int64_t ea_center_capacity(ea_handle h, int32_t stage) {
  if (!h || stage < 0 || stage >= h->cfg.n_stages) return -1;
  return h->p_pad[stage];
}

int64_t ea_shard_elems(ea_handle h, int32_t stage) {
  if (!h || stage < 0 || stage >= h->cfg.n_stages) return -1;
  return h->cfg.layout == EA_SPREAD ? h->p_pad[stage] / h->cfg.n_pipelines : h->p[stage];
}

ea_status ea_step(ea_handle h, int32_t stage, float* const* replica_ptrs, const float* const* grad_ptrs,
                  float* center_ptr, void* stream) {
  NvtxRange range("ea_step");
  if (!h) { set_err(nullptr, "handle is NULL"); return EA_EINVAL; }
  ea_status st = check_stage_ptrs(h, stage, replica_ptrs, grad_ptrs, center_ptr);
  if (st != EA_OK) return st;
  if (h->cfg.layout == EA_SPREAD && h->cfg.exchange == EA_XCHG_NCCL && !h->comm) {
    set_err(h, "EA_SPREAD handle created without an NCCL id: use ea_spread_local / ea_spread_apply");
    return EA_ESTATE;
  }
  cudaError_t e = cudaSetDevice(h->cfg.device);
  if (e != cudaSuccess) return cuda_fail(h, e, "cudaSetDevice");
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  if (h->cfg.layout == EA_COLOCATED) return colocated_launch(h, 1, &stage, replica_ptrs, grad_ptrs, &center_ptr, s);
  return spread_step(h, stage, replica_ptrs[0], grad_ptrs[0], center_ptr, s);
}

ea_status ea_step_many(ea_handle h, int32_t count, const int32_t* stages, float* const* replica_ptrs,
                       const float* const* grad_ptrs, float* const* center_ptrs, void* stream) {
  NvtxRange range("ea_step_many");
  if (!h) { set_err(nullptr, "handle is NULL"); return EA_EINVAL; }
  if (count < 0 || (count > 0 && (!stages || !replica_ptrs || !grad_ptrs || !center_ptrs))) {
    set_err(h, "ea_step_many: bad count or NULL array");
    return EA_EINVAL;
  }
  const int reps = replicas_here(h);
  for (int j = 0; j < count; ++j) {
    for (int k = 0; k < j; ++k)
      if (stages[k] == stages[j]) { set_err(h, "ea_step_many: stage %d listed twice", stages[j]); return EA_EINVAL; }
    ea_status st = check_stage_ptrs(h, stages[j], replica_ptrs + (size_t)j * reps, grad_ptrs + (size_t)j * reps,
                                    center_ptrs[j]);
    if (st != EA_OK) return st;
  }
  if (count == 0) return EA_OK;
  if (h->cfg.layout == EA_SPREAD && h->cfg.exchange == EA_XCHG_NCCL && !h->comm) {
    set_err(h, "EA_SPREAD handle created without an NCCL id: use ea_spread_local / ea_spread_apply");
    return EA_ESTATE;
  }
  cudaError_t e = cudaSetDevice(h->cfg.device);
  if (e != cudaSuccess) return cuda_fail(h, e, "cudaSetDevice");
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  if (h->cfg.layout == EA_COLOCATED) return colocated_launch(h, count, stages, replica_ptrs, grad_ptrs, center_ptrs, s);
  for (int j = 0; j < count; ++j) {
    ea_status st = spread_step(h, stages[j], replica_ptrs[j], grad_ptrs[j], center_ptrs[j], s);
    if (st != EA_OK) return st;
  }
  return EA_OK;
}

ea_status ea_step_many_host(ea_handle h, int32_t count, const int32_t* stages, float* const* replica_ptrs,
                            const float* const* host_grad_ptrs, float* const* center_ptrs,
                            float* const* host_center_out, void* stream) {
  NvtxRange range("ea_step_many_host");
  if (!h) { set_err(nullptr, "handle is NULL"); return EA_EINVAL; }
  if (h->cfg.layout != EA_COLOCATED) { set_err(h, "ea_step_many_host needs EA_COLOCATED"); return EA_ESTATE; }
  if (h->cfg.staleness != 0) { set_err(h, "ea_step_many_host does not support staleness 1"); return EA_ESTATE; }
  if (count < 0 || (count > 0 && (!stages || !replica_ptrs || !host_grad_ptrs || !center_ptrs || !host_center_out))) {
    set_err(h, "ea_step_many_host: bad count or NULL array");
    return EA_EINVAL;
  }
  const int n = h->cfg.n_pipelines;
  const int dev = h->cfg.device;
  for (int j = 0; j < count; ++j) {
    const int st = stages[j];
    if (st < 0 || st >= h->cfg.n_stages) { set_err(h, "stage %d out of range", st); return EA_EINVAL; }
    for (int k = 0; k < j; ++k)
      if (stages[k] == st) { set_err(h, "ea_step_many_host: stage %d listed twice", st); return EA_EINVAL; }
    if (!center_ptrs[j] || !aligned16(center_ptrs[j]) || !is_device_ptr(center_ptrs[j], dev) ||
        !host_center_out[j] || !is_host_ptr(host_center_out[j])) {
      set_err(h, "stage %d: center must be an aligned device pointer and host_center_out a host pointer", st);
      return EA_EINVAL;
    }
    for (int i = 0; i < n; ++i) {
      const float* x = replica_ptrs[(size_t)j * n + i];
      const float* g = host_grad_ptrs[(size_t)j * n + i];
      if (!x || !aligned16(x) || !is_device_ptr(x, dev) || !g || !is_host_ptr(g)) {
        set_err(h, "stage %d replica %d: replica must be an aligned device pointer, grad a host pointer", st, i);
        return EA_EINVAL;
      }
    }
  }
  if (count == 0) return EA_OK;
  cudaError_t e = cudaSetDevice(dev);
  if (e != cudaSuccess) return cuda_fail(h, e, "cudaSetDevice");
  ea_status rs = host_path_resources(h);
  if (rs != EA_OK) return rs;
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  const int opt = h->cfg.optimizer;
  const bool two = state_slots(h) == 2;
  // the copies must not overtake work already queued on the caller's stream
  if ((e = cudaEventRecord(h->ev_d2h, s)) != cudaSuccess) return cuda_fail(h, e, "cudaEventRecord");
  if ((e = cudaStreamWaitEvent(h->h2d, h->ev_d2h, 0)) != cudaSuccess) return cuda_fail(h, e, "cudaStreamWaitEvent");
  int64_t k = 0;  // chunk counter (staging buffer k % 2)
  for (int j = 0; j < count; ++j) {
    const int st = stages[j];
    ea_status st2 = advance(h, &stages[j], 1, s);
    if (st2 != EA_OK) return st2;
    const ea::StepCoef* sc = h->d_coef + st;
    const int64_t ps = h->p[st];
    const int64_t chunk = host_chunk();
    for (int64_t off = 0; off < ps; off += chunk, ++k) {
      const int64_t len = ps - off < chunk ? ps - off : chunk;
      const int b = static_cast<int>(k & 1);
      float* stage_buf = h->staging[b];
      // H2D of this chunk's gradients once the kernel that last read this buffer is done
      if (k >= 2 && (e = cudaStreamWaitEvent(h->h2d, h->ev_kern[b], 0)) != cudaSuccess)
        return cuda_fail(h, e, "cudaStreamWaitEvent");
      for (int i = 0; i < n; ++i) {
        e = cudaMemcpyAsync(stage_buf + (size_t)i * kHostChunk, host_grad_ptrs[(size_t)j * n + i] + off,
                            sizeof(float) * len, cudaMemcpyHostToDevice, h->h2d);
        if (e != cudaSuccess) return cuda_fail(h, e, "H2D gradients");
      }
      if ((e = cudaEventRecord(h->ev_h2d[b], h->h2d)) != cudaSuccess) return cuda_fail(h, e, "cudaEventRecord");
      if ((e = cudaStreamWaitEvent(s, h->ev_h2d[b], 0)) != cudaSuccess) return cuda_fail(h, e, "cudaStreamWaitEvent");
      // the fused step on [off, off+len) of the stage (elementwise: any chunk is a valid sub-problem)
      if (n > ea::kMaxFusedN) {
        ea::ReplicaTable t;
        for (int i = 0; i < n; ++i) {
          t.x[i] = replica_ptrs[(size_t)j * n + i] + off;
          t.g[i] = stage_buf + (size_t)i * kHostChunk;
          t.m[i] = state_ptr(h, 0, st, i) + off;
          t.v[i] = two ? state_ptr(h, 1, st, i) + off : nullptr;
        }
        e = ea::launch_colocated_wide(t, n, center_ptrs[j] + off, nullptr, len, h->hp, opt, sc, h->num_sms, s);
      } else {
        ea::StageBatch bt;
        bt.nstages = 1;
        ea::StageRefs& r = bt.st[0];
        for (int i = 0; i < ea::kMaxFusedN; ++i) {
          const bool on = i < n;
          r.x[i] = on ? replica_ptrs[(size_t)j * n + i] + off : nullptr;
          r.g[i] = on ? stage_buf + (size_t)i * kHostChunk : nullptr;
          r.m[i] = on ? state_ptr(h, 0, st, i) + off : nullptr;
          r.v[i] = (on && two) ? state_ptr(h, 1, st, i) + off : nullptr;
        }
        r.c = center_ptrs[j] + off;
        r.p = len;
        r.scp = sc;
        e = ea::launch_colocated_batch(bt, n, h->hp, opt, h->variant, h->num_sms, s);
      }
      if (e != cudaSuccess) return cuda_fail(h, e, "co-located kernel launch");
      if ((e = cudaEventRecord(h->ev_kern[b], s)) != cudaSuccess) return cuda_fail(h, e, "cudaEventRecord");
      // D2H of the updated center chunk
      if ((e = cudaStreamWaitEvent(h->d2h, h->ev_kern[b], 0)) != cudaSuccess)
        return cuda_fail(h, e, "cudaStreamWaitEvent");
      e = cudaMemcpyAsync(host_center_out[j] + off, center_ptrs[j] + off, sizeof(float) * len, cudaMemcpyDeviceToHost,
                          h->d2h);
      if (e != cudaSuccess) return cuda_fail(h, e, "D2H center");
    }
  }
  if ((e = cudaEventRecord(h->ev_d2h, h->d2h)) != cudaSuccess) return cuda_fail(h, e, "cudaEventRecord");
  if ((e = cudaStreamWaitEvent(s, h->ev_d2h, 0)) != cudaSuccess) return cuda_fail(h, e, "cudaStreamWaitEvent");
  return EA_OK;
}

ea_status ea_p2p_connect(ea_handle h, const ea_handle* peers, int32_t world) {
  if (!h) { set_err(nullptr, "handle is NULL"); return EA_EINVAL; }
  if (h->cfg.layout != EA_SPREAD || h->cfg.exchange != EA_XCHG_P2P) {
    set_err(h, "ea_p2p_connect needs EA_SPREAD with exchange EA_XCHG_P2P");
    return EA_ESTATE;
  }
  if (!peers || world != h->cfg.world) { set_err(h, "peers must list all %d ranks", h->cfg.world); return EA_EINVAL; }
  int same = 0;
  for (int q = 0; q < world; ++q) {
    const ea_ctx* o = peers[q];
    if (!o || o->cfg.rank != q || o->cfg.world != world || o->cfg.layout != EA_SPREAD ||
        o->cfg.exchange != EA_XCHG_P2P || o->cfg.n_stages != h->cfg.n_stages || o->p != h->p || !o->xbuf) {
      set_err(h, "peer %d is not a matching EA_SPREAD/EA_XCHG_P2P handle of rank %d", q, q);
      return EA_EINVAL;
    }
    if (o->cfg.device == h->cfg.device) {
      ++same;
    } else {
      int can = 0;
      cudaDeviceCanAccessPeer(&can, h->cfg.device, o->cfg.device);
      if (!can) { set_err(h, "device %d cannot access device %d", h->cfg.device, o->cfg.device); return EA_EINVAL; }
      cudaSetDevice(h->cfg.device);
      cudaError_t e = cudaDeviceEnablePeerAccess(o->cfg.device, 0);
      if (e != cudaSuccess && e != cudaErrorPeerAccessAlreadyEnabled) return cuda_fail(h, e, "cudaDeviceEnablePeerAccess");
      cudaGetLastError();
    }
  }
  if (h != peers[h->cfg.rank]) { set_err(h, "peers[rank] must be this handle"); return EA_EINVAL; }
  for (int q = 0; q < world; ++q) h->peer_base[q] = peers[q]->xbuf;
  h->same_device_ranks = same;
  h->p2p_ready = true;
  return EA_OK;
}

ea_status ea_p2p_export(ea_handle h, uint8_t* handle) {
  if (!h || !handle) { set_err(h, "NULL handle or output"); return EA_EINVAL; }
  if (h->cfg.layout != EA_SPREAD || h->cfg.exchange != EA_XCHG_P2P || !h->xbuf) {
    set_err(h, "ea_p2p_export needs EA_SPREAD with exchange EA_XCHG_P2P");
    return EA_ESTATE;
  }
  static_assert(sizeof(cudaIpcMemHandle_t) == EA_IPC_HANDLE_BYTES, "IPC handle size");
  cudaError_t e = cudaSetDevice(h->cfg.device);
  if (e == cudaSuccess) e = cudaIpcGetMemHandle(reinterpret_cast<cudaIpcMemHandle_t*>(handle), h->xbuf);
  if (e != cudaSuccess) return cuda_fail(h, e, "cudaIpcGetMemHandle");
  return EA_OK;
}

ea_status ea_p2p_open(ea_handle h, const uint8_t* handles, int32_t world) {
  if (!h || !handles) { set_err(h, "NULL handle or handle list"); return EA_EINVAL; }
  if (h->cfg.layout != EA_SPREAD || h->cfg.exchange != EA_XCHG_P2P || !h->xbuf) {
    set_err(h, "ea_p2p_open needs EA_SPREAD with exchange EA_XCHG_P2P");
    return EA_ESTATE;
  }
  if (world != h->cfg.world) { set_err(h, "handle list must have world = %d entries", h->cfg.world); return EA_EINVAL; }
  if (h->p2p_ready) { set_err(h, "peer exchange already connected"); return EA_ESTATE; }
  cudaError_t e = cudaSetDevice(h->cfg.device);
  if (e != cudaSuccess) return cuda_fail(h, e, "cudaSetDevice");
  return p2p_open_handles(h, handles);
}

ea_status ea_sync(ea_handle h, void* stream) {
  NvtxRange range("ea_sync");
  if (!h) { set_err(nullptr, "handle is NULL"); return EA_EINVAL; }
  cudaError_t e = cudaSetDevice(h->cfg.device);
  if (e != cudaSuccess) return cuda_fail(h, e, "cudaSetDevice");
  ea_status st = join_side(h, static_cast<cudaStream_t>(stream));
  if (st != EA_OK) return st;
  if (h->err_host && *reinterpret_cast<volatile uint32_t*>(h->err_host)) {
    set_err(h, "peer-memory exchange timed out (a rank did not reach the same step)");
    return EA_ECUDA;
  }
  if (h->comm) {
    ncclResult_t async_err = ncclSuccess;
    ncclResult_t r = ncclCommGetAsyncError(h->comm, &async_err);
    if (r != ncclSuccess) return nccl_fail(h, r, "ncclCommGetAsyncError");
    if (async_err != ncclSuccess && async_err != ncclInProgress) return nccl_fail(h, async_err, "NCCL async error");
  }
  e = cudaGetLastError();
  if (e != cudaSuccess) return cuda_fail(h, e, "asynchronous CUDA error");
  return EA_OK;
}

ea_status ea_spread_local(ea_handle h, int32_t stage, float* replica_ptr, const float* grad_ptr,
                          const float* center_ptr, float* contrib, void* stream) {
  if (!h) { set_err(nullptr, "handle is NULL"); return EA_EINVAL; }
  if (h->cfg.layout != EA_SPREAD) { set_err(h, "ea_spread_local needs EA_SPREAD"); return EA_ESTATE; }
  if (stage < 0 || stage >= h->cfg.n_stages) { set_err(h, "stage %d out of range", stage); return EA_EINVAL; }
  const int dev = h->cfg.device;
  const void* ptrs[4] = {replica_ptr, grad_ptr, center_ptr, contrib};
  for (const void* p : ptrs)
    if (!p || !aligned16(p) || !is_device_ptr(p, dev)) {
      set_err(h, "pointers must be 16-byte aligned device pointers on device %d", dev);
      return EA_EINVAL;
    }
  cudaError_t e = cudaSetDevice(dev);
  if (e != cudaSuccess) return cuda_fail(h, e, "cudaSetDevice");
  ea_status st2 = advance(h, &stage, 1, static_cast<cudaStream_t>(stream));
  if (st2 != EA_OK) return st2;
  e = ea::launch_spread_local(replica_ptr, grad_ptr, state_ptr(h, 0, stage, 0), state_ptr(h, 1, stage, 0), center_ptr,
                              contrib, h->p[stage], h->p_pad[stage], h->hp, h->cfg.optimizer, h->d_coef + stage,
                              h->num_sms, static_cast<cudaStream_t>(stream));
  if (e != cudaSuccess) return cuda_fail(h, e, "spread local kernel launch");
  return EA_OK;
}

ea_status ea_spread_apply(ea_handle h, int32_t stage, float* center_shard, const float* reduced, void* stream) {
  if (!h) { set_err(nullptr, "handle is NULL"); return EA_EINVAL; }
  if (h->cfg.layout != EA_SPREAD) { set_err(h, "ea_spread_apply needs EA_SPREAD"); return EA_ESTATE; }
  if (stage < 0 || stage >= h->cfg.n_stages) { set_err(h, "stage %d out of range", stage); return EA_EINVAL; }
  const int dev = h->cfg.device;
  if (!center_shard || !reduced || !aligned16(center_shard) || !aligned16(reduced) ||
      !is_device_ptr(center_shard, dev) || !is_device_ptr(reduced, dev)) {
    set_err(h, "pointers must be 16-byte aligned device pointers on device %d", dev);
    return EA_EINVAL;
  }
  cudaError_t e = cudaSetDevice(dev);
  if (e != cudaSuccess) return cuda_fail(h, e, "cudaSetDevice");
  e = ea::launch_spread_apply(center_shard, reduced, h->p_pad[stage] / h->cfg.n_pipelines, h->hp.inv_n, h->num_sms, 0,
                              static_cast<cudaStream_t>(stream));
  if (e != cudaSuccess) return cuda_fail(h, e, "spread apply kernel launch");
  return EA_OK;
}

ea_status ea_get_state(ea_handle h, int32_t stage, int32_t replica, int32_t slot, float** state_dev) {
  if (!h) { set_err(nullptr, "handle is NULL"); return EA_EINVAL; }
  if (!state_dev || !slot_ok(h, stage, replica, slot)) {
    set_err(h, "bad stage/replica/slot or NULL out pointer (this optimizer has %d state slot(s); "
               "EA_SLOT_CENTER_PREV needs staleness 1 and replica 0)", state_slots(h));
    return EA_EINVAL;
  }
  *state_dev = slot_ptr(h, stage, replica, slot);
  return EA_OK;
}

ea_status ea_set_state(ea_handle h, int32_t stage, int32_t replica, int32_t slot, const float* src, void* stream) {
  if (!h) { set_err(nullptr, "handle is NULL"); return EA_EINVAL; }
  if (!slot_ok(h, stage, replica, slot) || !src || !is_device_ptr(src, h->cfg.device)) {
    set_err(h, "bad stage/replica/slot or src is not a device pointer");
    return EA_EINVAL;
  }
  cudaError_t e = cudaSetDevice(h->cfg.device);
  if (e != cudaSuccess) return cuda_fail(h, e, "cudaSetDevice");
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  ea_status st = join_side(h, s);  // order after pending side-stream work on this state
  if (st != EA_OK) return st;
  e = cudaMemcpyAsync(slot_ptr(h, stage, replica, slot), src, sizeof(float) * h->p[stage], cudaMemcpyDeviceToDevice, s);
  if (e != cudaSuccess) return cuda_fail(h, e, "cudaMemcpyAsync");
  if (slot == EA_SLOT_CENTER_PREV) h->prev_init[stage] = 1;
  return EA_OK;
}

ea_status ea_get_step(ea_handle h, int32_t stage, int64_t* step) {
  if (!h) { set_err(nullptr, "handle is NULL"); return EA_EINVAL; }
  if (stage < 0 || stage >= h->cfg.n_stages || !step) { set_err(h, "bad stage or NULL out pointer"); return EA_EINVAL; }
  if (!device_steps(h)) {
    *step = h->steps[stage];
    return EA_OK;
  }
  cudaError_t e = cudaSetDevice(h->cfg.device);
  if (e == cudaSuccess) e = cudaDeviceSynchronize();
  if (e == cudaSuccess) e = cudaMemcpy(step, h->d_steps + stage, sizeof(int64_t), cudaMemcpyDeviceToHost);
  if (e != cudaSuccess) return cuda_fail(h, e, "reading the step counter");
  return EA_OK;
}

ea_status ea_set_step(ea_handle h, int32_t stage, int64_t step) {
  if (!h) { set_err(nullptr, "handle is NULL"); return EA_EINVAL; }
  if (stage < 0 || stage >= h->cfg.n_stages || step < 0) { set_err(h, "bad stage or negative step"); return EA_EINVAL; }
  h->steps[stage] = step;
  cudaError_t e = cudaSetDevice(h->cfg.device);
  if (e == cudaSuccess) e = cudaDeviceSynchronize();
  if (e == cudaSuccess) e = cudaMemcpy(h->d_steps + stage, &step, sizeof(int64_t), cudaMemcpyHostToDevice);
  if (e != cudaSuccess) return cuda_fail(h, e, "writing the step counter");
  return EA_OK;
}

ea_status ea_set_hyper(ea_handle h, const ea_config* cfg) {
  if (!h) { set_err(nullptr, "handle is NULL"); return EA_EINVAL; }
  if (!cfg) { set_err(h, "cfg is NULL"); return EA_EINVAL; }
  if (cfg->optimizer != h->cfg.optimizer || cfg->n_pipelines != h->cfg.n_pipelines || cfg->layout != h->cfg.layout) {
    set_err(h, "ea_set_hyper cannot change optimizer, n_pipelines or layout");
    return EA_EINVAL;
  }
  ea_status st = check_hyper(h, *cfg);
  if (st != EA_OK) return st;
  ea_config c = h->cfg;
  c.alpha = cfg->alpha; c.beta = cfg->beta; c.rho = cfg->rho; c.lr = cfg->lr;
  c.momentum = cfg->momentum; c.weight_decay = cfg->weight_decay; c.nesterov = cfg->nesterov;
  c.beta1 = cfg->beta1; c.beta2 = cfg->beta2; c.eps = cfg->eps;
  c.asgd_lambd = cfg->asgd_lambd; c.asgd_alpha = cfg->asgd_alpha; c.asgd_t0 = cfg->asgd_t0;
  h->cfg = c;
  h->hp = make_hyper(c);
  return EA_OK;
}

ea_status ea_destroy(ea_handle h) {
  if (!h) return EA_OK;
  free_ctx(h);
  return EA_OK;
}

const char* ea_last_error(ea_handle h) { return h ? h->err.c_str() : g_init_err.c_str(); }

}  // extern "C"

// C-ABI layer of the elastic-averaging library (declared in include/ea.h).
//
// Owns: the handle, per-stage momentum (zero-initialised, P:112 Step 1
// optimizer state), and for EA_SPREAD the side stream, events, contribution
// scratch and the NCCL communicator that replace the paper's reference
// process and message queues.  Validates every argument before
// enqueuing anything; never throws or aborts.
#include <cuda_runtime.h>
#include <nccl.h>
#include <stdint.h>

#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <new>
#include <string>
#include <vector>

#include "../../include/ea.h"
#include "ea_internal.h"

struct ea_ctx {
  ea_config cfg{};
  ea::Hyper hp{};
  int variant = 0;
  int num_sms = 148;
  std::vector<int64_t> p;       // P_s
  std::vector<int64_t> p_pad;   // center capacity
  std::vector<int64_t> stride;  // momentum row stride (floats)
  std::vector<float*> mom;      // per stage: [replicas][stride]
  // EA_SPREAD
  cudaStream_t side = nullptr;
  cudaEvent_t ev_in = nullptr, ev_local = nullptr, ev_done = nullptr;
  float* contrib = nullptr;  // max P_pad floats
  float* reduced = nullptr;  // max P_pad/N floats
  ncclComm_t comm = nullptr;
  std::string err;
};

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

ea_status check_hyper(ea_ctx* h, float alpha, float beta, float rho, float lr, float momentum, float wd, int nesterov) {
  auto finite = [](float v) { return v == v && v - v == 0.f; };
  if (!(alpha >= 0.f && alpha <= 1.f)) { set_err(h, "alpha must be in [0,1] (P:112), got %g", alpha); return EA_EINVAL; }
  if (!finite(beta) || !finite(rho) || !finite(lr)) { set_err(h, "beta, rho, lr must be finite"); return EA_EINVAL; }
  if (!(momentum >= 0.f && momentum < 1.f)) { set_err(h, "momentum must be in [0,1), got %g", momentum); return EA_EINVAL; }
  if (!(wd >= 0.f) || !finite(wd)) { set_err(h, "weight_decay must be finite and >= 0"); return EA_EINVAL; }
  if (nesterov != 0 && nesterov != 1) { set_err(h, "nesterov must be 0 or 1"); return EA_EINVAL; }
  if (nesterov && momentum <= 0.f) { set_err(h, "nesterov needs momentum > 0 (torch.optim.SGD rule)"); return EA_EINVAL; }
  return EA_OK;
}

ea::Hyper make_hyper(const ea_config& c) {
  ea::Hyper hp;
  hp.alpha = c.alpha; hp.beta = c.beta; hp.rho = c.rho; hp.lr = c.lr;
  hp.momentum = c.momentum; hp.wd = c.weight_decay; hp.nesterov = c.nesterov;
  hp.inv_n = 1.0f / static_cast<float>(c.n_pipelines);
  return hp;
}

ea_status cuda_fail(ea_ctx* h, cudaError_t e, const char* what) {
  set_err(h, "%s: %s", what, cudaGetErrorString(e));
  return e == cudaErrorMemoryAllocation ? EA_ENOMEM : EA_ECUDA;
}

ea_status nccl_fail(ea_ctx* h, ncclResult_t r, const char* what) {
  set_err(h, "%s: %s", what, ncclGetErrorString(r));
  return EA_ENCCL;
}

void free_ctx(ea_ctx* h) {
  if (!h) return;
  cudaSetDevice(h->cfg.device);
  if (h->side) cudaStreamSynchronize(h->side);
  if (h->comm) ncclCommDestroy(h->comm);
  for (float* m : h->mom) if (m) cudaFree(m);
  if (h->contrib) cudaFree(h->contrib);
  if (h->reduced) cudaFree(h->reduced);
  if (h->ev_in) cudaEventDestroy(h->ev_in);
  if (h->ev_local) cudaEventDestroy(h->ev_local);
  if (h->ev_done) cudaEventDestroy(h->ev_done);
  if (h->side) cudaStreamDestroy(h->side);
  delete h;
}

int replicas_here(const ea_ctx* h) { return h->cfg.layout == EA_SPREAD ? 1 : h->cfg.n_pipelines; }

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
  if (c.kernel_variant < 0 || c.kernel_variant > 3) { set_err(nullptr, "kernel_variant must be 0..3"); return EA_EINVAL; }
  ea_status st = check_hyper(nullptr, c.alpha, c.beta, c.rho, c.lr, c.momentum, c.weight_decay, c.nesterov);
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
  h->cfg.stage_params = nullptr;  // not retained
  e = cudaSetDevice(c.device);
  if (e != cudaSuccess) { ea_status r = cuda_fail(nullptr, e, "cudaSetDevice"); free_ctx(h); return r; }
  cudaDeviceGetAttribute(&h->num_sms, cudaDevAttrMultiProcessorCount, c.device);

  const int reps = replicas_here(h);
  int64_t max_pad = 0;
  for (int s = 0; s < c.n_stages; ++s) {
    const int64_t ps = h->p[s];
    const int64_t pad = c.layout == EA_SPREAD ? round_up(ps, 32LL * c.n_pipelines) : ps;
    h->p_pad.push_back(pad);
    if (pad > max_pad) max_pad = pad;
    const int64_t stride = round_up(ps, 64);
    h->stride.push_back(stride);
    float* m = nullptr;
    e = cudaMalloc(&m, sizeof(float) * stride * reps);
    if (e == cudaSuccess) e = cudaMemset(m, 0, sizeof(float) * stride * reps);
    if (e != cudaSuccess) {
      ea_status r = cuda_fail(nullptr, e, "momentum allocation");
      if (m) cudaFree(m);
      free_ctx(h);
      return r;
    }
    h->mom.push_back(m);
  }
  if (c.layout == EA_SPREAD) {
    if ((e = cudaStreamCreateWithFlags(&h->side, cudaStreamNonBlocking)) != cudaSuccess ||
        (e = cudaEventCreateWithFlags(&h->ev_in, cudaEventDisableTiming)) != cudaSuccess ||
        (e = cudaEventCreateWithFlags(&h->ev_local, cudaEventDisableTiming)) != cudaSuccess ||
        (e = cudaEventCreateWithFlags(&h->ev_done, cudaEventDisableTiming)) != cudaSuccess ||
        (e = cudaMalloc(&h->contrib, sizeof(float) * max_pad)) != cudaSuccess ||
        (e = cudaMalloc(&h->reduced, sizeof(float) * (max_pad / c.n_pipelines))) != cudaSuccess) {
      ea_status r = cuda_fail(nullptr, e, "spread resources");
      free_ctx(h);
      return r;
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

// Validates one stage's pointers (nothing enqueued on failure).
static ea_status check_stage_ptrs(ea_ctx* h, int32_t stage, float* const* replica_ptrs, const float* const* grad_ptrs,
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

// Co-located: `count` validated stages in as few launches as possible.
static ea_status colocated_launch(ea_ctx* h, int32_t count, const int32_t* stages, float* const* replica_ptrs,
                                  const float* const* grad_ptrs, float* const* center_ptrs, cudaStream_t s) {
  const int n = h->cfg.n_pipelines;
  cudaError_t e = cudaSuccess;
  if (n > ea::kMaxFusedN) {  // wide N: one launch per stage
    for (int j = 0; j < count; ++j) {
      const int st = stages[j];
      ea::ReplicaTable t;
      for (int i = 0; i < n; ++i) {
        t.x[i] = replica_ptrs[j * n + i];
        t.g[i] = grad_ptrs[j * n + i];
        t.m[i] = h->mom[st] + h->stride[st] * i;
      }
      e = ea::launch_colocated_wide(t, n, center_ptrs[j], h->p[st], h->hp, h->num_sms, s);
      if (e != cudaSuccess) return cuda_fail(h, e, "co-located kernel launch");
    }
    return EA_OK;
  }
  for (int j0 = 0; j0 < count; j0 += ea::kMaxLaunchStages) {
    ea::StageBatch b;
    b.nstages = 0;
    for (int j = j0; j < count && j < j0 + ea::kMaxLaunchStages; ++j) {
      const int st = stages[j];
      ea::StageRefs& r = b.st[b.nstages++];
      for (int i = 0; i < ea::kMaxFusedN; ++i) {
        const bool on = i < n;
        r.x[i] = on ? replica_ptrs[j * n + i] : nullptr;
        r.g[i] = on ? grad_ptrs[j * n + i] : nullptr;
        r.m[i] = on ? h->mom[st] + h->stride[st] * i : nullptr;
      }
      r.c = center_ptrs[j];
      r.p = h->p[st];
    }
    e = ea::launch_colocated_batch(b, n, h->hp, h->variant, h->num_sms, s);
    if (e != cudaSuccess) return cuda_fail(h, e, "co-located kernel launch");
  }
  return EA_OK;
}

// Spread: one stage's exchange on the side stream (rows a6-a8).
static ea_status spread_step(ea_ctx* h, int32_t stage, float* replica, const float* grad, float* center_ptr,
                             cudaStream_t s) {
  if (!h->comm) {
    set_err(h, "EA_SPREAD handle created without an NCCL id: use ea_spread_local / ea_spread_apply");
    return EA_ESTATE;
  }
  cudaError_t e;
  const int n = h->cfg.n_pipelines;
  const int64_t pad = h->p_pad[stage], shard = pad / n;
  float* own = center_ptr + shard * h->cfg.rank;
  if ((e = cudaEventRecord(h->ev_in, s)) != cudaSuccess) return cuda_fail(h, e, "cudaEventRecord");
  if ((e = cudaStreamWaitEvent(h->side, h->ev_in, 0)) != cudaSuccess) return cuda_fail(h, e, "cudaStreamWaitEvent");
  e = ea::launch_spread_local(replica, grad, h->mom[stage], center_ptr, h->contrib, h->p[stage], pad, h->hp,
                              h->num_sms, h->side);
  if (e != cudaSuccess) return cuda_fail(h, e, "spread local kernel launch");
  if ((e = cudaEventRecord(h->ev_local, h->side)) != cudaSuccess) return cuda_fail(h, e, "cudaEventRecord");
  ncclResult_t r = ncclReduceScatter(h->contrib, h->reduced, static_cast<size_t>(shard), ncclFloat, ncclSum, h->comm,
                                     h->side);
  if (r != ncclSuccess) return nccl_fail(h, r, "ncclReduceScatter");
  e = ea::launch_spread_apply(own, h->reduced, shard, h->hp.inv_n, h->num_sms, h->side);
  if (e != cudaSuccess) return cuda_fail(h, e, "spread apply kernel launch");
  r = ncclAllGather(own, center_ptr, static_cast<size_t>(shard), ncclFloat, h->comm, h->side);
  if (r != ncclSuccess) return nccl_fail(h, r, "ncclAllGather");
  // The caller's stream waits only for x_i (the next forward may start now).
  if ((e = cudaStreamWaitEvent(s, h->ev_local, 0)) != cudaSuccess) return cuda_fail(h, e, "cudaStreamWaitEvent");
  return EA_OK;
}

ea_status ea_step(ea_handle h, int32_t stage, float* const* replica_ptrs, const float* const* grad_ptrs,
                  float* center_ptr, void* stream) {
  if (!h) { set_err(nullptr, "handle is NULL"); return EA_EINVAL; }
  ea_status st = check_stage_ptrs(h, stage, replica_ptrs, grad_ptrs, center_ptr);
  if (st != EA_OK) return st;
  cudaError_t e = cudaSetDevice(h->cfg.device);
  if (e != cudaSuccess) return cuda_fail(h, e, "cudaSetDevice");
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  if (h->cfg.layout == EA_COLOCATED) return colocated_launch(h, 1, &stage, replica_ptrs, grad_ptrs, &center_ptr, s);
  return spread_step(h, stage, replica_ptrs[0], grad_ptrs[0], center_ptr, s);
}

ea_status ea_step_many(ea_handle h, int32_t count, const int32_t* stages, float* const* replica_ptrs,
                       const float* const* grad_ptrs, float* const* center_ptrs, void* stream) {
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

ea_status ea_sync(ea_handle h, void* stream) {
  if (!h) { set_err(nullptr, "handle is NULL"); return EA_EINVAL; }
  cudaError_t e = cudaSetDevice(h->cfg.device);
  if (e != cudaSuccess) return cuda_fail(h, e, "cudaSetDevice");
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  if (h->cfg.layout == EA_SPREAD) {
    if ((e = cudaEventRecord(h->ev_done, h->side)) != cudaSuccess) return cuda_fail(h, e, "cudaEventRecord");
    if ((e = cudaStreamWaitEvent(s, h->ev_done, 0)) != cudaSuccess) return cuda_fail(h, e, "cudaStreamWaitEvent");
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
  e = ea::launch_spread_local(replica_ptr, grad_ptr, h->mom[stage], center_ptr, contrib, h->p[stage], h->p_pad[stage],
                              h->hp, h->num_sms, static_cast<cudaStream_t>(stream));
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
  e = ea::launch_spread_apply(center_shard, reduced, h->p_pad[stage] / h->cfg.n_pipelines, h->hp.inv_n, h->num_sms,
                              static_cast<cudaStream_t>(stream));
  if (e != cudaSuccess) return cuda_fail(h, e, "spread apply kernel launch");
  return EA_OK;
}

ea_status ea_get_state(ea_handle h, int32_t stage, int32_t replica, float** momentum_dev) {
  if (!h) { set_err(nullptr, "handle is NULL"); return EA_EINVAL; }
  if (stage < 0 || stage >= h->cfg.n_stages || replica < 0 || replica >= replicas_here(h) || !momentum_dev) {
    set_err(h, "bad stage/replica/out pointer");
    return EA_EINVAL;
  }
  *momentum_dev = h->mom[stage] + h->stride[stage] * replica;
  return EA_OK;
}

ea_status ea_set_state(ea_handle h, int32_t stage, int32_t replica, const float* momentum_src, void* stream) {
  if (!h) { set_err(nullptr, "handle is NULL"); return EA_EINVAL; }
  if (stage < 0 || stage >= h->cfg.n_stages || replica < 0 || replica >= replicas_here(h) || !momentum_src ||
      !is_device_ptr(momentum_src, h->cfg.device)) {
    set_err(h, "bad stage/replica or momentum_src is not a device pointer");
    return EA_EINVAL;
  }
  cudaError_t e = cudaSetDevice(h->cfg.device);
  if (e != cudaSuccess) return cuda_fail(h, e, "cudaSetDevice");
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  if (h->cfg.layout == EA_SPREAD) {  // order after pending side-stream work on this momentum
    if ((e = cudaEventRecord(h->ev_done, h->side)) != cudaSuccess) return cuda_fail(h, e, "cudaEventRecord");
    if ((e = cudaStreamWaitEvent(s, h->ev_done, 0)) != cudaSuccess) return cuda_fail(h, e, "cudaStreamWaitEvent");
  }
  e = cudaMemcpyAsync(h->mom[stage] + h->stride[stage] * replica, momentum_src, sizeof(float) * h->p[stage],
                      cudaMemcpyDeviceToDevice, s);
  if (e != cudaSuccess) return cuda_fail(h, e, "cudaMemcpyAsync");
  return EA_OK;
}

ea_status ea_set_hyper(ea_handle h, float alpha, float beta, float rho, float lr, float momentum, float weight_decay,
                       int32_t nesterov) {
  if (!h) { set_err(nullptr, "handle is NULL"); return EA_EINVAL; }
  ea_status st = check_hyper(h, alpha, beta, rho, lr, momentum, weight_decay, nesterov);
  if (st != EA_OK) return st;
  h->cfg.alpha = alpha; h->cfg.beta = beta; h->cfg.rho = rho; h->cfg.lr = lr;
  h->cfg.momentum = momentum; h->cfg.weight_decay = weight_decay; h->cfg.nesterov = nesterov;
  h->hp = make_hyper(h->cfg);
  return EA_OK;
}

ea_status ea_destroy(ea_handle h) {
  if (!h) return EA_OK;
  free_ctx(h);
  return EA_OK;
}

const char* ea_last_error(ea_handle h) { return h ? h->err.c_str() : g_init_err.c_str(); }

}  // extern "C"

// Test infrastructure (NOT product code): an in-process emulation of the NCCL
// calls libavgpipe_ea.so makes, so that the library's own EA_SPREAD + NCCL
// exchange code path (ea_step -> ncclReduceScatter -> spread_apply -> in-place
// ncclAllGather on the side stream, rows a6/a7) runs with N > 1 ranks on ONE
// GPU.  Loaded with LD_PRELOAD ahead of the real libnccl.so.2; the N ranks are
// N handles driven by N host threads of one process, every rank on cuda:0.
//
// Semantics follow NCCL's documented ones: a collective is stream-ordered on
// each rank's stream; its output on rank r is complete when r's stream reaches
// the end of the call; a rank's send buffer may be reused once its own stream
// passes the call.  Emulation: every call is a host rendezvous of the N ranks
// (the k-th collective of every rank must match, as NCCL requires); each rank's
// stream waits for every rank's "inputs ready" event, computes its own output
// from the other ranks' buffers (same device) with a small kernel, and then
// waits for every rank's "done" event (so nobody overwrites an input another
// rank still reads).  Summation order over ranks is 0..N-1 (NCCL's is its
// ring/tree order; any order is correct, reading c14).
//
// NCCL_EMU_LOG=<path> appends one line per call: op rank world sendbuff
// recvbuff count dtype (pointers in hex) -- the tests check the library's
// arguments (counts, shard offsets, in-place all-gather aliasing) against
// parallel.shard_bounds.
#include <cuda_runtime.h>
#include <nccl.h>
#include <stdint.h>
#include <unistd.h>

#include <chrono>
#include <condition_variable>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <map>
#include <mutex>
#include <string>
#include <vector>

namespace {

constexpr int kMaxRanks = 64;

enum Kind { kRS = 0, kAG = 1, kAR = 2 };

struct Post {
  int kind = -1;
  const void* send = nullptr;
  void* recv = nullptr;
  size_t count = 0;
  int dtype = 0;
  cudaEvent_t ready = nullptr, done = nullptr;
};

struct Group {
  int n = 0;
  int joined = 0;
  std::mutex mu;
  std::condition_variable cv;
  int arrived = 0;
  uint64_t gen = 0;
  std::vector<Post> posts;
};

std::mutex g_mu;
std::map<std::string, Group*> g_groups;
uint64_t g_id_counter = 0;

int timeout_s() {
  const char* e = std::getenv("NCCL_EMU_TIMEOUT_S");
  const int v = e ? std::atoi(e) : 120;
  return v > 0 ? v : 120;
}

// Host barrier of the group's N ranks (generation counting); false on timeout.
bool barrier(Group* g) {
  std::unique_lock<std::mutex> lk(g->mu);
  const uint64_t gen = g->gen;
  if (++g->arrived == g->n) {
    g->arrived = 0;
    ++g->gen;
    g->cv.notify_all();
    return true;
  }
  return g->cv.wait_for(lk, std::chrono::seconds(timeout_s()), [&] { return g->gen != gen; });
}

void log_call(const char* op, int rank, int world, const void* s, const void* r, size_t count, int dtype) {
  const char* path = std::getenv("NCCL_EMU_LOG");
  if (!path) return;
  static std::mutex mu;
  std::lock_guard<std::mutex> lk(mu);
  FILE* f = std::fopen(path, "a");
  if (!f) return;
  std::fprintf(f, "%s %d %d %p %p %zu %d\n", op, rank, world, s, r, count, dtype);
  std::fclose(f);
}

size_t dtype_bytes(int dt) {
  switch (dt) {
    case ncclInt8: case ncclUint8: return 1;
    case ncclFloat16: case ncclBfloat16: return 2;
    case ncclInt32: case ncclUint32: case ncclFloat32: return 4;
    default: return 8;
  }
}

struct Ptrs {
  const void* p[kMaxRanks];
};

// Reduce-scatter (sum): out[i] = sum_q in_q[rank*count + i].
template <class T>
__global__ void rs_kernel(Ptrs in, int n, int rank, T* out, size_t count) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < count; i += (size_t)gridDim.x * blockDim.x) {
    T acc = T(0);
    for (int q = 0; q < n; ++q) acc += static_cast<const T*>(in.p[q])[rank * count + i];
    out[i] = acc;
  }
}

// All-reduce (sum): out[i] = sum_q in_q[i].
template <class T>
__global__ void ar_kernel(Ptrs in, int n, T* out, size_t count) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < count; i += (size_t)gridDim.x * blockDim.x) {
    T acc = T(0);
    for (int q = 0; q < n; ++q) acc += static_cast<const T*>(in.p[q])[i];
    out[i] = acc;
  }
}

// All-gather (bytes): out[q*bytes + i] = in_q[i].
__global__ void ag_kernel(Ptrs in, int n, unsigned char* out, size_t bytes) {
  const size_t total = bytes * n;
  for (size_t k = blockIdx.x * (size_t)blockDim.x + threadIdx.x; k < total; k += (size_t)gridDim.x * blockDim.x) {
    const size_t q = k / bytes, i = k % bytes;
    out[k] = static_cast<const unsigned char*>(in.p[q])[i];
  }
}

}  // namespace

struct ncclComm {
  Group* g;
  int rank;
  cudaEvent_t ready, done;
};

namespace {

ncclResult_t collective(ncclComm_t c, int kind, const void* send, void* recv, size_t count, ncclDataType_t dt,
                        ncclRedOp_t op, cudaStream_t s) {
  static const char* names[] = {"RS", "AG", "AR"};
  log_call(names[kind], c->rank, c->g->n, send, recv, count, (int)dt);
  if (kind != kAG && op != ncclSum) return ncclInvalidArgument;
  if (kind != kAG && dt != ncclFloat32 && dt != ncclInt32) return ncclInvalidArgument;
  Group* g = c->g;
  if (cudaEventRecord(c->ready, s) != cudaSuccess) return ncclUnhandledCudaError;
  {
    std::lock_guard<std::mutex> lk(g->mu);
    Post& p = g->posts[c->rank];
    p.kind = kind; p.send = send; p.recv = recv; p.count = count; p.dtype = (int)dt; p.ready = c->ready;
    p.done = c->done;
  }
  if (!barrier(g)) return ncclSystemError;  // every rank posted this collective
  Ptrs in{};
  for (int q = 0; q < g->n; ++q) {
    const Post& p = g->posts[q];
    if (p.kind != kind || p.count != count || p.dtype != (int)dt) {
      std::fprintf(stderr, "nccl_emu: rank %d posted a different collective than rank %d\n", q, c->rank);
      return ncclInvalidUsage;
    }
    in.p[q] = p.send;
    if (cudaStreamWaitEvent(s, p.ready, 0) != cudaSuccess) return ncclUnhandledCudaError;
  }
  const int threads = 256;
  const size_t work = kind == kAG ? count * dtype_bytes(dt) * g->n : count;
  const int blocks = static_cast<int>(work / threads + 1 < 1024 ? work / threads + 1 : 1024);
  if (kind == kRS) {
    if (dt == ncclFloat32) rs_kernel<float><<<blocks, threads, 0, s>>>(in, g->n, c->rank, (float*)recv, count);
    else rs_kernel<int><<<blocks, threads, 0, s>>>(in, g->n, c->rank, (int*)recv, count);
  } else if (kind == kAR) {
    if (dt == ncclFloat32) ar_kernel<float><<<blocks, threads, 0, s>>>(in, g->n, (float*)recv, count);
    else ar_kernel<int><<<blocks, threads, 0, s>>>(in, g->n, (int*)recv, count);
  } else {
    ag_kernel<<<blocks, threads, 0, s>>>(in, g->n, (unsigned char*)recv, count * dtype_bytes(dt));
  }
  if (cudaGetLastError() != cudaSuccess) return ncclUnhandledCudaError;
  if (cudaEventRecord(c->done, s) != cudaSuccess) return ncclUnhandledCudaError;
  if (!barrier(g)) return ncclSystemError;  // every rank's output kernel is enqueued
  for (int q = 0; q < g->n; ++q)
    if (cudaStreamWaitEvent(s, g->posts[q].done, 0) != cudaSuccess) return ncclUnhandledCudaError;
  if (!barrier(g)) return ncclSystemError;  // posts[] may be reused by the next collective
  return ncclSuccess;
}

}  // namespace

extern "C" {

ncclResult_t ncclGetUniqueId(ncclUniqueId* id) {
  if (!id) return ncclInvalidArgument;
  std::memset(id, 0, sizeof(*id));
  std::lock_guard<std::mutex> lk(g_mu);
  std::snprintf(id->internal, sizeof(id->internal), "nccl_emu:%d:%llu", (int)getpid(),
                (unsigned long long)++g_id_counter);
  return ncclSuccess;
}

ncclResult_t ncclCommInitRank(ncclComm_t* comm, int nranks, ncclUniqueId id, int rank) {
  if (!comm || nranks < 1 || nranks > kMaxRanks || rank < 0 || rank >= nranks) return ncclInvalidArgument;
  const std::string key(id.internal, strnlen(id.internal, sizeof(id.internal)));
  Group* g;
  {
    std::lock_guard<std::mutex> lk(g_mu);
    auto it = g_groups.find(key);
    if (it == g_groups.end()) {
      g = new Group;
      g->n = nranks;
      g->posts.resize(nranks);
      g_groups[key] = g;
    } else {
      g = it->second;
    }
  }
  if (g->n != nranks) return ncclInvalidUsage;
  ncclComm* c = new ncclComm{g, rank, nullptr, nullptr};
  if (cudaEventCreateWithFlags(&c->ready, cudaEventDisableTiming) != cudaSuccess ||
      cudaEventCreateWithFlags(&c->done, cudaEventDisableTiming) != cudaSuccess) {
    delete c;
    return ncclUnhandledCudaError;
  }
  log_call("INIT", rank, nranks, nullptr, nullptr, 0, 0);
  if (!barrier(g)) return ncclSystemError;  // blocking, like ncclCommInitRank
  *comm = c;
  return ncclSuccess;
}

ncclResult_t ncclCommDestroy(ncclComm_t c) {
  if (!c) return ncclSuccess;
  cudaEventDestroy(c->ready);
  cudaEventDestroy(c->done);
  delete c;  // the group stays registered (ids are never reused)
  return ncclSuccess;
}

ncclResult_t ncclCommGetAsyncError(ncclComm_t, ncclResult_t* e) {
  if (e) *e = ncclSuccess;
  return ncclSuccess;
}

const char* ncclGetErrorString(ncclResult_t r) { return r == ncclSuccess ? "success (nccl_emu)" : "error (nccl_emu)"; }

ncclResult_t ncclReduceScatter(const void* send, void* recv, size_t count, ncclDataType_t dt, ncclRedOp_t op,
                               ncclComm_t c, cudaStream_t s) {
  return collective(c, kRS, send, recv, count, dt, op, s);
}

ncclResult_t ncclAllGather(const void* send, void* recv, size_t count, ncclDataType_t dt, ncclComm_t c,
                           cudaStream_t s) {
  return collective(c, kAG, send, recv, count, dt, ncclSum, s);
}

ncclResult_t ncclAllReduce(const void* send, void* recv, size_t count, ncclDataType_t dt, ncclRedOp_t op,
                           ncclComm_t c, cudaStream_t s) {
  return collective(c, kAR, send, recv, count, dt, op, s);
}

}  // extern "C"

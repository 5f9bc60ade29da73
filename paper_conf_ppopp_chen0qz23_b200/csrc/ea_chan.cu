// Point-to-point activation channel (row f2): the transfers of the advance-forward pipeline runtime.
//
// Stage k of a parallel pipeline sends its output activations to stage k+1 and receives the activation
// gradients back ("a parallel pipeline launches a process on each GPU"; the order of the sends and
// receives is Algorithm 1's).  A channel is one direction between two processes -- two GPUs joined by
// NVLink, or two processes sharing one GPU.  It moves the bytes GPU to GPU with the copy engine over a CUDA IPC
// mapping of the receiver's memory and does the handshake with stream memory operations, so neither side's
// host ever waits for the other:
//
//   receiving end owns: slot[S] of slot_bytes (the message ring) and ready[S] (u32)
//   sending end owns:   ack[S] (u32)
//   send #k (slot q = k mod S, round u = k div S), on the sender's stream:
//       wait   ack[q]   >= u        (local word: the receiver freed message k - S of this slot)
//       copy   src -> slot[q]       (peer write over the IPC mapping)
//       write  ready[q] := u + 1    (peer word; the write is ordered after the copy)
//   recv #k, on the receiver's stream:
//       wait   ready[q] >= u + 1    (local word)
//       copy   slot[q] -> dst
//       write  ack[q]   := u + 1    (peer word)
//
// Every end waits only on its own memory and writes the other's.  Messages are matched in order, as the runtime's
// sends and receives of one (pipeline, direction) are (both follow the micro-batch order of Algorithm 1).
// Stream memory operations come from the driver through cudaGetDriverEntryPoint (no libcuda link).
#include <cuda.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <string>

#include "ea.h"

namespace {

using WaitFn = CUresult (*)(CUstream, CUdeviceptr, cuuint32_t, unsigned int);
using WriteFn = CUresult (*)(CUstream, CUdeviceptr, cuuint32_t, unsigned int);

struct MemOps {
  WaitFn wait = nullptr;
  WriteFn write = nullptr;
  bool ok = false;
};

const MemOps& memops() {
  static const MemOps m = [] {
    MemOps r;
    void* w = nullptr;
    void* v = nullptr;
    cudaDriverEntryPointQueryResult q1, q2;
    if (cudaGetDriverEntryPoint("cuStreamWaitValue32", &w, cudaEnableDefault, &q1) == cudaSuccess &&
        cudaGetDriverEntryPoint("cuStreamWriteValue32", &v, cudaEnableDefault, &q2) == cudaSuccess &&
        q1 == cudaDriverEntryPointSuccess && q2 == cudaDriverEntryPointSuccess && w && v) {
      r.wait = reinterpret_cast<WaitFn>(w);
      r.write = reinterpret_cast<WriteFn>(v);
      r.ok = true;
    }
    return r;
  }();
  return m;
}

}  // namespace

struct ea_chan_s {
  int device = 0;
  int role = 0;            // 0 = sending end, 1 = receiving end
  int64_t slot_bytes = 0;  // capacity of one message
  int64_t stride = 0;      // slot stride (256-B aligned)
  int32_t slots = 0;
  char* local = nullptr;   // this end's buffer (IPC-exported): recv = ring + ready words, send = ack words
  char* peer = nullptr;    // the other end's buffer (IPC-opened, or the other end's local buffer when paired)
  bool peer_ipc = false;   // peer opened with cudaIpcOpenMemHandle (closed at destroy)
  int64_t seq = 0;         // messages enqueued so far
  std::string err;
};

namespace {

thread_local std::string g_chan_err;  // ea_chan_create failures (no channel yet)

void set_err(ea_chan c, const char* fmt, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof(buf), fmt, ap);
  va_end(ap);
  (c ? c->err : g_chan_err) = buf;
}

ea_status cfail(ea_chan c, cudaError_t e, const char* what) {
  set_err(c, "%s: %s", what, cudaGetErrorString(e));
  return EA_ECUDA;
}

// receiving end: ring of slots, then the ready words; sending end: the ack words
int64_t local_bytes(const ea_chan_s* c) {
  const int64_t words = ((int64_t)c->slots * 4 + 255) / 256 * 256;
  return c->role == 1 ? c->stride * c->slots + words : words;
}
uint32_t* ready_words(ea_chan_s* c, char* recv_buf) {
  return reinterpret_cast<uint32_t*>(recv_buf + c->stride * c->slots);
}

bool capturing(cudaStream_t s) {
  cudaStreamCaptureStatus st = cudaStreamCaptureStatusNone;
  return cudaStreamIsCapturing(s, &st) == cudaSuccess && st != cudaStreamCaptureStatusNone;
}

ea_status check_io(ea_chan c, const void* p, int64_t bytes, cudaStream_t s, int want_role) {
  if (!c) return EA_EINVAL;
  if (c->role != want_role) {
    set_err(c, want_role == 0 ? "ea_chan_send on a receiving end" : "ea_chan_recv on a sending end");
    return EA_EINVAL;
  }
  if (!c->peer) { set_err(c, "channel not connected (ea_chan_connect / ea_chan_pair)"); return EA_ESTATE; }
  if (bytes < 0 || bytes > c->slot_bytes) {
    set_err(c, "message of %lld bytes does not fit a slot of %lld", (long long)bytes, (long long)c->slot_bytes);
    return EA_EINVAL;
  }
  if (bytes > 0 && !p) { set_err(c, "NULL buffer"); return EA_EINVAL; }
  if (capturing(s)) {  // the round numbers are host counters: a replayed graph would reuse them
    set_err(c, "channel operations cannot be captured into a CUDA graph");
    return EA_ESTATE;
  }
  if (!memops().ok) { set_err(c, "stream memory operations unavailable from the driver"); return EA_ECUDA; }
  return EA_OK;
}

}  // namespace

extern "C" {

EA_API ea_status ea_chan_create(int32_t device, int32_t role, int64_t slot_bytes, int32_t slots, ea_chan* out) {
  if (!out) { set_err(nullptr, "NULL output"); return EA_EINVAL; }
  *out = nullptr;
  if (role != 0 && role != 1) { set_err(nullptr, "role must be 0 (send) or 1 (recv)"); return EA_EINVAL; }
  if (slot_bytes <= 0 || slots <= 0) { set_err(nullptr, "slot_bytes and slots must be > 0"); return EA_EINVAL; }
  ea_chan c = new ea_chan_s;
  c->device = device;
  c->role = role;
  c->slot_bytes = slot_bytes;
  c->stride = (slot_bytes + 255) / 256 * 256;
  c->slots = slots;
  cudaError_t e = cudaSetDevice(device);
  if (e == cudaSuccess) e = cudaMalloc(&c->local, local_bytes(c));
  if (e == cudaSuccess) e = cudaMemset(c->local, 0, local_bytes(c));
  if (e == cudaSuccess) e = cudaDeviceSynchronize();
  if (e != cudaSuccess) {
    set_err(nullptr, "channel buffer of %lld bytes: %s", (long long)local_bytes(c), cudaGetErrorString(e));
    if (c->local) cudaFree(c->local);
    delete c;
    return e == cudaErrorMemoryAllocation ? EA_ENOMEM : EA_ECUDA;
  }
  *out = c;
  return EA_OK;
}

// Exported handle: the CUDA IPC handle of this end's buffer, then the end's geometry and role, so that
// ea_chan_connect can refuse a peer whose slots differ (its copies would overrun this end's ring).
struct ChanHandle {
  cudaIpcMemHandle_t ipc;
  int64_t slot_bytes;
  int32_t slots;
  int32_t role;
};
static_assert(sizeof(ChanHandle) == EA_CHAN_HANDLE_BYTES, "EA_CHAN_HANDLE_BYTES");

EA_API ea_status ea_chan_export(ea_chan c, uint8_t* handle) {
  if (!c || !handle) { set_err(c, "NULL channel or output"); return EA_EINVAL; }
  ChanHandle h;
  memset(&h, 0, sizeof(h));
  cudaError_t e = cudaSetDevice(c->device);
  if (e == cudaSuccess) e = cudaIpcGetMemHandle(&h.ipc, c->local);
  if (e != cudaSuccess) return cfail(c, e, "cudaIpcGetMemHandle");
  h.slot_bytes = c->slot_bytes;
  h.slots = c->slots;
  h.role = c->role;
  memcpy(handle, &h, sizeof(h));
  return EA_OK;
}

EA_API ea_status ea_chan_connect(ea_chan c, const uint8_t* peer_handle) {
  if (!c || !peer_handle) { set_err(c, "NULL channel or handle"); return EA_EINVAL; }
  if (c->peer) { set_err(c, "channel already connected"); return EA_ESTATE; }
  ChanHandle ph;
  memcpy(&ph, peer_handle, sizeof(ph));
  if (ph.role != 1 - c->role) { set_err(c, "the peer end must have the opposite role"); return EA_EINVAL; }
  if (ph.slot_bytes != c->slot_bytes || ph.slots != c->slots) {
    set_err(c, "peer geometry (%lld bytes x %d slots) differs from this end's (%lld x %d)", (long long)ph.slot_bytes,
            ph.slots, (long long)c->slot_bytes, c->slots);
    return EA_EINVAL;
  }
  const cudaIpcMemHandle_t h = ph.ipc;
  void* p = nullptr;
  cudaError_t e = cudaSetDevice(c->device);
  if (e == cudaSuccess) e = cudaIpcOpenMemHandle(&p, h, cudaIpcMemLazyEnablePeerAccess);
  if (e != cudaSuccess) return cfail(c, e, "cudaIpcOpenMemHandle");
  c->peer = static_cast<char*>(p);
  c->peer_ipc = true;
  return EA_OK;
}

EA_API ea_status ea_chan_pair(ea_chan send_end, ea_chan recv_end) {
  if (!send_end || !recv_end) { set_err(nullptr, "NULL channel"); return EA_EINVAL; }
  if (send_end->role != 0 || recv_end->role != 1) { set_err(send_end, "ea_chan_pair(send end, recv end)"); return EA_EINVAL; }
  if (send_end->slots != recv_end->slots || send_end->slot_bytes != recv_end->slot_bytes) {
    set_err(send_end, "the two ends differ in slots or slot_bytes");
    return EA_EINVAL;
  }
  if (send_end->peer || recv_end->peer) { set_err(send_end, "channel already connected"); return EA_ESTATE; }
  send_end->peer = recv_end->local;
  recv_end->peer = send_end->local;
  return EA_OK;
}

EA_API ea_status ea_chan_send(ea_chan c, const void* src, int64_t bytes, void* stream) {
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  ea_status st = check_io(c, src, bytes, s, 0);
  if (st != EA_OK) return st;
  const int32_t q = static_cast<int32_t>(c->seq % c->slots);
  const uint32_t u = static_cast<uint32_t>(c->seq / c->slots);
  cudaError_t e = cudaSetDevice(c->device);
  if (e != cudaSuccess) return cfail(c, e, "cudaSetDevice");
  const MemOps& m = memops();
  uint32_t* ack = reinterpret_cast<uint32_t*>(c->local) + q;
  if (m.wait(s, reinterpret_cast<CUdeviceptr>(ack), u, CU_STREAM_WAIT_VALUE_GEQ) != CUDA_SUCCESS) {
    set_err(c, "cuStreamWaitValue32 (slot free)");
    return EA_ECUDA;
  }
  if (bytes > 0 && (e = cudaMemcpyAsync(c->peer + c->stride * q, src, bytes, cudaMemcpyDeviceToDevice, s)) != cudaSuccess)
    return cfail(c, e, "peer copy into the receiver's slot");
  uint32_t* ready = ready_words(c, c->peer) + q;
  if (m.write(s, reinterpret_cast<CUdeviceptr>(ready), u + 1, CU_STREAM_WRITE_VALUE_DEFAULT) != CUDA_SUCCESS) {
    set_err(c, "cuStreamWriteValue32 (ready)");
    return EA_ECUDA;
  }
  ++c->seq;
  return EA_OK;
}

EA_API ea_status ea_chan_recv(ea_chan c, void* dst, int64_t bytes, void* stream) {
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  ea_status st = check_io(c, dst, bytes, s, 1);
  if (st != EA_OK) return st;
  const int32_t q = static_cast<int32_t>(c->seq % c->slots);
  const uint32_t u = static_cast<uint32_t>(c->seq / c->slots);
  cudaError_t e = cudaSetDevice(c->device);
  if (e != cudaSuccess) return cfail(c, e, "cudaSetDevice");
  const MemOps& m = memops();
  uint32_t* ready = ready_words(c, c->local) + q;
  if (m.wait(s, reinterpret_cast<CUdeviceptr>(ready), u + 1, CU_STREAM_WAIT_VALUE_GEQ) != CUDA_SUCCESS) {
    set_err(c, "cuStreamWaitValue32 (message ready)");
    return EA_ECUDA;
  }
  if (bytes > 0 && (e = cudaMemcpyAsync(dst, c->local + c->stride * q, bytes, cudaMemcpyDeviceToDevice, s)) != cudaSuccess)
    return cfail(c, e, "copy out of the slot");
  uint32_t* ack = reinterpret_cast<uint32_t*>(c->peer) + q;
  if (m.write(s, reinterpret_cast<CUdeviceptr>(ack), u + 1, CU_STREAM_WRITE_VALUE_DEFAULT) != CUDA_SUCCESS) {
    set_err(c, "cuStreamWriteValue32 (ack)");
    return EA_ECUDA;
  }
  ++c->seq;
  return EA_OK;
}

EA_API int64_t ea_chan_count(ea_chan c) { return c ? c->seq : -1; }

EA_API ea_status ea_chan_destroy(ea_chan c) {
  if (!c) return EA_OK;
  cudaSetDevice(c->device);
  cudaDeviceSynchronize();
  if (c->peer_ipc && c->peer) cudaIpcCloseMemHandle(c->peer);
  if (c->local) cudaFree(c->local);
  delete c;
  return EA_OK;
}

EA_API const char* ea_chan_last_error(ea_chan c) { return c ? c->err.c_str() : g_chan_err.c_str(); }

}  // extern "C"

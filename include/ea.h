/*
 * ea.h -- C ABI of the B200-native elastic-averaging step of AvgPipe
 * (Chen, Xu, Qian, Zhou, "Elastic Averaging for Efficient Pipelined DNN
 * Training", PPoPP'23).  Citations "P:<line> §<sec>" are to the paper text.
 *
 * What the library computes (per pipeline stage s, per iteration; §3.2):
 *
 *   N parallel pipelines each hold a replica x_i of every stage; a
 *   reference ("center") model x~ is co-partitioned with them.  For
 *   every element j, with x~ = x~_t and all right-hand sides at step t:
 *
 *     Step 1  local update of a user-specified optimizer (ea_optimizer),
 *                     PyTorch conventions:
 *                     SGD+momentum (buffer starts at 0, dampening 0):
 *                       g' = g_i + lambda*x_i;  m_i <- mu*m_i + g';
 *                       Delta_i = -lr * (nesterov ? g' + mu*m_i : m_i)
 *                     Adam / AdamW (t = the stage's step count; DESIGN.md c21):
 *                       m <- b1 m + (1-b1) g';  v <- b2 v + (1-b2) g'^2;
 *                       Delta_i = -(lr/(1-b1^t)) m / (sqrt(v)/sqrt(1-b2^t) + eps)
 *                       (Adam: g' = g + lambda x;  AdamW: g' = g, Delta -= lr lambda x)
 *                     ASGD (averaged SGD, the AWD-LSTM run's optimizer; torch.optim.ASGD;
 *                     DESIGN.md c29; t = the stage's step count):
 *                       eta_t = lr / (1 + l*lr*(t-1))^a;  mu_t = 1 / max(1, t-1-t0)
 *                       Delta_i = -eta_t * (g + lambda x + l x)      (l = asgd_lambd decay term)
 *                       ax_i <- mu_t == 1 ? x_i + Delta_i : ax_i + mu_t*(x_i + Delta_i - ax_i)
 *     Step 2  dilution in the ratio (1-alpha):alpha plus the local update:
 *                       x_i <- (1-alpha)*x_i + alpha*x~ + Delta_i
 *     Step 3/4  send and accumulate the contribution
 *                       R = sum_i r_i,  r_i = rho*Delta_i + beta*(x_i - x~)
 *     Step 5  normalise and apply:  x~ <- x~ + R / N
 *
 *   (alpha, beta, rho) = (1/N, 0, 1) is the paper's own mode ("stays the
 *   average"); (alpha, 0, N*alpha) is EASGD's center pull (refs [35],
 *   [18]); see DESIGN.md "Readings" c1-c14 for every reading of the prose.
 *
 * Layouts (ea_config.layout):
 *   EA_COLOCATED  all N replicas of each hosted stage live on this GPU (the
 *                 paper's placement: one GPU per stage).  One
 *                 fused kernel per ea_step; no communication.
 *   EA_SPREAD     one replica per GPU per stage; world == N ranks; the center
 *                 of each stage is sharded 1/N over the ranks.  ea_step runs
 *                 the fused local kernel, an NCCL reduce-scatter of the
 *                 contributions into the owning shard, the shard update and an
 *                 in-place NCCL all-gather, all on a library-owned side stream
 *                 (the reference process "so as to not block the parallel
 *                 pipelines").
 *
 * Data: fp32, flat, contiguous, device-resident, 16-byte aligned.  The caller
 * owns x_i, g_i and x~ (e.g. torch tensors); the library owns momentum,
 * scratch, streams, events and the NCCL communicator.
 *
 * Errors: every call returns an ea_status; nothing throws or aborts.  On
 * EA_EINVAL nothing was enqueued.  ea_last_error(h) returns a message for the
 * last failing call on h (thread-local message for h == NULL / ea_init).
 * Threading: a handle is not thread-safe; use one per (process, device).
 */
#ifndef AVGPIPE_EA_H_
#define AVGPIPE_EA_H_

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#if defined(__GNUC__)
#define EA_API __attribute__((visibility("default")))
#else
#define EA_API
#endif

#define EA_ABI_VERSION 6
#define EA_MAX_REPLICAS 64     /* co-located N limit (kernel parameter table) */
#define EA_UNIQUE_ID_BYTES 128 /* == sizeof(ncclUniqueId) */
#define EA_IPC_HANDLE_BYTES 64 /* == sizeof(cudaIpcMemHandle_t) */
#define EA_CHAN_HANDLE_BYTES 80 /* ea_chan_export: the IPC handle + the end's slot_bytes, slots and role */
#define EA_SLOT_CENTER_PREV 2  /* ea_get_state / ea_set_state slot of the stale center x~_{t-1} (staleness 1) */

typedef enum {
  EA_OK = 0,
  EA_EINVAL = 1,  /* bad argument: null/misaligned pointer, N<1, alpha not in [0,1], ... */
  EA_ECUDA = 2,   /* CUDA launch / runtime error (also async, reported at ea_sync) */
  EA_ENCCL = 3,   /* NCCL error (init, enqueue, or async at ea_sync) */
  EA_ESTATE = 4,  /* call not valid in the handle's current state/layout */
  EA_ENOMEM = 5   /* device or host allocation failed */
} ea_status;

typedef enum { EA_COLOCATED = 0, EA_SPREAD = 1 } ea_layout;

/* Local optimizer of Step 1 ("a user-specified optimizer"; the paper
 * trains GNMT/BERT with Adam and AWD with SGD/ASGD).  State slots
 * (ea_get_state): SGD 1 (momentum), Adam/AdamW 2 (m, v), ASGD 1 (the
 * average ax). */
typedef enum { EA_OPT_SGD = 0, EA_OPT_ADAM = 1, EA_OPT_ADAMW = 2, EA_OPT_ASGD = 3 } ea_optimizer;

/* How EA_SPREAD exchanges contributions and the center (rows a6/a7). */
typedef enum {
  EA_XCHG_NCCL = 0,  /* ncclReduceScatter -> shard update kernel -> in-place ncclAllGather on a side stream */
  EA_XCHG_P2P = 1    /* the library's own peer-memory kernels (CUDA IPC mappings over NVLink): p2p_push
                        on the caller's stream (local update, contributions stored straight into the
                        owners' inboxes), p2p_exchange on the side stream (owner reduction + center
                        update, center chunks pulled back), see ea_p2p.cu */
} ea_exchange;

typedef struct {
  int32_t n_pipelines;          /* N >= 1 parallel pipelines */
  int32_t n_stages;             /* stages hosted by this process, >= 1 */
  const int64_t* stage_params;  /* n_stages entries, P_s >= 1 (copied by ea_init) */
  float alpha;                  /* dilution rate in [0,1], P:112 (default 1/N) */
  float beta;                   /* center pull (EASGD); 0 in the paper's mode */
  float rho;                    /* weight of Delta_i in the contribution; 1 in the paper's mode */
  float lr;                     /* learning rate eta */
  float momentum;               /* SGD: mu in [0,1) */
  float weight_decay;           /* lambda >= 0 (SGD/Adam: L2 added to the gradient; AdamW: decoupled) */
  int32_t nesterov;             /* SGD: 0/1 */
  int32_t layout;               /* ea_layout */
  int32_t rank;                 /* EA_SPREAD: 0 <= rank < world; ignored otherwise */
  int32_t world;                /* EA_SPREAD: must equal n_pipelines; ignored otherwise */
  int32_t device;               /* CUDA device ordinal the handle binds to */
  int32_t kernel_variant;       /* EA_COLOCATED kernel (N <= 8; larger N has one kernel):
                                   0 = library default, 1 = register-resident replica loop,
                                   2 = lane-per-replica, center tile staged by cp.async.bulk,
                                   warp-shuffle reduction, 3 = bulk-copy pipeline (every input
                                   tile by cp.async.bulk into an mbarrier ring), 4 = split
                                   register loop (two lanes per center column, N/2 replicas
                                   each, shuffle reduction), 5 = warp per replica (contributions
                                   reduced through shared memory), 6 = warp-specialised warp per
                                   replica (N replica warps + a reducer warp over an mbarrier ring
                                   of contribution tiles; no block barrier).  Same results
                                   up to fp32 summation order (DESIGN.md c14); the default picks per N and optimizer
                                   (DESIGN.md §7). */
  int32_t optimizer;            /* ea_optimizer */
  double beta1, beta2;          /* Adam(W): moment rates in [0,1) (torch defaults 0.9, 0.999); double so
                                   that 1-beta2 keeps full precision (0.999f would be off by 1.3e-5) */
  float eps;                    /* Adam(W): denominator epsilon > 0 (torch default 1e-8) */
  int32_t exchange;             /* EA_SPREAD: ea_exchange (ignored for EA_COLOCATED) */
  int32_t staleness;            /* 0: synchronous center (c3); 1: the replicas see the center one step
                                   late, x~_{t-1}, as with the paper's asynchronous queues (
                                   reading c28, row f4).  Any optimizer; EA_COLOCATED, or EA_SPREAD with
                                   EA_XCHG_NCCL (there the local step of iteration t waits only for the
                                   snapshot of x~_t taken at the start of exchange t-1, so that exchange
                                   overlaps the whole iteration t).  The library keeps x~_{t-1} (P_s
                                   floats per stage, slot EA_SLOT_CENTER_PREV); x~_{-1} := x~_0 at the
                                   stage's first step, which must not be taken while the stream is
                                   capturing a CUDA graph (EA_ESTATE) unless the slot was set. */
  double asgd_lambd;            /* ASGD: decay term l >= 0 (torch default 1e-4) */
  double asgd_alpha;            /* ASGD: power a of the eta schedule (torch default 0.75) */
  double asgd_t0;               /* ASGD: step after which averaging starts, >= 0 (torch default 1e6) */
} ea_config;

typedef struct ea_ctx* ea_handle;

/* One op of the micro-batch order (Algorithm 1): kind 0 = forward,
 * 1 = backward; micro_batch is 0-based. */
typedef struct {
  int32_t kind;
  int32_t micro_batch;
} ea_op;

/* ABI version compiled into the library (EA_ABI_VERSION). */
EA_API int32_t ea_abi_version(void);

/* Fill id[EA_UNIQUE_ID_BYTES] with a fresh NCCL unique id (call on rank 0 and
 * broadcast it, e.g. over a torch process group).  EA_ENCCL on failure. */
EA_API ea_status ea_get_unique_id(uint8_t* id);

/* Create a handle.  Validates cfg (EA_EINVAL, nothing allocated), binds
 * cfg->device, allocates zero-initialised momentum for every hosted stage and
 * replica (N per stage co-located, 1 per stage spread) and, for EA_SPREAD,
 * the side stream, events, contribution scratch and -- if nccl_id is not
 * NULL -- the NCCL communicator of `world` ranks built from nccl_id (a
 * collective call: every rank must call ea_init).  EA_SPREAD with nccl_id ==
 * NULL is the external-collective mode: ea_step returns EA_ESTATE and the
 * caller drives ea_spread_local / its own reduce-scatter / ea_spread_apply /
 * its own all-gather.  nccl_id is ignored for EA_COLOCATED.  *out is NULL on
 * failure. */
EA_API ea_status ea_init(const ea_config* cfg, const uint8_t* nccl_id, ea_handle* out);

/* Number of fp32 elements the center buffer of `stage` must hold:
 * P_s for EA_COLOCATED; P_pad = round_up(P_s, 32*N) for EA_SPREAD (the
 * padding must be zero-initialised by the caller and stays zero).
 * Returns -1 for a bad handle or stage. */
EA_API int64_t ea_center_capacity(ea_handle h, int32_t stage);

/* Number of center elements owned by this rank (EA_SPREAD: P_pad/N; the
 * shard starts at element rank*P_pad/N).  EA_COLOCATED: P_s.  -1 on error. */
EA_API int64_t ea_shard_elems(ea_handle h, int32_t stage);

/* One elastic-averaging iteration of `stage` (0-based, < n_stages).
 *   replica_ptrs: EA_COLOCATED: N device pointers x_0..x_{N-1}, each P_s
 *                 floats, updated in place; EA_SPREAD: 1 pointer (this
 *                 rank's replica).
 *   grad_ptrs:    matching gradient pointers (read only).
 *   center_ptr:   x~ of the stage (ea_center_capacity floats), updated in place.
 *   stream:       caller's stream (cudaStream_t); NULL = legacy default stream.
 * EA_COLOCATED: one fused kernel on `stream`.  EA_SPREAD with EA_XCHG_NCCL:
 * the local kernel (x_i, optimizer state, contribution) runs on `stream`
 * after this stage's previous all-gather; the exchange (reduce-scatter ->
 * shard update -> all-gather) runs on the library's side stream and `stream`
 * does NOT wait for it -- the next forward and the other stages' local steps
 * proceed while the center is exchanged (never block the
 * pipelines).  EA_XCHG_P2P: the same split -- the push kernel (local update,
 * contributions pushed to the owners over peer memory) on `stream`, the
 * owner reduction and the pull of the other shards on the side stream.  Call
 * ea_sync before reading x~ on any stream.  All ranks must
 * call ea_step for the same stages in the same order (collective ordering).
 * Pointers must stay valid until the work completes. */
EA_API ea_status ea_step(ea_handle h, int32_t stage, float* const* replica_ptrs,
                  const float* const* grad_ptrs, float* center_ptr, void* stream);

/* Several stages in one call, in the given order (e.g. all stages hosted
 * here once the last backward is done).  stages: `count` distinct stage
 * indices; replica_ptrs / grad_ptrs: count*R pointers, stage-major (R = N
 * co-located, 1 spread); center_ptrs: `count` pointers.  EA_COLOCATED with
 * N <= 8 updates up to 8 stages with ONE kernel launch whose persistent grid
 * splits the concatenated work of all of them evenly; otherwise the stages
 * are stepped one after another exactly as by ea_step.  Every argument is
 * validated before anything is enqueued. */
EA_API ea_status ea_step_many(ea_handle h, int32_t count, const int32_t* stages, float* const* replica_ptrs,
                              const float* const* grad_ptrs, float* const* center_ptrs, void* stream);

/* End-to-end variant of ea_step_many for callers whose gradients live in HOST
 * memory (EA_COLOCATED): host_grad_ptrs are count*N host pointers (pinned
 * memory gives asynchronous, full-duplex copies), replica_ptrs / center_ptrs
 * device pointers as in ea_step_many, host_center_out `count` host buffers of
 * P_s floats that receive the updated centers.  The library streams the
 * gradients through double-buffered device staging in chunks of 4 Mi
 * elements on its own copy streams, runs the fused kernel on each chunk as it
 * lands (on `stream`) and copies each finished center chunk back on a second
 * copy stream, so H2D, kernel and D2H overlap.  When `stream` reaches the end
 * of this work, host_center_out is complete.  EA_ESTATE for EA_SPREAD. */
EA_API ea_status ea_step_many_host(ea_handle h, int32_t count, const int32_t* stages, float* const* replica_ptrs,
                                   const float* const* host_grad_ptrs, float* const* center_ptrs,
                                   float* const* host_center_out, void* stream);

/* EA_XCHG_P2P between handles of ONE process (e.g. N ranks on one device, or
 * N devices driven by one process): peers[q] is rank q's handle (peers[rank]
 * == h); every handle must call this with the same list.  Ranks created with
 * an NCCL id are connected by ea_init itself (CUDA IPC handles all-gathered
 * over NCCL) and need no call.  The ranks' exchange kernels wait for one
 * another's push kernels, so each rank must drive its own stream; ranks that
 * share a device split its SMs, and since each rank uses two streams (its
 * caller's and the library's side stream) the process must run with
 * CUDA_DEVICE_MAX_CONNECTIONS >= 2 * ranks + 1 (set before the CUDA context
 * exists): with fewer hardware queues a spinning exchange kernel can sit
 * ahead of a push it waits for in the same queue, and the wait times out.
 * EA_ESTATE for other layouts/exchanges. */
EA_API ea_status ea_p2p_connect(ea_handle h, const ea_handle* peers, int32_t world);

/* EA_XCHG_P2P between processes without an NCCL id (the caller moves the
 * handles, e.g. over a torch process group): ea_p2p_export writes this rank's
 * exchange-buffer IPC handle (EA_IPC_HANDLE_BYTES); ea_p2p_open takes all
 * ranks' handles (world x EA_IPC_HANDLE_BYTES, rank-major) and maps the peers
 * (cudaIpcOpenMemHandle).  Ranks created with an NCCL id do this inside ea_init. */
EA_API ea_status ea_p2p_export(ea_handle h, uint8_t* handle);
EA_API ea_status ea_p2p_open(ea_handle h, const uint8_t* handles, int32_t world);

/* Make `stream` wait until every center update enqueued so far is complete,
 * then report any asynchronous CUDA/NCCL error seen so far.  Does not block
 * the host. */
EA_API ea_status ea_sync(ea_handle h, void* stream);

/* ---- Phases of the EA_SPREAD step, for callers that run their own
 * collective (and for single-GPU verification of the decomposition). ---- */

/* Local phase of EA_SPREAD on `stream`: updates x (this rank's replica) and
 * this rank's momentum in place and writes the contribution
 * r = rho*Delta + beta*(x - x~) into contrib[0..P_s) and zeros into
 * contrib[P_s..P_pad).  center_ptr is read only. */
EA_API ea_status ea_spread_local(ea_handle h, int32_t stage, float* replica_ptr, const float* grad_ptr,
                          const float* center_ptr, float* contrib, void* stream);

/* Shard phase of EA_SPREAD on `stream`: center_shard[k] += reduced[k] / N for
 * k < ea_shard_elems (reduced = this rank's shard of sum_i r_i). */
EA_API ea_status ea_spread_apply(ea_handle h, int32_t stage, float* center_shard, const float* reduced,
                          void* stream);

/* ---- Optimizer state (checkpoint / resume) ---- */

/* *state_dev = device pointer to optimizer-state slot `slot` of (stage,
 * replica): P_s floats, owned by the library, valid until ea_destroy.
 * slot 0 = SGD momentum / Adam first moment / ASGD average, slot 1 = Adam second moment
 * (EA_EINVAL for SGD and ASGD), slot EA_SLOT_CENTER_PREV = the stale center
 * x~_{t-1} of a staleness-1 handle (replica 0; defined after the stage's first
 * step or an ea_set_state of the slot).  EA_SPREAD: replica must be 0. */
EA_API ea_status ea_get_state(ea_handle h, int32_t stage, int32_t replica, int32_t slot, float** state_dev);

/* Copy P_s floats from device pointer src into state slot `slot` of (stage,
 * replica), ordered on `stream` (after pending EA_SPREAD side-stream work).
 * Setting EA_SLOT_CENTER_PREV marks x~_{t-1} as given (checkpoint resume; no
 * x~_{-1} := x~_0 initialisation at the next step). */
EA_API ea_status ea_set_state(ea_handle h, int32_t stage, int32_t replica, int32_t slot, const float* src,
                              void* stream);

/* Step count t of `stage` (number of ea_step / ea_spread_local calls so far;
 * Adam's bias correction uses t+1 for the next step).  ea_set_step changes
 * only the optimizer's t (resume); the peer-memory exchange keeps its own
 * epoch counter, which every rank advances once per ea_step. */
EA_API ea_status ea_get_step(ea_handle h, int32_t stage, int64_t* step);
EA_API ea_status ea_set_step(ea_handle h, int32_t stage, int64_t step);

/* Replace the hyper-parameters (alpha, beta, rho, lr, momentum, weight_decay,
 * nesterov, beta1, beta2, eps, asgd_lambd, asgd_alpha, asgd_t0) from cfg,
 * e.g. for a learning-rate schedule; same validation as ea_init; optimizer,
 * n_pipelines and layout must equal the handle's (other fields are ignored).
 * Takes effect for steps enqueued afterwards (ASGD: eta_t of the next step is
 * computed from the new lr; torch.optim.ASGD would use the eta it computed
 * at the end of the previous step with the old lr). */
EA_API ea_status ea_set_hyper(ea_handle h, const ea_config* cfg);

/* Wait for outstanding work, free everything the library owns, destroy the
 * communicator.  EA_XCHG_P2P with an NCCL communicator: a barrier over the
 * communicator precedes freeing the IPC-exported exchange buffer, so every
 * rank must call ea_destroy (collective); handles wired with ea_p2p_open /
 * ea_p2p_connect must be destroyed after a caller-side barrier of all ranks.
 * NULL is a no-op. */
EA_API ea_status ea_destroy(ea_handle h);

/* Message of the last failing call on h (h == NULL: this thread's last
 * ea_init / handle-less failure).  Never NULL; "" if none. */
EA_API const char* ea_last_error(ea_handle h);

/* Advance-forward-propagation order of one batch on one stage (Algorithm 1,
 * P:140-162, plus the implied cool-down -- DESIGN.md c15).  K stages, M
 * micro-batches, stage 0-based (< K), advance = forwards run in advance
 * (clamped to [0, M]; K-1-stage is 1F1B, M is AFAB).  Writes 2M ops to out
 * (cap >= 2M) and returns 2M; returns -EA_EINVAL for K < 1, M < 0, stage out
 * of range, cap < 2M or out == NULL (with M > 0).  Host only; no GPU needed. */
EA_API int32_t ea_schedule(int32_t K, int32_t M, int32_t stage, int32_t advance, ea_op* out, int32_t cap);

/* ---- Point-to-point activation channel (row f2; csrc/ea_chan.cu) ----
 * The transfers of the pipeline runtime: stage k sends activations to stage k+1 and receives activation
 * gradients back, in Algorithm 1's order ("a parallel pipeline launches a process on each GPU",
 * P:140-162).  A channel is ONE direction between two processes (NVLink peers, or two processes sharing a GPU).
 * The receiving end owns a ring of `slots` message slots of `slot_bytes` and one ready word per slot, the
 * sending end one acknowledgement word per slot, all in device memory on `device`.  Each end exports its buffer
 * (ea_chan_export: EA_CHAN_HANDLE_BYTES = the cudaIpcMemHandle_t plus the end's geometry and role) and opens the
 * other's (ea_chan_connect: EA_EINVAL unless the peer has the opposite role and the same slot_bytes and slots);
 * two ends in ONE process are wired with ea_chan_pair instead (CUDA IPC cannot open a handle of its own process).
 *
 * ea_chan_send / ea_chan_recv enqueue on `stream` (cudaStream_t; NULL = legacy default stream) and never block
 * the host: send = wait until the slot is free (stream wait on the local ack word) -> copy-engine copy of
 * `bytes` from device pointer src into the receiver's slot over the peer mapping -> stream write of the
 * receiver's ready word; recv = stream wait on the local ready word -> copy into device pointer dst -> stream
 * write of the sender's ack word.  The k-th send matches the k-th recv (k counts calls on each end).  src must
 * stay unmodified, and dst unread, until the stream reaches that point.  Errors: bytes > slot_bytes, a NULL
 * buffer or the wrong end -> EA_EINVAL; not connected, or the stream is capturing a CUDA graph (the slot and
 * round are host counters) -> EA_ESTATE; CUDA / driver failures -> EA_ECUDA.  Nothing is enqueued on error.
 * ea_chan_destroy synchronises the device, closes the peer mapping and frees this end's buffer: both ends
 * must be past their last operation (a caller-side barrier) before either is destroyed.
 * Caution: a stream that waits for a message blocks until the peer sends it; anything that synchronises the
 * whole context meanwhile (cudaDeviceSynchronize, and the FIRST launch of a kernel under CUDA's lazy module
 * loading) waits for it too.  If the peer sends that message only after this process enqueues more work, use
 * CUDA_MODULE_LOADING=EAGER (the pipeline runtime requires it) and no device-wide synchronisation while
 * messages are outstanding. */
typedef struct ea_chan_s* ea_chan;
EA_API ea_status ea_chan_create(int32_t device, int32_t role /* 0 = send, 1 = recv */, int64_t slot_bytes,
                                int32_t slots, ea_chan* out);
EA_API ea_status ea_chan_export(ea_chan c, uint8_t* handle);
EA_API ea_status ea_chan_connect(ea_chan c, const uint8_t* peer_handle);
EA_API ea_status ea_chan_pair(ea_chan send_end, ea_chan recv_end);
EA_API ea_status ea_chan_send(ea_chan c, const void* src, int64_t bytes, void* stream);
EA_API ea_status ea_chan_recv(ea_chan c, void* dst, int64_t bytes, void* stream);
/* Messages enqueued so far on this end (-1 for NULL). */
EA_API int64_t ea_chan_count(ea_chan c);
EA_API ea_status ea_chan_destroy(ea_chan c);
/* Message of the last failing call on c (c == NULL: this thread's last ea_chan_create failure). */
EA_API const char* ea_chan_last_error(ea_chan c);

/* ---- Run-time advance adjustment (Algorithm 1 lines 1, 9-10) ---- */

/* Controller state (plain data, caller-owned; DESIGN.md c27). */
typedef struct {
  int32_t K, M;          /* pipeline depth and micro-batches per batch */
  int32_t advance_num;   /* forwards in advance on the first stage (starts at K-1: 1F1B) */
  int32_t has_last;      /* a previous batch time is recorded */
  double last_time;      /* previous batch time */
} ea_advance_ctl;

/* Line 1: advance_num = min(K-1, M).  EA_EINVAL for K < 1, M < 0 or ctl == NULL. */
EA_API ea_status ea_advance_init(ea_advance_ctl* ctl, int32_t K, int32_t M);

/* Lines 9-10 after one batch: if the batch was faster than the previous one
 * (the first batch counts as faster) and peak_mem + mem_per_microbatch <=
 * mem_limit, advance_num++ (capped at M).  Returns the new advance_num, or
 * -EA_EINVAL on NULL / NaN arguments. */
EA_API int32_t ea_advance_update(ea_advance_ctl* ctl, double batch_time, double peak_mem, double mem_per_microbatch,
                                 double mem_limit);

/* Advance of `stage` (0-based): min(M, K-1-stage + advance_num - min(K-1, M)) (c15); -EA_EINVAL if out of range. */
EA_API int32_t ea_advance_for_stage(const ea_advance_ctl* ctl, int32_t stage);

/* ---- Profiling-based tuning predictor (§5.2, Eqs. (1)-(8); host only) ---- */

/* One profiled setting: M = m micro-batches, N = n parallel pipelines, K GPUs. */
typedef struct {
  int32_t n_gpus;         /* K >= 1 */
  int32_t m, n;           /* profiled micro-batches per batch and pipelines, >= 1 */
  int32_t n_samples;      /* samples per utilisation curve (>= 0) */
  double dt;              /* seconds between samples */
  const double* phi;      /* K x n_samples, row-major: GPU k's utilisation phi^k(t) in [0, 1] */
  const double* t_gpu;    /* K: computation time per batch T_gpu^k (s) */
  const double* t_comm;   /* K: total communication time per batch TT^k (s) */
  const double* f_mod;    /* K: parallel + reference model footprint F_mod^k (bytes) */
  const double* f_dat;    /* K: data / intermediate-result footprint F_dat^k (bytes) */
} ea_profile;

/* Prediction for one GPU at a candidate (m*, n*). */
typedef struct {
  double t_gpu;    /* Eq. (2) */
  double t_com;    /* Eq. (4) */
  double t_up;     /* Eq. (6) */
  double t_down;   /* Eq. (7) */
  double t_bub;    /* Eq. (5) */
  double t_total;  /* Eq. (1) */
  double mem;      /* Eq. (8) */
} ea_gpu_prediction;

typedef enum { EA_TUNE_THROUGHPUT = 0, EA_TUNE_TIME = 1 } ea_tune_objective;

/* Predict every GPU's time decomposition and memory at (m_star, n_star).
 * out: K entries (may be NULL); *iter_time = max_k t_total; *peak_mem =
 * max_k mem (either may be NULL).  EA_EINVAL on a malformed profile (NULL
 * arrays, negative or non-finite values, phi outside [0, 1]) or m*, n* < 1. */
EA_API ea_status ea_predict(const ea_profile* prof, int32_t m_star, int32_t n_star, ea_gpu_prediction* out,
                            double* iter_time, double* peak_mem);

/* Choose (m*, n*) from the candidate lists: the highest throughput
 * n* / T* (EA_TUNE_THROUGHPUT) or the lowest T* (EA_TUNE_TIME) among settings
 * whose peak memory <= mem_limit; ties go to lower memory, then smaller n*,
 * then smaller m*.  EA_ESTATE (best = -1) if nothing fits the limit. */
EA_API ea_status ea_tune(const ea_profile* prof, const int32_t* m_cands, int32_t n_m, const int32_t* n_cands,
                         int32_t n_n, double mem_limit, int32_t objective, int32_t* best_m, int32_t* best_n,
                         double* best_iter_time);

#ifdef __cplusplus
}
#endif

#endif /* AVGPIPE_EA_H_ */

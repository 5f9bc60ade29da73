// Internal declarations shared by the C-ABI layer (ea_api.cu) and the
// kernels (ea_kernels.cu).  Not part of the public ABI (include/ea.h).
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

namespace ea {

// Local optimizer of Step 1 (DESIGN.md c7 SGD-momentum, c21 Adam/AdamW, c29 ASGD).
enum Opt : int { kOptSGD = 0, kOptAdam = 1, kOptAdamW = 2, kOptASGD = 3 };

// Adam(W) keep two state vectors (m, v); SGD-momentum and ASGD one (momentum / the average ax), so they
// move the same bytes and share the kernels' 3-stream geometry.
__host__ __device__ constexpr bool two_state(int opt) { return opt == kOptAdam || opt == kOptAdamW; }
// Optimizers with per-step coefficients (StepCoef): Adam(W)'s bias corrections, ASGD's eta_t and mu_t.
__host__ __device__ constexpr bool has_coef(int opt) { return opt != kOptSGD; }

// Hyper-parameters in the form the kernels consume (fp32).
struct Hyper {
  float alpha;     // dilution rate
  float beta;      // center pull (EASGD)
  float rho;       // weight of Delta_i in the contribution
  float lr;        // learning rate
  float momentum;  // mu (SGD)
  float wd;        // weight decay lambda (SGD/Adam: L2 on the gradient; AdamW: decoupled)
  int nesterov;    // 0/1 (SGD)
  float inv_n;     // 1/N (step 5 normalisation)
  float beta1, one_minus_beta1;  // Adam
  float beta2, one_minus_beta2;
  float eps;
  float lr_wd;     // lr * wd (AdamW decoupled decay)
  float asgd_lambd;  // ASGD decay term l (Delta = -eta_t (g + wd x + l x))
};

// Per-stage Adam bias corrections for the step being taken (t = the stage's
// step count).  They live in device memory, written by advance_steps() on the
// stream right before the step's kernel, so a captured CUDA graph advances t
// on every replay.
struct StepCoef {
  float step_size;     // Adam: lr / (1 - beta1^t);     ASGD: eta_t = lr / (1 + l lr (t-1))^a
  float inv_sqrt_bc2;  // Adam: 1 / sqrt(1 - beta2^t);  ASGD: mu_t = 1 / max(1, t-1-t0)
};

// What advance_steps needs to compute StepCoef for the handle's optimizer.
struct CoefParams {
  int opt;
  double beta1, beta2, lr;          // Adam(W)
  double lambd, asgd_alpha, t0;     // ASGD
};

// Stage list of one advance_steps launch.
struct StageList {
  int idx[8];
  int count;
};

// On `s`: for every listed stage, ++steps[stage], ++xepoch[stage] (if xepoch is not null: the peer-memory
// exchange's epoch) and recompute coef[stage] (double precision).
cudaError_t launch_advance_steps(int64_t* steps, uint32_t* xepoch, StepCoef* coef, const StageList& list,
                                 const CoefParams& cp, cudaStream_t s);

constexpr int kMaxReplicas = 64;      // EA_MAX_REPLICAS
constexpr int kMaxFusedN = 8;         // replicas handled by the compile-time-N kernels
constexpr int kMaxLaunchStages = 8;   // stages fused into one launch

// One co-located stage as the kernels see it.
struct StageRefs {
  float* x[kMaxFusedN];
  const float* g[kMaxFusedN];
  float* m[kMaxFusedN];  // SGD momentum / Adam first moment
  float* v[kMaxFusedN];  // Adam second moment (unused by SGD)
  float* c;
  int64_t p;             // elements
  const StepCoef* scp;   // device: this stage's Adam coefficients (unused by SGD)
  float* prev = nullptr; // staleness 1 (row f4): x~_{t-1}, read by the replicas, then set to x~_t
};

// Up to kMaxLaunchStages stages updated by ONE launch (same N).
struct StageBatch {
  StageRefs st[kMaxLaunchStages];
  int nstages;
};

// Pointer table of one stage with up to kMaxReplicas replicas (N > 8 path).
struct ReplicaTable {
  float* x[kMaxReplicas];
  const float* g[kMaxReplicas];
  float* m[kMaxReplicas];
  float* v[kMaxReplicas];
};

enum KernelVariant : int {
  kVariantAuto = 0,      // library picks (lane/shuffle, the measured best)
  kVariantRegLoop = 1,   // one thread per float4 of center, loops over N replicas in registers (SGD)
  kVariantLaneShfl = 2,  // lanes = (replica, float4 chunk); center tile staged by cp.async.bulk
                         // into shared memory; replica reduction by warp shuffles (SGD, Adam)
  kVariantBulkPipe = 3,  // every input tile streamed by cp.async.bulk into a multi-stage smem
                         // ring (producer warp + mbarriers); consumers store from registers (SGD)
  kVariantSplit = 4,     // split register loop: 2 lanes per center column, N/2 replicas each, shuffle reduction
  kVariantWarpRep = 5,   // warp per replica, 512 B rows, contributions reduced through shared memory
  kVariantWarpSpec = 6,  // warp-specialised: N replica warps + a reducer warp, mbarrier ring of contribution tiles
};

// Co-located fused step (rows a1-a5) for a batch of stages with the same N
// (N <= kMaxFusedN): updates x_i, optimizer state and x~ of every stage in
// place, one launch.  Adam/AdamW always use the lane kernel.
cudaError_t launch_colocated_batch(const StageBatch& b, int n, const Hyper& hp, int opt, int variant, int num_sms,
                                   cudaStream_t s);

// Stale center (row f4) for a batch of stages with N <= 5, every st[].prev set: for 2 <= N <= kMaxStaleLaneN the
// lane kernel with x~_{t-1} staged beside x~_t, for N = 1 and 5 the bulk-copy pipeline with x~_{t-1} as one more
// stream (replicas use x~_{t-1}, x~_{t+1} = x~_t + R/N, prev <- x~_t).
constexpr int kMaxStaleLaneN = 4;
// variant kVariantWarpRep / kVariantWarpSpec: the warp-per-replica kernels with x~_{t-1} for any N <= kMaxFusedN.
cudaError_t launch_colocated_batch_stale(const StageBatch& b, int n, const Hyper& hp, int opt, int variant,
                                         int num_sms, cudaStream_t s);

// Co-located step for one stage with any N <= kMaxReplicas (replica loop).  prev != nullptr: stale
// center (row f4): replicas use prev (x~_{t-1}), center is updated from x~_t, prev <- x~_t.
cudaError_t launch_colocated_wide(const ReplicaTable& t, int n, float* center, float* prev, int64_t p, const Hyper& hp,
                                  int opt, const StepCoef* scp, int num_sms, cudaStream_t s);

// Spread local step (rows a1-a4 for one replica): updates x and the optimizer
// state in place and writes r = rho*Delta + beta*(x - x~) into contrib[0..p),
// zeros into contrib[p..p_pad).
cudaError_t launch_spread_local(float* x, const float* g, float* m, float* v, const float* center, float* contrib,
                                int64_t p, int64_t p_pad, const Hyper& hp, int opt, const StepCoef* scp, int num_sms,
                                cudaStream_t s);

// ---- fused peer-memory spread step (ea_p2p.cu)
constexpr int kMaxWorld = 16;

// Addresses of every rank's exchange buffers for one stage, as seen from this GPU.
struct P2PView {
  float* inbox[kMaxWorld];     // rank o: [N][slots][chunk] contributions for the chunks o owns
  float* outbox[kMaxWorld];    // rank o: [slots][chunk] updated center of the chunks o owns
  uint32_t* arrive[kMaxWorld]; // rank o: [slots] cumulative arrival counters
  uint32_t* ready[kMaxWorld];  // rank o: [slots] epoch at which the outbox chunk is final
};

struct P2PArgs {
  float* x;            // this rank's replica (p floats)
  const float* g;      // its gradient
  float* m;            // optimizer state slot 0
  float* v;            // optimizer state slot 1 (Adam) or null
  float* center;       // this rank's copy of x~ (p_pad floats, zero padding)
  int64_t p, p_pad;    // elements / padded elements
  int64_t chunk;       // floats per chunk (multiple of 4)
  int64_t nchunks, slots;
  int rank, world;
  const uint32_t* epochp;  // device: this stage's exchange epoch (>= 1; advanced on the stream, never by ea_set_step)
  uint32_t* tickets;   // device: this stage's work-item ticket of p2p_exchange (zeroed before each launch)
  uint32_t* abort;     // device: set by the first timed-out wait; later waits fail at once
  Hyper hp;
  const StepCoef* scp;   // device: the step's optimizer coefficients
  uint32_t* err;       // host-mapped error flag (timeouts)
  uint64_t timeout_ns;
  int sc_fence;        // 1: fence.sc.sys before each release (knob AVGPIPE_EA_P2P_FENCE=1; default 0)
};

// Phase A (local update, contributions pushed into the owners' inboxes): never waits.  Default: the bulk-copy
// ring kernel, one CTA per SM on at most max_sms SMs; knob AVGPIPE_EA_P2P_PUSH=plain: the register loop with up
// to max_ctas CTAs.
cudaError_t launch_p2p_push(const P2PArgs& a, const P2PView& v, int opt, int max_ctas, int max_sms, cudaStream_t s);
// Phases B (owner reduction + center update) and C (pull the other owners' chunks), ticket-ordered.
cudaError_t launch_p2p_exchange(const P2PArgs& a, const P2PView& v, int max_ctas, cudaStream_t s);
int p2p_blocks_per_sm(int opt);

// Spread shard epilogue (row a5): shard[k] += reduced[k] * inv_n for k < count.  max_ctas > 0 caps the grid
// (the library's side stream runs it beside the caller's compute).
cudaError_t launch_spread_apply(float* shard, const float* reduced, int64_t count, float inv_n, int num_sms,
                                int max_ctas, cudaStream_t s);

}  // namespace ea

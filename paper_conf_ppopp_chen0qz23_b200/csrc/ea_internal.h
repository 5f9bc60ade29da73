// Internal declarations shared by the C-ABI layer (ea_api.cu) and the
// kernels (ea_kernels.cu).  Not part of the public ABI (include/ea.h).
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

namespace ea {

// Hyper-parameters in the form the kernels consume (fp32, P:112 / DESIGN.md c7).
struct Hyper {
  float alpha;     // dilution rate
  float beta;      // center pull (EASGD)
  float rho;       // weight of Delta_i in the contribution
  float lr;        // SGD learning rate
  float momentum;  // mu
  float wd;        // L2 weight decay lambda
  int nesterov;    // 0/1
  float inv_n;     // 1/N (step 5 normalisation)
};

constexpr int kMaxReplicas = 64;      // EA_MAX_REPLICAS
constexpr int kMaxFusedN = 8;         // replicas handled by the compile-time-N kernels
constexpr int kMaxLaunchStages = 8;   // stages fused into one launch

// One co-located stage as the kernels see it.
struct StageRefs {
  float* x[kMaxFusedN];
  const float* g[kMaxFusedN];
  float* m[kMaxFusedN];
  float* c;
  int64_t p;  // elements
};

// Up to kMaxLaunchStages stages updated by ONE launch (same N): the work of
// all stages is concatenated and split evenly over the persistent grid.
struct StageBatch {
  StageRefs st[kMaxLaunchStages];
  int nstages;
};

// Pointer table of one stage with up to kMaxReplicas replicas (N > 8 path).
struct ReplicaTable {
  float* x[kMaxReplicas];
  const float* g[kMaxReplicas];
  float* m[kMaxReplicas];
};

enum KernelVariant : int {
  kVariantAuto = 0,      // library picks (see launch_colocated_batch)
  kVariantRegLoop = 1,   // one thread per float4 of center, loops over N replicas in registers
  kVariantLaneShfl = 2,  // lanes = (replica, float4 chunk); center tile staged by cp.async.bulk
                         // into shared memory; replica reduction by warp shuffles
  kVariantBulkPipe = 3,  // every input tile streamed by cp.async.bulk into a multi-stage smem
                         // ring (producer warp + mbarriers); consumers store from registers
};

// Co-located fused step (rows a1-a5) for a batch of stages with the same N
// (N <= kMaxFusedN): updates x_i, m_i and x~ of every stage in place, one launch.
cudaError_t launch_colocated_batch(const StageBatch& b, int n, const Hyper& hp, int variant, int num_sms,
                                   cudaStream_t s);

// Co-located step for one stage with any N <= kMaxReplicas (N > 8 path).
cudaError_t launch_colocated_wide(const ReplicaTable& t, int n, float* center, int64_t p, const Hyper& hp,
                                  int num_sms, cudaStream_t s);

// Spread local step (rows a1-a4 for one replica): updates x, m in place and
// writes r = rho*Delta + beta*(x - x~) into contrib[0..p), zeros into
// contrib[p..p_pad).
cudaError_t launch_spread_local(float* x, const float* g, float* m, const float* center, float* contrib,
                                int64_t p, int64_t p_pad, const Hyper& hp, int num_sms, cudaStream_t s);

// Spread shard epilogue (row a5): shard[k] += reduced[k] * inv_n for k < count.
cudaError_t launch_spread_apply(float* shard, const float* reduced, int64_t count, float inv_n, int num_sms,
                                cudaStream_t s);

}  // namespace ea

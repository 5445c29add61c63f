// Launch accounting / per-class event timing hooks (prof.cu).
#pragma once
#include <cuda_runtime.h>

namespace adainf {

enum ProfClass {
  PC_CONV_FWD = 0,
  PC_CONV_DGRAD,
  PC_CONV_WGRAD,
  PC_WGRAD_REDUCE,
  PC_BIAS_COLSUM,
  PC_PACK,
  PC_POOL_FWD,
  PC_POOL_BWD,
  PC_EXIT_HEAD,
  PC_COMPACT,
  PC_EXIT_LOSS,
  PC_HEAD_GRADS,
  PC_GRAD_FINALIZE,
  PC_SUM,
  PC_SGD,
  PC_SHADOW_PACK,
  PC_SELECT_PROJ,
  PC_SELECT_COSINE,
  PC_SELECT_TOPK,
  PC_DET_ROUTE,
  PC_CROP,
  PC_ROUTE_CLASS,
  PC_GATHER,
  PC_STEM_FWD,
  PC_STEM_WGRAD,
  PC_STEM_AUX,
  PC_CONV_DGRAD_PREP,
  PC_SURVIVOR_GATHER,
  PC_EXIT_HEAD_TRAIN,
  PC_VERSION_AVG,
  PC_DW,
  PC_SHUFFLE,
  PROF_NCLASS
};

// RAII: counts `n` kernel launches of class `cls` on `st`; when profiling is enabled, brackets them with
// CUDA events recorded on the same stream.
struct ProfScope {
  ProfScope(int cls, cudaStream_t st, int n = 1);
  ~ProfScope();
  int cls_;
  cudaStream_t st_;
  void* ev_;
};

}  // namespace adainf

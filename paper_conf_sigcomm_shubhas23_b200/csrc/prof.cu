// Launch accounting and optional per-kernel-class CUDA-event timing (used by bench.py for the roofline
// leg: the dominant kernel's average launch duration measured live, on the launching stream).
#include <mutex>
#include <vector>

#include "../../include/adainf_debug.h"
#include "api_common.h"
#include "prof.h"

namespace adainf {

static const char* kNames[PROF_NCLASS] = {"conv_fwd",     "conv_dgrad", "conv_wgrad", "wgrad_reduce", "bias_colsum",
                                          "pack_input",   "maxpool_fwd", "maxpool_bwd", "exit_head",    "compact",
                                          "exit_loss",    "head_grads",  "grad_finalize", "sum",        "sgd_update",
                                          "shadow_pack",  "select_proj", "select_cosine", "select_topk", "det_route",
                                          "crop",         "route_class", "gather_rows", "stem_fwd",   "stem_wgrad",
                                          "stem_aux",     "dgrad_sp_prep", "survivor_gather", "exit_head_train",
                                          "version_average", "depthwise", "shufflenet_aux"};

struct Prof {
  std::mutex mu;
  bool on = false;
  long long launches = 0;
  struct Rec {
    int cls;
    cudaEvent_t a, b;
  };
  std::vector<Rec> recs;
  std::vector<cudaEvent_t> pool;
  long long n_launch[PROF_NCLASS] = {0};
  double ms[PROF_NCLASS] = {0};
};
static Prof g;

static cudaEvent_t get_ev() {
  if (!g.pool.empty()) {
    cudaEvent_t e = g.pool.back();
    g.pool.pop_back();
    return e;
  }
  cudaEvent_t e;
  CK(cudaEventCreate(&e));
  return e;
}

ProfScope::ProfScope(int cls, cudaStream_t st, int n) : cls_(cls), st_(st), ev_(nullptr) {
  std::lock_guard<std::mutex> l(g.mu);
  g.launches += n;
  g.n_launch[cls] += n;
  if (g.on) {
    cudaEvent_t a = get_ev();
    CK(cudaEventRecord(a, st));
    ev_ = a;
  }
}
ProfScope::~ProfScope() {
  if (!ev_) return;
  std::lock_guard<std::mutex> l(g.mu);
  cudaEvent_t b = get_ev();
  cudaEventRecord(b, st_);
  g.recs.push_back({cls_, (cudaEvent_t)ev_, b});
}

static void drain() {
  for (auto& r : g.recs) {
    cudaEventSynchronize(r.b);
    float t = 0.f;
    cudaEventElapsedTime(&t, r.a, r.b);
    g.ms[r.cls] += t;
    g.pool.push_back(r.a);
    g.pool.push_back(r.b);
  }
  g.recs.clear();
}

}  // namespace adainf

using namespace adainf;

extern "C" adainf_status adainf_prof_enable(int32_t on) {
  return guard([&] {
    std::lock_guard<std::mutex> l(g.mu);
    drain();
    g.on = on != 0;
  });
}
extern "C" adainf_status adainf_prof_reset(void) {
  return guard([&] {
    std::lock_guard<std::mutex> l(g.mu);
    drain();
    for (int i = 0; i < PROF_NCLASS; ++i) {
      g.ms[i] = 0;
      g.n_launch[i] = 0;
    }
  });
}
extern "C" int64_t adainf_launch_count(void) {
  std::lock_guard<std::mutex> l(g.mu);
  return g.launches;
}
extern "C" adainf_status adainf_prof_query(adainf_prof_entry* out, int32_t max_entries, int32_t* n_out) {
  return guard([&] {
    std::lock_guard<std::mutex> l(g.mu);
    drain();
    int n = 0;
    for (int i = 0; i < PROF_NCLASS && n < max_entries; ++i) {
      out[n].name = kNames[i];
      out[n].launches = g.n_launch[i];
      out[n].total_ms = g.ms[i];
      n++;
    }
    if (n_out) *n_out = n;
  });
}

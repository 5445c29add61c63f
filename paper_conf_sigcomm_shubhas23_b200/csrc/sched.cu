// Incremental-retraining support (include/adainf_sched.h): spare-time split
// (example P:51), retraining setting from a measured step profile, version averaging
// (P:241), disjoint-sample marking, prediction accuracy counts.
#include <cmath>
#include <vector>

#include "../../include/adainf_sched.h"
#include "api_common.h"
#include "api_handles.h"
#include "prof.h"

using namespace adainf;

namespace {

bool finite_nonneg(double v) { return std::isfinite(v) && v >= 0.0; }

// up to 16 versions: the pointer table travels as a kernel parameter (no host->device copy, no synchronization:
// the call can be captured in a CUDA graph)
struct SrcTable {
  const float* p[16];
  __device__ const float* operator[](int v) const { return p[v]; }
};

// dst = (sum_v src_v in order) / n, fp32; one thread per 4 parameters
template <class Tab>
__global__ void average_kernel(float* __restrict__ dst, Tab srcs, int n, long long count) {
  const long long i = (blockIdx.x * (long long)blockDim.x + threadIdx.x) * 4;
  if (i >= count) return;
  if (i + 4 <= count) {
    float4 acc = __ldg((const float4*)(srcs[0] + i));
    for (int v = 1; v < n; ++v) {
      const float4 x = __ldg((const float4*)(srcs[v] + i));
      acc.x = __fadd_rn(acc.x, x.x);
      acc.y = __fadd_rn(acc.y, x.y);
      acc.z = __fadd_rn(acc.z, x.z);
      acc.w = __fadd_rn(acc.w, x.w);
    }
    const float fn = (float)n;
    *(float4*)(dst + i) = make_float4(__fdiv_rn(acc.x, fn), __fdiv_rn(acc.y, fn), __fdiv_rn(acc.z, fn),
                                      __fdiv_rn(acc.w, fn));
  } else {
    for (long long j = i; j < count; ++j) {
      float acc = srcs[0][j];
      for (int v = 1; v < n; ++v) acc = __fadd_rn(acc, srcs[v][j]);
      dst[j] = __fdiv_rn(acc, (float)n);
    }
  }
}

__global__ void scale_kernel(float* __restrict__ x, long long count, float div) {
  const long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x;
  if (i < count) x[i] = __fdiv_rn(x[i], div);
}

__global__ void mark_used_kernel(uint8_t* __restrict__ exclude, const int32_t* __restrict__ idx, const int32_t* count,
                                 int n_static) {
  const int n = count ? min(*count, n_static) : n_static;
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) exclude[idx[i]] = 1;
}

__global__ void count_correct_kernel(const int32_t* __restrict__ pred, const int32_t* __restrict__ labels, int n,
                                     int32_t* __restrict__ correct) {
  __shared__ int wsum[32];
  int c = 0;
  for (int i = threadIdx.x; i < n; i += blockDim.x) c += pred[i] == labels[i];
  for (int o = 16; o > 0; o >>= 1) c += __shfl_xor_sync(0xffffffffu, c, o);
  if ((threadIdx.x & 31) == 0) wsum[threadIdx.x >> 5] = c;
  __syncthreads();
  if (threadIdx.x == 0) {
    int t = 0;
    for (int w = 0; w < (int)(blockDim.x >> 5); ++w) t += wsum[w];
    *correct = t;
  }
}

}  // namespace

extern "C" adainf_status adainf_time_split(double slo_ms, const double* infer_ms, int32_t n_infer,
                                           const double* impact, int32_t n_retrain, double* out_spare_ms,
                                           double* out_alloc_ms) {
  return guard([&] {
    if (n_infer < 0 || n_retrain < 0) throw InvalidError("time_split: negative count");
    if ((n_infer > 0 && !infer_ms) || (n_retrain > 0 && (!impact || !out_alloc_ms)) || !out_spare_ms)
      throw InvalidError("time_split: null array");
    if (!finite_nonneg(slo_ms)) throw InvalidError("time_split: SLO must be finite and >= 0");
    double used = 0.0;
    for (int k = 0; k < n_infer; ++k) {
      if (!finite_nonneg(infer_ms[k])) throw InvalidError("time_split: inference latency must be finite and >= 0");
      used += infer_ms[k];
    }
    double dsum = 0.0;
    for (int j = 0; j < n_retrain; ++j) {
      if (!finite_nonneg(impact[j])) throw InvalidError("time_split: impact degree must be finite and >= 0");
      dsum += impact[j];
    }
    const double tr = slo_ms > used ? slo_ms - used : 0.0;  // T_r^i = L_s^i - sum_k l_k^i
    *out_spare_ms = tr;
    for (int j = 0; j < n_retrain; ++j) out_alloc_ms[j] = dsum > 0.0 ? tr * impact[j] / dsum : 0.0;
  });
}

extern "C" adainf_status adainf_retrain_setting(double alloc_ms, const adainf_retrain_profile* prof, int64_t eligible,
                                                int32_t max_batch, adainf_retrain_plan* out) {
  return guard([&] {
    if (!prof || !out || prof->n < 1 || !prof->batch || !prof->step_ms) throw InvalidError("retrain_setting: bad profile");
    if (!finite_nonneg(alloc_ms) || eligible < 0 || max_batch < 1) throw InvalidError("retrain_setting: bad arguments");
    adainf_retrain_plan best{0, 0, 0, 0, 0.0};
    long long best_visits = 0;
    for (int i = 0; i < prof->n; ++i) {
      const int b = prof->batch[i];
      const double t = prof->step_ms[i];
      if (b < 1 || !(t > 0.0) || !std::isfinite(t)) throw InvalidError("retrain_setting: profile entries need batch >= 1, ms > 0");
      if (b > max_batch || (long long)b > eligible) continue;  // a step needs b distinct eligible samples
      const long long steps = (long long)std::floor(alloc_ms / t);
      if (steps < 1) continue;
      const long long visits = steps * b;
      if (visits > best_visits || (visits == best_visits && b > best.batch)) {
        best_visits = visits;
        best.batch = b;
        best.steps = (int32_t)std::min<long long>(steps, 1LL << 30);
        best.est_ms = (double)best.steps * t;
      }
    }
    if (best_visits > 0) {
      const long long r = std::min<long long>(eligible, best_visits);
      best.samples = (int32_t)std::min<long long>(r, 1LL << 30);
      best.epochs = (int32_t)((best_visits + r - 1) / r);
    }
    *out = best;
  });
}

extern "C" adainf_status adainf_model_average(adainf_model_t dst, const adainf_model_t* versions, int32_t n,
                                              adainf_stream_t stream) {
  return guard([&] {
    if (!dst || !versions || n < 1) throw InvalidError("model_average: need dst and n >= 1 versions");
    require_device();
    Model& d = dst->m;
    std::vector<const float*> srcs(n);
    for (int v = 0; v < n; ++v) {
      if (!versions[v]) throw InvalidError("model_average: null version");
      const Model& m = versions[v]->m;
      if (m.nparams != d.nparams || m.device != d.device)
        throw ShapeError("model_average: versions must share the architecture and device of dst");
      srcs[v] = m.params.as<float>();
    }
    cudaStream_t st = (cudaStream_t)stream;
    CK(cudaSetDevice(d.device));
    const long long cnt = d.nparams;
    const long long threads = (cnt + 3) / 4;
    const unsigned blocks = (unsigned)((threads + 255) / 256);
    if (n <= 16) {
      SrcTable t{};
      for (int v = 0; v < n; ++v) t.p[v] = srcs[v];
      ProfScope ps(PC_VERSION_AVG, st);
      average_kernel<<<blocks, 256, 0, st>>>(d.params.as<float>(), t, n, cnt);
      CK(cudaGetLastError());
    } else {
      const float** dsrc = nullptr;
      CK(cudaMallocAsync((void**)&dsrc, sizeof(float*) * n, st));
      CK(cudaMemcpyAsync(dsrc, srcs.data(), sizeof(float*) * n, cudaMemcpyHostToDevice, st));
      {
        ProfScope ps(PC_VERSION_AVG, st);
        average_kernel<<<blocks, 256, 0, st>>>(d.params.as<float>(), (const float* const*)dsrc, n, cnt);
        CK(cudaGetLastError());
      }
      CK(cudaFreeAsync(dsrc, st));
      CK(cudaStreamSynchronize(st));  // the host pointer table must outlive the copy
    }
    CK(cudaMemsetAsync(d.mom.p, 0, d.mom.bytes, st));  // reading Q23: momentum restarts from the averaged version
    d.refresh_shadows(st);
  });
}

extern "C" adainf_status adainf_dp_average(adainf_model_t mh, adainf_stream_t stream) {
  adainf_status s = guard([&] {
    if (!mh) throw InvalidError("null model");
    require_device();
    Model& m = mh->m;
    cudaStream_t st = (cudaStream_t)stream;
    CK(cudaSetDevice(m.device));
#ifdef ADAINF_WITH_NCCL
    if (m.comm && m.dp_world > 1) {
      ncclResult_t r = ncclAllReduce(m.params.p, m.params.p, (size_t)m.nparams, ncclFloat, ncclSum, m.comm, st);
      if (r != ncclSuccess) throw std::runtime_error(std::string("nccl: ") + ncclGetErrorString(r));
      scale_kernel<<<(unsigned)((m.nparams + 255) / 256), 256, 0, st>>>(m.params.as<float>(), m.nparams,
                                                                         (float)m.dp_world);
      CK(cudaGetLastError());
    }
#endif
    CK(cudaMemsetAsync(m.mom.p, 0, m.mom.bytes, st));
    m.refresh_shadows(st);
  });
  if (s == ADAINF_ERR_INVALID && std::string(adainf_last_error()).rfind("nccl", 0) == 0) return ADAINF_ERR_NCCL;
  return s;
}

extern "C" adainf_status adainf_mark_used(uint8_t* exclude, const int32_t* idx, const int32_t* count, int32_t n_static,
                                          adainf_stream_t stream) {
  return guard([&] {
    if (!exclude || !idx || n_static < 0) throw InvalidError("mark_used: bad arguments");
    require_device();
    if (n_static == 0) return;
    cudaStream_t st = (cudaStream_t)stream;
    ProfScope ps(PC_GATHER, st);
    mark_used_kernel<<<(n_static + 255) / 256, 256, 0, st>>>(exclude, idx, count, n_static);
    CK(cudaGetLastError());
  });
}

extern "C" adainf_status adainf_count_correct(const int32_t* pred, const int32_t* labels, int32_t n, int32_t* correct,
                                              adainf_stream_t stream) {
  return guard([&] {
    if (!pred || !labels || !correct || n < 0) throw InvalidError("count_correct: bad arguments");
    require_device();
    cudaStream_t st = (cudaStream_t)stream;
    ProfScope ps(PC_EXIT_LOSS, st);
    count_correct_kernel<<<1, 1024, 0, st>>>(pred, labels, n, correct);
    CK(cudaGetLastError());
  });
}

extern "C" adainf_status adainf_drift_should_stop(const uint64_t* results, int32_t n_steps, int32_t n,
                                                  int32_t* out_stop) {
  return guard([&] {
    if (!out_stop || n < 1 || n_steps < 0 || (n_steps > 0 && !results)) throw InvalidError("drift_should_stop: bad arguments");
    int stop = n_steps >= n;
    for (int i = n_steps - n; stop && i < n_steps; ++i) stop = results[i] == results[n_steps - 1];
    *out_stop = stop;
  });
}

// ------------------------------------------------------------------------------------------------
// NEXT-4 (P:118-134 Obs. 5-6): worst-case latency W(b) = per_batch_ms(b) * ceil(R / b)
namespace {
void check_profile(const adainf_latency_profile* p) {
  if (!p || p->n < 1 || !p->batch || !p->per_batch_ms) throw InvalidError("latency profile: empty");
  for (int i = 0; i < p->n; ++i)
    if (p->batch[i] < 1 || !(p->per_batch_ms[i] > 0.0) || !std::isfinite(p->per_batch_ms[i]))
      throw InvalidError("latency profile: entries need batch >= 1 and finite ms > 0");
}
double worst_ms(const adainf_latency_profile* p, int i, long long requests) {
  const long long nb = (requests + p->batch[i] - 1) / p->batch[i];
  return p->per_batch_ms[i] * (double)nb;
}
void pick_batch_impl(const adainf_latency_profile* p, long long requests, int32_t* batch, double* w) {
  check_profile(p);
  if (requests < 1) throw InvalidError("pick_batch: requests must be >= 1");
  int best = -1;
  double bw = 0.0;
  for (int i = 0; i < p->n; ++i) {
    const double wi = worst_ms(p, i, requests);
    if (best < 0 || wi < bw || (wi == bw && p->batch[i] < p->batch[best])) {
      best = i;
      bw = wi;
    }
  }
  *batch = p->batch[best];
  *w = bw;
}
}  // namespace

extern "C" adainf_status adainf_pick_batch(const adainf_latency_profile* profile, int64_t requests, int32_t* out_batch,
                                           double* out_worst_ms) {
  return guard([&] {
    if (!out_batch || !out_worst_ms) throw InvalidError("pick_batch: null output");
    pick_batch_impl(profile, requests, out_batch, out_worst_ms);
  });
}

extern "C" adainf_status adainf_pick_structure(int32_t n, const adainf_latency_profile* profiles, const double* accuracy,
                                               double a_min, int32_t has_retraining, int32_t full_index, int32_t batch0,
                                               int64_t requests, int32_t* out_structure, int32_t* out_batch,
                                               double* out_worst_ms) {
  return guard([&] {
    if (n < 1 || !profiles || !accuracy || !out_structure || !out_batch || !out_worst_ms)
      throw InvalidError("pick_structure: bad arguments");
    if (full_index < 0 || full_index >= n) throw InvalidError("pick_structure: full_index out of range");
    if (!std::isfinite(a_min)) throw InvalidError("pick_structure: a_min must be finite");
    int chosen = full_index;
    if (has_retraining) {
      double best_ms = 0.0;
      int best = -1;
      for (int s = 0; s < n; ++s) {
        check_profile(&profiles[s]);
        if (!std::isfinite(accuracy[s])) throw InvalidError("pick_structure: accuracy must be finite");
        if (accuracy[s] < a_min) continue;
        int at = -1;
        for (int i = 0; i < profiles[s].n; ++i)
          if (profiles[s].batch[i] == batch0) at = i;
        if (at < 0) throw InvalidError("pick_structure: batch0 missing from a structure's profile");
        const double ms = profiles[s].per_batch_ms[at];
        if (best < 0 || ms < best_ms) {
          best = s;
          best_ms = ms;
        }
      }
      if (best >= 0) chosen = best;
    }
    *out_structure = chosen;
    pick_batch_impl(&profiles[chosen], requests, out_batch, out_worst_ms);
  });
}

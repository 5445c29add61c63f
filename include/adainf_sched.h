/*
 * adainf_sched.h — incremental-retraining support of libadainf.so:
 * the spare-time split of a job's SLO, the retraining setting a time allocation affords, averaging of
 * concurrent model versions, and the disjoint-sample bookkeeping between jobs.
 *
 * P:L = line L of the paper text.  Readings Q.. are listed in DESIGN.md.
 * Host-only calls (adainf_time_split, adainf_retrain_setting) do plain double-precision arithmetic and
 * need no device; the device calls follow the conventions of adainf.h (stream-ordered, caller-owned
 * buffers, no CPU fallback).
 */
#ifndef ADAINF_SCHED_H_
#define ADAINF_SCHED_H_
#include "adainf.h"

#ifdef __cplusplus
extern "C" {
#endif

/* Spare time of job i and its split among retraining tasks (worked example P:51):
 *   T_r = L_s - sum_k l_k            (clamped at 0: an SLO shorter than the inference leaves no retraining)
 *   alloc_j = T_r * d_j / sum_j d_j  (impact degrees d_j >= 0; all zero -> every alloc_j = 0)
 * slo_ms: the job's latency SLO L_s.  infer_ms[n_infer]: inference-task latencies l_k (host).
 * impact[n_retrain]: impact degrees (host).  out_spare_ms: T_r.  out_alloc_ms[n_retrain] (host).
 * Errors: ADAINF_ERR_INVALID on NULL arrays with n > 0, negative counts, or negative / non-finite values. */
adainf_status adainf_time_split(double slo_ms, const double* infer_ms, int32_t n_infer, const double* impact,
                                int32_t n_retrain, double* out_spare_ms, double* out_alloc_ms);

/* Retraining setting for a time allocation ("number of retraining samples, retraining data batch size,
 * and the number of epochs"), from a per-step latency profile measured on this GPU (NEXT-4).  The paper picks
 * the setting with an accuracy regression it does not give; reading: maximise the sample visits
 * steps * batch that fit, steps = floor(alloc_ms / step_ms(batch)), ties -> larger batch; samples =
 * min(eligible, steps * batch) (distinct samples first), epochs = ceil(steps * batch / samples).
 * profile: n entries of (batch, measured ms per retrain_step at that batch), batch in 1..max_batch.
 * out: samples R (0 when nothing fits), batch b, steps, epochs and the estimated time steps * step_ms(b). */
typedef struct {
  int32_t n;
  const int32_t* batch;   /* host [n] */
  const double* step_ms;  /* host [n], > 0 */
} adainf_retrain_profile;
typedef struct {
  int32_t samples, batch, steps, epochs;
  double est_ms;
} adainf_retrain_plan;
adainf_status adainf_retrain_setting(double alloc_ms, const adainf_retrain_profile* profile, int64_t eligible,
                                     int32_t max_batch, adainf_retrain_plan* out);

/* Version averaging: dst's fp32 parameters become the unweighted mean of the versions' parameters
 * (reading Q23: summed in the given order in fp32, then divided by n), its momentum is reset to 0 and its bf16
 * GEMM shadows are refreshed.  versions[n] (n >= 1) may include dst; all models must share dst's architecture
 * (same parameter count) and device.  Stream-ordered; with n <= 16 it neither copies from the host nor
 * synchronizes (CUDA-graph capturable), with n > 16 it synchronizes the stream. */
adainf_status adainf_model_average(adainf_model_t dst, const adainf_model_t* versions, int32_t n,
                                   adainf_stream_t stream);

/* Cross-GPU version averaging: NCCL all-reduce (sum, then / world) of the fp32 parameters over the
 * communicator attached with adainf_dp_attach, momentum reset, shadows refreshed (P:241 across replicas).
 * world == 1: no-op apart from the momentum reset.  ADAINF_ERR_NCCL on NCCL failure. */
adainf_status adainf_dp_average(adainf_model_t m, adainf_stream_t stream);

/* Disjoint samples between jobs: exclude[idx[i]] = 1 for i < min(*count, n_static) (count: device
 * pointer or NULL -> n_static).  exclude: device [pool] bytes, idx: device int32.  Stream-ordered. */
adainf_status adainf_mark_used(uint8_t* exclude, const int32_t* idx, const int32_t* count, int32_t n_static,
                               adainf_stream_t stream);

/* Accuracy of predictions (NEXT-2, P:195 I'_m): *correct = #{i < n : pred[i] == labels[i]} (device int32
 * arrays, device int32 output).  Integer count, stream-ordered. */
adainf_status adainf_count_correct(const int32_t* pred, const int32_t* labels, int32_t n, int32_t* correct,
                                   adainf_stream_t stream);

/* Stop rule of the drift-impact detection ("gradually increases the value of S each time to repeat the
 * process. It stops when there is no change in the results for consecutive n (e.g., 4) times"; Table 2,
 * the impacted set settles at S = 9% and the process stops at S = 18%).  results[n_steps] holds the
 * impacted-model set found at each S so far (bit m = model m impacted).  *out_stop = 1 iff n_steps >= n and
 * the last n results are identical (the current one and the n - 1 before it), else 0.  Host-only. */
adainf_status adainf_drift_should_stop(const uint64_t* results, int32_t n_steps, int32_t n, int32_t* out_stop);

/* ---- NEXT-4: request batch size and early-exit structure from B200 latency profiles ------------------------
 * A latency profile holds the per-batch inference latency (ms; measured with CUDA events on the launching stream,
 * whole GPU) of one early-exit structure at each profiled request batch size (P:118 Obs. 5).
 * Worst-case latency of a job of `requests` requests at batch b ("the product of the per-batch
 * inference latency and the total number of batches"):  W(b) = per_batch_ms(b) * ceil(requests / b).
 * The GPU-space scaling regressions of §3.3.1 ([3], MPS space fractions) are prior art that B200 placement
 * replaces: the profiles are whole-GPU. Host arithmetic, no device. */
typedef struct {
  int32_t n;
  const int32_t* batch;        /* host [n], >= 1 */
  const double* per_batch_ms;  /* host [n], > 0  */
} adainf_latency_profile;

/* The batch with the lowest worst-case latency W(b) (ties -> the smaller batch), and W there.
 * Errors: ADAINF_ERR_INVALID on an empty / malformed profile or requests < 1. */
adainf_status adainf_pick_batch(const adainf_latency_profile* profile, int64_t requests, int32_t* out_batch,
                                double* out_worst_ms);

/* Early-exit structure of one inference task:
 *   - no retraining task for the model (has_retraining == 0): the full structure `full_index`;
 *   - else, among the structures whose accuracy >= a_min (the application's A_m), the one with the lowest
 *     per-batch latency at the job's current batch size batch0 (reading: §3.3.1 picked batch0 from the initial
 *     DAG's profile; ties -> lower index); none qualifies -> the full structure (the most accurate one);
 * then the batch size is re-picked for the chosen structure (Obs. 6: "adjusts the batch size ... given the
 * chosen early-exit structure") with adainf_pick_batch.
 * profiles[n_structures] (each must contain batch0), accuracy[n_structures] host.  Outputs: structure index,
 * batch size, worst-case latency W(batch) of the chosen structure.  ADAINF_ERR_INVALID on bad arguments. */
adainf_status adainf_pick_structure(int32_t n_structures, const adainf_latency_profile* profiles,
                                    const double* accuracy, double a_min, int32_t has_retraining,
                                    int32_t full_index, int32_t batch0, int64_t requests, int32_t* out_structure,
                                    int32_t* out_batch, double* out_worst_ms);

#ifdef __cplusplus
}
#endif
#endif

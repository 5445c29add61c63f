/*
 * adainf.h — C ABI of the B200-native AdaInf hot path (libadainf.so, sm_100a).
 *
 * What it computes (Shubha & Shen, "AdaInf", SIGCOMM'23; P:L = /root/reference/PAPER.md line L):
 *   - batched early-exit inference of an application's model DAG on a request batch
 *     (multi-model DAG P:29 / Fig. 1; early-exit structures P:96; one layer for the whole batch
 *     at once P:251)                                                     -> adainf_infer_dag
 *   - retraining-sample selection: PCA projection, cosine distance to the mean feature vector of the
 *     old training samples, the k most divergent new samples, never reusing samples
 *     used by other jobs                                         -> adainf_select_retrain
 *   - the incremental-retraining SGD step   -> adainf_retrain_step
 * Unspecified details follow the readings listed in DESIGN.md §Readings (Q1..Q27).
 *
 * Conventions
 *   - Tensors are NHWC, bf16 (uint16 bit patterns, RNE) unless stated; labels int32.
 *   - Pointers documented "device" must be CUDA device memory of the model's device; "host" pointers
 *     are ordinary host memory.  The caller owns every input/output buffer; the library owns
 *     parameters, momentum, bf16 shadows and workspaces (allocated at create, sized by max_batch).
 *   - Calls enqueue work on `stream` and return without synchronizing (except *_get_params /
 *     *_set_params / create / destroy, which synchronize).  Device-side counts are written to device
 *     memory; the library never reads them back on the hot path.
 *   - Errors: every call returns an adainf_status; 0 = OK.  Argument/shape validation is synchronous.
 *     CUDA errors map to ADAINF_ERR_CUDA with text in adainf_last_error() (thread-local).  No C++
 *     exception crosses the ABI.  NCCL errors map to ADAINF_ERR_NCCL.  A capacity overflow on the device
 *     (more routed crops than max_routed_per_dst) clamps deterministically in index order and reports the
 *     required count in n_routed (device: n_routed[e] > max_routed_per_dst is the overflow signal, valid
 *     under CUDA-graph replay too); the library also raises a mapped host flag that makes the next
 *     adainf_infer_dag or adainf_app_poll on the app return ADAINF_ERR_CAPACITY.  Graph replay does not run
 *     the host-side check of adainf_infer_dag: callers that replay a captured step poll with adainf_app_poll.
 *   - Thread safety: one handle = one thread + one stream at a time; distinct handles are independent.
 *   - There is no CPU fallback: without an sm_100 device every compute call returns
 *     ADAINF_ERR_UNSUPPORTED.
 */
#ifndef ADAINF_H_
#define ADAINF_H_
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef int32_t adainf_status;
enum {
  ADAINF_OK = 0,
  ADAINF_ERR_INVALID = -1,
  ADAINF_ERR_SHAPE = -2,
  ADAINF_ERR_CAPACITY = -3,
  ADAINF_ERR_OOM = -4,
  ADAINF_ERR_CUDA = -5,
  ADAINF_ERR_NCCL = -6,
  ADAINF_ERR_UNSUPPORTED = -7
};
const char* adainf_last_error(void);
int32_t adainf_version(void);

typedef struct adainf_model* adainf_model_t; /* opaque, library-owned */
typedef struct adainf_app* adainf_app_t;
typedef void* adainf_stream_t; /* cudaStream_t (NULL = legacy default stream) */

/* ---- Model description (the "exit-layer spec" of north_star) ----------------------------------
 * A model is a sequence of ops applied to the current tensor:
 *   CONV     kh x kw conv, stride, pad, cout; act 0 none / 1 ReLU / 2 leaky-ReLU(0.1) / 3 ReLU6; BN folded
 *            (reading Q10).  residual=1: add the innermost open BLOCK's shortcut before the act and
 *            close that block; residual=2: close it by concatenating [shortcut, conv] along channels, act
 *            applied to both parts (ShuffleNet stride-2 unit; output channels = shortcut's + cout).
 *            A CONV directly followed by DET_HEAD writes fp32 (no bf16 rounding).
 *   UPSAMPLE nearest-neighbour x`stride` of the current tensor (TinyYOLOv3's second scale); must feed a ROUTE.
 *   ROUTE    the current tensor becomes the output of op `kh` (absolute op index), concatenated along channels with
 *            op `kw`'s output when kw >= 0 (same H, W; only the first source may be an UPSAMPLE).  Models with
 *            UPSAMPLE / ROUTE are inference-only (detectors are not retrained): retraining them returns
 *            ADAINF_ERR_UNSUPPORTED.  A second DET_HEAD (same anchors per cell, classes, nms_iou) adds a scale: its
 *            grid cells follow the first head's in each frame's candidate order (det_table `cell` column), and NMS
 *            runs over both scales together (two-scale TinyYOLOv3, NEXT-3, reading Q18c).
 *   SHUFFLE  ShuffleNet channel shuffle of the current tensor with `groups` g (view (g, C/g), transpose,
 *            flatten; NEXT-3).  It must directly follow a non-depthwise CONV whose output has no other
 *            reader yet: the permutation is folded into that conv's output channel order (weights and bias),
 *            so no data moves (ADAINF_ERR_UNSUPPORTED otherwise).
 *   MAXPOOL  kh x kw window, stride, pad (padding = -inf).
 *   BLOCK    opens a residual block on the current tensor; cout > 0 -> 1x1 projection shortcut with
 *            `stride` (no activation); pool = 1 -> kh x kw average-pool shortcut (stride, pad; zero padding
 *            counted in the divisor, ShuffleNet); else identity.
 *   EXIT     early-exit head on the current tensor: GAP -> FC (num_classes) -> softmax (reading Q4);
 *            exit criterion max-softmax confidence >= tau (readings Q1/Q5); the last EXIT is the
 *            final classifier and is unconditional.  All EXITs of a model share num_classes.
 *            loss_weight w_k weights its cross-entropy in retraining (reading Q8).
 *   DET_HEAD TinyYOLOv3-style single-scale decode of the current fp32 tensor (reading Q18):
 *            `anchors` anchors x (5 + det_classes) channels, grid stride `grid_stride`, anchor_wh; with
 *            nms_iou > 0 the detections then go through greedy NMS per (frame, class): visited by score
 *            descending (ties -> lower candidate index), dropped if their fp32 IoU with a kept detection exceeds
 *            nms_iou; det_table / n_det / routing then list the kept detections (ascending candidate index).
 * Parameter layout (flat fp32, op order): CONV W[cout][kh][kw][cin / groups] then b[cout]; BLOCK with cout>0:
 * W[cout][1][1][cin] then b[cout]; EXIT: Wk[cin][num_classes] then bk[num_classes].            */
typedef enum {
  ADAINF_OP_CONV = 0,
  ADAINF_OP_MAXPOOL = 1,
  ADAINF_OP_BLOCK = 2,
  ADAINF_OP_EXIT = 3,
  ADAINF_OP_DET_HEAD = 4,
  ADAINF_OP_SHUFFLE = 5,
  ADAINF_OP_UPSAMPLE = 6,
  ADAINF_OP_ROUTE = 7
} adainf_op_kind;

typedef struct {
  int32_t kind; /* adainf_op_kind */
  int32_t kh, kw, stride, pad, cout;
  int32_t act;
  int32_t residual;
  int32_t num_classes;
  float loss_weight;
  int32_t anchors, det_classes, grid_stride;
  float anchor_wh[16];
  float nms_iou;      /* DET_HEAD: > 0 -> greedy per-(frame, class) NMS at this IoU threshold before routing
                         (NEXT-3, reading Q18b); 0 -> none */
  int32_t groups;     /* CONV: 0 / 1 dense; == cin == cout: depthwise 3x3 (MobileNetV2, NEXT-3); 1 < groups < cin:
                         grouped conv (ShuffleNet, NEXT-3; cin, cout multiples of groups), run as one tensor-core GEMM
                         over a block-diagonal weight.  Weights [cout][kh][kw][cin / groups].  SHUFFLE: g */
  int32_t pool;       /* BLOCK: 1 -> average-pool shortcut (kh, kw, stride, pad) */
} adainf_op;

typedef struct {
  int32_t in_h, in_w, in_c;   /* input tensor (NHWC); in_c need not be a multiple of 8 */
  int32_t max_batch;          /* capacity of inference rows AND of retraining samples per step */
  int32_t n_ops;
  const adainf_op* ops;       /* host, copied at create */
  float momentum, weight_decay; /* SGD (PyTorch semantics, reading Q9) */
  uint64_t seed;              /* LeCun-normal init when init_params == NULL */
  const float* init_params;   /* host, num_params fp32, or NULL */
  int32_t device;             /* CUDA device ordinal */
} adainf_model_spec;

adainf_status adainf_model_create(const adainf_model_spec* spec, adainf_model_t* out);
adainf_status adainf_model_destroy(adainf_model_t m);
adainf_status adainf_model_num_params(adainf_model_t m, int64_t* n);
adainf_status adainf_model_num_exits(adainf_model_t m, int32_t* n);
/* host <-> library fp32 master parameters (flat layout above); synchronizing; set_params also
 * refreshes the bf16 shadow and resets momentum to 0. */
adainf_status adainf_model_get_params(adainf_model_t m, float* host_dst, int64_t n);
adainf_status adainf_model_set_params(adainf_model_t m, const float* host_src, int64_t n);
/* device pointer to the flat fp32 gradient of the last retrain step (num_params floats), for
 * inspection and for callers that reduce gradients themselves. */
adainf_status adainf_model_grad_ptr(adainf_model_t m, float** dev_ptr);
/* host copy of that gradient (synchronizing) */
adainf_status adainf_model_get_grads(adainf_model_t m, float* host_dst, int64_t n);

/* ---- Application DAG (Fig. 1): root model first, routing edges between models ---------- */
typedef enum {
  ADAINF_ROUTE_DET_CROP = 0,    /* detector detections of class src_class -> crops for dst (Q19); at most one
                                   DET_CROP edge per (source, class): ADAINF_ERR_INVALID otherwise */
  ADAINF_ROUTE_CLASS_WHOLE = 1  /* whole input of samples predicted src_class -> dst (audio, Q24) */
} adainf_route_kind;

typedef struct {
  int32_t src_model, dst_model;
  int32_t kind;       /* adainf_route_kind */
  int32_t src_class;
  int32_t crop_h, crop_w; /* DET_CROP: must equal the dst model's in_h / in_w */
} adainf_edge;

typedef struct {
  int32_t n_models;
  const adainf_model_t* models; /* host array; models are borrowed, not owned */
  int32_t n_edges;
  const adainf_edge* edges;
  int32_t max_routed_per_dst;   /* capacity of each destination's routed batch */
} adainf_app_spec;

adainf_status adainf_app_create(const adainf_app_spec* spec, adainf_app_t* out);
adainf_status adainf_app_destroy(adainf_app_t app);
/* Synchronizes `stream`, then returns ADAINF_ERR_CAPACITY (and clears the flag) if any infer_dag since the last
 * check routed more crops than max_routed_per_dst; ADAINF_OK otherwise. */
adainf_status adainf_app_poll(adainf_app_t app, adainf_stream_t stream);

/* Per-model outputs of adainf_infer_dag (all DEVICE pointers, caller-allocated; any may be NULL).
 * Rows refer to the model's input rows in original order (root: the request batch; routed model:
 * its routed batch, in route order).  R = rows capacity (batch for the root, max_routed_per_dst
 * otherwise), E = number of exits, NC = num_classes, C0 = channels at exit 0.                   */
typedef struct {
  int8_t* exit_id;      /* [R] exit taken (0..E-1)                                       */
  int32_t* pred;        /* [R] argmax class at the exit taken (lowest index on ties)     */
  float* conf;          /* [R] max softmax probability at the exit taken                 */
  float* entropy;       /* [R] softmax entropy (nats) at the exit taken                  */
  float* logits;        /* [R * NC] logits at the exit taken                             */
  int32_t* exit_counts; /* [E] samples leaving at each exit                              */
  int32_t* surv_idx;    /* [(E-1) * R] row k: ascending original rows alive after exit k, count = R - sum(counts[0..k]) */
  float* embed;         /* [R * C0] exit-0 pooled features (selection embeddings, Q12)   */
  /* detector models (DET_HEAD): */
  int32_t* n_det;       /* [1] true number of detections (may exceed capacity)           */
  float* det_table;     /* [max_det * 9] frame, cell, anchor, class, score, x0, y0, x1, y1 (ascending candidate index) */
  int32_t max_det;      /* capacity of det_table rows                                    */
  int32_t* route_idx;   /* [n_out_edges * max_routed_per_dst] detection numbers per out-edge, ascending */
  int32_t* n_routed;    /* [n_out_edges] required count per out-edge (clamped use if > capacity) */
} adainf_model_out;

/* Early-exit inference of the whole DAG on one request batch (device bf16 NHWC, batch rows).
 * exit_thresholds (HOST) are concatenated in model order: an early-exit model with E exits takes
 * E-1 taus (tau_k <= 0: every sample exits at k; tau_k > 1: exit k disabled — the "full structure"
 * of P:229 is all taus > 1); a detector takes 1 tau_det; a model with 1 exit takes none.
 * outs[n_models].  Survivors are compacted on the device between stages (no host round trip). */
adainf_status adainf_infer_dag(adainf_app_t app, const void* batch_bf16_nhwc, int32_t batch,
                               const float* exit_thresholds, int32_t n_thresholds,
                               adainf_model_out* outs, adainf_stream_t stream);

/* ---- Retraining-sample selection ---------------------------------------
 * d_i = min_r (1 - cos(X_i W, ref_r W)) (uncentred projection, reading Q13/Q14; zero norm -> d = 1,
 * Q17); excluded samples are never selected; the k largest d are returned (ties -> lower index),
 * as an ascending index set with their distances (Q15); count = min(k, #eligible).               */
typedef struct {
  const void* X_bf16;     /* device [N * D] bf16 candidate features                    */
  int64_t N;
  int32_t D;              /* multiple of 8, <= 1024                                     */
  const void* W_bf16;     /* device [D * P] bf16 PCA basis (row-major), or NULL -> identity (P == D) */
  int32_t P;              /* 16..256, multiple of 16                                    */
  const float* ref;       /* device [M * D] fp32 reference rows (M = 1: mean of old samples) */
  int32_t M;              /* 1..4096 (M > 4: lanes stride the reference rows) */
  const uint8_t* exclude; /* device [N] nonzero = already used / in use, or NULL */
} adainf_select_in;

adainf_status adainf_select_retrain(const adainf_select_in* in, int32_t k, int32_t* out_idx,
                                    float* out_dist, int32_t* out_count, float* dist_all,
                                    adainf_stream_t stream);
/* out_idx, out_dist: device [k]; out_count: device [1]; dist_all: device [N] or NULL (excluded -> -1) */

/* Sharded selection: each of G shards of the candidate pool runs adainf_select_retrain on its
 * own rows with the same k; the G (out_dist, out_idx, out_count) lists are gathered (e.g. an NCCL all-gather) into
 * dist / idx [n_blocks * block_len] and block_count [n_blocks] (device; NULL -> every block full), and this call
 * returns the global top-k exactly as adainf_select_retrain on the whole pool would (ties -> lower GLOBAL index,
 * ascending output, count = min(k, #eligible)): local index i of block b is global index i * idx_mul + b * block_off
 * (contiguous shards: idx_mul = 1, block_off = rows per shard; index-mod-G shards: idx_mul = G,
 * block_off = 1), n_total = the global pool size.  Entries with dist < 0 or a global index outside [0, n_total) are
 * ignored.  Workspace n_total * 4 bytes, stream-ordered.  Errors: ADAINF_ERR_SHAPE on bad sizes. */
adainf_status adainf_select_merge(const float* dist, const int32_t* idx, const int32_t* block_count, int32_t n_blocks,
                                  int32_t block_len, int64_t idx_mul, int64_t block_off, int64_t n_total, int32_t k,
                                  int32_t* out_idx, float* out_dist, int32_t* out_count, adainf_stream_t stream);

/* ---- Incremental-retraining SGD step (readings Q8, Q9, Q22) -----------------------
 * One SGD-with-momentum step on n_local samples (device bf16 NHWC, labels device int32):
 * forward at full depth (all exits), loss L = (1/n_global) sum_n sum_k w_k CE(softmax(l_k(n)), y_n),
 * backward, (data-parallel: gradient all-reduce over the attached communicator), update
 * v <- mu v + (g + lambda w); w <- w - lr v (fp32 master), bf16 shadow refreshed.
 * stats_dev (device, optional): {loss (this replica's partial sum), grad_norm (of the reduced grad)}. */
typedef struct {
  float loss;
  float grad_norm;
} adainf_step_stats;

adainf_status adainf_retrain_step(adainf_model_t m, const void* samples_bf16_nhwc, const int32_t* labels,
                                  int32_t n_local, int64_t n_global, float lr,
                                  adainf_step_stats* stats_dev, adainf_stream_t stream);

/* The retraining step on rows of a device-resident window pool (samples collected in the previous
 * period), without materialising the batch.  pool: device bf16 NHWC [pool_rows][in_h][in_w][in_c];
 * pool_labels: device int32 [pool_rows]; row_idx: device int32 [n_local]; count: device int32 [1] or NULL.
 * Sample r of the step is pool row row_idx[r] with label pool_labels[row_idx[r]] when r < *count (count == NULL:
 * every r < n_local) and 0 <= row_idx[r] < pool_rows; any other row contributes nothing (zero input, no loss, no
 * gradient), so adainf_select_retrain's (out_idx, out_count) can be passed as is even when fewer than k samples
 * were eligible (exclusions accumulate) — the unwritten tail of out_idx is never read as a row.
 * A label outside [0, num_classes) likewise contributes nothing (here and in adainf_retrain_step).
 * The rows are read once, straight into the model's packed input layout.  Same semantics, results and errors
 * as adainf_retrain_step on the gathered batch; models whose input is used unpacked (in_c a multiple of 8)
 * return ADAINF_ERR_UNSUPPORTED; pool_rows <= 0 -> ADAINF_ERR_SHAPE. */
adainf_status adainf_retrain_step_rows(adainf_model_t m, const void* pool_bf16_nhwc, int64_t pool_rows,
                                       const int32_t* pool_labels, const int32_t* row_idx, const int32_t* count,
                                       int32_t n_local, int64_t n_global, float lr,
                                       adainf_step_stats* stats_dev, adainf_stream_t stream);

/* The two halves of a retraining step, for callers that reduce gradients themselves (SURVEY §8(c.1) step 13:
 * each replica's gradient scaled by 1/n_global, summed over replicas):
 *   adainf_retrain_grad[_rows]: forward + losses + backward only — the replica's gradient is left in the
 *     model's gradient buffer (adainf_model_grad_ptr), no all-reduce, no update; stats_dev->loss written.
 *   adainf_model_update: the update of adainf_retrain_step on whatever the gradient buffer holds (all-reduced
 *     first over an attached communicator), stats_dev->grad_norm written.  ADAINF_ERR_INVALID if no gradient
 *     was ever computed on the model.
 * adainf_retrain_step == adainf_retrain_grad + adainf_model_update, bit for bit. */
adainf_status adainf_retrain_grad(adainf_model_t m, const void* samples_bf16_nhwc, const int32_t* labels,
                                  int32_t n_local, int64_t n_global, adainf_step_stats* stats_dev,
                                  adainf_stream_t stream);
adainf_status adainf_retrain_grad_rows(adainf_model_t m, const void* pool_bf16_nhwc, int64_t pool_rows,
                                       const int32_t* pool_labels, const int32_t* row_idx, const int32_t* count,
                                       int32_t n_local, int64_t n_global, adainf_step_stats* stats_dev,
                                       adainf_stream_t stream);
adainf_status adainf_model_update(adainf_model_t m, float lr, adainf_step_stats* stats_dev, adainf_stream_t stream);

/* Assemble the retraining batch from the device-resident window pool (samples collected in the
 * previous period): dst[r] = src[idx[r]] for r < min(*count, n) (count device int or NULL -> n);
 * rows of row_bytes bytes (multiple of 4; 16 for 128-bit copies).  Pairs with adainf_select_retrain's out_idx/out_count. */
adainf_status adainf_gather_rows(const void* src, const int32_t* idx, const int32_t* count, int32_t n,
                                 int64_t row_bytes, void* dst, adainf_stream_t stream);

/* Data-parallel retraining: attach an NCCL communicator created from a 128-byte
 * ncclUniqueId (broadcast by the caller, e.g. over torch.distributed); retrain_step then sums the
 * replicas' gradients (each scaled by 1/n_global) with ncclAllReduce before the update, so all
 * replicas stay bit-identical.  world == 1 detaches. */
adainf_status adainf_dp_attach(adainf_model_t m, const void* nccl_unique_id, int32_t rank, int32_t world);
adainf_status adainf_nccl_unique_id(void* out128);

#ifdef __cplusplus
}
#endif
#endif /* ADAINF_H_ */

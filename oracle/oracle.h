/*
 * AdaInf hot-path ORACLE — TEST INFRASTRUCTURE ONLY.
 *
 * A plain, slow, obviously-correct CPU implementation of what the AdaInf GPU hot path computes
 * (Shubha & Shen, SIGCOMM'23; `PAPER.md` line numbers cited as P:L).  Only tests/,
 * __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference leg may load it.  It shares
 * no code, header, helper or constant generator with the CUDA path
 * (paper_conf_sigcomm_shubhas23_b200/csrc); neither includes the other.
 *
 * Every floating-point sum is accumulated in fp64 (exact bf16 x bf16 products) and cast to fp32 at
 * the storage points listed in DESIGN.md "Numerics contract"; bf16 rounding is round-to-nearest-even
 * on the fp32 bit pattern.  Tensors are NHWC, one sample at a time, held as float arrays whose values
 * are bf16-representable where the GPU stores bf16.
 *
 * Pins (tests/test_oracle_*.py): brute-force / closed-form / torch-fp64 / finite-difference checks
 * listed per function below and in DESIGN.md §Oracle pins.
 */
#pragma once
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* Op kinds of the oracle's own model description (same meaning as the ABI's, declared separately). */
enum { OR_CONV = 0, OR_MAXPOOL = 1, OR_BLOCK = 2, OR_EXIT = 3, OR_DET_HEAD = 4, OR_SHUFFLE = 5, OR_UPSAMPLE = 6,
       OR_ROUTE = 7 };
/* UPSAMPLE: nearest-neighbour x`stride` of the current tensor.  ROUTE (TinyYOLOv3's two-scale branch): the current
 * tensor becomes the output of op `kh` (absolute op index), concatenated along channels with the output of op `kw`
 * when kw >= 0 (same H, W).  Models with UPSAMPLE / ROUTE are inference-only (the detector is not retrained).
 * Several DET_HEADs may appear; det_raw then holds, per frame, each head's G*G*(A*(5+nc)) values in op order. */

typedef struct {
  int32_t kind;
  int32_t kh, kw, stride, pad, cout; /* CONV; MAXPOOL uses kh,kw,stride,pad; BLOCK: cout>0 -> 1x1 projection shortcut with `stride` */
  int32_t act;                       /* CONV: 0 none, 1 ReLU, 2 leaky-ReLU(0.1), 3 ReLU6 (MobileNetV2) */
  int32_t residual;                  /* CONV: 1 = add the innermost open BLOCK's shortcut before act; 2 = concat
                                        [shortcut, conv] along channels, act applied to both parts (ShuffleNet
                                        stride-2 unit); either closes the block */
  int32_t num_classes;               /* EXIT */
  float loss_weight;                 /* EXIT */
  int32_t anchors, det_classes, grid_stride; /* DET_HEAD */
  float anchor_wh[16];               /* DET_HEAD: (w,h) per anchor, pixels */
  int32_t groups;                    /* CONV: channel groups (1 dense, = Cin = Cout depthwise); 0 is read as 1;
                                        SHUFFLE: g of the channel shuffle (ShuffleNet: view (g, C/g) -> transpose) */
  int32_t pool;                      /* BLOCK with cout == 0: 1 = shortcut is an average pool kh x kw / stride / pad
                                        of the block input, zero padding counted in the divisor (ShuffleNet) */
} or_op;

typedef struct {
  int32_t in_h, in_w, in_c;
  int32_t n_ops;
  const or_op* ops;
} or_model;

/* --- primitives (each pinned on its own) ------------------------------------------------------ */
float or_bf16(float x);                                  /* RNE to bf16, returned as float */
void or_bf16_array(const float* x, float* y, int64_t n);

/* conv forward for ONE sample, NHWC: acc[ho][wo][co] = sum x*w (fp64) -> fp32 (no epilogue).
 * x: H*W*C, w: Co*KH*KW*C (values used as given). Pinned: brute force + torch conv2d fp64. */
void or_conv_acc(const float* x, int H, int W, int C, const float* w, int Co, int KH, int KW, int s,
                 int p, float* acc, int* Ho, int* Wo);
void or_maxpool(const float* x, int H, int W, int C, int K, int s, int p, float* y, int* Ho, int* Wo);
/* exit head on one sample: pooled[C], logits[ncls], conf, entropy, pred (P:96 exit head, SURVEY c.1 step 3) */
void or_exit_head(const float* fmap, int H, int W, int C, const float* Wk, const float* bk, int ncls,
                  float* pooled, float* logits, float* conf, float* entropy, int32_t* pred);
/* softmax confidence / entropy / argmax of a logit vector */
void or_softmax_stats(const float* logits, int ncls, float* conf, float* entropy, int32_t* pred);

/* --- model-level ------------------------------------------------------------------------------ */
int64_t or_num_params(const or_model* m);
int32_t or_num_exits(const or_model* m);
/* output (H,W,C) of the op at index op_idx (C of the EXIT / DET input) */
int or_tensor_shape(const or_model* m, int op_idx, int* H, int* W, int* C);

/* Full-depth forward of B samples (all exits evaluated, no early exit).
 * x: B*H*W*C bf16 values as float.  Outputs (any may be NULL):
 *   conf, ent: B*E; pred: B*E; logits: B*E*ncls (all exits share ncls);
 *   pooled0: B*C0 (exit-0 pooled features); det_raw: B*G*G*(A*(5+nc)) fp32 (DET_HEAD input).
 * OpenMP over samples.  Returns 0 on success. */
int or_forward(const or_model* m, const float* params, const float* x, int B, float* conf, float* ent,
               int32_t* pred, float* logits, float* pooled0, float* det_raw);

/* Exit rule + stable compaction (SURVEY c.1 steps 4-5), brute force.
 * conf: B*E (all exits), tau: E-1 thresholds. exit_id[B]; surv: (E-1)*B, row k = ascending original
 * indices still alive after exit k; counts[E]. */
void or_exit_assign(const float* conf, int B, int E, const float* tau, int8_t* exit_id, int32_t* surv,
                    int32_t* counts);

/* Detector decode (SURVEY c.1 step 6; TinyYOLOv3-style): det_raw B*G*G*(A*(5+NC)) fp32.
 * Writes up to max_det rows of det_table (9 floats: frame, cell, anchor, class, score, x0,y0,x1,y1)
 * in ascending linear index; returns the true number of detections. */
int32_t or_detect(const float* det_raw, int B, int G, int A, int NC, const float* anchor_wh, int stride,
                  int img_w, int img_h, float tau_det, float* det_table, int32_t max_det);
/* Greedy non-maximum suppression (NEXT-3; reading Q18b): det rows as written by or_detect (ascending
 * candidate index).  Within each (frame, class), detections are visited by score descending (ties -> lower row);
 * a detection is kept unless its IoU with an already kept one exceeds iou_thr.  IoU in fp32, every op rounded:
 *   iw = max(0, min(x1a, x1b) - max(x0a, x0b)), ih likewise, inter = iw * ih,
 *   union = (x1a - x0a) * (y1a - y0a) + (x1b - x0b) * (y1b - y0b) - inter   (area_a + area_b, then - inter),
 *   iou = union > 0 ? inter / union : 0.
 * keep[n] out (0/1); returns the number kept. */
int32_t or_nms(const float* det, int32_t n, float iou_thr, uint8_t* keep);
float or_iou(const float* a, const float* b); /* boxes x0, y0, x1, y1 */

/* Bilinear crop-resize of one box from a bf16 (as float) NHWC frame -> crop_h*crop_w*C, bf16-rounded
 * (SURVEY c.1 step 7 / Q19). */
void or_crop(const float* frame, int H, int W, int C, float x0, float y0, float x1, float y1, int crop_h,
             int crop_w, float* out);

/* Retraining-sample selection (SURVEY c.1 step 8).
 * X: N*D (bf16 values as float), Wp: D*P (NULL -> identity, requires P == D), ref: M*D fp32,
 * exclude: N bytes or NULL.  dist[N] out (all samples, excluded get -1), out_idx/out_dist: k entries
 * ascending index; returns count = min(k, #eligible). */
int32_t or_select(const float* X, int64_t N, int D, const float* Wp, int P, const float* ref, int M,
                  const uint8_t* exclude, int32_t k, float* dist, int32_t* out_idx, float* out_dist);

/* One incremental-retraining SGD step (SURVEY c.1 steps 9-12) on n samples whose
 * gradients are scaled by 1/n_global.  params/momentum updated in place (fp32).
 * grads (optional, num_params) receives the gradient; loss (optional) the summed loss / n_global. */
int or_retrain_step(const or_model* m, float* params, float* momentum, const float* x,
                    const int32_t* labels, int n, int64_t n_global, float lr, float mu, float wd,
                    float* grads, double* loss);
/* loss only (fp64 forward without bf16 rounding when exact==1) for finite-difference pins */
double or_loss(const or_model* m, const double* params, const float* x, const int32_t* labels, int n,
               int64_t n_global, int exact);
/* gradient with exact (no bf16) arithmetic, for finite-difference pins */
int or_grad_exact(const or_model* m, const double* params, const float* x, const int32_t* labels, int n,
                  int64_t n_global, double* grads);

void or_set_threads(int n);
int or_get_threads(void);

#ifdef __cplusplus
}
#endif

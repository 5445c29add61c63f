// Declarations of the CUDA-core kernels' host launchers (HBM / latency-bound steps of the hot path).
#pragma once
#include "prof.h"
#include <cuda_runtime.h>
#include <stdint.h>

#include "runtime.h"

namespace adainf {

// pad channels Cin -> Cpad (zeros), optional row map / device count (a1 ingest)
void launch_pack_input(const bf16* x, const int* map, const int* count, int n_static, int H, int W, int Cin, int Cpad,
                       bf16* y, cudaStream_t st);

// argmax code of a window whose ReLU producer output is not > 0: routes no gradient (act' = 0)
constexpr uint8_t AMAX_MASKED = 0xFF;
// maxpool fwd (NHWC bf16); optional input map; optional argmax offsets (uint8, kh*K+kw of the FIRST maximum)
// for backward; fold_relu (producer activation ReLU) stores AMAX_MASKED where the window max is not > 0
void launch_maxpool_fwd(const bf16* x, const int* map, const int* count, int n_static, int H, int W, int C, int K,
                        int s, int p, int Ho, int Wo, bf16* y, uint8_t* argmax, int fold_relu, cudaStream_t st);
// maxpool bwd fused with the producer's activation mask: dz = bf16(sum_windows dT * [first argmax]) * act'(y).
// act == 1 (ReLU): the mask is folded into the argmax codes (AMAX_MASKED) and `pooled` is not read;
// otherwise the mask is taken from the pooled output P (= y at the selected position)
void launch_maxpool_bwd(const bf16* dT, const uint8_t* argmax, const bf16* pooled, int act, int n, int H, int W, int C,
                        int K, int s, int p, int Ho, int Wo, bf16* dz, cudaStream_t st);

// ---- depthwise conv (groups == channels; NEXT-3 MobileNetV2), dwconv.cu ----
struct DwArgs {
  const bf16* x;        // fwd / wgrad: input [n][H][W][C]; dgrad: dZ [n][Ho][Wo][C]
  const bf16* dz;       // wgrad: dZ
  const int* map;       // fwd: input row map (inference stages) or nullptr
  const int* count;     // fwd: device row count or nullptr
  int n_static;
  int H, W, C, Ho, Wo, KH, KW, s, p;
  const bf16* w;        // [taps][C] (dw_prep)
  const float* bias;    // fwd
  int act;              // fwd
  const float* bcast;   // dgrad: exit broadcast [n][C] or nullptr
  const bf16* sc;       // dgrad: shortcut term [n][H][W][C] or nullptr
  const bf16* yact;     // dgrad: producer output for the activation mask, or nullptr
  int mask_act;
  bf16* y;              // fwd: output; dgrad: dX
};
bool dw_ok(const ConvGeom& g, int groups);
void dw_prep(const bf16* shadow, int ldb, int C, int taps, bf16* wdw, cudaStream_t st);
void dw_fwd(const DwArgs& a, cudaStream_t st);
void dw_dgrad(const DwArgs& a, cudaStream_t st);
size_t dw_wgrad_ws_bytes(const ConvGeom& g, int n);
void dw_wgrad(const DwArgs& a, float* ws, size_t ws_bytes, float* dw, float* db, cudaStream_t st);

// ---- ShuffleNet pieces (NEXT-3), shuffle.cu: channel-shuffle fold (permuted bias), grouped weight-gradient gather,
// stride-2 unit's average-pool shortcut + concat
struct AvgPoolArgs {
  const bf16* x;       // [n][H][W][C] (rows through map)
  const int* map;
  const int* count;
  int n_static, H, W, C, K, s, p, Ho, Wo;
  bf16* y;             // [n][Ho][Wo][C]
};
void permute_bias(const float* b, int Cout, int g, float* out, cudaStream_t st);
void grouped_wgrad_gather(const float* dense, const float* dbs, int Cout, int taps, int Cin, int groups, int shuf_g,
                          float* dw, float* db, cudaStream_t st);
void avgpool_fwd(const AvgPoolArgs& a, cudaStream_t st);
void concat_fwd(const bf16* S, const bf16* Y, const int* count, int n_static, int HW, int Cs, int Co, int act, bf16* Z,
                cudaStream_t st);
// TinyYOLOv3 ROUTE of two sources: [A upsampled by f (nearest), B] along channels (inference)
void route_concat(const bf16* A, int HA, int WA, int CA, int f, const bf16* B, int CB, const int* count, int n_static,
                  int H, int W, bf16* out, cudaStream_t st);
void concat_bwd(const bf16* dZ, int n, int H, int W, int Cs, int Co, int K, int s, int p, int Ho, int Wo, bf16* dY,
                bf16* sc, cudaStream_t st);

// ---- 3x3/1 conv + bias + act + 2x2/2 max-pool in one tensor-core kernel (inference), conv3pool.cu: the detector's
// few-channel early layers; first = the model's first layer on the space-to-depth packed input (<= 4 channels)
bool conv3_pool_ok(const ConvGeom& g, bool first, int cin_real, int pk, int ps, int pp);
size_t conv3_pool_wexp_bytes(const ConvGeom& g, bool first);
void conv3_pool(const ConvGeom& g, bool first, const bf16* x, const int* count, int n_static, const bf16* shadow,
                int ldb, int cin_real, const float* bias, int act, bf16* wexp, bf16* y, cudaStream_t st);

// ---- exit head (K4) ----
struct ExitHeadArgs {
  const bf16* fmap;     // dense [rows][HW][C]
  const int* count;     // device rows count (nullptr -> n_static)
  int n_static;
  int HW, C, ncls;
  const float* Wk;      // [C][ncls]
  const float* bk;
  float tau;            // exit iff conf >= tau (ignored if is_final)
  int is_final;
  const int* orig;      // dense row -> original row (nullptr = identity)
  // outputs scattered to original rows (written only when the row exits here)
  int8_t* exit_id;
  int exit_index;
  int32_t* pred;
  float* conf;
  float* entropy;
  float* logits;        // [R][ncls]
  float* embed;         // exit-0 pooled features [R][C], all rows
  uint8_t* alive;       // [rows] 1 = survives past this exit
  // training mode: all rows, saved pooled / logits
  float* pooled_save;   // [rows][C]
  float* logits_save;   // [rows][ncls]
};
void launch_exit_head(const ExitHeadArgs& a, cudaStream_t st, int prof_class = PC_EXIT_HEAD);

// K4 + K5 fused: exit head + decision + decoupled look-back compaction (+ survivor row copy when src != nullptr);
// ws: exit_fused_ws_bytes(max_batch) of device scratch (zeroed by the launcher)
size_t exit_fused_ws_bytes(int max_batch);
void launch_exit_fused(const ExitHeadArgs& h, unsigned* ws, int* pos_next, int* orig_next, int* count_next,
                       int32_t* counts_out, int32_t* surv_out, int32_t* last_count_out, int last_index,
                       const bf16* src, bf16* dense_next, long long row_elems, cudaStream_t st);

// stable compaction of alive rows: pos_next[j'] = j, orig_next[j'] = orig[j]; count_next; counts[k] += exited;
// surv_out (optional, user): ascending original rows
void launch_compact(const uint8_t* alive, const int* count, int n_static, const int* orig, int* pos_next,
                    int* orig_next, int* count_next, int32_t* counts_out, int exit_index, int32_t* surv_out,
                    int32_t* last_count_out, int last_index, cudaStream_t st);

// ---- retraining (K8, K9, K10) ----
// per exit: dl = w (softmax - onehot) / n_global ; loss_rows[n] += w CE
void launch_sanitize_rows(const int32_t* pool_labels, const int32_t* idx, const int32_t* count, int n,
                          long long pool_rows, int32_t* map, int32_t* labels, cudaStream_t st);
void launch_exit_loss(const float* logits, const int32_t* labels, int n, int ncls, float w, float inv_n, float* dl,
                      float* loss_rows, int accumulate, cudaStream_t st);
// head grads: dW[c][j] = sum_n pooled[n][c] dl[n][j]; db[j] = sum_n dl[n][j]; bcast[n][c] = (sum_j dl W[c][j]) / HW
// exit-head gradients: dW = pooled^T dl, db = colsum(dl) (deterministic split over samples, partials in `ws`
// of head_grads_ws_bytes), bcast = dl Wk^T / HW (the GAP broadcast added to the exit tensor's gradient)
size_t head_grads_ws_bytes(int n, int C, int ncls);
void launch_head_grads(const float* pooled, const float* dl, const float* Wk, int n, int C, int ncls, int HW,
                       float* dW, float* db, float* bcast, float* ws, cudaStream_t st);
// dz = bf16((bcast[n][c] + sc) * act'(y))
void launch_grad_finalize(const float* bcast, const bf16* sc, const bf16* yact, int act, int n, int HW, int C,
                          bf16* dz, cudaStream_t st);
// fixed-order sum of a float vector into out[0] (single block)
void launch_sum(const float* x, int n, float* out, float scale, cudaStream_t st);
// *p = v, stream-ordered (no pageable host source, so it can be captured into a CUDA graph)
void launch_fill_i32(int32_t* p, int32_t v, cudaStream_t st);

struct SgdSeg {
  long long off;       // flat offset
  long long count;
  bf16* shadow;        // conv weight shadow [Cout][ldb] or nullptr
  int taps, cin, cin_pad, ldb;
  int cog;             // grouped conv: output channels per group (weight (co, tap, ci) -> column tap*cin_pad +
                       // (co / cog) * cin + ci of the block-diagonal shadow); 0 = dense
  int shuf_g, cout;    // folded channel shuffle: master row co -> shadow row (co % (cout/shuf_g)) * shuf_g + co / ...
};
// elements per sgd_kernel block (the host partitions the parameter segments into units of this size)
constexpr int SGD_BLOCK_ELEMS = 256 * 4 * 2;
void launch_sgd(float* w, float* v, const float* g, long long n, float lr, float mu, float wd, const SgdSeg* segs_dev,
                int nseg, const int* block_seg_dev, const long long* block_start_dev, int nblocks, float* sq_partial,
                cudaStream_t st);
void launch_shadow_pack(const float* w, const SgdSeg* segs_dev, int nseg, cudaStream_t st);
void launch_gather_rows(const void* src, const int32_t* idx, const int32_t* count, int n_static, long long row_bytes,
                        void* dst, cudaStream_t st, int prof_class = PC_GATHER);

}  // namespace adainf

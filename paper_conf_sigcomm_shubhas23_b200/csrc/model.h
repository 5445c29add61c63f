// Model / app runtime of libadainf.so: the model IR resolved into tensors + GEMM/pool nodes + exit heads,
// device-resident parameters (fp32 master, momentum, bf16 GEMM-ready shadows) and workspaces sized for
// max_batch at create time, and the stream-ordered orchestration of inference (stage by stage with
// device-side survivor counts) and of the retraining step (forward, losses, reverse walk, update).
#pragma once
#include <cuda_runtime.h>

#include <memory>
#include <string>
#include <vector>

#include "../../include/adainf.h"
#include "kernels.cuh"
#include "runtime.h"

#ifdef ADAINF_WITH_NCCL
#include <nccl.h>
#endif

namespace adainf {

// N_AVGPOOL: a BLOCK's average-pool shortcut; N_CONCAT: [shortcut, conv] join closing such a block (ShuffleNet)
// N_ROUTE: TinyYOLOv3 route of two sources (concat, the first optionally read through an upsampling factor)
enum NodeKind { N_CONV = 0, N_POOL = 1, N_PROJ = 2, N_AVGPOOL = 3, N_CONCAT = 4, N_ROUTE = 5 };

struct DevBuf {  // owning device allocation
  void* p = nullptr;
  size_t bytes = 0;
  DevBuf() = default;
  DevBuf(const DevBuf&) = delete;  // owning: a copy would free the allocation twice
  DevBuf& operator=(const DevBuf&) = delete;
  DevBuf(DevBuf&& o) noexcept : p(o.p), bytes(o.bytes) { o.p = nullptr; o.bytes = 0; }
  DevBuf& operator=(DevBuf&& o) noexcept {
    std::swap(p, o.p);
    std::swap(bytes, o.bytes);
    return *this;
  }
  void alloc(size_t b);
  void zero(cudaStream_t st = 0);
  ~DevBuf();
  template <class T>
  T* as() const { return (T*)p; }
};

struct TensorRt {
  int H, W, C;
  int producer = -1;  // node index, -1 = model input
  int act = 0;        // activation of the producing conv (mask for gradients)
  int stage = 0;
  bool f32 = false;
  bf16* buf = nullptr;   // activations (max_batch rows)
  DevBuf own;
  // training
  bf16* grad = nullptr;  // stored gradient (dZ of a conv output / dT of a pool output)
  DevBuf own_grad;
  int primary = -1;      // node reading it as main input (conv or pool)
  int proj = -1;         // projection node reading it
  int res_of = -1;       // conv node adding it as identity shortcut
  int exit_k = -1;       // exit attached
  int avgpool = -1;      // N_AVGPOOL node reading it as a block input (its shortcut term comes from there)
  bool routed = false;   // read again by a ROUTE (inference-only detectors): its producer may not fuse it away
  int alias_of = -1;     // single-source ROUTE: the same buffer as that tensor
  int up_src = -1, up = 1;  // UPSAMPLE: virtual (never materialised) nearest x`up` view of tensor up_src
  size_t row_elems() const { return (size_t)H * W * C; }
};

struct NodeRt {
  int kind;
  int op;
  int in, out, res = -1;
  int stage;
  ConvGeom g{};
  int act = 0;
  int cin_real = 0;            // input channels per group of the weights (first layer: the unpadded in_c)
  int groups = 1;              // > 1: depthwise (groups == Cin == Cout, dwconv.cu) or, with gdense, grouped
  bool gdense = false;         // grouped conv as one dense GEMM over a block-diagonal shadow (shuffle.cu)
  int shuf_g = 0;              // > 1: channel shuffle folded into the output channel order (shadow rows, bias)
  DevBuf bias_perm;            // shuf_g: bias in the physical (shuffled) order, rebuilt every forward
  int fuse_pool = -1;          // inference: the 2x2/2 max-pool node computed by this conv's conv3_pool kernel
  DevBuf wexp;                 // its expanded weights (conv3pool.cu), rebuilt from the shadow every forward
  DevBuf pool_sc;              // N_AVGPOOL (training): shortcut term of the block input, bf16 [max_batch][H][W][C]
  DevBuf wdw;                  // depthwise weights [taps][C] bf16, rebuilt from the shadow every forward
  long long w_off = 0, b_off = 0;
  int ldb = 0;
  DevBuf shadow;  // bf16 [Cout][ldb]
  bool fp32_out = false;
  int pk = 0, ps = 0, pp = 0;  // pool
  DevBuf argmax;               // pool (training)
  DevBuf proj_dx;              // proj (training): dgrad into the block input, added as shortcut term
  bool proj_compact = false;   // proj: proj_dx stored on the output grid (only the (0,0) phase is nonzero),
                               // consumed by the sibling's sub-pixel dgrad epilogue
  bool sp = false;             // stride-2 3x3 conv whose dgrad runs as one sub-pixel GEMM (MODE_DGRAD_SP)
  DevBuf wsp;                  // its packed sub-pixel weights bf16 [4*Cin][4*Cout]
};

struct ExitRt {
  int op, tensor, ncls, stage;
  float lw;
  long long w_off, b_off;
  DevBuf pooled, logits, dl, bcast;  // training
  // inference: the survivors' rows of this exit's tensor gathered densely after the compaction, so the next
  // stage's convolutions read a dense source (TMA im2col operands) instead of gathering through the row map
  DevBuf dense_next;
};

struct DetRt {
  int tensor = -1;
  int tensor2 = -1, stride2 = 0;  // second head (two-scale TinyYOLOv3, NEXT-3)
  float anchor_wh2[16];
  int anchors = 0, classes = 0, stride = 0;
  float anchor_wh[16];
  float nms_iou = 0.f;  // > 0: greedy NMS before routing (NEXT-3)
};

struct Model {
  int device = 0;
  int in_h, in_w, in_c, cin_pad, max_batch;
  bool pack = false;
  std::vector<adainf_op> ops;
  std::vector<TensorRt> T;
  std::vector<NodeRt> nodes;
  std::vector<int> op_node;  // op index -> node index (or -1)
  std::vector<ExitRt> exits;
  DetRt det;
  int nstages = 1;
  long long nparams = 0;
  float momentum = 0.9f, weight_decay = 0.f;

  DevBuf params, mom, grads;
  DevBuf packed_in;           // [max_batch][H][W][cin_pad], or S2D [max_batch][H/2][W/2][16] (stem_s2d)
  // ResNet stem (7x7/2 conv + ReLU + 3x3/2 max-pool) run by the fused space-to-depth kernels (stem.cuh)
  bool stem_s2d = false;
  int stem_pool = -1;         // node index of the pool fused into the stem
  DevBuf stem_wprep;          // per-tap bf16 weights [16][2][64][8], rebuilt from the shadow every forward
  bool inference_only = false;  // UPSAMPLE / ROUTE present (detectors are not retrained)
  bool first_s2d = false;     // inference: the first conv runs fused with its pool on the s2d-packed input (conv3pool.cu)
  // inference stage bookkeeping
  DevBuf pos, orig, counts, alive;  // pos/orig: [nstages][max_batch] int; counts [nstages] int
  DevBuf exit_ws;                   // fused exit kernel: ticket + look-back status words
  // training
  bool train_ready = false;
  DevBuf wgrad_ws, loss_rows, stats_tmp, sq_partial;
  DevBuf gw_dense;  // grouped / shuffled convs: dense weight-gradient scratch [Cout][taps][Cin] + [Cout]
  size_t wgrad_ws_bytes = 0;
  DevBuf sgd_segs, sgd_block_seg, sgd_block_start;
  int sgd_nblocks = 0, sgd_nseg = 0;
  int n_out_det_edges = 0;
#ifdef ADAINF_WITH_NCCL
  ncclComm_t comm = nullptr;
#endif
  int dp_world = 1, dp_rank = 0;

  void build(const adainf_model_spec& s);
  void refresh_shadows(cudaStream_t st);
  void ingest(const bf16* x, const int* map, const int* count, int n_static, cudaStream_t st, bool s2d = false);
  void ensure_training();
  // inference of one (possibly routed / device-counted) batch
  void infer(const bf16* x, const int* in_map, const int* in_count, int n_static, const float* taus,
             const adainf_model_out& out, cudaStream_t st, bool x_padded = false);
  void train_step(const bf16* x, const int32_t* labels, int n, long long n_global, float lr,
                  adainf_step_stats* stats, cudaStream_t st, bool update = true);
  // the same step on pool rows idx[0..n) (packed straight from the pool; labels gathered from pool_labels);
  // rows r >= *count (count device, nullable) and indices outside [0, pool_rows) contribute nothing
  void train_step_rows(const bf16* pool, long long pool_rows, const int32_t* pool_labels, const int32_t* idx,
                       const int32_t* count, int n, long long n_global, float lr, adainf_step_stats* stats,
                       cudaStream_t st, bool update = true);
  DevBuf row_labels, row_map;  // sanitised labels / pool rows of train_step_rows
  // forward + losses + backward: the gradient of this replica's samples (scaled by 1/n_global) in `grads`
  void train_grad_impl(const bf16* x, const int32_t* row_map, const int32_t* labels, int n, long long n_global,
                       adainf_step_stats* stats, cudaStream_t st);
  // (data-parallel: gradient all-reduce over the attached communicator) + fused SGD / momentum / shadow refresh
  void update_impl(float lr, adainf_step_stats* stats, cudaStream_t st);

 private:
  void forward_nodes(const bf16* x0, const int* map0, const int* count0, int n_static, bool train, const float* taus,
                     const adainf_model_out* out, cudaStream_t st, bool in_s2d = false);
};

struct App {
  std::vector<Model*> models;
  std::vector<adainf_edge> edges;
  int max_routed = 0;
};

// detector decode / routing / crop (detect.cu)
struct DetRouteArgs {
  const float* raw;  // [B][G][G][A*(5+NC)]
  const int* count;  // frames count (device) or nullptr
  int n_static, G, A, NC, stride, img_w, img_h;
  float anchor_wh[16];
  // optional second head (two-scale TinyYOLOv3, NEXT-3): [B][G2][G2][A*(5+NC)], its cells follow the first
  // head's G*G cells of the same frame in the candidate order
  const float* raw2;
  int G2, stride2;
  float anchor_wh2[16];
  float tau;
  int n_edges;
  int edge_class[8];
  int cap;
  float* det_table;      // internal, capacity = all candidates
  float* user_table;     // caller's copy (first user_max rows) or nullptr
  int user_max;
  int32_t* n_det;
  int32_t* route_idx;    // [n_edges][cap]
  int32_t* n_routed;     // [n_edges] required
  int32_t* count_clamped;  // [n_edges]
  int32_t* cap_flag;
  float nms_iou;           // > 0: NMS between decode and routing
};
size_t det_route_ws_bytes(int n_static, int cells_per_frame, int A, bool nms);
void launch_det_route(const DetRouteArgs& a, void* ws, cudaStream_t st);
void launch_crops(const bf16* frames, int H, int W, int C, const float* det_table, const int32_t* route_idx,
                  const int32_t* count_clamped, int edge, int cap, int crop_h, int crop_w, int cout_pad, bf16* dst,
                  cudaStream_t st, bool s2d = false);
// CLASS_WHOLE routing: stable compaction of rows with pred == cls
void launch_route_class(const int32_t* pred, const int* count, int n_static, int cls, int32_t* list,
                        int32_t* count_out, int cap, int32_t* cap_flag, cudaStream_t st);

}  // namespace adainf

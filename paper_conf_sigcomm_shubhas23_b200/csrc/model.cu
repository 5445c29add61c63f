// Model runtime: IR resolution, parameter storage, inference and retraining orchestration.
#include <algorithm>
#include <cmath>
#include <cstring>
#include <random>

#include "api_common.h"
#include "model.h"
#include "stem.cuh"

namespace adainf {

void DevBuf::alloc(size_t b) {
  if (p) cudaFree(p);
  p = nullptr;
  bytes = b;
  if (b) {
    cudaError_t e = cudaMalloc(&p, b);
    if (e != cudaSuccess) {
      cudaGetLastError();
      p = nullptr;
      throw CudaError(std::string("cudaMalloc(") + std::to_string(b) + "): " + cudaGetErrorString(e));
    }
  }
}
void DevBuf::zero(cudaStream_t st) {
  if (p) CK(cudaMemsetAsync(p, 0, bytes, st));
}
DevBuf::~DevBuf() {
  if (p) cudaFree(p);
}

static int pad8(int c) { return (c + 7) / 8 * 8; }

// ------------------------------------------------------------------------------------------------
void Model::build(const adainf_model_spec& s) {
  if (s.n_ops <= 0 || !s.ops) throw InvalidError("model: empty op list");
  if (s.in_h <= 0 || s.in_w <= 0 || s.in_c <= 0 || s.max_batch <= 0) throw ShapeError("model: bad input shape");
  in_h = s.in_h;
  in_w = s.in_w;
  in_c = s.in_c;
  max_batch = s.max_batch;
  // few-channel inputs (images 3, spectrograms 1) are padded to 4 channels (8-byte pixels) and gathered
  // by the conv producers with 8-byte cp.async (one tap per half chunk); others to a multiple of 8
  cin_pad = in_c <= 4 ? 4 : pad8(in_c);
  pack = cin_pad != in_c;
  momentum = s.momentum;
  weight_decay = s.weight_decay;
  ops.assign(s.ops, s.ops + s.n_ops);
  device = s.device;

  TensorRt t0;
  t0.H = in_h;
  t0.W = in_w;
  t0.C = cin_pad;
  T.push_back(std::move(t0));
  int cur = 0, stage = 0;
  std::vector<int> blocks;
  op_node.assign(ops.size(), -1);
  int n_exit_ops = 0;
  for (auto& o : ops)
    if (o.kind == ADAINF_OP_EXIT) n_exit_ops++;
  int seen_exits = 0;
  long long off = 0;
  std::vector<int> op_tensor;  // current tensor after each op (ROUTE sources)
  for (size_t i = 0; i < ops.size(); ++i) {
    if (i > 0) op_tensor.push_back(cur);
    const adainf_op& o = ops[i];
    if (T[cur].up_src >= 0 && o.kind != ADAINF_OP_ROUTE)
      throw UnsupportedError("UPSAMPLE must feed a ROUTE (it is read through the concat, never materialised)");
    if (o.kind == ADAINF_OP_UPSAMPLE) {
      if (o.stride < 1 || o.stride > 8) throw ShapeError("upsample: factor in 1..8");
      TensorRt V;
      V.H = T[cur].H * o.stride;
      V.W = T[cur].W * o.stride;
      V.C = T[cur].C;
      V.f32 = T[cur].f32;
      V.stage = stage;
      V.up_src = cur;
      V.up = o.stride;
      if (V.f32) throw UnsupportedError("upsample of an fp32 tensor");
      T.push_back(std::move(V));
      cur = (int)T.size() - 1;
      inference_only = true;
      continue;
    }
    if (o.kind == ADAINF_OP_ROUTE) {
      if (o.kh < 0 || o.kh >= (int)i || o.kw >= (int)i) throw InvalidError("route: sources must be earlier ops");
      const int ta = op_tensor[o.kh];
      inference_only = true;
      if (o.kw < 0) {  // the earlier output itself: an alias of its buffer
        if (T[ta].up_src >= 0) throw UnsupportedError("route of an upsampled tensor alone");
        TensorRt Z;
        Z.H = T[ta].H;
        Z.W = T[ta].W;
        Z.C = T[ta].C;
        Z.f32 = T[ta].f32;
        Z.stage = stage;
        Z.alias_of = T[ta].alias_of >= 0 ? T[ta].alias_of : ta;
        T[Z.alias_of].routed = true;
        T.push_back(std::move(Z));
        cur = (int)T.size() - 1;
        continue;
      }
      const int tb = op_tensor[o.kw];
      const TensorRt& A = T[ta];
      const TensorRt& Bt = T[tb];
      if (Bt.up_src >= 0 || A.f32 || Bt.f32) throw UnsupportedError("route: only the first source may be upsampled");
      if (A.H != Bt.H || A.W != Bt.W || A.C % 8 || Bt.C % 8) throw ShapeError("route: sources must share H, W");
      NodeRt nd;
      nd.kind = N_ROUTE;
      nd.op = (int)i;
      nd.in = ta;
      nd.res = tb;
      nd.stage = stage;
      TensorRt Z;
      Z.H = A.H;
      Z.W = A.W;
      Z.C = A.C + Bt.C;
      Z.stage = stage;
      Z.producer = (int)nodes.size();
      T[A.up_src >= 0 ? A.up_src : (A.alias_of >= 0 ? A.alias_of : ta)].routed = true;
      T[Bt.alias_of >= 0 ? Bt.alias_of : tb].routed = true;
      T.push_back(std::move(Z));
      nd.out = (int)T.size() - 1;
      cur = nd.out;
      op_node[i] = (int)nodes.size();
      nodes.push_back(std::move(nd));
      continue;
    }
    if (o.kind == ADAINF_OP_BLOCK && o.cout <= 0 && o.pool) {
      // average-pool shortcut (ShuffleNet stride-2 unit): its own node and tensor, closed by a concat
      NodeRt nd;
      nd.kind = N_AVGPOOL;
      nd.op = (int)i;
      nd.in = cur;
      nd.stage = stage;
      const TensorRt& X = T[cur];
      if (X.f32 || X.C % 8) throw ShapeError("pool shortcut: bf16 input with a multiple of 8 channels");
      if (o.kh <= 0 || o.kh != o.kw || o.stride <= 0 || o.pad < 0 || o.pad >= o.kh)
        throw ShapeError("pool shortcut: bad window");
      nd.pk = o.kh;
      nd.ps = o.stride;
      nd.pp = o.pad;
      nd.g.H = X.H;
      nd.g.W = X.W;
      nd.g.Cin = nd.g.Cout = X.C;
      nd.g.Ho = (X.H + 2 * o.pad - o.kh) / o.stride + 1;
      nd.g.Wo = (X.W + 2 * o.pad - o.kw) / o.stride + 1;
      if (T[cur].avgpool >= 0) throw InvalidError("tensor used by two pool shortcuts");
      TensorRt Y;
      Y.H = nd.g.Ho;
      Y.W = nd.g.Wo;
      Y.C = X.C;
      Y.producer = (int)nodes.size();
      Y.stage = stage;
      T[cur].avgpool = (int)nodes.size();
      T.push_back(std::move(Y));
      nd.out = (int)T.size() - 1;
      blocks.push_back(nd.out);
      op_node[i] = (int)nodes.size();
      nodes.push_back(std::move(nd));
      continue;
    }
    if (o.kind == ADAINF_OP_SHUFFLE) {
      // channel shuffle folded into the producing conv's output order (shadow rows + bias): no data moves
      const int pr = T[cur].producer;
      bool ok = pr >= 0 && nodes[pr].kind == N_CONV && nodes[pr].out == cur && nodes[pr].in != 0 &&
                !nodes[pr].fp32_out && nodes[pr].shuf_g == 0 && nodes[pr].res < 0 &&
                (nodes[pr].groups == 1 || nodes[pr].gdense) && T[cur].primary < 0 && T[cur].exit_k < 0 &&
                T[cur].res_of < 0 && T[cur].proj < 0 && T[cur].avgpool < 0;
      for (int b : blocks) ok = ok && b != cur;
      if (!ok) throw UnsupportedError("SHUFFLE must directly follow a dense / grouped conv whose output has no other reader");
      if (o.groups <= 1 || T[cur].C % o.groups) throw ShapeError("shuffle: groups must divide the channels");
      nodes[pr].shuf_g = o.groups;
      continue;
    }
    if (o.kind == ADAINF_OP_CONV || o.kind == ADAINF_OP_BLOCK) {
      const bool proj = o.kind == ADAINF_OP_BLOCK;
      if (proj && o.cout <= 0) {
        blocks.push_back(cur);
        continue;
      }
      NodeRt nd;
      nd.kind = proj ? N_PROJ : N_CONV;
      nd.op = (int)i;
      nd.in = cur;
      nd.stage = stage;
      const TensorRt& X = T[cur];
      if (X.f32) throw InvalidError("conv on an fp32 tensor");
      const int KH = proj ? 1 : o.kh, KW = proj ? 1 : o.kw, st = o.stride, pd = proj ? 0 : o.pad;
      if (KH <= 0 || KW <= 0 || st <= 0 || pd < 0 || o.cout <= 0) throw ShapeError("conv: bad geometry");
      if (KH * KW > 49) throw ShapeError("conv: at most 49 taps");
      if (o.cout % 8 && !(i + 1 < ops.size() && ops[i + 1].kind == ADAINF_OP_DET_HEAD))
        throw ShapeError("conv: cout must be a multiple of 8");
      nd.g.Cin = X.C;
      nd.g.Cout = o.cout;
      nd.g.KH = KH;
      nd.g.KW = KW;
      nd.g.stride = st;
      nd.g.pad = pd;
      nd.g.H = X.H;
      nd.g.W = X.W;
      nd.g.Ho = (X.H + 2 * pd - KH) / st + 1;
      nd.g.Wo = (X.W + 2 * pd - KW) / st + 1;
      if (nd.g.Ho <= 0 || nd.g.Wo <= 0) throw ShapeError("conv: empty output");
      nd.groups = (!proj && o.groups > 1) ? o.groups : 1;
      if (nd.groups > 1) {
        if (cur == 0) throw UnsupportedError("grouped conv on the model input");
        if (!dw_ok(nd.g, nd.groups)) {
          // grouped (ShuffleNet): one dense GEMM over a block-diagonal weight
          if (X.C % nd.groups || o.cout % nd.groups || nd.groups >= X.C)
            throw UnsupportedError("grouped conv: groups must divide cin and cout (depthwise: 3x3, groups == cin == cout)");
          nd.gdense = true;
        }
      }
      if (!proj && (o.act < 0 || o.act > 3)) throw InvalidError("conv: act must be 0..3");
      nd.cin_real = (cur == 0) ? in_c : X.C / nd.groups;
      nd.act = proj ? 0 : o.act;
      nd.w_off = off;
      off += (long long)o.cout * KH * KW * nd.cin_real;
      nd.b_off = off;
      off += o.cout;
      // 16-byte aligned shadow rows (4-channel stems: 49*4 -> 200); grouped-dense rows span all input channels
      nd.ldb = pad8(KH * KW * X.C / (nd.gdense ? 1 : nd.groups));
      nd.fp32_out = !proj && (i + 1 < ops.size() && ops[i + 1].kind == ADAINF_OP_DET_HEAD);
      TensorRt Y;
      Y.H = nd.g.Ho;
      Y.W = nd.g.Wo;
      Y.C = o.cout;
      Y.producer = (int)nodes.size();
      Y.act = nd.act;
      Y.stage = stage;
      Y.f32 = nd.fp32_out;
      T.push_back(std::move(Y));
      nd.out = (int)T.size() - 1;
      int concat_src = -1;
      if (!proj && o.residual == 2) {  // concat join: [shortcut, this conv] (ShuffleNet stride-2 unit)
        if (blocks.empty()) throw InvalidError("concat conv without an open block");
        concat_src = blocks.back();
        blocks.pop_back();
        const TensorRt& R = T[concat_src];
        const TensorRt& Yo = T[nd.out];
        if (R.H != Yo.H || R.W != Yo.W || R.f32) throw ShapeError("concat shape mismatch");
        if (R.stage != stage) throw InvalidError("a residual block may not span an exit");
        if (nd.fp32_out) throw UnsupportedError("concat into a detector head");
      } else if (!proj && o.residual) {
        if (blocks.empty()) throw InvalidError("residual conv without an open block");
        nd.res = blocks.back();
        blocks.pop_back();
        const TensorRt& R = T[nd.res];
        const TensorRt& Yo = T[nd.out];
        if (R.H != Yo.H || R.W != Yo.W || R.C != Yo.C) throw ShapeError("residual shape mismatch");
        if (R.stage != stage) throw InvalidError("a residual block may not span an exit");
      }
      const int ni = (int)nodes.size();
      if (proj) {
        if (T[cur].proj >= 0) throw InvalidError("tensor used by two projections");
        T[cur].proj = ni;
        blocks.push_back(nd.out);
      } else {
        if (T[cur].primary >= 0) throw InvalidError("tensor consumed twice on the main path");
        T[cur].primary = ni;
        if (nd.res >= 0 && T[nd.res].producer >= 0 && nodes[T[nd.res].producer].kind == N_PROJ) {
          // shortcut tensor produced by a projection: its gradient is this conv's dZ (handled by the walk)
        } else if (nd.res >= 0) {
          T[nd.res].res_of = ni;
        }
        cur = nd.out;
      }
      op_node[i] = ni;
      nodes.push_back(std::move(nd));
      if (concat_src >= 0) {
        const int yi = cur;
        NodeRt cn;
        cn.kind = N_CONCAT;
        cn.op = (int)i;
        cn.in = yi;
        cn.res = concat_src;
        cn.stage = stage;
        cn.act = o.act;
        TensorRt Z;
        Z.H = T[yi].H;
        Z.W = T[yi].W;
        Z.C = T[concat_src].C + T[yi].C;
        Z.producer = (int)nodes.size();
        Z.act = o.act;
        Z.stage = stage;
        T[yi].primary = (int)nodes.size();
        T[concat_src].primary = (int)nodes.size();
        T.push_back(std::move(Z));
        cn.out = (int)T.size() - 1;
        cur = cn.out;
        nodes.push_back(std::move(cn));
      }
    } else if (o.kind == ADAINF_OP_MAXPOOL) {
      NodeRt nd;
      nd.kind = N_POOL;
      nd.op = (int)i;
      nd.in = cur;
      nd.stage = stage;
      const TensorRt& X = T[cur];
      nd.pk = o.kh;
      nd.ps = o.stride;
      nd.pp = o.pad;
      if (o.kh <= 0 || o.kh != o.kw || o.kh * o.kw > 255 || o.stride <= 0) throw ShapeError("maxpool: bad window");
      nd.g.H = X.H;
      nd.g.W = X.W;
      nd.g.Cin = nd.g.Cout = X.C;
      nd.g.Ho = (X.H + 2 * o.pad - o.kh) / o.stride + 1;
      nd.g.Wo = (X.W + 2 * o.pad - o.kw) / o.stride + 1;
      TensorRt Y;
      Y.H = nd.g.Ho;
      Y.W = nd.g.Wo;
      Y.C = X.C;
      Y.producer = (int)nodes.size();
      Y.act = 0;
      Y.stage = stage;
      T.push_back(std::move(Y));
      nd.out = (int)T.size() - 1;
      if (T[cur].primary >= 0) throw InvalidError("tensor consumed twice on the main path");
      T[cur].primary = (int)nodes.size();
      cur = nd.out;
      op_node[i] = (int)nodes.size();
      nodes.push_back(std::move(nd));
    } else if (o.kind == ADAINF_OP_EXIT) {
      if (!blocks.empty()) throw InvalidError("an exit may not sit inside an open residual block");
      if (o.num_classes <= 0 || o.num_classes > 64) throw ShapeError("exit: num_classes in 1..64");
      ExitRt e;
      e.op = (int)i;
      e.tensor = cur;
      e.ncls = o.num_classes;
      e.stage = stage;
      e.lw = o.loss_weight;
      const int C = T[cur].C;
      if (C % 8 || C / 8 > 1024) throw ShapeError("exit: channels must be a multiple of 8, <= 8192");
      e.w_off = off;
      off += (long long)C * o.num_classes;
      e.b_off = off;
      off += o.num_classes;
      if (!exits.empty() && exits[0].ncls != e.ncls) throw ShapeError("all exits of a model share num_classes");
      if (T[cur].exit_k >= 0) throw InvalidError("two exits on one tensor");
      T[cur].exit_k = (int)exits.size();
      exits.push_back(std::move(e));
      seen_exits++;
      if (seen_exits < n_exit_ops) stage++;
    } else if (o.kind == ADAINF_OP_DET_HEAD && det.tensor >= 0) {  // second scale (two-scale TinyYOLOv3)
      if (!T[cur].f32) throw InvalidError("DET_HEAD must follow a conv");
      if (det.tensor2 >= 0) throw UnsupportedError("at most two DET_HEADs");
      if (o.anchors != det.anchors || o.det_classes != det.classes || o.nms_iou != det.nms_iou ||
          T[cur].C != o.anchors * (5 + o.det_classes))
        throw ShapeError("det_head: both scales share anchors per cell, classes and nms_iou");
      det.tensor2 = cur;
      det.stride2 = o.grid_stride;
      memcpy(det.anchor_wh2, o.anchor_wh, sizeof(det.anchor_wh2));
    } else if (o.kind == ADAINF_OP_DET_HEAD) {
      if (!T[cur].f32) throw InvalidError("DET_HEAD must follow a conv");
      det.tensor = cur;
      if (!(o.nms_iou >= 0.f) || o.nms_iou > 1.f) throw InvalidError("DET_HEAD: nms_iou must be in [0, 1]");
      det.nms_iou = o.nms_iou;
      det.anchors = o.anchors;
      det.classes = o.det_classes;
      det.stride = o.grid_stride;
      if (o.anchors <= 0 || o.anchors > 8 || o.det_classes <= 0 || T[cur].C != o.anchors * (5 + o.det_classes))
        throw ShapeError("det_head: channels must be anchors*(5+classes)");
      memcpy(det.anchor_wh, o.anchor_wh, sizeof(det.anchor_wh));
    } else {
      throw InvalidError("unknown op kind");
    }
  }
  if (!blocks.empty()) throw InvalidError("unclosed residual block");
  if (exits.empty() && det.tensor < 0) throw InvalidError("model needs at least one EXIT or a DET_HEAD");
  if (!exits.empty() && exits.back().op != (int)ops.size() - 1) throw InvalidError("the final EXIT must be the last op");
  for (auto& nd : nodes)
    if (nd.kind == N_POOL && (T[nd.in].exit_k >= 0 || T[nd.in].res_of >= 0 || T[nd.in].proj >= 0))
      throw InvalidError("a pooled tensor may not feed an exit or a shortcut");
  for (size_t i = 0; i < nodes.size(); ++i) {
    const NodeRt& nd = nodes[i];
    if (T[nd.in].stage + 1 < nd.stage) throw InvalidError("tensor read across two exits");
  }
  nstages = stage + 1;
  nparams = off;

  // fused space-to-depth stem: conv 7x7/2 (ReLU) whose only consumer is a 3x3/2 pad-1 max-pool
  stem_s2d = false;
  if (!nodes.empty() && nodes[0].kind == N_CONV && nodes[0].in == 0 && win_mode() != 8) {
    const NodeRt& c0 = nodes[0];
    const TensorRt& Y = T[c0.out];
    const int po = Y.primary;
    if (po >= 0 && nodes[po].kind == N_POOL && nodes[po].pk == 3 && nodes[po].ps == 2 && nodes[po].pp == 1 &&
        nodes[po].stage == c0.stage && c0.act == 1 && !c0.fp32_out && c0.res < 0 && Y.exit_k < 0 &&
        Y.res_of < 0 && Y.proj < 0 && !Y.routed && stem_s2d_ok(in_h, in_w, in_c, c0.g.Cout, c0.g.KH, c0.g.KW, c0.g.stride, c0.g.pad)) {
      stem_s2d = true;
      stem_pool = po;
      pack = true;
    }
  }
  // 3x3/1 convs whose only reader is a 2x2/2 max-pool (the TinyYOLOv3-like detector's few-channel layers): conv +
  // pool in one tensor-core kernel in inference (conv3pool.cu); the first layer on the space-to-depth packed input
  first_s2d = false;
  const char* c3p_env = getenv("ADAINF_CONV3POOL");
  if (!c3p_env || atoi(c3p_env) != 0) {
    for (size_t ni = 0; ni < nodes.size(); ++ni) {
      NodeRt& nd = nodes[ni];
      if (nd.kind != N_CONV || nd.groups != 1 || nd.shuf_g || nd.res >= 0 || nd.fp32_out) continue;
      if (stem_s2d && ni == 0) continue;
      const TensorRt& Y = T[nd.out];
      const int po = Y.primary;
      if (po < 0 || nodes[po].kind != N_POOL || nodes[po].stage != nd.stage || Y.exit_k >= 0 || Y.res_of >= 0 ||
          Y.proj >= 0 || Y.avgpool >= 0 || Y.routed)
        continue;
      const bool first = nd.in == 0;
      if (first && cin_pad != 4) continue;
      if (!conv3_pool_ok(nd.g, first, nd.cin_real, nodes[po].pk, nodes[po].ps, nodes[po].pp)) continue;
      nd.fuse_pool = po;
      if (first) first_s2d = true;
    }
  }

  CK(cudaSetDevice(device));
  // activations
  for (size_t t = 1; t < T.size(); ++t) {
    if (stem_s2d && (int)t == nodes[0].out) continue;  // the fused stem never materialises its conv output
    if (T[t].up_src >= 0 || T[t].alias_of >= 0) continue;  // upsampling views / route aliases own no memory
    const size_t b = (size_t)max_batch * T[t].row_elems() * (T[t].f32 ? 4 : 2);
    T[t].own.alloc(b);
    T[t].buf = T[t].own.as<bf16>();
  }
  if (pack) {
    packed_in.alloc((size_t)max_batch * T[0].row_elems() * 2);
    T[0].buf = packed_in.as<bf16>();
  }
  for (size_t t = 1; t < T.size(); ++t) {
    if (T[t].alias_of >= 0) T[t].buf = T[T[t].alias_of].buf;
    if (T[t].up_src >= 0) T[t].buf = T[T[t].up_src].buf;
  }
  for (auto& nd : nodes)
    if (nd.kind == N_CONV || nd.kind == N_PROJ) {
      nd.shadow.alloc((size_t)nd.g.Cout * nd.ldb * 2);
      nd.shadow.zero();  // grouped-dense: the off-diagonal blocks stay zero
      if (nd.groups > 1 && !nd.gdense) nd.wdw.alloc((size_t)nd.g.KH * nd.g.KW * nd.g.Cin * 2);
      if (nd.shuf_g) nd.bias_perm.alloc((size_t)nd.g.Cout * 4);
      if (nd.fuse_pool >= 0) nd.wexp.alloc(conv3_pool_wexp_bytes(nd.g, nd.in == 0));
    }
  if (stem_s2d) stem_wprep.alloc(16 * 2 * 64 * 8 * 2);
  for (size_t k = 0; k + 1 < exits.size(); ++k) {  // dense survivor copies of the stage-boundary tensors
    const TensorRt& X = T[exits[k].tensor];
    if (!X.f32 && exits[k].tensor > 0 && (X.row_elems() * 2) % 16 == 0)
      exits[k].dense_next.alloc((size_t)max_batch * X.row_elems() * 2);
  }
  params.alloc(nparams * 4);
  mom.alloc(nparams * 4);
  grads.alloc(nparams * 4);
  mom.zero();
  grads.zero();
  pos.alloc((size_t)nstages * max_batch * 4);
  orig.alloc((size_t)nstages * max_batch * 4);
  counts.alloc((size_t)nstages * 4 + 16);
  alive.alloc((size_t)max_batch);
  exit_ws.alloc(exit_fused_ws_bytes(max_batch));

  // SGD segment tables (shadow layout per conv weight)
  std::vector<SgdSeg> segs;
  auto add_seg = [&](long long o, long long c, bf16* sh, int taps, int cin, int cin_p, int ldb) {
    SgdSeg s{};
    s.off = o;
    s.count = c;
    s.shadow = sh;
    s.taps = taps;
    s.cin = cin;
    s.cin_pad = cin_p;
    s.ldb = ldb;
    segs.push_back(s);
  };
  // segments in flat order
  std::vector<std::pair<long long, int>> order;  // (offset, kind/index)
  for (size_t i = 0; i < nodes.size(); ++i)
    if (nodes[i].kind == N_CONV || nodes[i].kind == N_PROJ) order.push_back({nodes[i].w_off, (int)i});
  for (size_t k = 0; k < exits.size(); ++k) order.push_back({exits[k].w_off, -1 - (int)k});
  std::sort(order.begin(), order.end());
  for (auto& pr : order) {
    if (pr.second >= 0) {
      NodeRt& nd = nodes[pr.second];
      add_seg(nd.w_off, (long long)nd.g.Cout * nd.g.KH * nd.g.KW * nd.cin_real, nd.shadow.as<bf16>(),
              nd.g.KH * nd.g.KW, nd.cin_real, nd.gdense ? nd.g.Cin : nd.g.Cin / nd.groups, nd.ldb);
      segs.back().cog = nd.gdense ? nd.g.Cout / nd.groups : 0;
      segs.back().shuf_g = nd.shuf_g;
      segs.back().cout = nd.g.Cout;
      add_seg(nd.b_off, nd.g.Cout, nullptr, 0, 0, 0, 0);
    } else {
      ExitRt& e = exits[-1 - pr.second];
      add_seg(e.w_off, e.b_off + e.ncls - e.w_off, nullptr, 0, 0, 0, 0);
    }
  }
  std::vector<int> bseg;
  std::vector<long long> bstart;
  const long long PER = SGD_BLOCK_ELEMS;
  for (size_t si = 0; si < segs.size(); ++si)
    for (long long st = segs[si].off; st < segs[si].off + segs[si].count; st += PER) {
      bseg.push_back((int)si);
      bstart.push_back(st);
    }
  sgd_nseg = (int)segs.size();
  sgd_nblocks = (int)bseg.size();
  sgd_segs.alloc(segs.size() * sizeof(SgdSeg));
  sgd_block_seg.alloc(bseg.size() * 4);
  sgd_block_start.alloc(bstart.size() * 8);
  CK(cudaMemcpy(sgd_segs.p, segs.data(), segs.size() * sizeof(SgdSeg), cudaMemcpyHostToDevice));
  CK(cudaMemcpy(sgd_block_seg.p, bseg.data(), bseg.size() * 4, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(sgd_block_start.p, bstart.data(), bstart.size() * 8, cudaMemcpyHostToDevice));
  sq_partial.alloc((size_t)sgd_nblocks * 4 + 64);

  // parameters: caller's, or He-normal from seed (exit heads x4)
  std::vector<float> host(nparams);
  if (s.init_params) {
    memcpy(host.data(), s.init_params, nparams * 4);
  } else {
    std::mt19937_64 rng(s.seed);
    std::normal_distribution<float> nd01(0.f, 1.f);
    for (auto& nd : nodes) {
      if (nd.kind != N_CONV && nd.kind != N_PROJ) continue;
      const float sd = std::sqrt(1.0f / (float)(nd.g.KH * nd.g.KW * nd.cin_real));
      for (long long j = nd.w_off; j < nd.b_off; ++j) host[j] = nd01(rng) * sd;
      for (int j = 0; j < nd.g.Cout; ++j) host[nd.b_off + j] = 0.01f * nd01(rng);
    }
    for (auto& e : exits) {
      const int C = T[e.tensor].C;
      const float sd = 4.0f / std::sqrt((float)C);
      for (long long j = e.w_off; j < e.b_off; ++j) host[j] = nd01(rng) * sd;
      for (int cls = 0; cls < e.ncls; ++cls) {  // zero-mean over channels (see synth.init_params)
        double mean = 0;
        for (int c = 0; c < C; ++c) mean += host[e.w_off + (long long)c * e.ncls + cls];
        mean /= C;
        for (int c = 0; c < C; ++c) host[e.w_off + (long long)c * e.ncls + cls] -= (float)mean;
      }
      for (int j = 0; j < e.ncls; ++j) host[e.b_off + j] = 0.1f * nd01(rng);
    }
  }
  CK(cudaMemcpy(params.p, host.data(), nparams * 4, cudaMemcpyHostToDevice));
  refresh_shadows(0);
  CK(cudaDeviceSynchronize());
}

// a1 ingest: channel padding (to 4 for few-channel inputs, else to a multiple of 8)
void Model::ingest(const bf16* x, const int* map, const int* count, int n_static, cudaStream_t st, bool s2d) {
  if (stem_s2d || s2d) {
    launch_pack_s2d(x, map, count, n_static, in_h, in_w, in_c, packed_in.as<bf16>(), st);
    return;
  }
  launch_pack_input(x, map, count, n_static, in_h, in_w, in_c, cin_pad, packed_in.as<bf16>(), st);
}

void Model::refresh_shadows(cudaStream_t st) {
  launch_shadow_pack(params.as<float>(), sgd_segs.as<SgdSeg>(), sgd_nseg, st);
}

void Model::ensure_training() {
  if (train_ready) return;
  if (exits.empty()) throw UnsupportedError("retraining needs an early-exit classifier (detector is not retrained, P:86)");
  if (inference_only) throw UnsupportedError("UPSAMPLE / ROUTE models are inference-only (detectors, P:86)");
  for (size_t t = 1; t < T.size(); ++t) {
    if (T[t].f32) continue;
    T[t].own_grad.alloc((size_t)max_batch * T[t].row_elems() * 2);
    T[t].grad = T[t].own_grad.as<bf16>();
  }
  size_t ws = 0;
  for (auto& nd : nodes)
    if (nd.kind == N_CONV && nd.in != 0 && nd.groups == 1 && dgrad_sp_ok(nd.g)) {
      nd.sp = true;
      nd.wsp.alloc(dgrad_sp_ws_bytes(nd.g));
    }
  size_t gd = 0;  // dense weight-gradient scratch of grouped / shuffled convs (gathered into the master layout)
  for (auto& nd : nodes) {
    if (nd.kind == N_CONCAT) continue;
    if (nd.kind == N_AVGPOOL) {
      if (nd.in != 0) nd.pool_sc.alloc((size_t)max_batch * T[nd.in].row_elems() * 2);
      continue;
    }
    if (nd.gdense || nd.shuf_g)
      gd = std::max(gd, ((size_t)nd.g.Cout * nd.g.KH * nd.g.KW * nd.g.Cin + nd.g.Cout) * 4);
    if (nd.kind == N_POOL) {
      nd.argmax.alloc((size_t)max_batch * T[nd.out].row_elems());
    } else {
      ws = std::max(ws, (nd.groups > 1 && !nd.gdense) ? dw_wgrad_ws_bytes(nd.g, max_batch) : ::adainf::wgrad_ws_bytes(nd.g, max_batch));
      if (stem_s2d && &nd == &nodes[0]) ws = std::max(ws, stem_wgrad_ws_bytes(max_batch));
      if (nd.kind == N_PROJ && nd.in != 0) {
        for (const auto& c : nodes)
          if (c.kind == N_CONV && c.in == nd.in && c.sp && c.g.Ho == nd.g.Ho && c.g.Wo == nd.g.Wo) nd.proj_compact = true;
        const size_t rows = nd.proj_compact ? (size_t)nd.g.Ho * nd.g.Wo * nd.g.Cin : T[nd.in].row_elems();
        nd.proj_dx.alloc((size_t)max_batch * rows * 2);
      }
    }
  }
  for (auto& e : exits) ws = std::max(ws, head_grads_ws_bytes(max_batch, T[e.tensor].C, e.ncls));
  wgrad_ws.alloc(ws);
  wgrad_ws_bytes = ws;
  gw_dense.alloc(gd);
  for (auto& e : exits) {
    const int C = T[e.tensor].C;
    e.pooled.alloc((size_t)max_batch * C * 4);
    e.logits.alloc((size_t)max_batch * e.ncls * 4);
    e.dl.alloc((size_t)max_batch * e.ncls * 4);
    e.bcast.alloc((size_t)max_batch * C * 4);
  }
  loss_rows.alloc((size_t)max_batch * 4);
  stats_tmp.alloc(64);
  train_ready = true;
}

// ------------------------------------------------------------------------------------------------
// Forward over all ops.  Inference: stage s>0 reads tensors of stage s-1 through pos[s] (dense survivor
// positions) and works on count[s] rows (device-side), outputs are scattered through orig[s].
// Training: all rows, no exits taken, heads evaluated for every row (SURVEY c.1 step 9).
void Model::forward_nodes(const bf16* x0, const int* map0, const int* count0, int n_static, bool train,
                          const float* taus, const adainf_model_out* out, cudaStream_t st, bool in_s2d) {
  std::vector<char> pool_done(nodes.size(), 0);  // max-pools already produced by their conv (conv3_pool)
  int* posb = pos.as<int>();
  int* origb = orig.as<int>();
  int* cnt = counts.as<int>();
  auto stage_count = [&](int s) -> const int* { return s == 0 ? count0 : cnt + s; };
  auto stage_orig = [&](int s) -> const int* { return s == 0 ? nullptr : origb + (size_t)s * max_batch; };
  // inference: stage-boundary tensors whose survivors have been gathered densely (per tensor, after compaction)
  std::vector<const bf16*> dense_t(T.size(), nullptr);
  auto buf_of = [&](int t) -> const bf16* { return t == 0 ? x0 : (dense_t[t] ? dense_t[t] : T[t].buf); };
  // map used by a node of stage `ns` reading tensor t
  auto map_for = [&](int t, int ns) -> const int* {
    if (train) return nullptr;
    if (t == 0) return ns == 0 ? map0 : nullptr;
    if (dense_t[t]) return nullptr;
    if (T[t].stage < ns) return posb + (size_t)ns * max_batch;
    return nullptr;
  };
  const int E = (int)exits.size();
  for (size_t i = 0; i < ops.size(); ++i) {
    const int ni = op_node[i];
    if (ni >= 0) {
      NodeRt& nd = nodes[ni];
      const int ns = train ? 0 : nd.stage;
      const int* c = train ? nullptr : stage_count(ns);
      if (stem_s2d && ni == 0) {
        if (map_for(0, ns)) throw InvalidError("stem: mapped input rows must be ingested first");
        const NodeRt& pl = nodes[stem_pool];
        launch_stem_wprep(nd.shadow.as<bf16>(), nd.ldb, stem_wprep.as<bf16>(), st);
        stem_fwd(buf_of(0), c, n_static, in_h / 2, in_w / 2, stem_wprep.as<bf16>(), params.as<float>() + nd.b_off,
                 T[pl.out].buf, train ? pl.argmax.as<uint8_t>() : nullptr, st);
        continue;
      }
      if (!train && nd.kind == N_CONV && nd.fuse_pool >= 0 && !map_for(nd.in, ns) && (nd.in != 0 || in_s2d)) {
        // conv + its 2x2 max-pool in one kernel (inference only: training keeps the pre-pool tensor)
        const NodeRt& pl = nodes[nd.fuse_pool];
        conv3_pool(nd.g, nd.in == 0, buf_of(nd.in), c, n_static, nd.shadow.as<bf16>(), nd.ldb, nd.cin_real,
                   params.as<float>() + nd.b_off, nd.act, nd.wexp.as<bf16>(), T[pl.out].buf, st);
        pool_done[nd.fuse_pool] = 1;
        continue;
      }
      if (nd.kind == N_ROUTE) {
        const TensorRt& A = T[nd.in];
        const TensorRt& Z = T[nd.out];
        const int asrc = A.up_src >= 0 ? A.up_src : nd.in;
        route_concat(buf_of(asrc), T[asrc].H, T[asrc].W, A.C, A.up_src >= 0 ? A.up : 1, buf_of(nd.res), T[nd.res].C, c,
                     n_static, Z.H, Z.W, Z.buf, st);
        continue;
      }
      if (nd.kind == N_AVGPOOL) {
        AvgPoolArgs ap{};
        ap.x = buf_of(nd.in);
        ap.map = map_for(nd.in, ns);
        ap.count = c;
        ap.n_static = n_static;
        ap.H = nd.g.H;
        ap.W = nd.g.W;
        ap.C = nd.g.Cin;
        ap.K = nd.pk;
        ap.s = nd.ps;
        ap.p = nd.pp;
        ap.Ho = nd.g.Ho;
        ap.Wo = nd.g.Wo;
        ap.y = T[nd.out].buf;
        avgpool_fwd(ap, st);
        continue;
      }
      if (nd.kind == N_POOL) {
        if (stem_s2d && ni == stem_pool) continue;  // produced by the fused stem
        if (pool_done[ni]) continue;  // produced by its conv (conv3_pool)
        launch_maxpool_fwd(buf_of(nd.in), map_for(nd.in, ns), c, n_static, nd.g.H, nd.g.W, nd.g.Cin, nd.pk, nd.ps,
                           nd.pp, nd.g.Ho, nd.g.Wo, T[nd.out].buf, train ? nd.argmax.as<uint8_t>() : nullptr,
                           nd.in > 0 && T[nd.in].act == 1, st);
      } else if (nd.groups > 1 && !nd.gdense) {
        if (nd.res >= 0) throw UnsupportedError("depthwise conv closing a residual block");
        dw_prep(nd.shadow.as<bf16>(), nd.ldb, nd.g.Cin, nd.g.KH * nd.g.KW, nd.wdw.as<bf16>(), st);
        DwArgs d{};
        d.x = buf_of(nd.in);
        d.map = map_for(nd.in, ns);
        d.count = c;
        d.n_static = n_static;
        d.H = nd.g.H;
        d.W = nd.g.W;
        d.C = nd.g.Cin;
        d.Ho = nd.g.Ho;
        d.Wo = nd.g.Wo;
        d.KH = nd.g.KH;
        d.KW = nd.g.KW;
        d.s = nd.g.stride;
        d.p = nd.g.pad;
        d.w = nd.wdw.as<bf16>();
        d.bias = params.as<float>() + nd.b_off;
        d.act = nd.act;
        d.y = T[nd.out].buf;
        dw_fwd(d, st);
      } else {
        const float* bias = params.as<float>() + nd.b_off;
        if (nd.shuf_g) {  // folded channel shuffle: bias in the physical output order
          permute_bias(bias, nd.g.Cout, nd.shuf_g, nd.bias_perm.as<float>(), st);
          bias = nd.bias_perm.as<float>();
        }
        const bf16* res = nd.res >= 0 ? buf_of(nd.res) : nullptr;
        const int* rmap = nd.res >= 0 ? map_for(nd.res, ns) : nullptr;
        conv_fwd(nd.g, buf_of(nd.in), map_for(nd.in, ns), c, n_static, nd.shadow.as<bf16>(), nd.ldb, bias, res, rmap,
                 nd.act, T[nd.out].buf, nd.fp32_out, st);
        if (ni + 1 < (int)nodes.size() && nodes[ni + 1].kind == N_CONCAT && nodes[ni + 1].in == nd.out) {
          const NodeRt& cn = nodes[ni + 1];  // [shortcut, conv] join right after its conv (same stage rows)
          const TensorRt& Z = T[cn.out];
          concat_fwd(T[cn.res].buf, T[nd.out].buf, c, n_static, Z.H * Z.W, T[cn.res].C, nd.g.Cout, cn.act, Z.buf, st);
        }
      }
      continue;
    }
    if (ops[i].kind != ADAINF_OP_EXIT) continue;
    int k = -1;
    for (int q = 0; q < E; ++q)
      if (exits[q].op == (int)i) k = q;
    ExitRt& e = exits[k];
    const TensorRt& X = T[e.tensor];
    ExitHeadArgs a{};
    a.fmap = buf_of(e.tensor);
    a.HW = X.H * X.W;
    a.C = X.C;
    a.ncls = e.ncls;
    a.Wk = params.as<float>() + e.w_off;
    a.bk = params.as<float>() + e.b_off;
    a.n_static = n_static;
    if (train) {
      a.is_final = 1;
      a.pooled_save = e.pooled.as<float>();
      a.logits_save = e.logits.as<float>();
      launch_exit_head(a, st, PC_EXIT_HEAD_TRAIN);
      continue;
    }
    const int s = e.stage;
    a.count = stage_count(s);
    a.orig = stage_orig(s);
    a.is_final = (k == E - 1);
    a.tau = a.is_final ? 0.f : taus[k];
    a.exit_index = k;
    a.exit_id = out->exit_id;
    a.pred = out->pred;
    a.conf = out->conf;
    a.entropy = out->entropy;
    a.logits = out->logits;
    a.embed = k == 0 ? out->embed : nullptr;
    a.alive = a.is_final ? nullptr : alive.as<uint8_t>();
    if (e.tensor == 0 && map0) throw InvalidError("exit directly on a mapped input is not supported");
    static int fused_env = -1;
    if (fused_env < 0) {
      const char* ev = getenv("ADAINF_EXIT_FUSED");
      fused_env = ev ? atoi(ev) : 1;
    }
    if (fused_env) {
      // K4 + K5: head, decision, look-back compaction and the survivors' dense copy in one kernel
      a.alive = nullptr;
      const bool copy = !a.is_final && e.dense_next.p;
      launch_exit_fused(a, exit_ws.as<unsigned>(), posb + (size_t)(s + 1) * max_batch,
                        origb + (size_t)(s + 1) * max_batch, cnt + s + 1, out->exit_counts,
                        (!a.is_final && out->surv_idx) ? out->surv_idx + (size_t)k * n_static : nullptr,
                        (k == E - 2) ? out->exit_counts : nullptr, E - 1, copy ? T[e.tensor].buf : nullptr,
                        copy ? e.dense_next.as<bf16>() : nullptr, (long long)X.row_elems(), st);
      if (copy) dense_t[e.tensor] = e.dense_next.as<bf16>();
      continue;
    }
    launch_exit_head(a, st);
    if (!a.is_final) {
      // survivors of exit k -> stage s+1 (stable, ascending original rows)
      launch_compact(alive.as<uint8_t>(), a.count, n_static, a.orig, posb + (size_t)(s + 1) * max_batch,
                     origb + (size_t)(s + 1) * max_batch, cnt + s + 1, out->exit_counts, k,
                     out->surv_idx ? out->surv_idx + (size_t)k * n_static : nullptr,
                     (k == E - 2) ? out->exit_counts : nullptr, E - 1, st);
      if (e.dense_next.p) {
        launch_gather_rows(T[e.tensor].buf, posb + (size_t)(s + 1) * max_batch, cnt + s + 1, n_static,
                           (long long)X.row_elems() * 2, e.dense_next.p, st, PC_SURVIVOR_GATHER);
        dense_t[e.tensor] = e.dense_next.as<bf16>();
      }
    }
  }
}

void Model::infer(const bf16* x, const int* in_map, const int* in_count, int n_static, const float* taus,
                  const adainf_model_out& out, cudaStream_t st, bool x_padded) {
  if (n_static <= 0) return;
  if (n_static > max_batch) throw ShapeError("batch exceeds max_batch");
  const bf16* x0 = x;
  bool in_s2d = false;
  const int* map0 = in_map;
  if (pack && !x_padded) {
    ingest(x, in_map, in_count, n_static, st, first_s2d);
    in_s2d = first_s2d;
    x0 = packed_in.as<bf16>();
    map0 = nullptr;
  }
  if (exits.size() == 1 && out.exit_counts) {
    // single-exit model: every row leaves at exit 0 -> counts[0] = rows (device count or static)
    if (in_count)
      CK(cudaMemcpyAsync(out.exit_counts, in_count, 4, cudaMemcpyDeviceToDevice, st));
    else
      launch_fill_i32(out.exit_counts, n_static, st);
  }
  forward_nodes(x0, map0, in_count, n_static, false, taus, &out, st, in_s2d);
}

// ------------------------------------------------------------------------------------------------
void Model::train_step_rows(const bf16* pool, long long pool_rows, const int32_t* pool_labels, const int32_t* idx,
                            const int32_t* count, int n, long long n_global, float lr, adainf_step_stats* stats,
                            cudaStream_t st, bool update) {
  if (!pack) throw UnsupportedError("retrain_step_rows: the model reads its input unpacked (in_c % 8 == 0)");
  if (n <= 0 || n > max_batch) throw ShapeError("retrain: n_local must be in 1..max_batch");
  if (pool_rows <= 0) throw ShapeError("retrain_step_rows: pool_rows must be positive");
  if (!row_labels.p) {
    row_labels.alloc((size_t)max_batch * 4);
    row_map.alloc((size_t)max_batch * 4);
  }
  // rows past the device count / out-of-range indices -> map -1 (zero input) and label -1 (no loss, no gradient)
  launch_sanitize_rows(pool_labels, idx, count, n, pool_rows, row_map.as<int32_t>(), row_labels.as<int32_t>(), st);
  train_grad_impl(pool, row_map.as<int32_t>(), row_labels.as<int32_t>(), n, n_global, stats, st);
  if (update) update_impl(lr, stats, st);
}

void Model::train_step(const bf16* x, const int32_t* labels, int n, long long n_global, float lr,
                       adainf_step_stats* stats, cudaStream_t st, bool update) {
  train_grad_impl(x, nullptr, labels, n, n_global, stats, st);
  if (update) update_impl(lr, stats, st);
}

void Model::train_grad_impl(const bf16* x, const int32_t* row_map, const int32_t* labels, int n, long long n_global,
                            adainf_step_stats* stats, cudaStream_t st) {
  if (n <= 0 || n > max_batch) throw ShapeError("retrain: n_local must be in 1..max_batch");
  if (n_global < n) throw ShapeError("retrain: n_global < n_local");
  ensure_training();
  const bf16* x0 = x;
  if (pack) {
    ingest(x, row_map, nullptr, n, st);  // row_map: rows of a pool, packed straight into the model layout
    x0 = packed_in.as<bf16>();
  } else if (row_map) {
    throw UnsupportedError("retrain: row-mapped input needs a packed model input");
  }
  forward_nodes(x0, nullptr, nullptr, n, true, nullptr, nullptr, st);
  float* G = grads.as<float>();
  const float* P = params.as<float>();
  const float inv_n = (float)(1.0 / (double)n_global);
  // exit losses and head gradients (K8)
  for (size_t k = 0; k < exits.size(); ++k) {
    ExitRt& e = exits[k];
    const TensorRt& X = T[e.tensor];
    launch_exit_loss(e.logits.as<float>(), labels, n, e.ncls, e.lw, inv_n, e.dl.as<float>(), loss_rows.as<float>(),
                     k > 0, st);
    launch_head_grads(e.pooled.as<float>(), e.dl.as<float>(), P + e.w_off, n, X.C, e.ncls, X.H * X.W, G + e.w_off,
                      G + e.b_off, e.bcast.as<float>(), wgrad_ws.as<float>(), st);
  }
  auto buf_of = [&](int t) -> const bf16* { return t == 0 ? x0 : T[t].buf; };
  auto bcast_of = [&](int t) -> const float* { return T[t].exit_k >= 0 ? exits[T[t].exit_k].bcast.as<float>() : nullptr; };
  auto sc_of = [&](int t) -> const bf16* {
    if (T[t].res_of >= 0) return T[nodes[T[t].res_of].out].grad;  // identity shortcut: dZ of the residual conv
    if (T[t].proj >= 0) return nodes[T[t].proj].proj_dx.as<bf16>();
    if (T[t].avgpool >= 0) return nodes[T[t].avgpool].pool_sc.as<bf16>();  // average-pool shortcut's backward
    return nullptr;
  };
  // tensors with no main-path consumer (the final exit's input): gradient = broadcast (+ shortcut)
  for (size_t t = 1; t < T.size(); ++t)
    if (T[t].primary < 0 && !T[t].f32 && T[t].producer >= 0 && nodes[T[t].producer].kind != N_PROJ &&
        nodes[T[t].producer].kind != N_AVGPOOL)
      launch_grad_finalize(bcast_of((int)t), sc_of((int)t), T[t].buf, T[t].act, n, T[t].H * T[t].W, T[t].C,
                           T[t].grad, st);
  // reverse walk (K2, K3, K9)
  // the stem's max-pool backward is fused into its weight gradient when the stem output feeds only the pool
  static int fuse_env = -1;
  if (fuse_env < 0) {
    const char* e = getenv("ADAINF_STEM_POOL_FUSE");
    fuse_env = e ? atoi(e) : 1;
  }
  bool stem_pool_fused = false;
  if (stem_s2d && fuse_env) {
    const NodeRt& pl = nodes[stem_pool];
    const TensorRt& X = T[pl.in];
    stem_pool_fused = pl.in == nodes[0].out && pl.pk == 3 && pl.ps == 2 && pl.pp == 1 && X.C == 64 &&
                      (X.act == 0 || X.act == 1) && X.exit_k < 0 && X.res_of < 0 && X.proj < 0;
  }
  auto conv_backward = [&](NodeRt& nd, const bf16* dz) {
    if (stem_s2d && &nd == &nodes[0]) {
      if (stem_pool_fused) {
        const NodeRt& pl = nodes[stem_pool];
        stem_wgrad_pooled(buf_of(0), T[pl.out].grad, pl.argmax.as<uint8_t>(), pl.g.Ho, pl.g.Wo, n, in_h / 2,
                          in_w / 2, nd.cin_real, wgrad_ws.as<float>(), wgrad_ws_bytes, G + nd.w_off, G + nd.b_off, st);
      } else {
        stem_wgrad(buf_of(0), dz, n, in_h / 2, in_w / 2, nd.cin_real, wgrad_ws.as<float>(), wgrad_ws_bytes,
                   G + nd.w_off, G + nd.b_off, st);
      }
      return;
    }
    if (nd.groups > 1 && !nd.gdense) {  // depthwise: weight / bias gradient, then the input gradient (dwconv.cu)
      DwArgs d{};
      d.x = buf_of(nd.in);
      d.dz = dz;
      d.n_static = n;
      d.H = nd.g.H;
      d.W = nd.g.W;
      d.C = nd.g.Cin;
      d.Ho = nd.g.Ho;
      d.Wo = nd.g.Wo;
      d.KH = nd.g.KH;
      d.KW = nd.g.KW;
      d.s = nd.g.stride;
      d.p = nd.g.pad;
      dw_wgrad(d, wgrad_ws.as<float>(), wgrad_ws_bytes, G + nd.w_off, G + nd.b_off, st);
      if (nd.in == 0) return;
      const TensorRt& X = T[nd.in];
      const int prod = X.producer;
      const int mask = (prod >= 0 && (nodes[prod].kind == N_CONV || nodes[prod].kind == N_CONCAT)) ? X.act : 0;
      d.x = dz;
      d.w = nd.wdw.as<bf16>();
      d.bcast = bcast_of(nd.in);
      d.sc = sc_of(nd.in);
      d.yact = mask ? X.buf : nullptr;
      d.mask_act = mask;
      d.y = T[nd.in].grad;
      dw_dgrad(d, st);
      return;
    }
    if (nd.gdense || nd.shuf_g) {
      // dense weight gradient over the block-diagonal / row-permuted shadow, then its diagonal blocks gathered
      // back into the master layout (shuffle.cu)
      float* dense = gw_dense.as<float>();
      float* dbs = dense + (size_t)nd.g.Cout * nd.g.KH * nd.g.KW * nd.g.Cin;
      conv_wgrad(nd.g, buf_of(nd.in), dz, n, nd.g.Cin, wgrad_ws.as<float>(), wgrad_ws_bytes, dense, dbs, st);
      grouped_wgrad_gather(dense, dbs, nd.g.Cout, nd.g.KH * nd.g.KW, nd.g.Cin, nd.gdense ? nd.groups : 1, nd.shuf_g,
                           G + nd.w_off, G + nd.b_off, st);
    } else {
      conv_wgrad(nd.g, buf_of(nd.in), dz, n, nd.cin_real, wgrad_ws.as<float>(), wgrad_ws_bytes, G + nd.w_off,
                 G + nd.b_off, st);
    }
    if (nd.in == 0) return;  // no input gradient for the first layer
    const TensorRt& X = T[nd.in];
    if (nd.kind == N_PROJ) {
      ConvGeom g = nd.g;
      if (nd.proj_compact) {  // only the even input positions receive gradient: a plain 1x1 GEMM on the dZ grid
        g.stride = 1;
        g.H = g.Ho;
        g.W = g.Wo;
      }
      conv_dgrad(g, dz, nd.shadow.as<bf16>(), nd.ldb, n, nullptr, nullptr, nullptr, 0, nd.proj_dx.as<bf16>(), st);
    } else {
      const int prod = X.producer;
      const int mask = (prod >= 0 && (nodes[prod].kind == N_CONV || nodes[prod].kind == N_CONCAT)) ? X.act : 0;
      if (nd.sp) {
        const bool sc_compact = X.res_of < 0 && X.proj >= 0 && nodes[X.proj].proj_compact;
        conv_dgrad_sp(nd.g, dz, nd.shadow.as<bf16>(), nd.ldb, nd.wsp.as<bf16>(), n, bcast_of(nd.in), sc_of(nd.in),
                      sc_compact, mask ? X.buf : nullptr, mask, T[nd.in].grad, st);
      } else {
        conv_dgrad(nd.g, dz, nd.shadow.as<bf16>(), nd.ldb, n, bcast_of(nd.in), sc_of(nd.in), mask ? X.buf : nullptr,
                   mask, T[nd.in].grad, st);
      }
    }
  };
  for (int ni = (int)nodes.size() - 1; ni >= 0; --ni) {
    NodeRt& nd = nodes[ni];
    if (nd.kind == N_PROJ || nd.kind == N_AVGPOOL) continue;  // projection: right after its residual conv;
                                                              // avg-pool shortcut: inside its concat's backward
    if (nd.kind == N_CONCAT) {
      // T[out].grad = the consumer's gradient of [shortcut, conv], already masked by act'(Z) and bf16: its conv
      // part is the conv's dZ, its shortcut part goes through the average-pool backward into the block input's
      // shortcut term
      const NodeRt& ap = nodes[T[nd.res].producer];
      const TensorRt& Z = T[nd.out];
      bf16* sc = ap.in != 0 ? nodes[T[nd.res].producer].pool_sc.as<bf16>() : nullptr;
      if (!sc) throw UnsupportedError("pool shortcut on the model input");
      concat_bwd(Z.grad, n, ap.g.H, ap.g.W, T[nd.res].C, T[nd.in].C, ap.pk, ap.ps, ap.pp, Z.H, Z.W, T[nd.in].grad, sc,
                 st);
      continue;
    }
    if (nd.kind == N_POOL) {
      const TensorRt& X = T[nd.in];
      if (nd.in == 0) continue;
      if (stem_pool_fused && ni == stem_pool) continue;  // inside the stem weight gradient
      launch_maxpool_bwd(T[nd.out].grad, nd.argmax.as<uint8_t>(), T[nd.out].buf, X.act, n, X.H, X.W, X.C, nd.pk, nd.ps, nd.pp,
                         nd.g.Ho, nd.g.Wo, T[nd.in].grad, st);
      continue;
    }
    const bf16* dz = T[nd.out].grad;
    if (nd.res >= 0 && T[nd.res].producer >= 0 && nodes[T[nd.res].producer].kind == N_PROJ) {
      // projection shortcut: its output gradient is this conv's dZ; do it before the block's first conv
      conv_backward(nd, dz);
      conv_backward(nodes[T[nd.res].producer], dz);
    } else {
      conv_backward(nd, dz);
    }
  }
  if (stats) launch_sum(loss_rows.as<float>(), n, &stats->loss, 0.f, st);
}

void Model::update_impl(float lr, adainf_step_stats* stats, cudaStream_t st) {
  if (!train_ready) throw InvalidError("update: no gradient has been computed on this model");
  float* G = grads.as<float>();
#ifdef ADAINF_WITH_NCCL
  if (comm && dp_world > 1) {
    ncclResult_t r = ncclAllReduce(G, G, (size_t)nparams, ncclFloat, ncclSum, comm, st);
    if (r != ncclSuccess) throw NcclError(std::string("NCCL all-reduce: ") + ncclGetErrorString(r));
  }
#endif
  // fused SGD + momentum + shadow refresh (K10)
  launch_sgd(params.as<float>(), mom.as<float>(), G, nparams, lr, momentum, weight_decay, sgd_segs.as<SgdSeg>(),
             sgd_nseg, sgd_block_seg.as<int>(), sgd_block_start.as<long long>(), sgd_nblocks, sq_partial.as<float>(),
             st);
  if (stats) launch_sum(sq_partial.as<float>(), sgd_nblocks, &stats->grad_norm, -1.f, st);
}

}  // namespace adainf

// AdaInf hot-path ORACLE — TEST INFRASTRUCTURE ONLY (see oracle.h header comment).
//
// Plain direct loops, fp64 accumulation, bf16 rounding (RNE) at the storage points of DESIGN.md
// "Numerics contract".  Citations: P:L = /root/reference/PAPER.md line L; "c.1 step N" = the
// step-by-step definition in SURVEY.md §8(c).  Built with -O2 -ffp-contract=off -fno-fast-math.
#include "oracle.h"

#include <math.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include <algorithm>
#include <vector>
#ifdef _OPENMP
#include <omp.h>
#endif

using std::vector;

// ------------------------------------------------------------------------------------------------
// bf16: round-to-nearest-even on the fp32 bit pattern (c.1 step 1).  Pinned by tests against
// torch.Tensor.to(torch.bfloat16) on hand-picked ties and random values.
extern "C" float or_bf16(float x) {
  uint32_t u;
  memcpy(&u, &x, 4);
  if ((u & 0x7f800000u) == 0x7f800000u) return x;  // inf / nan untouched (never on valid inputs)
  u += 0x7fffu + ((u >> 16) & 1u);
  u &= 0xffff0000u;
  float y;
  memcpy(&y, &u, 4);
  return y;
}
extern "C" void or_bf16_array(const float* x, float* y, int64_t n) {
  for (int64_t i = 0; i < n; ++i) y[i] = or_bf16(x[i]);
}

static int g_threads = 0;
extern "C" void or_set_threads(int n) {
  g_threads = n;
#ifdef _OPENMP
  if (n > 0) omp_set_num_threads(n);
#endif
}
extern "C" int or_get_threads(void) {
#ifdef _OPENMP
  return omp_get_max_threads();
#else
  return 1;
#endif
}

// ------------------------------------------------------------------------------------------------
// Conv forward accumulation (c.1 step 2): acc[ho][wo][co] = sum_{kh,kw,ci} x[ho*s-p+kh][wo*s-p+kw][ci]
// * w[co][kh][kw][ci], zero padding, fp64 sum of exact products, cast to fp32.
extern "C" void or_conv_acc(const float* x, int H, int W, int C, const float* w, int Co, int KH, int KW,
                            int s, int p, float* acc, int* pHo, int* pWo) {
  const int Ho = (H + 2 * p - KH) / s + 1, Wo = (W + 2 * p - KW) / s + 1;
  if (pHo) *pHo = Ho;
  if (pWo) *pWo = Wo;
  for (int ho = 0; ho < Ho; ++ho)
    for (int wo = 0; wo < Wo; ++wo)
      for (int co = 0; co < Co; ++co) {
        double a = 0.0;
        for (int kh = 0; kh < KH; ++kh) {
          const int ih = ho * s - p + kh;
          if (ih < 0 || ih >= H) continue;
          for (int kw = 0; kw < KW; ++kw) {
            const int iw = wo * s - p + kw;
            if (iw < 0 || iw >= W) continue;
            const float* xp = x + ((int64_t)ih * W + iw) * C;
            const float* wp = w + (((int64_t)co * KH + kh) * KW + kw) * C;
            for (int ci = 0; ci < C; ++ci) a += (double)xp[ci] * (double)wp[ci];
          }
        }
        acc[((int64_t)ho * Wo + wo) * Co + co] = (float)a;
      }
}

// Max pooling on stored values, padding = -inf (c.1 step 2, "optional maxpool").
extern "C" void or_maxpool(const float* x, int H, int W, int C, int K, int s, int p, float* y, int* pHo,
                           int* pWo) {
  const int Ho = (H + 2 * p - K) / s + 1, Wo = (W + 2 * p - K) / s + 1;
  if (pHo) *pHo = Ho;
  if (pWo) *pWo = Wo;
  for (int ho = 0; ho < Ho; ++ho)
    for (int wo = 0; wo < Wo; ++wo)
      for (int c = 0; c < C; ++c) {
        float m = -INFINITY;
        for (int kh = 0; kh < K; ++kh)
          for (int kw = 0; kw < K; ++kw) {
            const int ih = ho * s - p + kh, iw = wo * s - p + kw;
            if (ih < 0 || ih >= H || iw < 0 || iw >= W) continue;
            const float v = x[((int64_t)ih * W + iw) * C + c];
            if (v > m) m = v;
          }
        y[((int64_t)ho * Wo + wo) * C + c] = m;
      }
}

// Softmax statistics (c.1 step 3; exit criterion reading Q1/Q5/Q6/Q7): m = max l, s = sum exp(l-m),
// conf = 1/s, H = log s - sum exp(l-m)(l-m)/s, pred = lowest argmax.  fp64, cast to fp32.
extern "C" void or_softmax_stats(const float* l, int n, float* conf, float* ent, int32_t* pred) {
  int am = 0;
  for (int j = 1; j < n; ++j)
    if (l[j] > l[am]) am = j;
  const double m = l[am];
  double s = 0.0, t = 0.0;
  for (int j = 0; j < n; ++j) {
    const double e = exp((double)l[j] - m);
    s += e;
    t += e * ((double)l[j] - m);
  }
  if (conf) *conf = (float)(1.0 / s);
  if (ent) *ent = (float)(log(s) - t / s);
  if (pred) *pred = am;
}

// Exit head ("early-exit structures", reading Q4): GAP -> FC (fp32 weights) -> softmax stats.
extern "C" void or_exit_head(const float* f, int H, int W, int C, const float* Wk, const float* bk,
                             int ncls, float* pooled, float* logits, float* conf, float* ent,
                             int32_t* pred) {
  vector<double> acc(C, 0.0);
  for (int i = 0; i < H * W; ++i)
    for (int c = 0; c < C; ++c) acc[c] += (double)f[(int64_t)i * C + c];
  for (int c = 0; c < C; ++c) pooled[c] = (float)(acc[c] / (double)(H * W));
  for (int j = 0; j < ncls; ++j) {
    double a = (double)bk[j];
    for (int c = 0; c < C; ++c) a += (double)pooled[c] * (double)Wk[(int64_t)c * ncls + j];
    logits[j] = (float)a;
  }
  or_softmax_stats(logits, ncls, conf, ent, pred);
}

// ------------------------------------------------------------------------------------------------
// Model description walk.  Parameter layout (flat fp32, in op order — same documented layout as the
// ABI header, re-derived here): CONV W[co][kh][kw][ci] then b[co]; BLOCK with cout>0: W[co][1][1][ci]
// then b[co]; EXIT: Wk[C][ncls] then bk[ncls]; MAXPOOL/DET_HEAD: none.
namespace {

struct Shape3 {
  int H, W, C;
};

struct Walk {
  vector<Shape3> in_shape;   // per op: shape of the current tensor entering the op
  vector<Shape3> out_shape;  // per op: shape of its output (CONV/MAXPOOL), shortcut (BLOCK), input (EXIT)
  vector<int64_t> poff;      // per op: parameter offset
  vector<Shape3> cur_after;  // per op: the current tensor after the op (ROUTE sources)
  bool inference_only = false;  // UPSAMPLE / ROUTE present
  int64_t nparams = 0;
  int nexits = 0;
  int ncls = 0;
  bool ok = true;
};

Walk walk(const or_model* m) {
  Walk w;
  Shape3 cur{m->in_h, m->in_w, m->in_c};
  vector<Shape3> blocks;
  for (int i = 0; i < m->n_ops; ++i) {
    const or_op& op = m->ops[i];
    w.in_shape.push_back(cur);
    w.poff.push_back(w.nparams);
    struct After {  // record the current tensor after this op, whichever branch ran
      Walk& w;
      Shape3& cur;
      ~After() { w.cur_after.push_back(cur); }
    } after{w, cur};
    switch (op.kind) {
      case OR_CONV: {
        Shape3 o{(cur.H + 2 * op.pad - op.kh) / op.stride + 1, (cur.W + 2 * op.pad - op.kw) / op.stride + 1,
                 op.cout};
        const int g = op.groups > 0 ? op.groups : 1;
        if (cur.C % g || op.cout % g) w.ok = false;
        w.nparams += (int64_t)op.cout * op.kh * op.kw * (cur.C / g) + op.cout;
        if (op.residual) {
          if (blocks.empty()) w.ok = false;
          else {
            const Shape3 b = blocks.back();
            if (op.residual == 2) {  // concat [shortcut, conv] (ShuffleNet stride-2 unit)
              if (b.H != o.H || b.W != o.W) w.ok = false;
              o.C = b.C + op.cout;
            } else if (b.H != o.H || b.W != o.W || b.C != o.C) {
              w.ok = false;
            }
            blocks.pop_back();
          }
        }
        cur = o;
        w.out_shape.push_back(o);
        break;
      }
      case OR_MAXPOOL: {
        Shape3 o{(cur.H + 2 * op.pad - op.kh) / op.stride + 1, (cur.W + 2 * op.pad - op.kw) / op.stride + 1,
                 cur.C};
        cur = o;
        w.out_shape.push_back(o);
        break;
      }
      case OR_BLOCK: {
        if (op.cout > 0) {
          Shape3 o{(cur.H - 1) / op.stride + 1, (cur.W - 1) / op.stride + 1, op.cout};
          w.nparams += (int64_t)op.cout * cur.C + op.cout;
          blocks.push_back(o);
          w.out_shape.push_back(o);
        } else if (op.pool) {  // average-pool shortcut (ShuffleNet)
          Shape3 o{(cur.H + 2 * op.pad - op.kh) / op.stride + 1, (cur.W + 2 * op.pad - op.kw) / op.stride + 1, cur.C};
          blocks.push_back(o);
          w.out_shape.push_back(o);
        } else {
          blocks.push_back(cur);
          w.out_shape.push_back(cur);
        }
        break;
      }
      case OR_SHUFFLE: {
        if (op.groups <= 0 || cur.C % op.groups) w.ok = false;
        w.out_shape.push_back(cur);
        break;
      }
      case OR_EXIT: {
        w.nparams += (int64_t)cur.C * op.num_classes + op.num_classes;
        if (w.nexits == 0) w.ncls = op.num_classes;
        else if (w.ncls != op.num_classes) w.ok = false;
        w.nexits++;
        w.out_shape.push_back(cur);
        break;
      }
      case OR_DET_HEAD:
        w.out_shape.push_back(cur);
        break;
      case OR_UPSAMPLE: {
        if (op.stride < 1) w.ok = false;
        cur = Shape3{cur.H * op.stride, cur.W * op.stride, cur.C};
        w.out_shape.push_back(cur);
        w.inference_only = true;
        break;
      }
      case OR_ROUTE: {
        if (op.kh < 0 || op.kh >= i || op.kw >= i) {
          w.ok = false;
          w.out_shape.push_back(cur);
          break;
        }
        Shape3 o = w.cur_after[op.kh];
        if (op.kw >= 0) {
          const Shape3 b = w.cur_after[op.kw];
          if (b.H != o.H || b.W != o.W) w.ok = false;
          o.C += b.C;
        }
        cur = o;
        w.out_shape.push_back(o);
        w.inference_only = true;
        break;
      }
      default:
        w.ok = false;
        w.out_shape.push_back(cur);
    }
  }
  return w;
}

inline double act_f(int act, double v, bool exact) {
  if (act == 1) return v > 0 ? v : 0.0;
  if (act == 3) return v > 0 ? (v < 6.0 ? v : 6.0) : 0.0;  // ReLU6 (MobileNetV2, NEXT-3)
  if (act == 2) return v > 0 ? v : (exact ? 0.1 * v : (double)(0.1f * (float)v));  // fp32 0.1f*x (c.1 step 2)
  return v;
}
inline double act_d(int act, double y) {  // derivative from the stored output (ReLU'(0) = 0)
  if (act == 1) return y > 0 ? 1.0 : 0.0;
  if (act == 3) return (y > 0 && y < 6.0) ? 1.0 : 0.0;  // ReLU6: 0 at both clamps
  if (act == 2) return y > 0 ? 1.0 : 0.1;
  return 1.0;
}

// Forward/backward engine for ONE sample.  `exact` = pure fp64 (no bf16 / fp32 casts), used only by
// the finite-difference pins; otherwise rounding follows DESIGN.md "Numerics contract".
struct Engine {
  const or_model* m;
  const Walk& w;
  bool exact;
  Engine(const or_model* m_, const Walk& w_, bool exact_) : m(m_), w(w_), exact(exact_) {}

  double R(double v) const { return exact ? v : (double)or_bf16((float)v); }  // bf16 storage
  double F(double v) const { return exact ? v : (double)(float)v; }           // fp32 storage

  struct Tensor {
    int H = 0, W = 0, C = 0;
    vector<double> d;
  };
  struct Node {  // forward node, in op order
    int kind;    // OR_CONV, OR_MAXPOOL, OR_BLOCK(projection only)
    int op;
    int in, out, res;
  };
  vector<Tensor> T;
  vector<Node> nodes;
  vector<int> exit_tensor, exit_op;  // per exit
  vector<vector<double>> pooled, logits;
  vector<int> det_tensors;  // DET_HEAD inputs, op order
  vector<int> op_tensor;    // current tensor after each op (ROUTE sources)

  // conv with weights taken from params (bf16-rounded unless exact)
  // grouped conv (groups = 1: dense): output channel co reads input channels [g*Cg, (g+1)*Cg) of its group
  // g = co / (Co / groups), weights [Co][KH][KW][Cg]
  void conv(const Tensor& x, const double* Wf, const double* bf, int Co, int KH, int KW, int s, int p,
            vector<double>& acc, int& Ho, int& Wo, int groups = 1) const {
    const int Cg = x.C / groups, Cog = Co / groups;
    Ho = (x.H + 2 * p - KH) / s + 1;
    Wo = (x.W + 2 * p - KW) / s + 1;
    acc.assign((size_t)Ho * Wo * Co, 0.0);
    for (int ho = 0; ho < Ho; ++ho)
      for (int wo = 0; wo < Wo; ++wo)
        for (int co = 0; co < Co; ++co) {
          double a = 0.0;
          for (int kh = 0; kh < KH; ++kh) {
            const int ih = ho * s - p + kh;
            if (ih < 0 || ih >= x.H) continue;
            for (int kw = 0; kw < KW; ++kw) {
              const int iw = wo * s - p + kw;
              if (iw < 0 || iw >= x.W) continue;
              const double* xp = &x.d[((size_t)ih * x.W + iw) * x.C + (size_t)(co / Cog) * Cg];
              const double* wp = Wf + (((int64_t)co * KH + kh) * KW + kw) * Cg;
              if (exact)
                for (int ci = 0; ci < Cg; ++ci) a += xp[ci] * wp[ci];
              else
                for (int ci = 0; ci < Cg; ++ci) a += xp[ci] * (double)or_bf16((float)wp[ci]);
            }
          }
          // epilogue step 1: fp32 accumulator, then "+ b" in fp32
          acc[((size_t)ho * Wo + wo) * Co + co] = F(F(a) + (double)bf[co]);
        }
  }

  void forward(const double* params, const float* x) {
    T.clear();
    nodes.clear();
    exit_tensor.clear();
    exit_op.clear();
    pooled.clear();
    logits.clear();
    Tensor in;
    in.H = m->in_h;
    in.W = m->in_w;
    in.C = m->in_c;
    in.d.resize((size_t)in.H * in.W * in.C);
    for (size_t i = 0; i < in.d.size(); ++i) in.d[i] = exact ? (double)x[i] : (double)or_bf16(x[i]);
    T.push_back(std::move(in));
    det_tensors.clear();
    op_tensor.clear();
    int cur = 0;
    vector<int> blocks;
    for (int i = 0; i < m->n_ops; ++i) {
      const or_op& op = m->ops[i];
      const double* P = params + w.poff[i];
      if (op.kind == OR_CONV) {
        const Tensor& X = T[cur];
        const int Cin = X.C;
        Tensor Y;
        vector<double> acc;
        const int grp = op.groups > 0 ? op.groups : 1;
        conv(X, P, P + (int64_t)op.cout * op.kh * op.kw * (Cin / grp), op.cout, op.kh, op.kw, op.stride, op.pad, acc,
             Y.H, Y.W, grp);
        Y.C = op.cout;
        int res = -1;
        if (op.residual) {
          res = blocks.back();
          blocks.pop_back();
          const Tensor& S = T[res];
          if (op.residual == 1)
            for (size_t e = 0; e < acc.size(); ++e) acc[e] = F(acc[e] + S.d[e]);  // "+ float(residual)"
        }
        // det-head input (act none, followed by DET_HEAD) stays fp32; everything else bf16
        const bool fp32_out = (i + 1 < m->n_ops && m->ops[i + 1].kind == OR_DET_HEAD);
        if (op.residual == 2) {
          // concat along channels: [act(shortcut), act(conv)] (ShuffleNet: ReLU after the concat), bf16
          const Tensor& S = T[res];
          const int Cs = S.C, Co = op.cout;
          Y.C = Cs + Co;
          Y.d.resize((size_t)Y.H * Y.W * Y.C);
          for (int e = 0; e < Y.H * Y.W; ++e) {
            for (int c = 0; c < Cs; ++c) Y.d[(size_t)e * Y.C + c] = R(F(act_f(op.act, S.d[(size_t)e * Cs + c], exact)));
            for (int c = 0; c < Co; ++c)
              Y.d[(size_t)e * Y.C + Cs + c] = R(F(act_f(op.act, acc[(size_t)e * Co + c], exact)));
          }
        } else {
          Y.d.resize(acc.size());
          for (size_t e = 0; e < acc.size(); ++e) {
            const double v = F(act_f(op.act, acc[e], exact));
            Y.d[e] = fp32_out ? v : R(v);
          }
        }
        T.push_back(std::move(Y));
        nodes.push_back({OR_CONV, i, cur, (int)T.size() - 1, res});
        cur = (int)T.size() - 1;
      } else if (op.kind == OR_MAXPOOL) {
        const Tensor& X = T[cur];
        Tensor Y;
        Y.H = (X.H + 2 * op.pad - op.kh) / op.stride + 1;
        Y.W = (X.W + 2 * op.pad - op.kw) / op.stride + 1;
        Y.C = X.C;
        Y.d.assign((size_t)Y.H * Y.W * Y.C, 0.0);
        for (int ho = 0; ho < Y.H; ++ho)
          for (int wo = 0; wo < Y.W; ++wo)
            for (int c = 0; c < Y.C; ++c) {
              double mx = -INFINITY;
              for (int kh = 0; kh < op.kh; ++kh)
                for (int kw = 0; kw < op.kw; ++kw) {
                  const int ih = ho * op.stride - op.pad + kh, iw = wo * op.stride - op.pad + kw;
                  if (ih < 0 || ih >= X.H || iw < 0 || iw >= X.W) continue;
                  mx = std::max(mx, X.d[((size_t)ih * X.W + iw) * X.C + c]);
                }
              Y.d[((size_t)ho * Y.W + wo) * Y.C + c] = mx;
            }
        T.push_back(std::move(Y));
        nodes.push_back({OR_MAXPOOL, i, cur, (int)T.size() - 1, -1});
        cur = (int)T.size() - 1;
      } else if (op.kind == OR_BLOCK) {
        if (op.cout > 0) {  // 1x1 projection shortcut, no activation, stored bf16
          const Tensor& X = T[cur];
          Tensor Y;
          vector<double> acc;
          conv(X, P, P + (int64_t)op.cout * X.C, op.cout, 1, 1, op.stride, 0, acc, Y.H, Y.W);
          Y.C = op.cout;
          Y.d.resize(acc.size());
          for (size_t e = 0; e < acc.size(); ++e) Y.d[e] = R(acc[e]);
          T.push_back(std::move(Y));
          nodes.push_back({OR_BLOCK, i, cur, (int)T.size() - 1, -1});
          blocks.push_back((int)T.size() - 1);
        } else if (op.pool) {
          // average-pool shortcut: fp64 sum of the window (zero padding), fp32, / (kh*kw) in fp32, bf16
          const Tensor& X = T[cur];
          Tensor Y;
          Y.H = (X.H + 2 * op.pad - op.kh) / op.stride + 1;
          Y.W = (X.W + 2 * op.pad - op.kw) / op.stride + 1;
          Y.C = X.C;
          Y.d.assign((size_t)Y.H * Y.W * Y.C, 0.0);
          for (int ho = 0; ho < Y.H; ++ho)
            for (int wo = 0; wo < Y.W; ++wo)
              for (int c = 0; c < Y.C; ++c) {
                double a = 0.0;
                for (int kh = 0; kh < op.kh; ++kh)
                  for (int kw = 0; kw < op.kw; ++kw) {
                    const int ih = ho * op.stride - op.pad + kh, iw = wo * op.stride - op.pad + kw;
                    if (ih < 0 || ih >= X.H || iw < 0 || iw >= X.W) continue;
                    a += X.d[((size_t)ih * X.W + iw) * X.C + c];
                  }
                Y.d[((size_t)ho * Y.W + wo) * Y.C + c] = R(F(F(a) / (double)(op.kh * op.kw)));
              }
          T.push_back(std::move(Y));
          nodes.push_back({OR_BLOCK, i, cur, (int)T.size() - 1, -1});
          blocks.push_back((int)T.size() - 1);
        } else {
          blocks.push_back(cur);
        }
      } else if (op.kind == OR_SHUFFLE) {
        // channel shuffle: channel c = gi*(C/g) + j of the input moves to position j*g + gi (view (g, C/g),
        // transpose, flatten); values unchanged
        const Tensor& X = T[cur];
        Tensor Y;
        Y.H = X.H;
        Y.W = X.W;
        Y.C = X.C;
        Y.d.assign(X.d.size(), 0.0);
        const int g = op.groups, Cg = X.C / g;
        for (int e = 0; e < X.H * X.W; ++e)
          for (int gi = 0; gi < g; ++gi)
            for (int j = 0; j < Cg; ++j) Y.d[(size_t)e * X.C + j * g + gi] = X.d[(size_t)e * X.C + gi * Cg + j];
        T.push_back(std::move(Y));
        nodes.push_back({OR_SHUFFLE, i, cur, (int)T.size() - 1, -1});
        cur = (int)T.size() - 1;
      } else if (op.kind == OR_EXIT) {
        const Tensor& X = T[cur];
        const int ncls = op.num_classes;
        vector<double> pl(X.C), lg(ncls);
        for (int c = 0; c < X.C; ++c) {
          double a = 0.0;
          for (int e = 0; e < X.H * X.W; ++e) a += X.d[(size_t)e * X.C + c];
          pl[c] = F(a / (double)(X.H * X.W));
        }
        const double* Wk = P;
        const double* bk = P + (int64_t)X.C * ncls;
        for (int j = 0; j < ncls; ++j) {
          double a = (double)bk[j];
          for (int c = 0; c < X.C; ++c) a += pl[c] * (double)Wk[(int64_t)c * ncls + j];
          lg[j] = F(a);
        }
        pooled.push_back(pl);
        logits.push_back(lg);
        exit_tensor.push_back(cur);
        exit_op.push_back(i);
      } else if (op.kind == OR_DET_HEAD) {
        det_tensors.push_back(cur);
      } else if (op.kind == OR_UPSAMPLE) {  // nearest: Y[h][w] = X[h / s][w / s]
        const Tensor& X = T[cur];
        Tensor Y;
        Y.H = X.H * op.stride;
        Y.W = X.W * op.stride;
        Y.C = X.C;
        Y.d.resize((size_t)Y.H * Y.W * Y.C);
        for (int h = 0; h < Y.H; ++h)
          for (int ww = 0; ww < Y.W; ++ww)
            for (int c = 0; c < Y.C; ++c)
              Y.d[((size_t)h * Y.W + ww) * Y.C + c] = X.d[((size_t)(h / op.stride) * X.W + ww / op.stride) * X.C + c];
        T.push_back(std::move(Y));
        cur = (int)T.size() - 1;
      } else if (op.kind == OR_ROUTE) {  // [output of op kh, output of op kw] along channels
        const int ta = op_tensor[op.kh];
        if (op.kw < 0) {
          cur = ta;
        } else {
          const int tb = op_tensor[op.kw];
          Tensor Y;
          Y.H = T[ta].H;
          Y.W = T[ta].W;
          Y.C = T[ta].C + T[tb].C;
          Y.d.resize((size_t)Y.H * Y.W * Y.C);
          for (int e = 0; e < Y.H * Y.W; ++e) {
            for (int c = 0; c < T[ta].C; ++c) Y.d[(size_t)e * Y.C + c] = T[ta].d[(size_t)e * T[ta].C + c];
            for (int c = 0; c < T[tb].C; ++c) Y.d[(size_t)e * Y.C + T[ta].C + c] = T[tb].d[(size_t)e * T[tb].C + c];
          }
          T.push_back(std::move(Y));
          cur = (int)T.size() - 1;
        }
      }
      op_tensor.push_back(cur);
    }
  }

  // Backward (c.1 steps 10-11) for one sample; accumulates param grads (fp64) into g.
  // Returns this sample's loss contribution sum_k w_k CE_k / n_global.
  double backward(const double* params, int label, double inv_n, double* g) {
    const int nt = (int)T.size();
    vector<vector<double>> prim(nt), bc(nt), sc(nt);
    auto ensure = [&](vector<double>& v, int t) {
      if (v.empty()) v.assign(T[t].d.size(), 0.0);
    };
    double loss = 0.0;
    // exit heads first: loss, head grads, broadcast of dpooled/(H*W) into the exit's input tensor
    for (size_t k = 0; k < exit_op.size(); ++k) {
      const or_op& op = m->ops[exit_op[k]];
      const int t = exit_tensor[k];
      const Tensor& X = T[t];
      const int ncls = op.num_classes;
      const double* Wk = params + w.poff[exit_op[k]];
      double* gW = g + w.poff[exit_op[k]];
      double* gb = gW + (int64_t)X.C * ncls;
      const vector<double>& lg = logits[k];
      double mx = lg[0];
      for (int j = 1; j < ncls; ++j) mx = std::max(mx, lg[j]);
      double s = 0.0;
      for (int j = 0; j < ncls; ++j) s += exp(lg[j] - mx);
      const double lw = (double)op.loss_weight;
      loss += lw * (-(lg[label] - mx - log(s))) * inv_n;
      vector<double> dl(ncls);
      for (int j = 0; j < ncls; ++j) dl[j] = F(lw * (exp(lg[j] - mx) / s - (j == label ? 1.0 : 0.0)) * inv_n);
      for (int c = 0; c < X.C; ++c)
        for (int j = 0; j < ncls; ++j) gW[(int64_t)c * ncls + j] += pooled[k][c] * dl[j];
      for (int j = 0; j < ncls; ++j) gb[j] += dl[j];
      ensure(bc[t], t);
      const double inv_hw = F(1.0 / (double)(X.H * X.W));
      for (int c = 0; c < X.C; ++c) {
        double dp = 0.0;
        for (int j = 0; j < ncls; ++j) dp += dl[j] * (double)Wk[(int64_t)c * ncls + j];
        const double v = F(F(dp) * inv_hw);
        for (int e = 0; e < X.H * X.W; ++e) bc[t][(size_t)e * X.C + c] = F(bc[t][(size_t)e * X.C + c] + v);
      }
    }
    // total incoming gradient of tensor t, in the GPU epilogue's order: prim + bcast + shortcut
    auto total = [&](int t) {
      vector<double> r(T[t].d.size(), 0.0);
      for (size_t e = 0; e < r.size(); ++e) {
        double v = prim[t].empty() ? 0.0 : F(prim[t][e]);
        if (!bc[t].empty()) v = F(v + bc[t][e]);
        if (!sc[t].empty()) v = F(v + sc[t][e]);
        r[e] = v;
      }
      return r;
    };
    for (int ni = (int)nodes.size() - 1; ni >= 0; --ni) {
      const Node& nd = nodes[ni];
      const or_op& op = m->ops[nd.op];
      const Tensor& X = T[nd.in];
      const Tensor& Y = T[nd.out];
      if (nd.kind == OR_MAXPOOL) {
        vector<double> dT = total(nd.out);
        for (auto& v : dT) v = R(v);
        ensure(prim[nd.in], nd.in);
        // route each window's gradient to its FIRST maximal element (row-major window order)
        for (int ho = 0; ho < Y.H; ++ho)
          for (int wo = 0; wo < Y.W; ++wo)
            for (int c = 0; c < Y.C; ++c) {
              double mx = -INFINITY;
              int best = -1;
              for (int kh = 0; kh < op.kh; ++kh)
                for (int kw = 0; kw < op.kw; ++kw) {
                  const int ih = ho * op.stride - op.pad + kh, iw = wo * op.stride - op.pad + kw;
                  if (ih < 0 || ih >= X.H || iw < 0 || iw >= X.W) continue;
                  const int idx = (ih * X.W + iw) * X.C + c;
                  if (X.d[idx] > mx) {
                    mx = X.d[idx];
                    best = idx;
                  }
                }
              prim[nd.in][best] += dT[((size_t)ho * Y.W + wo) * Y.C + c];
            }
        continue;
      }
      if (nd.kind == OR_SHUFFLE) {  // a permutation: the gradient moves back unchanged
        const vector<double> dT = total(nd.out);
        ensure(prim[nd.in], nd.in);
        const int g = op.groups, Cg = X.C / g;
        for (int e = 0; e < X.H * X.W; ++e)
          for (int gi = 0; gi < g; ++gi)
            for (int j = 0; j < Cg; ++j) prim[nd.in][(size_t)e * X.C + gi * Cg + j] += dT[(size_t)e * X.C + j * g + gi];
        continue;
      }
      if (nd.kind == OR_BLOCK && op.pool) {
        // average-pool shortcut backward: each window's gradient / (kh*kw) to its in-range taps, summed in fp64,
        // divided in fp32 and stored bf16, then added as the block input's shortcut term (like a projection's dgrad)
        const vector<double> dS = total(nd.out);
        vector<double> a(X.d.size(), 0.0);
        for (int ho = 0; ho < Y.H; ++ho)
          for (int wo = 0; wo < Y.W; ++wo)
            for (int c = 0; c < Y.C; ++c)
              for (int kh = 0; kh < op.kh; ++kh)
                for (int kw = 0; kw < op.kw; ++kw) {
                  const int ih = ho * op.stride - op.pad + kh, iw = wo * op.stride - op.pad + kw;
                  if (ih < 0 || ih >= X.H || iw < 0 || iw >= X.W) continue;
                  a[((size_t)ih * X.W + iw) * X.C + c] += dS[((size_t)ho * Y.W + wo) * Y.C + c];
                }
        if (nd.in != 0) {
          ensure(sc[nd.in], nd.in);
          for (size_t e = 0; e < a.size(); ++e)
            sc[nd.in][e] = F(sc[nd.in][e] + R(F(F(a[e]) / (double)(op.kh * op.kw))));
        }
        continue;
      }
      // CONV or BLOCK projection
      const int KH = nd.kind == OR_CONV ? op.kh : 1, KW = nd.kind == OR_CONV ? op.kw : 1;
      const bool concat = nd.kind == OR_CONV && op.residual == 2;
      const int Cs = concat ? T[nd.res].C : 0;  // concat: the conv's channels sit after the shortcut's
      const int s = op.stride, p = nd.kind == OR_CONV ? op.pad : 0, Co = Y.C - Cs, Ci = X.C;
      const int act = nd.kind == OR_CONV ? op.act : 0;
      const int grp = (nd.kind == OR_CONV && op.groups > 0) ? op.groups : 1;
      const int Cg = Ci / grp, Cog = Co / grp;
      const vector<double> dY = total(nd.out);
      vector<double> dZ((size_t)Y.H * Y.W * Co);
      for (int e = 0; e < Y.H * Y.W; ++e)
        for (int c = 0; c < Co; ++c) {
          const size_t yi = (size_t)e * Y.C + Cs + c;
          dZ[(size_t)e * Co + c] = R(F(dY[yi] * act_d(act, Y.d[yi])));
        }
      if (concat) {  // shortcut part: masked by the act of the stored concat output, bf16, into the shortcut tensor
        ensure(sc[nd.res], nd.res);
        for (int e = 0; e < Y.H * Y.W; ++e)
          for (int c = 0; c < Cs; ++c) {
            const size_t yi = (size_t)e * Y.C + c;
            sc[nd.res][(size_t)e * Cs + c] = F(sc[nd.res][(size_t)e * Cs + c] + R(F(dY[yi] * act_d(act, Y.d[yi]))));
          }
      }
      const double* Wf = params + w.poff[nd.op];
      double* gW = g + w.poff[nd.op];
      double* gb = gW + (int64_t)Co * KH * KW * Cg;
      const bool need_dx = nd.in != 0;
      vector<double> dX;
      if (need_dx) dX.assign(X.d.size(), 0.0);
      for (int ho = 0; ho < Y.H; ++ho)
        for (int wo = 0; wo < Y.W; ++wo)
          for (int co = 0; co < Co; ++co) {
            const double dz = dZ[((size_t)ho * Y.W + wo) * Co + co];
            if (dz == 0.0) continue;
            gb[co] += dz;
            for (int kh = 0; kh < KH; ++kh) {
              const int ih = ho * s - p + kh;
              if (ih < 0 || ih >= X.H) continue;
              for (int kw = 0; kw < KW; ++kw) {
                const int iw = wo * s - p + kw;
                if (iw < 0 || iw >= X.W) continue;
                const size_t xo = ((size_t)ih * X.W + iw) * Ci + (size_t)(co / Cog) * Cg;
                const int64_t wo_ = (((int64_t)co * KH + kh) * KW + kw) * Cg;
                for (int ci = 0; ci < Cg; ++ci) {
                  gW[wo_ + ci] += dz * X.d[xo + ci];
                  if (need_dx) dX[xo + ci] += dz * (exact ? Wf[wo_ + ci] : (double)or_bf16((float)Wf[wo_ + ci]));
                }
              }
            }
          }
      if (need_dx) {
        if (nd.kind == OR_BLOCK) {  // projection dgrad stored bf16, then added as the shortcut term
          ensure(sc[nd.in], nd.in);
          for (size_t e = 0; e < dX.size(); ++e) sc[nd.in][e] = F(sc[nd.in][e] + R(F(dX[e])));
        } else {
          ensure(prim[nd.in], nd.in);
          for (size_t e = 0; e < dX.size(); ++e) prim[nd.in][e] += dX[e];
        }
      }
      if (nd.kind == OR_CONV && nd.res >= 0 && !concat) {  // residual add: dZ flows unchanged into the shortcut
        ensure(sc[nd.res], nd.res);
        for (size_t e = 0; e < dZ.size(); ++e) sc[nd.res][e] = F(sc[nd.res][e] + dZ[e]);
      }
    }
    return loss;
  }
};

}  // namespace

extern "C" int64_t or_num_params(const or_model* m) { return walk(m).nparams; }
extern "C" int32_t or_num_exits(const or_model* m) { return walk(m).nexits; }
extern "C" int or_tensor_shape(const or_model* m, int op_idx, int* H, int* W, int* C) {
  Walk w = walk(m);
  if (!w.ok || op_idx < 0 || op_idx >= m->n_ops) return -1;
  *H = w.out_shape[op_idx].H;
  *W = w.out_shape[op_idx].W;
  *C = w.out_shape[op_idx].C;
  return 0;
}

extern "C" int or_forward(const or_model* m, const float* params, const float* x, int B, float* conf,
                          float* ent, int32_t* pred, float* logits, float* pooled0, float* det_raw) {
  Walk w = walk(m);
  if (!w.ok) return -1;
  const int E = w.nexits, ncls = w.ncls;
  const int64_t in_sz = (int64_t)m->in_h * m->in_w * m->in_c;
  const vector<double> pd(params, params + w.nparams);
  int rc = 0;
#pragma omp parallel for schedule(dynamic, 1)
  for (int n = 0; n < B; ++n) {
    Engine eng(m, w, false);
    eng.forward(pd.data(), x + n * in_sz);
    for (int k = 0; k < E; ++k) {
      float c, h;
      int32_t pr;
      vector<float> lg(ncls);
      for (int j = 0; j < ncls; ++j) lg[j] = (float)eng.logits[k][j];
      or_softmax_stats(lg.data(), ncls, &c, &h, &pr);
      if (conf) conf[(int64_t)n * E + k] = c;
      if (ent) ent[(int64_t)n * E + k] = h;
      if (pred) pred[(int64_t)n * E + k] = pr;
      if (logits)
        for (int j = 0; j < ncls; ++j) logits[((int64_t)n * E + k) * ncls + j] = lg[j];
    }
    if (pooled0 && E > 0) {
      const int C0 = (int)eng.pooled[0].size();
      for (int c = 0; c < C0; ++c) pooled0[(int64_t)n * C0 + c] = (float)eng.pooled[0][c];
    }
    if (det_raw) {
      if (eng.det_tensors.empty()) {
        rc = -2;
      } else {
        size_t per = 0;
        for (int t : eng.det_tensors) per += eng.T[t].d.size();
        size_t o = (size_t)n * per;
        for (int t : eng.det_tensors)
          for (double v : eng.T[t].d) det_raw[o++] = (float)v;
      }
    }
  }
  return rc;
}

// Exit rule (reading Q1/Q5: exit at the smallest k < E-1 with conf_k >= tau_k, else the final exit)
// and stable compaction (c.1 step 5), brute force.
extern "C" void or_exit_assign(const float* conf, int B, int E, const float* tau, int8_t* exit_id,
                               int32_t* surv, int32_t* counts) {
  for (int k = 0; k < E; ++k) counts[k] = 0;
  for (int n = 0; n < B; ++n) {
    int e = E - 1;
    for (int k = 0; k < E - 1; ++k)
      if (conf[(int64_t)n * E + k] >= tau[k]) {
        e = k;
        break;
      }
    exit_id[n] = (int8_t)e;
    counts[e]++;
  }
  for (int k = 0; k + 1 < E; ++k) {
    int w = 0;
    for (int n = 0; n < B; ++n)
      if (exit_id[n] > k) surv[(int64_t)k * B + w++] = n;
    for (; w < B; ++w) surv[(int64_t)k * B + w] = -1;
  }
}

// ------------------------------------------------------------------------------------------------
// Detector decode (reading Q18): per candidate i = ((frame*G+row)*G+col)*A+a, channel block
// [tx, ty, tw, th, obj, cls_0..cls_{NC-1}] at a*(5+NC).
static double sigm(double x) { return 1.0 / (1.0 + exp(-x)); }
extern "C" int32_t or_detect(const float* raw, int B, int G, int A, int NC, const float* anchor_wh, int stride,
                             int img_w, int img_h, float tau_det, float* det, int32_t max_det) {
  int32_t n = 0;
  const int CH = A * (5 + NC);
  for (int f = 0; f < B; ++f)
    for (int row = 0; row < G; ++row)
      for (int col = 0; col < G; ++col)
        for (int a = 0; a < A; ++a) {
          const float* v = raw + (((int64_t)f * G + row) * G + col) * CH + a * (5 + NC);
          int cs = 0;
          for (int c = 1; c < NC; ++c)
            if (v[5 + c] > v[5 + cs]) cs = c;
          const float score = (float)(sigm(v[4]) * sigm(v[5 + cs]));
          if (!(score >= tau_det)) continue;
          if (n < max_det) {
            const double cx = (col + sigm(v[0])) * stride, cy = (row + sigm(v[1])) * stride;
            const double bw = anchor_wh[2 * a] * exp(std::min((double)v[2], 4.0));
            const double bh = anchor_wh[2 * a + 1] * exp(std::min((double)v[3], 4.0));
            float* d = det + (int64_t)n * 9;
            d[0] = (float)f;
            d[1] = (float)(row * G + col);
            d[2] = (float)a;
            d[3] = (float)cs;
            d[4] = score;
            d[5] = (float)std::min(std::max(cx - bw / 2, 0.0), (double)img_w);
            d[6] = (float)std::min(std::max(cy - bh / 2, 0.0), (double)img_h);
            d[7] = (float)std::min(std::max(cx + bw / 2, 0.0), (double)img_w);
            d[8] = (float)std::min(std::max(cy + bh / 2, 0.0), (double)img_h);
          }
          n++;
        }
  return n;
}

// Non-maximum suppression (NEXT-3 of SURVEY §8(f): TinyYOLOv3 post-processing; the paper gives no
// parameters: reading Q18b in DESIGN.md).  Plain greedy definition, per (frame, class).
extern "C" float or_iou(const float* a, const float* b) {
  const float iw = std::max(0.0f, std::min(a[2], b[2]) - std::max(a[0], b[0]));
  const float ih = std::max(0.0f, std::min(a[3], b[3]) - std::max(a[1], b[1]));
  const float inter = iw * ih;
  const float area_a = (a[2] - a[0]) * (a[3] - a[1]);
  const float area_b = (b[2] - b[0]) * (b[3] - b[1]);
  const float uni = (area_a + area_b) - inter;
  return uni > 0.0f ? inter / uni : 0.0f;
}

extern "C" int32_t or_nms(const float* det, int32_t n, float iou_thr, uint8_t* keep) {
  vector<int> order(n);
  for (int i = 0; i < n; ++i) order[i] = i;
  // visit order: frame, class, score descending, row ascending
  std::stable_sort(order.begin(), order.end(), [&](int x, int y) {
    const float* a = det + (int64_t)x * 9;
    const float* b = det + (int64_t)y * 9;
    if (a[0] != b[0]) return a[0] < b[0];
    if (a[3] != b[3]) return a[3] < b[3];
    return a[4] > b[4];
  });
  int32_t kept = 0;
  vector<int> kept_rows;
  for (int i = 0; i < n; ++i) keep[i] = 0;
  for (int q = 0; q < n; ++q) {
    const int i = order[q];
    const float* a = det + (int64_t)i * 9;
    bool ok = true;
    for (int k : kept_rows) {
      const float* b = det + (int64_t)k * 9;
      if (b[0] == a[0] && b[3] == a[3] && or_iou(a + 5, b + 5) > iou_thr) {
        ok = false;
        break;
      }
    }
    if (ok) {
      keep[i] = 1;
      kept_rows.push_back(i);
      kept++;
    }
  }
  return kept;
}

// Crop-resize (reading Q19): half-pixel centres, clamped edges, every fp32 op rounded separately (no
// FMA contraction: compiled with -ffp-contract=off), result rounded to bf16.
extern "C" void or_crop(const float* fr, int H, int W, int C, float x0, float y0, float x1, float y1, int ch,
                        int cw, float* out) {
  const float sxs = (x1 - x0) / (float)cw;
  const float sys = (y1 - y0) / (float)ch;
  for (int v = 0; v < ch; ++v) {
    float sy = y0 + ((float)v + 0.5f) * sys - 0.5f;
    sy = std::min(std::max(sy, 0.0f), (float)(H - 1));
    const int yl = (int)floorf(sy);
    const int yh = std::min(yl + 1, H - 1);
    const float fy = sy - (float)yl;
    for (int u = 0; u < cw; ++u) {
      float sx = x0 + ((float)u + 0.5f) * sxs - 0.5f;
      sx = std::min(std::max(sx, 0.0f), (float)(W - 1));
      const int xl = (int)floorf(sx);
      const int xh = std::min(xl + 1, W - 1);
      const float fx = sx - (float)xl;
      for (int c = 0; c < C; ++c) {
        const float p00 = fr[((int64_t)yl * W + xl) * C + c], p01 = fr[((int64_t)yl * W + xh) * C + c];
        const float p10 = fr[((int64_t)yh * W + xl) * C + c], p11 = fr[((int64_t)yh * W + xh) * C + c];
        const float wx0 = 1.0f - fx, wy0 = 1.0f - fy;
        const float top = wx0 * p00 + fx * p01;
        const float bot = wx0 * p10 + fx * p11;
        out[((int64_t)v * cw + u) * C + c] = or_bf16(wy0 * top + fy * bot);
      }
    }
  }
}

// ------------------------------------------------------------------------------------------------
// Selection ("Cosine distance of the feature vector of every new sample with the mean feature
// vector of the old training samples ... after PCA"; P:239 R_j^i samples; P:243 never reuse samples).
// Readings Q13 (uncentred projection), Q14 (min over M reference rows), Q15 (ties -> lower index,
// output ascending), Q17 (zero norm -> d = 1).
extern "C" int32_t or_select(const float* X, int64_t N, int D, const float* Wp, int P, const float* ref, int M,
                             const uint8_t* exclude, int32_t k, float* dist, int32_t* out_idx, float* out_dist) {
  vector<double> mu((size_t)M * P, 0.0), mun(M, 0.0);
  for (int r = 0; r < M; ++r) {
    for (int p = 0; p < P; ++p) {
      double a = 0.0;
      if (Wp)
        for (int d = 0; d < D; ++d) a += (double)ref[(int64_t)r * D + d] * (double)Wp[(int64_t)d * P + p];
      else
        a = ref[(int64_t)r * D + p];
      mu[(size_t)r * P + p] = a;
    }
    double s = 0.0;
    for (int p = 0; p < P; ++p) s += mu[(size_t)r * P + p] * mu[(size_t)r * P + p];
    mun[r] = sqrt(s);
  }
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < N; ++i) {
    vector<double> y(P);
    for (int p = 0; p < P; ++p) {
      double a = 0.0;
      if (Wp)
        for (int d = 0; d < D; ++d) a += (double)X[i * D + d] * (double)Wp[(int64_t)d * P + p];
      else
        a = X[i * D + p];
      y[p] = a;
    }
    double yn = 0.0;
    for (int p = 0; p < P; ++p) yn += y[p] * y[p];
    yn = sqrt(yn);
    double best = INFINITY;
    for (int r = 0; r < M; ++r) {
      double dot = 0.0;
      for (int p = 0; p < P; ++p) dot += y[p] * mu[(size_t)r * P + p];
      const double cs = dot / std::max(yn * mun[r], 1e-12);
      best = std::min(best, 1.0 - cs);
    }
    dist[i] = (exclude && exclude[i]) ? -1.0f : (float)best;
  }
  vector<int64_t> el;
  for (int64_t i = 0; i < N; ++i)
    if (!(exclude && exclude[i])) el.push_back(i);
  std::stable_sort(el.begin(), el.end(), [&](int64_t a, int64_t b) { return dist[a] > dist[b]; });
  const int32_t cnt = (int32_t)std::min<int64_t>(k, (int64_t)el.size());
  vector<int64_t> pick(el.begin(), el.begin() + cnt);
  std::sort(pick.begin(), pick.end());
  for (int32_t j = 0; j < cnt; ++j) {
    out_idx[j] = (int32_t)pick[j];
    if (out_dist) out_dist[j] = dist[pick[j]];
  }
  return cnt;
}

// ------------------------------------------------------------------------------------------------
// Incremental retraining step ("retrains a model as much as possible every time before it is
// used"; readings Q8 loss = sum_k w_k CE over all exits, Q9 SGD+momentum (PyTorch semantics), Q10 no
// BN, Q22 grads scaled by 1/N_global).
static int grads_of(const or_model* m, const double* params, const float* x, const int32_t* labels, int n,
                    int64_t n_global, bool exact, vector<double>& g, double* loss) {
  Walk w = walk(m);
  if (!w.ok || w.inference_only) return -1;  // detectors (UPSAMPLE / ROUTE) are not retrained
  g.assign(w.nparams, 0.0);
  const int64_t in_sz = (int64_t)m->in_h * m->in_w * m->in_c;
  const double inv_n = 1.0 / (double)n_global;
  double L = 0.0;
  int nt = 1;
#ifdef _OPENMP
  nt = omp_get_max_threads();
#endif
  vector<vector<double>> gl(nt, vector<double>(w.nparams, 0.0));
  vector<double> Ll(nt, 0.0);
#pragma omp parallel for schedule(dynamic, 1)
  for (int i = 0; i < n; ++i) {
    int tid = 0;
#ifdef _OPENMP
    tid = omp_get_thread_num();
#endif
    Engine eng(m, w, exact);
    eng.forward(params, x + i * in_sz);
    Ll[tid] += eng.backward(params, labels[i], inv_n, gl[tid].data());
  }
  for (int t = 0; t < nt; ++t) {
    L += Ll[t];
    for (int64_t j = 0; j < w.nparams; ++j) g[j] += gl[t][j];
  }
  if (loss) *loss = L;
  return 0;
}

extern "C" int or_retrain_step(const or_model* m, float* params, float* mom, const float* x,
                               const int32_t* labels, int n, int64_t n_global, float lr, float mu, float wd,
                               float* grads, double* loss) {
  vector<double> g;
  const vector<double> pd(params, params + or_num_params(m));
  int rc = grads_of(m, pd.data(), x, labels, n, n_global, false, g, loss);
  if (rc) return rc;
  // SGD with momentum, PyTorch semantics (dampening 0, no Nesterov), all fp32 (c.1 step 12)
  for (size_t j = 0; j < g.size(); ++j) {
    const float gj = (float)g[j];
    if (grads) grads[j] = gj;
    const float d = gj + wd * params[j];
    mom[j] = mu * mom[j] + d;
    params[j] = params[j] - lr * mom[j];
  }
  return 0;
}

extern "C" double or_loss(const or_model* m, const double* params, const float* x, const int32_t* labels, int n,
                          int64_t n_global, int exact) {
  Walk w = walk(m);
  const int64_t in_sz = (int64_t)m->in_h * m->in_w * m->in_c;
  double L = 0.0;
  for (int i = 0; i < n; ++i) {
    Engine eng(m, w, exact != 0);
    eng.forward(params, x + i * in_sz);
    for (size_t k = 0; k < eng.exit_op.size(); ++k) {
      const auto& lg = eng.logits[k];
      double mx = lg[0];
      for (double v : lg) mx = std::max(mx, v);
      double s = 0.0;
      for (double v : lg) s += exp(v - mx);
      L += (double)m->ops[eng.exit_op[k]].loss_weight * (-(lg[labels[i]] - mx - log(s))) / (double)n_global;
    }
  }
  return L;
}

extern "C" int or_grad_exact(const or_model* m, const double* params, const float* x, const int32_t* labels,
                             int n, int64_t n_global, double* grads) {
  vector<double> g;
  int rc = grads_of(m, params, x, labels, n, n_global, true, g, nullptr);
  if (rc) return rc;
  for (size_t j = 0; j < g.size(); ++j) grads[j] = g[j];
  return 0;
}

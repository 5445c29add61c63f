// Detector decode + DAG routing + on-device crop-resize (Fig. 1 DAG, P:146/P:162
// "the output of the detector is reused by the next model ... it must not leave the GPU").
//
//   1. count : per block of candidates, detections and per-edge routed counts (score = sigmoid(obj) *
//              sigmoid(cls*) >= tau_det, reading Q18)
//   2. scan  : single CTA exclusive scan of the block counts -> global offsets, n_det, n_routed, clamps
//   3. emit  : stable in-order writes of det_table rows and per-edge route lists
//   4. crops : bilinear crop-resize of every routed box into the destination model's input batch
//              (half-pixel centres, clamped edges, every fp32 op rounded on its own, reading Q19)
#include "common.cuh"
#include "model.h"
#include "prof.h"

namespace adainf {

constexpr int DET_THREADS = 256, DET_PER_THREAD = 4, DET_PER_BLOCK = DET_THREADS * DET_PER_THREAD;
constexpr int MAX_EDGES = 8;

struct Cand {
  bool det;
  int cls;
};

__device__ __forceinline__ float sigmoidf_(float x) { return __fdiv_rn(1.0f, __fadd_rn(1.0f, expf(-x))); }

// candidate i = (frame * CPF + cell) * A + anchor, CPF = G*G (+ G2*G2): cells of head 0 first, then head 1
struct CandPos {
  int f, head, row, col, cell, an;
  const float* v;
};
__device__ __forceinline__ CandPos cand_pos(const DetRouteArgs& a, long long i) {
  CandPos p;
  const long long cpf = (long long)a.G * a.G + (long long)a.G2 * a.G2;
  p.an = (int)(i % a.A);
  const long long cg = i / a.A;
  p.f = (int)(cg / cpf);
  p.cell = (int)(cg - (long long)p.f * cpf);
  p.head = p.cell >= a.G * a.G;
  const int G = p.head ? a.G2 : a.G;
  const int lc = p.head ? p.cell - a.G * a.G : p.cell;
  p.row = lc / G;
  p.col = lc - p.row * G;
  const float* raw = p.head ? a.raw2 : a.raw;
  p.v = raw + (((long long)p.f * G * G + lc) * a.A + p.an) * (5 + a.NC);
  return p;
}

__device__ __forceinline__ Cand eval_cand(const DetRouteArgs& a, long long i, int nframes) {
  Cand c{false, 0};
  const long long ncand = (long long)nframes * ((long long)a.G * a.G + (long long)a.G2 * a.G2) * a.A;
  if (i >= ncand) return c;
  const float* v = cand_pos(a, i).v;
  int cs = 0;
  for (int k = 1; k < a.NC; ++k)
    if (v[5 + k] > v[5 + cs]) cs = k;
  const float score = __fmul_rn(sigmoidf_(v[4]), sigmoidf_(v[5 + cs]));
  c.det = score >= a.tau;
  c.cls = cs;
  return c;
}

__device__ __forceinline__ int edge_of(const DetRouteArgs& a, int cls) {
  for (int e = 0; e < a.n_edges; ++e)
    if (a.edge_class[e] == cls) return e;
  return -1;
}

__global__ void det_count_kernel(const DetRouteArgs a, int* __restrict__ blk) {
  const int nframes = a.count ? *a.count : a.n_static;
  __shared__ int s[1 + MAX_EDGES];
  if (threadIdx.x <= MAX_EDGES) s[threadIdx.x] = 0;
  __syncthreads();
  int d = 0, r[MAX_EDGES] = {0};
  for (int q = 0; q < DET_PER_THREAD; ++q) {
    const long long i = (long long)blockIdx.x * DET_PER_BLOCK + q * DET_THREADS + threadIdx.x;
    const Cand c = eval_cand(a, i, nframes);
    if (c.det) {
      d++;
      const int e = edge_of(a, c.cls);
      if (e >= 0) r[e]++;
    }
  }
  atomicAdd(&s[0], d);  // integer: order-independent
  for (int e = 0; e < a.n_edges; ++e) atomicAdd(&s[1 + e], r[e]);
  __syncthreads();
  if (threadIdx.x <= a.n_edges) blk[(long long)blockIdx.x * (1 + MAX_EDGES) + threadIdx.x] = s[threadIdx.x];
}

__global__ void det_scan_kernel(const DetRouteArgs a, int nblocks, int* __restrict__ blk) {
  // one warp per column, sequential over blocks in chunks of 32 (exclusive scan in place)
  const int col = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (col > a.n_edges) return;
  int run = 0;
  for (int b0 = 0; b0 < nblocks; b0 += 32) {
    const int b = b0 + lane;
    const int v = b < nblocks ? blk[(long long)b * (1 + MAX_EDGES) + col] : 0;
    int x = v;
    for (int o = 1; o < 32; o <<= 1) {
      const int u = __shfl_up_sync(0xffffffffu, x, o);
      if (lane >= o) x += u;
    }
    if (b < nblocks) blk[(long long)b * (1 + MAX_EDGES) + col] = run + x - v;
    run += __shfl_sync(0xffffffffu, x, 31);
  }
  if (lane == 0) {
    if (col == 0) {
      if (a.n_det) *a.n_det = run;
    } else {
      const int e = col - 1;
      if (a.n_routed) a.n_routed[e] = run;
      a.count_clamped[e] = min(run, a.cap);
      if (run > a.cap && a.cap_flag) atomicExch(a.cap_flag, 1);
    }
  }
}

__global__ void det_emit_kernel(const DetRouteArgs a, const int* __restrict__ blk) {
  const int nframes = a.count ? *a.count : a.n_static;
  __shared__ int wd[DET_THREADS / 32][1 + MAX_EDGES];
  __shared__ int run[1 + MAX_EDGES];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  if (threadIdx.x <= MAX_EDGES) run[threadIdx.x] = blk[(long long)blockIdx.x * (1 + MAX_EDGES) + threadIdx.x];
  __syncthreads();
  for (int q = 0; q < DET_PER_THREAD; ++q) {
    const long long i = (long long)blockIdx.x * DET_PER_BLOCK + q * DET_THREADS + threadIdx.x;
    const Cand c = eval_cand(a, i, nframes);
    const int e = c.det ? edge_of(a, c.cls) : -1;
    // column 0: detections; columns 1+e: routed per edge
    unsigned bal[1 + MAX_EDGES];
    bal[0] = __ballot_sync(0xffffffffu, c.det);
    for (int k = 0; k < a.n_edges; ++k) bal[1 + k] = __ballot_sync(0xffffffffu, e == k);
    if (lane == 0)
      for (int k = 0; k <= a.n_edges; ++k) wd[w][k] = __popc(bal[k]);
    __syncthreads();
    if (c.det) {
      const unsigned lt = (1u << lane) - 1u;
      int pre0 = run[0] + __popc(bal[0] & lt);
      for (int ww = 0; ww < w; ++ww) pre0 += wd[ww][0];
      {
        const CandPos cp = cand_pos(a, i);
        const int an = cp.an, row = cp.row, col = cp.col, f = cp.f;
        const float* v = cp.v;
        const float stride = (float)(cp.head ? a.stride2 : a.stride);
        const float* aw = cp.head ? a.anchor_wh2 : a.anchor_wh;
        const float score = __fmul_rn(sigmoidf_(v[4]), sigmoidf_(v[5 + c.cls]));
        const float cx = __fmul_rn(__fadd_rn((float)col, sigmoidf_(v[0])), stride);
        const float cy = __fmul_rn(__fadd_rn((float)row, sigmoidf_(v[1])), stride);
        const float bw = __fmul_rn(aw[2 * an], expf(fminf(v[2], 4.f)));
        const float bh = __fmul_rn(aw[2 * an + 1], expf(fminf(v[3], 4.f)));
        float* d = a.det_table + (long long)pre0 * 9;
        d[0] = (float)f;
        d[1] = (float)cp.cell;
        d[2] = (float)an;
        d[3] = (float)c.cls;
        d[4] = score;
        d[5] = fminf(fmaxf(__fsub_rn(cx, __fmul_rn(bw, 0.5f)), 0.f), (float)a.img_w);
        d[6] = fminf(fmaxf(__fsub_rn(cy, __fmul_rn(bh, 0.5f)), 0.f), (float)a.img_h);
        d[7] = fminf(fmaxf(__fadd_rn(cx, __fmul_rn(bw, 0.5f)), 0.f), (float)a.img_w);
        d[8] = fminf(fmaxf(__fadd_rn(cy, __fmul_rn(bh, 0.5f)), 0.f), (float)a.img_h);
        if (a.user_table && pre0 < a.user_max)
          for (int q = 0; q < 9; ++q) a.user_table[(long long)pre0 * 9 + q] = d[q];
      }
      if (e >= 0) {
        int pre = run[1 + e] + __popc(bal[1 + e] & lt);
        for (int ww = 0; ww < w; ++ww) pre += wd[ww][1 + e];
        if (pre < a.cap) a.route_idx[(long long)e * a.cap + pre] = pre0;
      }
    }
    __syncthreads();
    if (threadIdx.x <= a.n_edges) {
      int tot = 0;
      for (int ww = 0; ww < DET_THREADS / 32; ++ww) tot += wd[ww][threadIdx.x];
      run[threadIdx.x] += tot;
    }
    __syncthreads();
  }
}

// ------------------------------------------------------------------------------------------------
// NMS (NEXT-3, reading Q18b): decode into a pre-NMS table (ascending candidate index, so each frame's rows are
// contiguous), then per frame one CTA sorts its detections by (class, score descending, row) with a bitonic sort
// in shared memory and one warp runs the greedy scan (fp32 IoU, every op rounded as in the oracle), then a single
// CTA compacts the kept rows in order into det_table and the per-edge route lists.
__device__ __forceinline__ float iou_rn(const float* a, const float* b) {
  const float iw = fmaxf(0.f, __fsub_rn(fminf(a[2], b[2]), fmaxf(a[0], b[0])));
  const float ih = fmaxf(0.f, __fsub_rn(fminf(a[3], b[3]), fmaxf(a[1], b[1])));
  const float inter = __fmul_rn(iw, ih);
  const float area_a = __fmul_rn(__fsub_rn(a[2], a[0]), __fsub_rn(a[3], a[1]));
  const float area_b = __fmul_rn(__fsub_rn(b[2], b[0]), __fsub_rn(b[3], b[1]));
  const float uni = __fsub_rn(__fadd_rn(area_a, area_b), inter);
  return uni > 0.f ? __fdiv_rn(inter, uni) : 0.f;
}

__global__ void __launch_bounds__(256) nms_kernel(const float* __restrict__ pre, const int* __restrict__ n_pre,
                                                  const int* frames_count, int n_static, int pow2, float thr,
                                                  uint8_t* __restrict__ keep) {
  extern __shared__ unsigned long long skey[];  // [pow2] keys, then boxes [pow2][4] fp32, sup [pow2] bytes
  float* sbox = (float*)(skey + pow2);
  uint8_t* sup = (uint8_t*)(sbox + 4 * pow2);
  const int f = blockIdx.x;
  const int nframes = frames_count ? min(*frames_count, n_static) : n_static;
  if (f >= nframes) return;
  const int n = *n_pre;
  // rows of frame f: [lo, hi) by binary search on the frame column (non-decreasing)
  __shared__ int s_lo, s_hi;
  if (threadIdx.x < 2) {
    const float key = (float)(f + threadIdx.x);
    int lo = 0, hi = n;
    while (lo < hi) {
      const int mid = (lo + hi) >> 1;
      if (pre[(long long)mid * 9] < key) lo = mid + 1;
      else hi = mid;
    }
    if (threadIdx.x == 0) s_lo = lo;
    else s_hi = lo;
  }
  __syncthreads();
  const int lo = s_lo, cnt = s_hi - s_lo;
  if (cnt <= 0) return;
  for (int i = threadIdx.x; i < pow2; i += blockDim.x) {
    unsigned long long k = ~0ull;
    if (i < cnt) {
      const float* r = pre + (long long)(lo + i) * 9;
      const unsigned cls = (unsigned)r[3];
      k = ((unsigned long long)cls << 56) | ((unsigned long long)(0xFFFFFFFFu - __float_as_uint(r[4])) << 24) |
          (unsigned long long)i;
    }
    skey[i] = k;
    if (i < cnt) keep[lo + i] = 0;
  }
  __syncthreads();
  for (int size = 2; size <= pow2; size <<= 1)
    for (int stride = size >> 1; stride > 0; stride >>= 1) {
      for (int i = threadIdx.x; i < pow2; i += blockDim.x) {
        const int j = i ^ stride;
        if (j > i) {
          const bool up = (i & size) == 0;
          const unsigned long long x = skey[i], y = skey[j];
          if ((x > y) == up) {
            skey[i] = y;
            skey[j] = x;
          }
        }
      }
      __syncthreads();
    }
  for (int i = threadIdx.x; i < cnt; i += blockDim.x) {
    const int row = (int)(skey[i] & 0xFFFFFFull);
    const float* r = pre + (long long)(lo + row) * 9;
#pragma unroll
    for (int q = 0; q < 4; ++q) sbox[i * 4 + q] = r[5 + q];
    sup[i] = 0;
  }
  __syncthreads();
  if (threadIdx.x < 32) {
    const int lane = threadIdx.x;
    for (int p = 0; p < cnt; ++p) {
      __syncwarp();
      if (sup[p]) continue;
      const unsigned cls = (unsigned)(skey[p] >> 56);
      if (lane == 0) keep[lo + (int)(skey[p] & 0xFFFFFFull)] = 1;
      for (int q = p + 1 + lane; q < cnt; q += 32) {
        if ((unsigned)(skey[q] >> 56) != cls) break;
        if (!sup[q] && iou_rn(sbox + p * 4, sbox + q * 4) > thr) sup[q] = 1;
      }
    }
  }
}

// stable compaction of the kept rows into det_table (+ the caller's copy) and the per-edge route lists
__global__ void __launch_bounds__(1024) nms_route_kernel(const DetRouteArgs a, const float* __restrict__ pre,
                                                         const int* __restrict__ n_pre, const uint8_t* __restrict__ keep) {
  __shared__ int wtot[32][1 + MAX_EDGES];
  __shared__ int run[1 + MAX_EDGES];
  const int t = threadIdx.x, lane = t & 31, w = t >> 5;
  const int n = *n_pre;
  const int ncol = 1 + a.n_edges;
  if (t < ncol) run[t] = 0;
  __syncthreads();
  for (int c0 = 0; c0 < n; c0 += 1024) {
    const int i = c0 + t;
    const bool f = i < n && keep[i];
    const int e = f ? edge_of(a, (int)pre[(long long)i * 9 + 3]) : -1;
    unsigned bal[1 + MAX_EDGES];
    bal[0] = __ballot_sync(0xffffffffu, f);
    for (int k = 0; k < a.n_edges; ++k) bal[1 + k] = __ballot_sync(0xffffffffu, e == k);
    if (lane == 0)
      for (int k = 0; k < ncol; ++k) wtot[w][k] = __popc(bal[k]);
    __syncthreads();
    if (f) {
      const unsigned lt = (1u << lane) - 1u;
      int p0 = run[0] + __popc(bal[0] & lt);
      for (int q = 0; q < w; ++q) p0 += wtot[q][0];
      const float* src = pre + (long long)i * 9;
      float* d = a.det_table + (long long)p0 * 9;
      for (int q = 0; q < 9; ++q) d[q] = src[q];
      if (a.user_table && p0 < a.user_max)
        for (int q = 0; q < 9; ++q) a.user_table[(long long)p0 * 9 + q] = src[q];
      if (e >= 0) {
        int pe = run[1 + e] + __popc(bal[1 + e] & lt);
        for (int q = 0; q < w; ++q) pe += wtot[q][1 + e];
        if (pe < a.cap) a.route_idx[(long long)e * a.cap + pe] = p0;
      }
    }
    __syncthreads();
    if (t < ncol) {
      int tot = 0;
      for (int q = 0; q < 32; ++q) tot += wtot[q][t];
      run[t] += tot;
    }
    __syncthreads();
  }
  if (t < ncol) {
    const int r = run[t];
    if (t == 0) {
      if (a.n_det) *a.n_det = r;
    } else {
      const int e = t - 1;
      if (a.n_routed) a.n_routed[e] = r;
      a.count_clamped[e] = min(r, a.cap);
      if (r > a.cap && a.cap_flag) atomicExch(a.cap_flag, 1);
    }
  }
}

size_t det_route_ws_bytes(int n_static, int cells_per_frame, int A, bool nms) {
  const long long ncand = (long long)n_static * cells_per_frame * A;
  const long long nb = (ncand + DET_PER_BLOCK - 1) / DET_PER_BLOCK;
  size_t b = (size_t)nb * (1 + MAX_EDGES) * sizeof(int) + 256;
  if (nms) b += 256 + (size_t)ncand * 9 * 4 + 256 + (size_t)ncand + 256 + 16;
  return b;
}

void launch_det_route(const DetRouteArgs& a, void* ws, cudaStream_t st) {
  if (a.n_edges > MAX_EDGES) throw ShapeError("at most 8 routing edges per detector");
  const long long ncand = (long long)a.n_static * ((long long)a.G * a.G + (long long)a.G2 * a.G2) * a.A;
  const int nb = (int)((ncand + DET_PER_BLOCK - 1) / DET_PER_BLOCK);
  int* blk = (int*)ws;
  if (a.nms_iou > 0.f) {
    char* p = (char*)ws + ((size_t)nb * (1 + MAX_EDGES) * sizeof(int) + 256 + 255) / 256 * 256;
    float* pre = (float*)p;
    p += ((size_t)ncand * 9 * 4 + 255) / 256 * 256;
    uint8_t* keep = (uint8_t*)p;
    p += ((size_t)ncand + 255) / 256 * 256;
    int* n_pre = (int*)p;
    DetRouteArgs b = a;  // decode only: every detection into the pre-NMS table, no routing yet
    b.n_edges = 0;
    b.det_table = pre;
    b.user_table = nullptr;
    b.user_max = 0;
    b.n_det = n_pre;
    b.n_routed = nullptr;
    const int per_frame = (a.G * a.G + a.G2 * a.G2) * a.A;
    int pow2 = 1;
    while (pow2 < per_frame) pow2 <<= 1;
    const size_t smem = (size_t)pow2 * (8 + 16 + 1) + 64;
    if (smem > 200 * 1024) throw ShapeError("NMS: too many candidates per frame");
    static size_t attr = 0;
    if (smem > 48 * 1024 && smem > attr) {
      CK(cudaFuncSetAttribute(nms_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
      attr = smem;
    }
    ProfScope ps(PC_DET_ROUTE, st, 5);
    det_count_kernel<<<nb, DET_THREADS, 0, st>>>(b, blk);
    det_scan_kernel<<<1, 32 * (1 + MAX_EDGES), 0, st>>>(b, nb, blk);
    det_emit_kernel<<<nb, DET_THREADS, 0, st>>>(b, blk);
    nms_kernel<<<a.n_static, 256, smem, st>>>(pre, n_pre, a.count, a.n_static, pow2, a.nms_iou, keep);
    nms_route_kernel<<<1, 1024, 0, st>>>(a, pre, n_pre, keep);
    CK(cudaGetLastError());
    return;
  }
  ProfScope ps(PC_DET_ROUTE, st, 3);
  det_count_kernel<<<nb, DET_THREADS, 0, st>>>(a, blk);
  det_scan_kernel<<<1, 32 * (1 + MAX_EDGES), 0, st>>>(a, nb, blk);
  det_emit_kernel<<<nb, DET_THREADS, 0, st>>>(a, blk);
  CK(cudaGetLastError());
}

// ------------------------------------------------------------------------------------------------
// crop-resize: dst[r][v][u][c] for routed detection r of edge e (c >= C zero-padded to cout_pad)
// One crop per CTA row-band (grid.y = routed detection r, grid.x = band of output rows): the per-column
// source coordinates (xl, xh, fx) of the crop are computed once into shared memory, each thread then emits two
// horizontally adjacent output pixels per row (3-channel crops: 12 contiguous bytes = three 32-bit stores instead
// of six 16-bit ones).  The per-pixel arithmetic is the oracle's, op for op (reading Q19): every value is bit-exact.
constexpr int CROP_BANDS = 8, CROP_MAXW = 512;
__global__ void __launch_bounds__(256) crop_kernel(const bf16* __restrict__ frames, int H, int W, int C,
                                                   const float* __restrict__ det, const int32_t* __restrict__ route_idx,
                                                   const int32_t* __restrict__ cnt, int edge, int cap, int ch, int cw,
                                                   int cpad, bf16* __restrict__ dst) {
  const int r = blockIdx.y;
  if (r >= cnt[edge]) return;
  __shared__ int s_xl[CROP_MAXW], s_xh[CROP_MAXW];
  __shared__ float s_fx[CROP_MAXW];
  const int di = route_idx[(long long)edge * cap + r];
  const float* d = det + (long long)di * 9;
  const int f = (int)d[0];
  const float x0 = d[5], y0 = d[6], x1 = d[7], y1 = d[8];
  const float sxs = __fdiv_rn(__fsub_rn(x1, x0), (float)cw);
  const float sys = __fdiv_rn(__fsub_rn(y1, y0), (float)ch);
  for (int u = threadIdx.x; u < cw; u += blockDim.x) {
    float sx = __fsub_rn(__fadd_rn(x0, __fmul_rn(__fadd_rn((float)u, 0.5f), sxs)), 0.5f);
    sx = fminf(fmaxf(sx, 0.f), (float)(W - 1));
    const int xl = (int)floorf(sx);
    s_xl[u] = xl;
    s_xh[u] = min(xl + 1, W - 1);
    s_fx[u] = __fsub_rn(sx, (float)xl);
  }
  __syncthreads();
  const bf16* fr = frames + (long long)f * H * W * C;
  const int rows_per = (ch + CROP_BANDS - 1) / CROP_BANDS;
  const int v0 = blockIdx.x * rows_per, v1 = min(ch, v0 + rows_per);
  const int pairs = (cw + 1) / 2;
  for (int idx = threadIdx.x; idx < (v1 - v0) * pairs; idx += blockDim.x) {
    const int v = v0 + idx / pairs, u0 = 2 * (idx % pairs);
    float sy = __fsub_rn(__fadd_rn(y0, __fmul_rn(__fadd_rn((float)v, 0.5f), sys)), 0.5f);
    sy = fminf(fmaxf(sy, 0.f), (float)(H - 1));
    const int yl = (int)floorf(sy);
    const int yh = min(yl + 1, H - 1);
    const float fy = __fsub_rn(sy, (float)yl);
    const float wy0 = __fsub_rn(1.0f, fy);
    const bf16* rl = fr + (long long)yl * W * C;
    const bf16* rh = fr + (long long)yh * W * C;
    __align__(4) bf16 out[2 * 4];
#pragma unroll
    for (int k = 0; k < 2; ++k) {
      const int u = min(u0 + k, cw - 1);
      const int xl = s_xl[u], xh = s_xh[u];
      const float fx = s_fx[u];
      const float wx0 = __fsub_rn(1.0f, fx);
#pragma unroll
      for (int c = 0; c < 4; ++c) {
        if (c >= cpad) break;
        float val = 0.f;
        if (c < C) {
          const float p00 = __bfloat162float(rl[xl * C + c]);
          const float p01 = __bfloat162float(rl[xh * C + c]);
          const float p10 = __bfloat162float(rh[xl * C + c]);
          const float p11 = __bfloat162float(rh[xh * C + c]);
          const float top = __fadd_rn(__fmul_rn(wx0, p00), __fmul_rn(fx, p01));
          const float bot = __fadd_rn(__fmul_rn(wx0, p10), __fmul_rn(fx, p11));
          val = __fadd_rn(__fmul_rn(wy0, top), __fmul_rn(fy, bot));
        }
        out[k * cpad + c] = __float2bfloat16_rn(val);
      }
    }
    bf16* o = dst + ((long long)r * ch * cw + (long long)v * cw + u0) * cpad;
    const int nv = min(2, cw - u0) * cpad;  // values of this pixel pair
    if (nv % 2 == 0 && (((uintptr_t)o) & 3) == 0) {
      for (int q = 0; q < nv / 2; ++q) ((uint32_t*)o)[q] = ((const uint32_t*)out)[q];
    } else {
      for (int q = 0; q < nv; ++q) o[q] = out[q];
    }
  }
}

// The same crops written straight into a space-to-depth destination's packed input (the ResNet stem's
// [n][ch/2][cw/2][16], channel (bh*2 + bw)*4 + c, c >= C zero): one 2x2 output block per thread, two 16-byte
// stores; the destination's own packing pass (a read and a write of every crop) disappears.
__global__ void __launch_bounds__(256) crop_s2d_kernel(const bf16* __restrict__ frames, int H, int W, int C,
                                                       const float* __restrict__ det,
                                                       const int32_t* __restrict__ route_idx,
                                                       const int32_t* __restrict__ cnt, int edge, int cap, int ch,
                                                       int cw, bf16* __restrict__ dst) {
  const int r = blockIdx.y;
  if (r >= cnt[edge]) return;
  __shared__ int s_xl[CROP_MAXW], s_xh[CROP_MAXW];
  __shared__ float s_fx[CROP_MAXW];
  const int di = route_idx[(long long)edge * cap + r];
  const float* d = det + (long long)di * 9;
  const int f = (int)d[0];
  const float x0 = d[5], y0 = d[6], x1 = d[7], y1 = d[8];
  const float sxs = __fdiv_rn(__fsub_rn(x1, x0), (float)cw);
  const float sys = __fdiv_rn(__fsub_rn(y1, y0), (float)ch);
  for (int u = threadIdx.x; u < cw; u += blockDim.x) {
    float sx = __fsub_rn(__fadd_rn(x0, __fmul_rn(__fadd_rn((float)u, 0.5f), sxs)), 0.5f);
    sx = fminf(fmaxf(sx, 0.f), (float)(W - 1));
    const int xl = (int)floorf(sx);
    s_xl[u] = xl;
    s_xh[u] = min(xl + 1, W - 1);
    s_fx[u] = __fsub_rn(sx, (float)xl);
  }
  __syncthreads();
  const bf16* fr = frames + (long long)f * H * W * C;
  const int hs = ch / 2, ws = cw / 2;
  const int rows_per = (hs + CROP_BANDS - 1) / CROP_BANDS;
  const int i0 = blockIdx.x * rows_per, i1 = min(hs, i0 + rows_per);
  for (int idx = threadIdx.x; idx < (i1 - i0) * ws; idx += blockDim.x) {
    const int i = i0 + idx / ws, j = idx % ws;
    __align__(16) bf16 out[16];
#pragma unroll
    for (int bh = 0; bh < 2; ++bh) {
      const int v = 2 * i + bh;
      float sy = __fsub_rn(__fadd_rn(y0, __fmul_rn(__fadd_rn((float)v, 0.5f), sys)), 0.5f);
      sy = fminf(fmaxf(sy, 0.f), (float)(H - 1));
      const int yl = (int)floorf(sy);
      const int yh = min(yl + 1, H - 1);
      const float fy = __fsub_rn(sy, (float)yl);
      const float wy0 = __fsub_rn(1.0f, fy);
      const bf16* rl = fr + (long long)yl * W * C;
      const bf16* rh = fr + (long long)yh * W * C;
#pragma unroll
      for (int bw = 0; bw < 2; ++bw) {
        const int u = 2 * j + bw;
        const int xl = s_xl[u], xh = s_xh[u];
        const float fx = s_fx[u];
        const float wx0 = __fsub_rn(1.0f, fx);
#pragma unroll
        for (int c = 0; c < 4; ++c) {
          float val = 0.f;
          if (c < C) {
            const float p00 = __bfloat162float(rl[xl * C + c]);
            const float p01 = __bfloat162float(rl[xh * C + c]);
            const float p10 = __bfloat162float(rh[xl * C + c]);
            const float p11 = __bfloat162float(rh[xh * C + c]);
            const float top = __fadd_rn(__fmul_rn(wx0, p00), __fmul_rn(fx, p01));
            const float bot = __fadd_rn(__fmul_rn(wx0, p10), __fmul_rn(fx, p11));
            val = __fadd_rn(__fmul_rn(wy0, top), __fmul_rn(fy, bot));
          }
          out[(bh * 2 + bw) * 4 + c] = __float2bfloat16_rn(val);
        }
      }
    }
    uint4* o = (uint4*)(dst + (((long long)r * hs + i) * ws + j) * 16);
    o[0] = ((const uint4*)out)[0];
    o[1] = ((const uint4*)out)[1];
  }
}

void launch_crops(const bf16* frames, int H, int W, int C, const float* det_table, const int32_t* route_idx,
                  const int32_t* count_clamped, int edge, int cap, int crop_h, int crop_w, int cout_pad, bf16* dst,
                  cudaStream_t st, bool s2d) {
  if (crop_w > CROP_MAXW || cout_pad > 4) throw ShapeError("crop: width <= 512 and <= 4 channels");
  if (s2d) {
    if (crop_h % 2 || crop_w % 2 || C > 4) throw ShapeError("crop (s2d): even crop size, <= 4 channels");
    ProfScope ps(PC_CROP, st);
    crop_s2d_kernel<<<dim3(CROP_BANDS, cap), 256, 0, st>>>(frames, H, W, C, det_table, route_idx, count_clamped, edge,
                                                           cap, crop_h, crop_w, dst);
    CK(cudaGetLastError());
    return;
  }
  dim3 grid(CROP_BANDS, cap);
  ProfScope ps(PC_CROP, st);
  crop_kernel<<<grid, 256, 0, st>>>(frames, H, W, C, det_table, route_idx, count_clamped, edge, cap, crop_h, crop_w,
                                     cout_pad, dst);
  CK(cudaGetLastError());
}

// ------------------------------------------------------------------------------------------------
// whole-input routing by predicted class (audio DAG, reading Q24): stable compaction, single CTA
__global__ void __launch_bounds__(1024) route_class_kernel(const int32_t* __restrict__ pred, const int* count,
                                                           int n_static, int cls, int32_t* __restrict__ list,
                                                           int32_t* count_out, int cap, int32_t* cap_flag) {
  __shared__ int wt[32];
  __shared__ int base_s;
  const int n = count ? *count : n_static;
  const int t = threadIdx.x, lane = t & 31, w = t >> 5;
  if (t == 0) base_s = 0;
  __syncthreads();
  for (int c0 = 0; c0 < n; c0 += 1024) {
    const int j = c0 + t;
    const bool f = j < n && pred[j] == cls;
    const unsigned bal = __ballot_sync(0xffffffffu, f);
    if (lane == 0) wt[w] = __popc(bal);
    __syncthreads();
    if (w == 0) {
      int v = wt[lane];
      for (int o = 1; o < 32; o <<= 1) {
        const int u = __shfl_up_sync(0xffffffffu, v, o);
        if (lane >= o) v += u;
      }
      wt[lane] = v;
    }
    __syncthreads();
    if (f) {
      const int o = base_s + (w ? wt[w - 1] : 0) + __popc(bal & ((1u << lane) - 1u));
      if (o < cap) list[o] = j;
    }
    __syncthreads();
    if (t == 0) base_s += wt[31];
    __syncthreads();
  }
  if (t == 0) {
    *count_out = min(base_s, cap);
    if (base_s > cap && cap_flag) atomicExch(cap_flag, 1);
  }
}
void launch_route_class(const int32_t* pred, const int* count, int n_static, int cls, int32_t* list,
                        int32_t* count_out, int cap, int32_t* cap_flag, cudaStream_t st) {
  ProfScope ps(PC_ROUTE_CLASS, st);
  route_class_kernel<<<1, 1024, 0, st>>>(pred, count, n_static, cls, list, count_out, cap, cap_flag);
  CK(cudaGetLastError());
}

}  // namespace adainf

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

__device__ __forceinline__ Cand eval_cand(const DetRouteArgs& a, long long i, int nframes) {
  Cand c{false, 0};
  const long long ncand = (long long)nframes * a.G * a.G * a.A;
  if (i >= ncand) return c;
  const int an = (int)(i % a.A);
  const long long cell = i / a.A;  // (frame*G + row)*G + col
  const float* v = a.raw + cell * (a.A * (5 + a.NC)) + an * (5 + a.NC);
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
        const int an = (int)(i % a.A);
        const long long cell = i / a.A;
        const int col = (int)(cell % a.G);
        const int row = (int)((cell / a.G) % a.G);
        const int f = (int)(cell / ((long long)a.G * a.G));
        const float* v = a.raw + cell * (a.A * (5 + a.NC)) + an * (5 + a.NC);
        const float score = __fmul_rn(sigmoidf_(v[4]), sigmoidf_(v[5 + c.cls]));
        const float cx = __fmul_rn(__fadd_rn((float)col, sigmoidf_(v[0])), (float)a.stride);
        const float cy = __fmul_rn(__fadd_rn((float)row, sigmoidf_(v[1])), (float)a.stride);
        const float bw = __fmul_rn(a.anchor_wh[2 * an], expf(fminf(v[2], 4.f)));
        const float bh = __fmul_rn(a.anchor_wh[2 * an + 1], expf(fminf(v[3], 4.f)));
        float* d = a.det_table + (long long)pre0 * 9;
        d[0] = (float)f;
        d[1] = (float)(row * a.G + col);
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

size_t det_route_ws_bytes(int n_static, int G, int A) {
  const long long ncand = (long long)n_static * G * G * A;
  const long long nb = (ncand + DET_PER_BLOCK - 1) / DET_PER_BLOCK;
  return (size_t)nb * (1 + MAX_EDGES) * sizeof(int) + 256;
}

void launch_det_route(const DetRouteArgs& a, void* ws, cudaStream_t st) {
  if (a.n_edges > MAX_EDGES) throw ShapeError("at most 8 routing edges per detector");
  const long long ncand = (long long)a.n_static * a.G * a.G * a.A;
  const int nb = (int)((ncand + DET_PER_BLOCK - 1) / DET_PER_BLOCK);
  int* blk = (int*)ws;
  ProfScope ps(PC_DET_ROUTE, st, 3);
  det_count_kernel<<<nb, DET_THREADS, 0, st>>>(a, blk);
  det_scan_kernel<<<1, 32 * (1 + MAX_EDGES), 0, st>>>(a, nb, blk);
  det_emit_kernel<<<nb, DET_THREADS, 0, st>>>(a, blk);
  CK(cudaGetLastError());
}

// ------------------------------------------------------------------------------------------------
// crop-resize: dst[r][v][u][c] for routed detection r of edge e (c >= C zero-padded to cout_pad)
__global__ void crop_kernel(const bf16* __restrict__ frames, int H, int W, int C, const float* __restrict__ det,
                            const int32_t* __restrict__ route_idx, const int32_t* __restrict__ cnt, int edge, int cap,
                            int ch, int cw, int cpad, bf16* __restrict__ dst) {
  const int r = blockIdx.y;
  if (r >= cnt[edge]) return;
  const int di = route_idx[(long long)edge * cap + r];
  const float* d = det + (long long)di * 9;
  const int f = (int)d[0];
  const float x0 = d[5], y0 = d[6], x1 = d[7], y1 = d[8];
  const float sxs = __fdiv_rn(__fsub_rn(x1, x0), (float)cw);
  const float sys = __fdiv_rn(__fsub_rn(y1, y0), (float)ch);
  const bf16* fr = frames + (long long)f * H * W * C;
  for (int pix = blockIdx.x * blockDim.x + threadIdx.x; pix < ch * cw; pix += gridDim.x * blockDim.x) {
    const int v = pix / cw, u = pix - v * cw;
    float sy = __fsub_rn(__fadd_rn(y0, __fmul_rn(__fadd_rn((float)v, 0.5f), sys)), 0.5f);
    sy = fminf(fmaxf(sy, 0.f), (float)(H - 1));
    const int yl = (int)floorf(sy);
    const int yh = min(yl + 1, H - 1);
    const float fy = __fsub_rn(sy, (float)yl);
    float sx = __fsub_rn(__fadd_rn(x0, __fmul_rn(__fadd_rn((float)u, 0.5f), sxs)), 0.5f);
    sx = fminf(fmaxf(sx, 0.f), (float)(W - 1));
    const int xl = (int)floorf(sx);
    const int xh = min(xl + 1, W - 1);
    const float fx = __fsub_rn(sx, (float)xl);
    const float wx0 = __fsub_rn(1.0f, fx), wy0 = __fsub_rn(1.0f, fy);
    bf16* o = dst + ((long long)r * ch * cw + pix) * cpad;
    for (int c = 0; c < cpad; ++c) {
      float val = 0.f;
      if (c < C) {
        const float p00 = __bfloat162float(fr[((long long)yl * W + xl) * C + c]);
        const float p01 = __bfloat162float(fr[((long long)yl * W + xh) * C + c]);
        const float p10 = __bfloat162float(fr[((long long)yh * W + xl) * C + c]);
        const float p11 = __bfloat162float(fr[((long long)yh * W + xh) * C + c]);
        const float top = __fadd_rn(__fmul_rn(wx0, p00), __fmul_rn(fx, p01));
        const float bot = __fadd_rn(__fmul_rn(wx0, p10), __fmul_rn(fx, p11));
        val = __fadd_rn(__fmul_rn(wy0, top), __fmul_rn(fy, bot));
      }
      o[c] = __float2bfloat16_rn(val);
    }
  }
}

void launch_crops(const bf16* frames, int H, int W, int C, const float* det_table, const int32_t* route_idx,
                  const int32_t* count_clamped, int edge, int cap, int crop_h, int crop_w, int cout_pad, bf16* dst,
                  cudaStream_t st) {
  dim3 grid((crop_h * crop_w + 255) / 256, cap);
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

// Depthwise convolution (groups == channels) for the paper's MobileNetV2 classifiers (NEXT-3: the video DAG's
// TinyYOLOv3 -> MobileNetV2 / ShuffleNet): forward, input gradient and weight gradient on NHWC bf16 tensors.
// There is no contraction to put on the tensor cores (one input channel per output channel, K = KH*KW): the kernels
// are bound by HBM traffic, so each thread owns one pixel x 8 channels (16-byte vectors, consecutive threads take
// consecutive channel groups then pixels: coalesced), the 9 taps hit L1, and fp32 accumulation runs in the fixed
// tap order (kh, kw).  Rounding points as the dense convs: forward fp32 + b -> act -> bf16;
// dgrad fp32 sum + exit broadcast + shortcut term -> x act' of the producer -> bf16; wgrad / bias fp32, reduced in a
// fixed order (per-CTA partials, then an ordered sum over the CTAs).
#include <algorithm>

#include "common.cuh"
#include "kernels.cuh"
#include "prof.h"

namespace adainf {

namespace {

__device__ __forceinline__ void ld8(const bf16* p, float* v) {
  const uint4 r = __ldg((const uint4*)p);
  const bf16* h = (const bf16*)&r;
#pragma unroll
  for (int q = 0; q < 8; ++q) v[q] = __bfloat162float(h[q]);
}

// shadow [C][ldb] (K = tap index, GEMM-ready rows) -> wdw [taps][C]
__global__ void dw_prep_kernel(const bf16* __restrict__ shadow, int ldb, int C, int taps, bf16* __restrict__ wdw) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= C * taps) return;
  const int c = i % C, t = i / C;
  wdw[i] = shadow[(long long)c * ldb + t];
}

__global__ void dw_fwd_kernel(DwArgs a) {
  const int n_rows = a.count ? *a.count : a.n_static;
  const int CG = a.C >> 3;
  const long long total = (long long)n_rows * a.Ho * a.Wo * CG;
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < total; i += (long long)gridDim.x * blockDim.x) {
    const int cg = (int)(i % CG);
    long long pix = i / CG;
    const int wo = (int)(pix % a.Wo);
    pix /= a.Wo;
    const int ho = (int)(pix % a.Ho);
    const int n = (int)(pix / a.Ho);
    const long long src = a.map ? a.map[n] : n;
    float acc[8];
#pragma unroll
    for (int q = 0; q < 8; ++q) acc[q] = 0.f;
    for (int kh = 0; kh < a.KH; ++kh) {
      const int ih = ho * a.s - a.p + kh;
      if (ih < 0 || ih >= a.H) continue;
      for (int kw = 0; kw < a.KW; ++kw) {
        const int iw = wo * a.s - a.p + kw;
        if (iw < 0 || iw >= a.W) continue;
        float xv[8], wv[8];
        ld8(a.x + ((src * a.H + ih) * a.W + iw) * a.C + cg * 8, xv);
        ld8(a.w + (kh * a.KW + kw) * a.C + cg * 8, wv);
#pragma unroll
        for (int q = 0; q < 8; ++q) acc[q] = fmaf(xv[q], wv[q], acc[q]);
      }
    }
    __align__(16) bf16 o[8];
#pragma unroll
    for (int q = 0; q < 8; ++q) o[q] = __float2bfloat16_rn(act_apply(a.act, __fadd_rn(acc[q], __ldg(a.bias + cg * 8 + q))));
    *(uint4*)(a.y + (((long long)n * a.Ho + ho) * a.Wo + wo) * a.C + cg * 8) = *(const uint4*)o;
  }
}

__global__ void dw_dgrad_kernel(DwArgs a) {
  const int CG = a.C >> 3;
  const long long total = (long long)a.n_static * a.H * a.W * CG;
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < total; i += (long long)gridDim.x * blockDim.x) {
    const int cg = (int)(i % CG);
    long long pix = i / CG;
    const int iw = (int)(pix % a.W);
    pix /= a.W;
    const int ih = (int)(pix % a.H);
    const int n = (int)(pix / a.H);
    float acc[8];
#pragma unroll
    for (int q = 0; q < 8; ++q) acc[q] = 0.f;
    for (int kh = 0; kh < a.KH; ++kh) {
      const int on = ih + a.p - kh;
      if (on < 0 || on % a.s) continue;
      const int oh = on / a.s;
      if (oh >= a.Ho) continue;
      for (int kw = 0; kw < a.KW; ++kw) {
        const int wn = iw + a.p - kw;
        if (wn < 0 || wn % a.s) continue;
        const int ow = wn / a.s;
        if (ow >= a.Wo) continue;
        float dv[8], wv[8];
        ld8(a.x + (((long long)n * a.Ho + oh) * a.Wo + ow) * a.C + cg * 8, dv);  // x = dZ here
        ld8(a.w + (kh * a.KW + kw) * a.C + cg * 8, wv);
#pragma unroll
        for (int q = 0; q < 8; ++q) acc[q] = fmaf(dv[q], wv[q], acc[q]);
      }
    }
    const long long o = (((long long)n * a.H + ih) * a.W + iw) * a.C + cg * 8;
    float sc[8], ya[8];
    if (a.sc) ld8(a.sc + o, sc);
    if (a.yact) ld8(a.yact + o, ya);
    __align__(16) bf16 r[8];
#pragma unroll
    for (int q = 0; q < 8; ++q) {
      float v = acc[q];
      if (a.bcast) v = __fadd_rn(v, a.bcast[(long long)n * a.C + cg * 8 + q]);
      if (a.sc) v = __fadd_rn(v, sc[q]);
      if (a.yact) v = __fmul_rn(v, act_grad(a.mask_act, ya[q]));
      r[q] = __float2bfloat16_rn(v);
    }
    *(uint4*)(a.y + o) = *(const uint4*)r;
  }
}

// weight + bias gradient, stage 1: CTA (chunk, channel group): 256 threads stride the chunk's output pixels, each
// accumulating 8 channels x (taps + 1 bias) in fp32; warp-shuffle then fixed-order cross-warp reduction ->
// part[chunk][C][taps + 1]
constexpr int DWW_THREADS = 256;
__global__ void __launch_bounds__(DWW_THREADS) dw_wgrad_partial_kernel(DwArgs a, long long pix_per_chunk, float* __restrict__ part) {
  const int cg = blockIdx.y;
  extern __shared__ float red[];  // [8 warps][8 ch][taps + 1]
  float acc[8][10];
#pragma unroll
  for (int q = 0; q < 8; ++q)
#pragma unroll
    for (int t = 0; t < 10; ++t) acc[q][t] = 0.f;
  const long long npix = (long long)a.n_static * a.Ho * a.Wo;
  const long long p0 = blockIdx.x * pix_per_chunk, p1 = min(npix, p0 + pix_per_chunk);
  for (long long pix = p0 + threadIdx.x; pix < p1; pix += DWW_THREADS) {
    const int wo = (int)(pix % a.Wo);
    const long long r = pix / a.Wo;
    const int ho = (int)(r % a.Ho);
    const long long n = r / a.Ho;
    float dv[8];
    ld8(a.dz + pix * a.C + cg * 8, dv);
#pragma unroll
    for (int q = 0; q < 8; ++q) acc[q][9] += dv[q];
#pragma unroll
    for (int kh = 0; kh < 3; ++kh) {
      const int ih = ho * a.s - a.p + kh;
#pragma unroll
      for (int kw = 0; kw < 3; ++kw) {
        const int iw = wo * a.s - a.p + kw;
        if (ih < 0 || ih >= a.H || iw < 0 || iw >= a.W) continue;
        float xv[8];
        ld8(a.x + ((n * a.H + ih) * a.W + iw) * a.C + cg * 8, xv);
#pragma unroll
        for (int q = 0; q < 8; ++q) acc[q][kh * 3 + kw] = fmaf(dv[q], xv[q], acc[q][kh * 3 + kw]);
      }
    }
  }
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
#pragma unroll
  for (int q = 0; q < 8; ++q)
#pragma unroll
    for (int t = 0; t < 10; ++t) {
      float v = acc[q][t];
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
      if (lane == 0) red[(w * 8 + q) * 10 + t] = v;
    }
  __syncthreads();
  if (threadIdx.x < 80) {
    const int q = threadIdx.x / 10, t = threadIdx.x % 10;
    float s = 0.f;
    for (int ww = 0; ww < DWW_THREADS / 32; ++ww) s += red[(ww * 8 + q) * 10 + t];
    part[((long long)blockIdx.x * a.C + cg * 8 + q) * 10 + t] = s;
  }
}

// stage 2: ordered sum over the chunks -> dw [C][taps] (master layout [C][KH][KW][1]), db [C]
__global__ void dw_wgrad_final_kernel(const float* __restrict__ part, int nchunks, int C, float* __restrict__ dw,
                                      float* __restrict__ db) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= C * 10) return;
  const int c = i / 10, t = i % 10;
  float s = 0.f;
  for (int k = 0; k < nchunks; ++k) s += part[((long long)k * C + c) * 10 + t];
  if (t < 9) dw[c * 9 + t] = s;
  else if (db) db[c] = s;
}

int grid_for(long long total) {
  return (int)std::min<long long>((total + 255) / 256, 32LL * num_sms());
}

}  // namespace

bool dw_ok(const ConvGeom& g, int groups) {
  return groups == g.Cin && groups == g.Cout && g.Cin % 8 == 0 && g.KH == 3 && g.KW == 3;
}

void dw_prep(const bf16* shadow, int ldb, int C, int taps, bf16* wdw, cudaStream_t st) {
  ProfScope ps(PC_DW, st);
  dw_prep_kernel<<<(C * taps + 255) / 256, 256, 0, st>>>(shadow, ldb, C, taps, wdw);
  CK(cudaGetLastError());
}

void dw_fwd(const DwArgs& a, cudaStream_t st) {
  const long long total = (long long)a.n_static * a.Ho * a.Wo * (a.C / 8);
  if (total <= 0) return;
  ProfScope ps(PC_DW, st);
  dw_fwd_kernel<<<grid_for(total), 256, 0, st>>>(a);
  CK(cudaGetLastError());
}

void dw_dgrad(const DwArgs& a, cudaStream_t st) {
  const long long total = (long long)a.n_static * a.H * a.W * (a.C / 8);
  if (total <= 0) return;
  ProfScope ps(PC_DW, st);
  dw_dgrad_kernel<<<grid_for(total), 256, 0, st>>>(a);
  CK(cudaGetLastError());
}

size_t dw_wgrad_ws_bytes(const ConvGeom& g, int n) {
  return (size_t)4 * num_sms() * g.Cout * 10 * 4 + 256;
}

void dw_wgrad(const DwArgs& a, float* ws, size_t ws_bytes, float* dw, float* db, cudaStream_t st) {
  const long long npix = (long long)a.n_static * a.Ho * a.Wo;
  if (npix <= 0) return;
  const int CG = a.C / 8;
  int nchunks = (int)std::max(1LL, std::min<long long>((4LL * num_sms() + CG - 1) / CG, (npix + 1023) / 1024));
  while ((size_t)nchunks * a.C * 10 * 4 > ws_bytes && nchunks > 1) nchunks /= 2;
  const long long per = (npix + nchunks - 1) / nchunks;
  ProfScope ps(PC_DW, st, 2);
  dw_wgrad_partial_kernel<<<dim3(nchunks, CG), DWW_THREADS, (DWW_THREADS / 32) * 8 * 10 * 4, st>>>(a, per, ws);
  dw_wgrad_final_kernel<<<(a.C * 10 + 255) / 256, 256, 0, st>>>(ws, nchunks, a.C, dw, db);
  CK(cudaGetLastError());
}

}  // namespace adainf

// CUDA-core kernels of the AdaInf hot path: input packing, max-pooling (fwd/bwd), the fused early-exit
// head (GAP -> FC -> softmax confidence / entropy / argmax -> threshold), the stable
// survivor compaction (ballot + block scan), exit losses and head gradients (a8-a9), and the fused
// SGD-momentum update with bf16-shadow refresh (a11).  All reductions use a fixed order (deterministic).
#include <cuda_bf16.h>

#include "common.cuh"
#include "kernels.cuh"
#include "pool_bwd.cuh"
#include "prof.h"

namespace adainf {

// ------------------------------------------------------------------------------------------------
__global__ void pack_input_kernel(const bf16* __restrict__ x, const int* __restrict__ map, const int* count,
                                  int n_static, int HW, int Cin, int Cpad, bf16* __restrict__ y) {
  const int n_rows = count ? *count : n_static;
  const long long total = (long long)n_rows * HW;
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < total; i += (long long)gridDim.x * blockDim.x) {
    const long long n = i / HW, pix = i - n * HW;
    const long long row = map ? map[n] : n;
    const long long src = row * (long long)HW + pix;
    bf16* o = y + i * Cpad;
    if (row < 0) {  // sanitised row (retrain_step_rows): zero input
      for (int c = 0; c < Cpad; ++c) o[c] = __float2bfloat16_rn(0.f);
      continue;
    }
    if (Cpad == 4) {
      __align__(8) bf16 v[4];
#pragma unroll
      for (int c = 0; c < 4; ++c) v[c] = c < Cin ? x[src * Cin + c] : __float2bfloat16_rn(0.f);
      *(uint2*)o = *(uint2*)v;
    } else {
      for (int c = 0; c < Cpad; ++c) o[c] = c < Cin ? x[src * Cin + c] : __float2bfloat16_rn(0.f);
    }
  }
}
void launch_pack_input(const bf16* x, const int* map, const int* count, int n_static, int H, int W, int Cin, int Cpad,
                       bf16* y, cudaStream_t st) {
  const long long total = (long long)n_static * H * W;
  const int blocks = (int)std::min<long long>((total + 255) / 256, 16LL * num_sms());
  if (blocks <= 0) return;
  ProfScope ps(PC_PACK, st);
  pack_input_kernel<<<blocks, 256, 0, st>>>(x, map, count, n_static, H * W, Cin, Cpad, y);
  CK(cudaGetLastError());
}

// ------------------------------------------------------------------------------------------------
__global__ void maxpool_fwd_kernel(const bf16* __restrict__ x, const int* __restrict__ map, const int* count,
                                   int n_static, int H, int W, int C, int K, int s, int p, int Ho, int Wo,
                                   bf16* __restrict__ y, uint8_t* __restrict__ amax, int fold_relu) {
  const int n_rows = count ? *count : n_static;
  const int CV = C / 8;
  const long long total = (long long)n_rows * Ho * Wo * CV;
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < total; i += (long long)gridDim.x * blockDim.x) {
    const int cv = (int)(i % CV);
    long long r = i / CV;
    const int wo = (int)(r % Wo);
    r /= Wo;
    const int ho = (int)(r % Ho);
    const long long n = r / Ho;
    const long long sn = map ? map[n] : n;
    float best[8];
    uint8_t arg[8];
#pragma unroll
    for (int q = 0; q < 8; ++q) {
      best[q] = -INFINITY;
      arg[q] = 0;
    }
    for (int kh = 0; kh < K; ++kh) {
      const int ih = ho * s - p + kh;
      if (ih < 0 || ih >= H) continue;
      for (int kw = 0; kw < K; ++kw) {
        const int iw = wo * s - p + kw;
        if (iw < 0 || iw >= W) continue;
        const uint4 raw = *(const uint4*)(x + ((sn * H + ih) * W + iw) * C + cv * 8);
        const bf16* h = (const bf16*)&raw;
#pragma unroll
        for (int q = 0; q < 8; ++q) {
          const float v = __bfloat162float(h[q]);
          if (v > best[q]) {  // strict: the FIRST maximal element in row-major window order
            best[q] = v;
            arg[q] = (uint8_t)(kh * K + kw);
          }
        }
      }
    }
    __align__(16) bf16 o[8];
#pragma unroll
    for (int q = 0; q < 8; ++q) o[q] = __float2bfloat16_rn(best[q]);
    const long long oi = ((n * Ho + ho) * Wo + wo) * C + cv * 8;
    *(uint4*)(y + oi) = *(uint4*)o;
    if (fold_relu)  // ReLU producer: a window whose max is not > 0 routes no gradient (act'(y) = 0)
#pragma unroll
      for (int q = 0; q < 8; ++q)
        if (!(best[q] > 0.f)) arg[q] = AMAX_MASKED;
    if (amax) *(uint2*)(amax + oi) = *(uint2*)arg;
  }
}
void launch_maxpool_fwd(const bf16* x, const int* map, const int* count, int n_static, int H, int W, int C, int K,
                        int s, int p, int Ho, int Wo, bf16* y, uint8_t* amax, int fold_relu, cudaStream_t st) {
  const long long total = (long long)n_static * Ho * Wo * (C / 8);
  const int blocks = (int)std::min<long long>((total + 255) / 256, 32LL * num_sms());
  if (blocks <= 0) return;
  ProfScope ps(PC_POOL_FWD, st);
  maxpool_fwd_kernel<<<blocks, 256, 0, st>>>(x, map, count, n_static, H, W, C, K, s, p, Ho, Wo, y, amax, fold_relu);
  CK(cudaGetLastError());
}

// Max-pool backward through the producer's activation: dz(pos) = act'(y(pos)) * sum of dT(w) over the windows
// w whose FIRST argmax is pos.  y(pos) equals the pooled value of any such window, so the activation mask
// is read from the pooled tensor P [n][Ho][Wo][C] (4x smaller than y for the 3x3/2 stem pool) instead of y.
// One thread per (n, ih, iw, 8-channel vector), fixed window order (ho, then wo ascending), 128-bit I/O.
__global__ void maxpool_bwd_kernel(const bf16* __restrict__ dT, const uint8_t* __restrict__ amax,
                                   const bf16* __restrict__ pooled, int act, long long n, int H, int W, int C, int K,
                                   int s, int p, int Ho, int Wo, bf16* __restrict__ dz) {
  const int CV = C / 8;
  const long long total = n * H * W * CV;
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < total; i += (long long)gridDim.x * blockDim.x) {
    const int cv = (int)(i % CV);
    long long r = i / CV;
    const int iw = (int)(r % W);
    r /= W;
    const int ih = (int)(r % H);
    const long long b = r / H;
    const int ho_lo = max(0, (ih + p - K + s) / s), ho_hi = min(Ho - 1, (ih + p) / s);
    const int wo_lo = max(0, (iw + p - K + s) / s), wo_hi = min(Wo - 1, (iw + p) / s);
    float acc[8], m[8];
#pragma unroll
    for (int q = 0; q < 8; ++q) acc[q] = 0.f, m[q] = 0.f;
    for (int ho = ho_lo; ho <= ho_hi; ++ho) {
      const int kh = ih - (ho * s - p);
      if (kh < 0 || kh >= K) continue;
      for (int wo = wo_lo; wo <= wo_hi; ++wo) {
        const int kw = iw - (wo * s - p);
        if (kw < 0 || kw >= K) continue;
        const long long oi = ((b * Ho + ho) * Wo + wo) * C + cv * 8;
        const uint2 am = __ldg((const uint2*)(amax + oi));
        const uint8_t* a8 = (const uint8_t*)&am;
        const uint4 dv = __ldg((const uint4*)(dT + oi));
        const bf16* d8 = (const bf16*)&dv;
        uint4 pv = make_uint4(0u, 0u, 0u, 0u);
        if (act != 1) pv = __ldg((const uint4*)(pooled + oi));  // ReLU: mask folded into the codes
        const bf16* p8 = (const bf16*)&pv;
        const uint8_t me = (uint8_t)(kh * K + kw);
#pragma unroll
        for (int q = 0; q < 8; ++q)
          if (a8[q] == me) {
            acc[q] = __fadd_rn(acc[q], __bfloat162float(d8[q]));
            m[q] = act == 1 ? 1.f : act_grad(act, __bfloat162float(p8[q]));
          }
      }
    }
    const long long xi = ((b * H + ih) * W + iw) * C + cv * 8;
    __align__(16) bf16 o[8];
#pragma unroll
    for (int q = 0; q < 8; ++q) o[q] = __float2bfloat16_rn(__fmul_rn(acc[q], m[q]));
    *(uint4*)(dz + xi) = *(uint4*)o;
  }
}
// stride-2 fast path: one thread per (n, 2x2 input block, 8-channel vector); each window touching the
// block is read once (argmax + dT + pooled value, 128-bit), its gradient routed to the block element it
// selected; the per-element window order is the same as the gather kernel's (ho, then wo ascending)
__global__ void maxpool_bwd_s2_kernel(const bf16* __restrict__ dT, const uint8_t* __restrict__ amax,
                                      const bf16* __restrict__ pooled, int act, long long n, int H, int W, int C,
                                      int K, int p, int Ho, int Wo, bf16* __restrict__ dz) {
  const int CV = C / 8;
  const int BH = (H + 1) / 2, BW = (W + 1) / 2;
  const long long total = n * BH * BW * CV;
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < total; i += (long long)gridDim.x * blockDim.x) {
    const int cv = (int)(i % CV);
    long long r = i / CV;
    const int bj = (int)(r % BW);
    r /= BW;
    const int bi = (int)(r % BH);
    const long long b = r / BH;
    const int ih0 = 2 * bi, iw0 = 2 * bj;
    float acc[2][2][8], m[2][2][8];
#pragma unroll
    for (int u = 0; u < 2; ++u)
#pragma unroll
      for (int v = 0; v < 2; ++v)
#pragma unroll
        for (int q = 0; q < 8; ++q) acc[u][v][q] = 0.f, m[u][v][q] = 0.f;
    const int ho_lo = max(0, (ih0 + p - K + 2) / 2), ho_hi = min(Ho - 1, (ih0 + 1 + p) / 2);
    const int wo_lo = max(0, (iw0 + p - K + 2) / 2), wo_hi = min(Wo - 1, (iw0 + 1 + p) / 2);
    for (int ho = ho_lo; ho <= ho_hi; ++ho)
      for (int wo = wo_lo; wo <= wo_hi; ++wo) {
        const long long oi = ((b * Ho + ho) * Wo + wo) * C + cv * 8;
        const uint2 am = __ldg((const uint2*)(amax + oi));
        const uint8_t* a8 = (const uint8_t*)&am;
        const uint4 dv = __ldg((const uint4*)(dT + oi));
        const bf16* d8 = (const bf16*)&dv;
        uint4 pv = make_uint4(0u, 0u, 0u, 0u);
        if (act != 1) pv = __ldg((const uint4*)(pooled + oi));  // ReLU: mask folded into the codes
        const bf16* p8 = (const bf16*)&pv;
#pragma unroll
        for (int q = 0; q < 8; ++q) {
          if (a8[q] == AMAX_MASKED) continue;
          const int kh = a8[q] / K, kw = a8[q] - (a8[q] / K) * K;
          const int u = ho * 2 - p + kh - ih0, v = wo * 2 - p + kw - iw0;
          const float g = __bfloat162float(d8[q]);
          const float mg = act == 1 ? 1.f : act_grad(act, __bfloat162float(p8[q]));
#pragma unroll
          for (int uu = 0; uu < 2; ++uu)
#pragma unroll
            for (int vv = 0; vv < 2; ++vv)
              if (u == uu && v == vv) {
                acc[uu][vv][q] = __fadd_rn(acc[uu][vv][q], g);
                m[uu][vv][q] = mg;
              }
        }
      }
#pragma unroll
    for (int u = 0; u < 2; ++u)
#pragma unroll
      for (int v = 0; v < 2; ++v) {
        const int ih = ih0 + u, iw = iw0 + v;
        if (ih >= H || iw >= W) continue;
        const long long xi = ((b * H + ih) * W + iw) * C + cv * 8;
        __align__(16) bf16 o[8];
#pragma unroll
        for (int q = 0; q < 8; ++q) o[q] = __float2bfloat16_rn(__fmul_rn(acc[u][v][q], m[u][v][q]));
        *(uint4*)(dz + xi) = *(uint4*)o;
      }
  }
}

// 3x3 / stride 2 / pad 1 (the ResNet stem pool) with the ReLU mask folded into the codes (or no activation):
// one thread per (n, 2x2 input block, 8-channel vector).  Block (bi, bj) is covered by windows (bi|bi+1, bj|bj+1)
// only; each of its four positions has a fixed set of (window, code) pairs that can select it:
//   (0,0): w00 code 4     (0,1): w00 5, w01 3     (1,0): w00 7, w10 1     (1,1): w00 8, w01 6, w10 2, w11 0
// summed in window order (ho, then wo ascending) like the generic kernels.  128-bit dT loads, 64-bit codes,
// no reads of the pooled tensor.
__global__ void __launch_bounds__(256) maxpool_bwd_k3s2_kernel(const bf16* __restrict__ dT,
                                                               const uint8_t* __restrict__ amax, long long n, int H,
                                                               int W, int C, int Ho, int Wo, bf16* __restrict__ dz) {
  const int CV = C / 8;
  const int BH = (H + 1) / 2, BW = (W + 1) / 2;
  const long long total = n * BH * BW * CV;
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < total; i += (long long)gridDim.x * blockDim.x) {
    const int cv = (int)(i % CV);
    long long r = i / CV;
    const int bj = (int)(r % BW);
    r /= BW;
    const int bi = (int)(r % BH);
    const long long b = r / BH;
    uint2 cw[4];
    uint4 gw[4];
    pool_bwd_k3s2_load(dT, amax, b, bi, bj, cv, C, Ho, Wo, cw, gw);
    uint4 ob[4];
    pool_bwd_k3s2_block(cw, gw, ob);
    const int ih = 2 * bi, iw = 2 * bj;
    bf16* d0 = dz + ((b * H + ih) * W + iw) * C + cv * 8;
    *(uint4*)d0 = ob[0];
    if (iw + 1 < W) *(uint4*)(d0 + C) = ob[1];
    if (ih + 1 < H) {
      bf16* d1 = d0 + (long long)W * C;
      *(uint4*)d1 = ob[2];
      if (iw + 1 < W) *(uint4*)(d1 + C) = ob[3];
    }
  }
}

void launch_maxpool_bwd(const bf16* dT, const uint8_t* amax, const bf16* pooled, int act, int n, int H, int W, int C,
                        int K, int s, int p, int Ho, int Wo, bf16* dz, cudaStream_t st) {
  ProfScope ps(PC_POOL_BWD, st);
  if (K == 3 && s == 2 && p == 1 && (act == 0 || act == 1)) {
    const long long total = (long long)n * ((H + 1) / 2) * ((W + 1) / 2) * (C / 8);
    const int blocks = (int)std::min<long long>((total + 255) / 256, 16LL * num_sms());
    maxpool_bwd_k3s2_kernel<<<blocks, 256, 0, st>>>(dT, amax, n, H, W, C, Ho, Wo, dz);
  } else if (s == 2) {
    const long long total = (long long)n * ((H + 1) / 2) * ((W + 1) / 2) * (C / 8);
    const int blocks = (int)std::min<long long>((total + 255) / 256, 64LL * num_sms());
    maxpool_bwd_s2_kernel<<<blocks, 256, 0, st>>>(dT, amax, pooled, act, n, H, W, C, K, p, Ho, Wo, dz);
  } else {
    const long long total = (long long)n * H * W * (C / 8);
    const int blocks = (int)std::min<long long>((total + 255) / 256, 64LL * num_sms());
    maxpool_bwd_kernel<<<blocks, 256, 0, st>>>(dT, amax, pooled, act, n, H, W, C, K, s, p, Ho, Wo, dz);
  }
  CK(cudaGetLastError());
}

// ------------------------------------------------------------------------------------------------
// Fused exit head: one CTA per dense row.  GAP over HW with 16-byte loads (channel vector v = t % (C/8),
// pixel group t / (C/8)), fixed-order reduction, FC in fp32, softmax statistics with IEEE expf/logf.
// EH_THREADS = 128 for large batches (a 1,024-row exit fits one wave, 12 CTAs / SM), 512 when the rows alone
// cannot fill the SMs (each row then has 4x the loads in flight)
template <int EH_THREADS>
__global__ void __launch_bounds__(EH_THREADS) exit_head_kernel(const ExitHeadArgs a) {
  const int n_rows = a.count ? *a.count : a.n_static;
  const int j = blockIdx.x;
  if (j >= n_rows) return;
  extern __shared__ float sh[];  // [EH_THREADS/CV][C] partials, then pooled[C], logits[ncls]
  const int C = a.C, CV = C / 8;
  const int groups = EH_THREADS / CV;
  const int t = threadIdx.x;
  float acc[8];
#pragma unroll
  for (int q = 0; q < 8; ++q) acc[q] = 0.f;
  const int v = t % CV, g0 = t / CV;
  if (g0 < groups) {
    const bf16* base = a.fmap + (long long)j * a.HW * C + v * 8;
    // eight independent 16-byte loads in flight per thread, accumulated in the same (ascending pixel) order
    int pix = g0;
    for (; pix + 7 * groups < a.HW; pix += 8 * groups) {
      uint4 raw[8];
#pragma unroll
      for (int u = 0; u < 8; ++u) raw[u] = __ldg((const uint4*)(base + (long long)(pix + u * groups) * C));
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        const bf16* h = (const bf16*)&raw[u];
#pragma unroll
        for (int q = 0; q < 8; ++q) acc[q] += __bfloat162float(h[q]);
      }
    }
    for (; pix < a.HW; pix += groups) {
      const uint4 raw = __ldg((const uint4*)(base + (long long)pix * C));
      const bf16* h = (const bf16*)&raw;
#pragma unroll
      for (int q = 0; q < 8; ++q) acc[q] += __bfloat162float(h[q]);
    }
#pragma unroll
    for (int q = 0; q < 8; ++q) sh[g0 * C + v * 8 + q] = acc[q];
  }
  __syncthreads();
  float* pooled = sh + groups * C;
  float* logits = pooled + C;
  const float inv_hw = 1.0f / (float)a.HW;
  for (int c = t; c < C; c += EH_THREADS) {
    float s = 0.f;
    for (int g = 0; g < groups; ++g) s += sh[g * C + c];
    pooled[c] = s * inv_hw;
  }
  __syncthreads();
  // FC: one warp per class, lanes stride the channels, fixed xor-tree reduction (deterministic)
  {
    const int wp = t >> 5, ln = t & 31;
    for (int k = wp; k < a.ncls; k += EH_THREADS / 32) {
      float l = 0.f;
      for (int c = ln; c < C; c += 32) l = fmaf(pooled[c], __ldg(a.Wk + c * a.ncls + k), l);
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) l += __shfl_xor_sync(0xffffffffu, l, o);
      if (ln == 0) logits[k] = __fadd_rn(l, a.bk[k]);
    }
  }
  __syncthreads();
  const int orig = a.orig ? a.orig[j] : j;
  if (a.embed)
    for (int c = t; c < C; c += EH_THREADS) a.embed[(long long)orig * C + c] = pooled[c];
  if (a.pooled_save)
    for (int c = t; c < C; c += EH_THREADS) a.pooled_save[(long long)j * C + c] = pooled[c];
  if (a.logits_save)
    for (int k = t; k < a.ncls; k += EH_THREADS) a.logits_save[(long long)j * a.ncls + k] = logits[k];
  __shared__ int s_exit;
  if (t == 0) {
    int am = 0;
    for (int k = 1; k < a.ncls; ++k)
      if (logits[k] > logits[am]) am = k;
    const float m = logits[am];
    float s = 0.f, tt = 0.f;
    for (int k = 0; k < a.ncls; ++k) {
      const float e = expf(logits[k] - m);
      s += e;
      tt += e * (logits[k] - m);
    }
    const float conf = 1.0f / s;
    const float ent = logf(s) - tt / s;
    const int ex = a.is_final || conf >= a.tau;
    s_exit = ex;
    if (a.alive) a.alive[j] = (uint8_t)(!ex);
    if (ex) {
      if (a.exit_id) a.exit_id[orig] = (int8_t)a.exit_index;
      if (a.pred) a.pred[orig] = am;
      if (a.conf) a.conf[orig] = conf;
      if (a.entropy) a.entropy[orig] = ent;
    }
  }
  __syncthreads();
  if (s_exit && a.logits)
    for (int k = t; k < a.ncls; k += EH_THREADS) a.logits[(long long)orig * a.ncls + k] = logits[k];
}
void launch_exit_head(const ExitHeadArgs& a, cudaStream_t st, int prof_class) {
  if (a.n_static <= 0) return;
  bool wide = a.n_static < 4 * num_sms();
  bool widest = a.n_static <= 2 * num_sms();  // a row per CTA cannot fill the SMs: 1,024 threads per row
  int T = widest ? 1024 : (wide ? 512 : 128);
  if (a.C % 8 || a.C / 8 > 1024) throw ShapeError("exit head: C must be a multiple of 8, <= 8192");
  while (a.C / 8 > T) T = T == 128 ? 512 : 1024;  // every 8-channel vector needs a thread
  widest = T == 1024;
  wide = T == 512;
  const int groups = T / (a.C / 8);
  const size_t smem = (size_t)(groups * a.C + a.C + a.ncls) * sizeof(float);
  ProfScope ps(prof_class, st);
  if (widest) exit_head_kernel<1024><<<a.n_static, 1024, smem, st>>>(a);
  else if (wide) exit_head_kernel<512><<<a.n_static, 512, smem, st>>>(a);
  else exit_head_kernel<128><<<a.n_static, 128, smem, st>>>(a);
  CK(cudaGetLastError());
}

// ------------------------------------------------------------------------------------------------
// K4 + K5 in one kernel (north_star "exit heads"): per row the exit head (GAP -> FC -> softmax confidence /
// entropy / argmax), the threshold decision, and the stable compaction of the survivors by a single-pass
// decoupled look-back scan over the rows (row order = ticket order, so every predecessor is resident or done:
// no deadlock), then each surviving CTA copies its own row of the stage tensor to its compacted slot of the next
// stage's dense input (the row was just streamed for the GAP, so the copy reads it back from L2).
// Status words: bits 31..30 = 1 (aggregate of this row) / 2 (inclusive prefix), bits 29..0 = value; the workspace
// ([0] ticket, [1..] status per row) is zeroed by a memset node before the kernel.
struct ExitFusedArgs {
  ExitHeadArgs h;
  unsigned* ws;
  int* pos_next;
  int* orig_next;
  int* count_next;
  int32_t* counts_out;
  int32_t* surv_out;
  int32_t* last_count_out;
  int last_index;
  const bf16* src;   // stage tensor rows [n][row_elems] (nullptr: no survivor copy)
  bf16* dense_next;  // [n][row_elems]
  long long row_elems;
};

__device__ __forceinline__ unsigned ld_acquire_u32(const unsigned* p) {
  unsigned v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release_u32(unsigned* p, unsigned v) {
  asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

template <int EH_THREADS>
__global__ void __launch_bounds__(EH_THREADS) exit_fused_kernel(const ExitFusedArgs F) {
  const ExitHeadArgs& a = F.h;
  __shared__ int s_row, s_exit, s_am, s_excl;
  __shared__ float s_conf, s_ent;
  const int t = threadIdx.x;
  if (t == 0) s_row = (int)atomicAdd(F.ws, 1u);
  __syncthreads();
  const int j = s_row;
  const int n_rows = a.count ? *a.count : a.n_static;
  if (j >= n_rows) {
    if (n_rows == 0 && j == 0 && t == 0 && !a.is_final) {  // empty stage: the counts still have to be written
      *F.count_next = 0;
      if (F.counts_out) {
        F.counts_out[a.exit_index] = 0;
        if (F.last_count_out) F.counts_out[F.last_index] = 0;
      }
    }
    return;
  }
  extern __shared__ float sh[];
  const int C = a.C, CV = C / 8;
  const int groups = EH_THREADS / CV;
  float acc[8];
#pragma unroll
  for (int q = 0; q < 8; ++q) acc[q] = 0.f;
  const int v = t % CV, g0 = t / CV;
  if (g0 < groups) {
    const bf16* base = a.fmap + (long long)j * a.HW * C + v * 8;
    int pix = g0;
    for (; pix + 7 * groups < a.HW; pix += 8 * groups) {
      uint4 raw[8];
#pragma unroll
      for (int u = 0; u < 8; ++u) raw[u] = __ldg((const uint4*)(base + (long long)(pix + u * groups) * C));
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        const bf16* hh = (const bf16*)&raw[u];
#pragma unroll
        for (int q = 0; q < 8; ++q) acc[q] += __bfloat162float(hh[q]);
      }
    }
    for (; pix < a.HW; pix += groups) {
      const uint4 raw = __ldg((const uint4*)(base + (long long)pix * C));
      const bf16* hh = (const bf16*)&raw;
#pragma unroll
      for (int q = 0; q < 8; ++q) acc[q] += __bfloat162float(hh[q]);
    }
#pragma unroll
    for (int q = 0; q < 8; ++q) sh[g0 * C + v * 8 + q] = acc[q];
  }
  __syncthreads();
  float* pooled = sh + groups * C;
  float* logits = pooled + C;
  const float inv_hw = 1.0f / (float)a.HW;
  for (int c = t; c < C; c += EH_THREADS) {
    float s = 0.f;
    for (int g = 0; g < groups; ++g) s += sh[g * C + c];
    pooled[c] = s * inv_hw;
  }
  __syncthreads();
  {
    const int wp = t >> 5, ln = t & 31;
    for (int k = wp; k < a.ncls; k += EH_THREADS / 32) {
      float l = 0.f;
      for (int c = ln; c < C; c += 32) l = fmaf(pooled[c], __ldg(a.Wk + c * a.ncls + k), l);
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) l += __shfl_xor_sync(0xffffffffu, l, o);
      if (ln == 0) logits[k] = __fadd_rn(l, a.bk[k]);
    }
  }
  __syncthreads();
  const int orig = a.orig ? a.orig[j] : j;
  if (a.embed)
    for (int c = t; c < C; c += EH_THREADS) a.embed[(long long)orig * C + c] = pooled[c];
  if (t == 0) {
    int am = 0;
    for (int k = 1; k < a.ncls; ++k)
      if (logits[k] > logits[am]) am = k;
    const float m = logits[am];
    float s = 0.f, tt = 0.f;
    for (int k = 0; k < a.ncls; ++k) {
      const float e = expf(logits[k] - m);
      s += e;
      tt += e * (logits[k] - m);
    }
    const float conf = 1.0f / s;
    s_conf = conf;
    s_ent = logf(s) - tt / s;
    s_am = am;
    s_exit = a.is_final || conf >= a.tau;
  }
  __syncthreads();
  const int ex = s_exit;
  if (ex) {
    if (t == 0) {
      if (a.exit_id) a.exit_id[orig] = (int8_t)a.exit_index;
      if (a.pred) a.pred[orig] = s_am;
      if (a.conf) a.conf[orig] = s_conf;
      if (a.entropy) a.entropy[orig] = s_ent;
    }
    if (a.logits)
      for (int k = t; k < a.ncls; k += EH_THREADS) a.logits[(long long)orig * a.ncls + k] = logits[k];
  }
  if (a.is_final) return;
  // ---- decoupled look-back: exclusive count of surviving rows before j ----
  unsigned* status = F.ws + 1;
  const unsigned mine = ex ? 0u : 1u;
  if (t < 32) {
    if (t == 0) st_release_u32(status + j, (1u << 30) | mine);
    int excl = 0;
    int k = j - 1;
    while (k >= 0) {
      const int idx = k - t;  // lane t looks at row k - t
      unsigned sv = 0;
      bool ready;
      do {
        sv = idx >= 0 ? ld_acquire_u32(status + idx) : (2u << 30);
        ready = (sv >> 30) != 0;
      } while (!__all_sync(0xffffffffu, ready));
      const unsigned incl_mask = __ballot_sync(0xffffffffu, idx >= 0 && (sv >> 30) == 2u);
      // lanes up to (and including) the first inclusive prefix contribute
      const int stop = incl_mask ? __ffs(incl_mask) - 1 : 31;
      int val = (t <= stop && idx >= 0) ? (int)(sv & 0x3FFFFFFFu) : 0;
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) val += __shfl_xor_sync(0xffffffffu, val, o);
      excl += val;
      if (incl_mask) break;
      k -= 32;
    }
    if (t == 0) {
      st_release_u32(status + j, (2u << 30) | (unsigned)(excl + (int)mine));
      s_excl = excl;
      if (j == n_rows - 1) {
        const int nn = excl + (int)mine;
        *F.count_next = nn;
        if (F.counts_out) {
          F.counts_out[a.exit_index] = n_rows - nn;
          if (F.last_count_out) F.counts_out[F.last_index] = nn;
        }
      }
    }
  }
  __syncthreads();
  if (ex) return;
  const int o = s_excl;
  if (t == 0) {
    F.pos_next[o] = j;
    F.orig_next[o] = orig;
    if (F.surv_out) F.surv_out[o] = orig;
  }
  if (F.src) {
    const uint4* sp = (const uint4*)(F.src + (long long)j * F.row_elems);
    uint4* dp = (uint4*)(F.dense_next + (long long)o * F.row_elems);
    const long long nv = F.row_elems / 8;
    for (long long i = t; i < nv; i += EH_THREADS) dp[i] = sp[i];
  }
}

size_t exit_fused_ws_bytes(int max_batch) { return (size_t)(max_batch + 1) * 4; }

void launch_exit_fused(const ExitHeadArgs& h, unsigned* ws, int* pos_next, int* orig_next, int* count_next,
                       int32_t* counts_out, int32_t* surv_out, int32_t* last_count_out, int last_index,
                       const bf16* src, bf16* dense_next, long long row_elems, cudaStream_t st) {
  if (h.n_static <= 0) return;
  bool wide = h.n_static < 4 * num_sms();
  bool widest = h.n_static <= 2 * num_sms();
  int T = widest ? 1024 : (wide ? 512 : 128);
  if (h.C % 8 || h.C / 8 > 1024) throw ShapeError("exit head: C must be a multiple of 8, <= 8192");
  while (h.C / 8 > T) T = T == 128 ? 512 : 1024;
  widest = T == 1024;
  wide = T == 512;
  if (src && (row_elems % 8)) throw ShapeError("exit_fused: row must be a multiple of 16 bytes");
  const int groups = T / (h.C / 8);
  const size_t smem = (size_t)(groups * h.C + h.C + h.ncls) * sizeof(float);
  ExitFusedArgs F{h, ws, pos_next, orig_next, count_next, counts_out, surv_out, last_count_out, last_index, src,
                  dense_next, row_elems};
  CK(cudaMemsetAsync(ws, 0, (size_t)(h.n_static + 1) * 4, st));
  ProfScope ps(PC_EXIT_HEAD, st);
  if (widest) exit_fused_kernel<1024><<<h.n_static, 1024, smem, st>>>(F);
  else if (wide) exit_fused_kernel<512><<<h.n_static, 512, smem, st>>>(F);
  else exit_fused_kernel<128><<<h.n_static, 128, smem, st>>>(F);
  CK(cudaGetLastError());
}

// ------------------------------------------------------------------------------------------------
// Stable compaction of alive rows (warp ballot + popc, block scan), single CTA, rows in chunks of 1024.
__global__ void __launch_bounds__(1024) compact_kernel(const uint8_t* __restrict__ alive, const int* count,
                                                       int n_static, const int* __restrict__ orig,
                                                       int* __restrict__ pos_next, int* __restrict__ orig_next,
                                                       int* count_next, int32_t* counts_out, int exit_index,
                                                       int32_t* surv_out, int32_t* last_count_out, int last_index) {
  __shared__ int warp_tot[32];
  __shared__ int base_s;
  const int n_rows = count ? *count : n_static;
  const int t = threadIdx.x, lane = t & 31, w = t >> 5;
  if (t == 0) base_s = 0;
  __syncthreads();
  for (int c0 = 0; c0 < n_rows; c0 += 1024) {
    const int j = c0 + t;
    const bool f = j < n_rows && alive[j];
    const unsigned bal = __ballot_sync(0xffffffffu, f);
    const int wpre = __popc(bal & ((1u << lane) - 1u));
    if (lane == 0) warp_tot[w] = __popc(bal);
    __syncthreads();
    if (w == 0) {
      int v = warp_tot[lane];
      for (int o = 1; o < 32; o <<= 1) {
        const int u = __shfl_up_sync(0xffffffffu, v, o);
        if (lane >= o) v += u;
      }
      warp_tot[lane] = v;  // inclusive
    }
    __syncthreads();
    const int base = base_s;
    const int wbase = w ? warp_tot[w - 1] : 0;
    if (f) {
      const int o = base + wbase + wpre;
      const int og = orig ? orig[j] : j;
      pos_next[o] = j;
      orig_next[o] = og;
      if (surv_out) surv_out[o] = og;
    }
    __syncthreads();
    if (t == 0) base_s = base + warp_tot[31];
    __syncthreads();
  }
  if (t == 0) {
    const int nn = base_s;
    *count_next = nn;
    if (counts_out) {
      counts_out[exit_index] = n_rows - nn;
      if (last_count_out) counts_out[last_index] = nn;
    }
  }
}
void launch_compact(const uint8_t* alive, const int* count, int n_static, const int* orig, int* pos_next,
                    int* orig_next, int* count_next, int32_t* counts_out, int exit_index, int32_t* surv_out,
                    int32_t* last_count_out, int last_index, cudaStream_t st) {
  ProfScope ps(PC_COMPACT, st);
  compact_kernel<<<1, 1024, 0, st>>>(alive, count, n_static, orig, pos_next, orig_next, count_next, counts_out,
                                     exit_index, surv_out, last_count_out, last_index);
  CK(cudaGetLastError());
}

// ------------------------------------------------------------------------------------------------
__global__ void exit_loss_kernel(const float* __restrict__ logits, const int32_t* __restrict__ labels, int n,
                                 int ncls, float w, float inv_n, float* __restrict__ dl, float* __restrict__ loss_rows,
                                 int accumulate) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  const float* l = logits + (long long)i * ncls;
  float m = l[0];
  for (int k = 1; k < ncls; ++k) m = fmaxf(m, l[k]);
  float s = 0.f;
  for (int k = 0; k < ncls; ++k) s += expf(l[k] - m);
  const int y = labels[i];
  if (y < 0 || y >= ncls) {  // ignored row (label outside [0, ncls), e.g. a sanitised pool row): no loss, no gradient
    for (int k = 0; k < ncls; ++k) dl[(long long)i * ncls + k] = 0.f;
    if (!accumulate) loss_rows[i] = 0.f;
    return;
  }
  for (int k = 0; k < ncls; ++k) {
    const float p = expf(l[k] - m) / s;
    dl[(long long)i * ncls + k] = w * (p - (k == y ? 1.f : 0.f)) * inv_n;
  }
  const float ce = (logf(s) - (l[y] - m)) * w * inv_n;
  loss_rows[i] = accumulate ? loss_rows[i] + ce : ce;
}
// retrain_step_rows: row r reads pool row idx[r] with label pool_labels[idx[r]] when r < *count (count nullable)
// and 0 <= idx[r] < pool_rows; otherwise map -1 (zero input) and label -1 (ignored by the loss)
__global__ void sanitize_rows_kernel(const int32_t* __restrict__ pool_labels, const int32_t* __restrict__ idx,
                                     const int32_t* __restrict__ count, int n, long long pool_rows,
                                     int32_t* __restrict__ map, int32_t* __restrict__ labels) {
  const int r = blockIdx.x * blockDim.x + threadIdx.x;
  if (r >= n) return;
  const int lim = count ? min(*count, n) : n;
  const int q = idx[r];
  const bool ok = r < lim && q >= 0 && (long long)q < pool_rows;
  map[r] = ok ? q : -1;
  labels[r] = ok ? pool_labels[q] : -1;
}
void launch_sanitize_rows(const int32_t* pool_labels, const int32_t* idx, const int32_t* count, int n,
                          long long pool_rows, int32_t* map, int32_t* labels, cudaStream_t st) {
  ProfScope ps(PC_GATHER, st);
  sanitize_rows_kernel<<<(n + 255) / 256, 256, 0, st>>>(pool_labels, idx, count, n, pool_rows, map, labels);
  CK(cudaGetLastError());
}

void launch_exit_loss(const float* logits, const int32_t* labels, int n, int ncls, float w, float inv_n, float* dl,
                      float* loss_rows, int accumulate, cudaStream_t st) {
  ProfScope ps(PC_EXIT_LOSS, st);
  exit_loss_kernel<<<(n + 127) / 128, 128, 0, st>>>(logits, labels, n, ncls, w, inv_n, dl, loss_rows, accumulate);
  CK(cudaGetLastError());
}

// dW[c][k] = sum_n pooled[n][c] dl[n][k] (+ db = sum_n dl[n][k]): stage 1, CTA (32-channel slab, sample split)
// writes fixed-order partials part[split][c][k] (c == C is the bias row); stage 2 sums the splits in order.
constexpr int HEAD_SPLIT_ROWS = 32;
__global__ void head_dw_partial_kernel(const float* __restrict__ pooled, const float* __restrict__ dl, int n, int C,
                                       int ncls, int chunk, float* __restrict__ part) {
  __shared__ float red[8][32][33];
  const int c = blockIdx.x * 32 + (threadIdx.x & 31);
  const int sl = threadIdx.x >> 5;  // 8 sample slices
  const bool bias_blk = blockIdx.x == (C + 31) / 32;
  const int i0 = blockIdx.y * chunk, i1 = min(n, i0 + chunk);
  float* out = part + (long long)blockIdx.y * (C + 1) * ncls;
  for (int k0 = 0; k0 < ncls; k0 += 32) {
    float acc[32];
#pragma unroll
    for (int k = 0; k < 32; ++k) acc[k] = 0.f;
    for (int i = i0 + sl; i < i1; i += 8) {
      const float pv = bias_blk ? 1.f : (c < C ? __ldg(pooled + (long long)i * C + c) : 0.f);
      const float* d = dl + (long long)i * ncls + k0;
#pragma unroll
      for (int k = 0; k < 32; ++k)
        if (k0 + k < ncls) acc[k] = fmaf(pv, __ldg(d + k), acc[k]);
    }
#pragma unroll
    for (int k = 0; k < 32; ++k) red[sl][threadIdx.x & 31][k] = acc[k];
    __syncthreads();
    for (int e = threadIdx.x; e < 32 * 32; e += 256) {
      const int cc = e >> 5, k = e & 31;
      const int ch = bias_blk ? C : blockIdx.x * 32 + cc;
      if (k0 + k >= ncls || (bias_blk ? cc != 0 : ch >= C)) continue;
      float sum = 0.f;
#pragma unroll
      for (int q = 0; q < 8; ++q) sum += red[q][cc][k];
      out[(long long)ch * ncls + k0 + k] = sum;
    }
    __syncthreads();
  }
}
__global__ void head_dw_final_kernel(const float* __restrict__ part, int splits, int C, int ncls,
                                     float* __restrict__ dW, float* __restrict__ db) {
  const int e = blockIdx.x * blockDim.x + threadIdx.x;
  const int per = (C + 1) * ncls;
  if (e >= per) return;
  float sum = 0.f;
  for (int sp = 0; sp < splits; ++sp) sum += __ldg(part + (long long)sp * per + e);
  if (e < C * ncls) dW[e] = sum;
  else db[e - C * ncls] = sum;
}
__global__ void head_bcast_kernel(const float* __restrict__ dl, const float* __restrict__ Wk, int n, int C, int ncls,
                                  float inv_hw, float* __restrict__ bcast) {
  const long long idx = blockIdx.x * (long long)blockDim.x + threadIdx.x;
  if (idx >= (long long)n * C) return;
  const int c = (int)(idx % C);
  const long long i = idx / C;
  float acc = 0.f;
  for (int k = 0; k < ncls; ++k) acc = fmaf(dl[i * ncls + k], Wk[c * ncls + k], acc);
  bcast[idx] = acc * inv_hw;
}
size_t head_grads_ws_bytes(int n, int C, int ncls) {
  const int splits = std::max(1, std::min(64, (n + HEAD_SPLIT_ROWS - 1) / HEAD_SPLIT_ROWS));
  return (size_t)splits * (C + 1) * ncls * sizeof(float);
}
void launch_head_grads(const float* pooled, const float* dl, const float* Wk, int n, int C, int ncls, int HW,
                       float* dW, float* db, float* bcast, float* ws, cudaStream_t st) {
  ProfScope ps(PC_HEAD_GRADS, st, 3);
  const int splits = std::max(1, std::min(64, (n + HEAD_SPLIT_ROWS - 1) / HEAD_SPLIT_ROWS));
  const int chunk = (n + splits - 1) / splits;
  head_dw_partial_kernel<<<dim3((C + 31) / 32 + 1, splits), 256, 0, st>>>(pooled, dl, n, C, ncls, chunk, ws);
  head_dw_final_kernel<<<((C + 1) * ncls + 255) / 256, 256, 0, st>>>(ws, splits, C, ncls, dW, db);
  const long long nb = ((long long)n * C + 255) / 256;
  head_bcast_kernel<<<(unsigned)nb, 256, 0, st>>>(dl, Wk, n, C, ncls, 1.0f / (float)HW, bcast);
  CK(cudaGetLastError());
}

// one thread per 8-channel vector (C % 8 == 0): 128-bit bf16 loads / stores, float4 bcast loads
__global__ void grad_finalize_kernel(const float* __restrict__ bcast, const bf16* __restrict__ sc,
                                     const bf16* __restrict__ yact, int act, long long n, int HW, int C,
                                     bf16* __restrict__ dz) {
  const int CV = C / 8;
  const long long total = n * HW * CV;
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < total; i += (long long)gridDim.x * blockDim.x) {
    const int cv = (int)(i % CV);
    const long long b = i / ((long long)HW * CV);
    float v[8];
#pragma unroll
    for (int q = 0; q < 8; ++q) v[q] = 0.f;
    if (bcast) {
      const float4 b0 = __ldg((const float4*)(bcast + b * C + cv * 8)), b1 = __ldg((const float4*)(bcast + b * C + cv * 8 + 4));
      v[0] = b0.x, v[1] = b0.y, v[2] = b0.z, v[3] = b0.w, v[4] = b1.x, v[5] = b1.y, v[6] = b1.z, v[7] = b1.w;
    }
    if (sc) {
      const uint4 r = __ldg((const uint4*)(sc + i * 8));
#pragma unroll
      for (int q = 0; q < 8; ++q) v[q] = __fadd_rn(v[q], __bfloat162float(((const bf16*)&r)[q]));
    }
    const uint4 y = __ldg((const uint4*)(yact + i * 8));
    __align__(16) bf16 o[8];
#pragma unroll
    for (int q = 0; q < 8; ++q) o[q] = __float2bfloat16_rn(__fmul_rn(v[q], act_grad(act, __bfloat162float(((const bf16*)&y)[q]))));
    *(uint4*)(dz + i * 8) = *(const uint4*)o;
  }
}
__global__ void grad_finalize_scalar_kernel(const float* __restrict__ bcast, const bf16* __restrict__ sc,
                                            const bf16* __restrict__ yact, int act, long long n, int HW, int C,
                                            bf16* __restrict__ dz) {
  const long long total = n * HW * C;
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < total; i += (long long)gridDim.x * blockDim.x) {
    const int c = (int)(i % C);
    const long long b = i / ((long long)HW * C);
    float v = 0.f;
    if (bcast) v = __fadd_rn(v, bcast[b * C + c]);
    if (sc) v = __fadd_rn(v, __bfloat162float(sc[i]));
    v = __fmul_rn(v, act_grad(act, __bfloat162float(yact[i])));
    dz[i] = __float2bfloat16_rn(v);
  }
}
void launch_grad_finalize(const float* bcast, const bf16* sc, const bf16* yact, int act, int n, int HW, int C,
                          bf16* dz, cudaStream_t st) {
  const long long total = (long long)n * HW * C;
  const int blocks = (int)std::min<long long>((total + 255) / 256, 32LL * num_sms());
  ProfScope ps(PC_GRAD_FINALIZE, st);
  if (C % 8 == 0) {
    const int vb = (int)std::min<long long>((total / 8 + 255) / 256, 32LL * num_sms());
    grad_finalize_kernel<<<vb, 256, 0, st>>>(bcast, sc, yact, act, n, HW, C, dz);
  } else {
    grad_finalize_scalar_kernel<<<blocks, 256, 0, st>>>(bcast, sc, yact, act, n, HW, C, dz);
  }
  CK(cudaGetLastError());
}

__global__ void sum_kernel(const float* __restrict__ x, int n, float* out, float scale) {
  __shared__ float sh[1024];
  float acc = 0.f;
  for (int i = threadIdx.x; i < n; i += blockDim.x) acc += x[i];
  sh[threadIdx.x] = acc;
  __syncthreads();
  for (int o = blockDim.x / 2; o > 0; o >>= 1) {
    if (threadIdx.x < o) sh[threadIdx.x] += sh[threadIdx.x + o];
    __syncthreads();
  }
  if (threadIdx.x == 0) *out = scale == 0.f ? sh[0] : (scale < 0.f ? sqrtf(sh[0]) : sh[0] * scale);
}
__global__ void fill_i32_kernel(int32_t* p, int32_t v) { *p = v; }
void launch_fill_i32(int32_t* p, int32_t v, cudaStream_t st) {
  fill_i32_kernel<<<1, 1, 0, st>>>(p, v);
  CK(cudaGetLastError());
}
void launch_sum(const float* x, int n, float* out, float scale, cudaStream_t st) {
  ProfScope ps(PC_SUM, st);
  sum_kernel<<<1, 1024, 0, st>>>(x, n, out, scale);
  CK(cudaGetLastError());
}

// ------------------------------------------------------------------------------------------------
// Fused SGD + momentum (PyTorch semantics, reading Q9), 128-bit loads/stores of w, v, g, and the bf16
// shadow written in the GEMM-ready [Cout][ldb] layout for conv weights.  Blocks map to parameter
// segments through host-built tables so every thread's float4 stays inside one segment.
constexpr int SGD_THREADS = 256, SGD_VEC = 4, SGD_ITEMS = 2;  // 2048-element units: < 10% last-wave tail
constexpr int SGD_PER_BLOCK = SGD_THREADS * SGD_VEC * SGD_ITEMS;
static_assert(SGD_PER_BLOCK == SGD_BLOCK_ELEMS, "host partition unit");

__device__ __forceinline__ void shadow_store(const SgdSeg& sg, long long local, const float* w4, int cnt) {
  const int K = sg.taps * sg.cin;
#pragma unroll
  for (int q = 0; q < 4; ++q) {  // fully unrolled with a predicate: w4 stays in registers
    if (q >= cnt) break;
    const unsigned l = (unsigned)(local + q);
    const unsigned co = l / (unsigned)K;
    const int rem = (int)(l - co * (unsigned)K);
    const int tap = rem / sg.cin, ci = rem - tap * sg.cin;
    int col = tap * sg.cin_pad + ci;
    if (sg.cog) col += (int)(co / (unsigned)sg.cog) * sg.cin;  // block-diagonal (grouped conv)
    unsigned row = co;
    if (sg.shuf_g) {  // folded channel shuffle
      const unsigned Cs = (unsigned)(sg.cout / sg.shuf_g);
      row = (co % Cs) * (unsigned)sg.shuf_g + co / Cs;
    }
    sg.shadow[(long long)row * sg.ldb + col] = __float2bfloat16_rn(w4[q]);
  }
}

__global__ void __launch_bounds__(SGD_THREADS) sgd_kernel(float* __restrict__ w, float* __restrict__ v,
                                                          const float* __restrict__ g, float lr, float mu, float wd,
                                                          const SgdSeg* __restrict__ segs,
                                                          const int* __restrict__ block_seg,
                                                          const long long* __restrict__ block_start,
                                                          float* __restrict__ sq_partial) {
  const SgdSeg sg = segs[block_seg[blockIdx.x]];
  const long long start = block_start[blockIdx.x];
  const long long end = min(sg.off + sg.count, start + (long long)SGD_PER_BLOCK);
  float sq = 0.f;
  const bool vec_ok = ((sg.off & 3) == 0);
  // issue every 128-bit load of the thread's items first (12 loads in flight), then update and store
  float4 wl[SGD_ITEMS], vl[SGD_ITEMS], gl[SGD_ITEMS];
#pragma unroll
  for (int it = 0; it < SGD_ITEMS; ++it) {
    const long long i = start + ((long long)it * SGD_THREADS + threadIdx.x) * SGD_VEC;
    if (vec_ok && i + SGD_VEC <= end) {
      wl[it] = *(const float4*)(w + i);
      vl[it] = *(const float4*)(v + i);
      gl[it] = __ldg((const float4*)(g + i));
    }
  }
#pragma unroll
  for (int it = 0; it < SGD_ITEMS; ++it) {
    const long long i = start + ((long long)it * SGD_THREADS + threadIdx.x) * SGD_VEC;
    if (i >= end) continue;
    const int cnt = (int)min((long long)SGD_VEC, end - i);
    const bool full = vec_ok && cnt == 4;
    float wr[4], vr[4], gr[4];
    if (full) {
      wr[0] = wl[it].x, wr[1] = wl[it].y, wr[2] = wl[it].z, wr[3] = wl[it].w;
      vr[0] = vl[it].x, vr[1] = vl[it].y, vr[2] = vl[it].z, vr[3] = vl[it].w;
      gr[0] = gl[it].x, gr[1] = gl[it].y, gr[2] = gl[it].z, gr[3] = gl[it].w;
    } else {
#pragma unroll
      for (int q = 0; q < 4; ++q) {  // unrolled + predicated (a runtime trip count would demote wr/vr/gr to local memory)
        wr[q] = q < cnt ? w[i + q] : 0.f;
        vr[q] = q < cnt ? v[i + q] : 0.f;
        gr[q] = q < cnt ? g[i + q] : 0.f;
      }
    }
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      if (q < cnt) {
        sq = fmaf(gr[q], gr[q], sq);
        const float d = __fadd_rn(gr[q], __fmul_rn(wd, wr[q]));
        vr[q] = __fadd_rn(__fmul_rn(mu, vr[q]), d);
        wr[q] = __fsub_rn(wr[q], __fmul_rn(lr, vr[q]));
      }
    }
    if (full) {
      *(float4*)(w + i) = make_float4(wr[0], wr[1], wr[2], wr[3]);
      *(float4*)(v + i) = make_float4(vr[0], vr[1], vr[2], vr[3]);
    } else {
#pragma unroll
      for (int q = 0; q < 4; ++q)
        if (q < cnt) w[i + q] = wr[q], v[i + q] = vr[q];
    }
    if (sg.shadow) {
      const long long local = i - sg.off;
      if (sg.cin == sg.cin_pad && !sg.shuf_g && (sg.cin & 3) == 0 && cnt == 4 && (local & 3) == 0) {
        const unsigned K = (unsigned)(sg.taps * sg.cin);  // segment-local offsets < 2^31: 32-bit division
        const unsigned co = (unsigned)local / K;
        const int rem = (int)((unsigned)local - co * K);
        __align__(8) bf16 h[4];
#pragma unroll
        for (int q = 0; q < 4; ++q) h[q] = __float2bfloat16_rn(wr[q]);
        *(uint2*)(sg.shadow + (long long)co * sg.ldb + rem) = *(uint2*)h;
      } else {
        shadow_store(sg, local, wr, cnt);
      }
    }
  }
  // fixed-order block reduction of sum g^2 (for the grad-norm statistic)
  __shared__ float red[SGD_THREADS];
  red[threadIdx.x] = sq;
  __syncthreads();
  for (int o = SGD_THREADS / 2; o > 0; o >>= 1) {
    if (threadIdx.x < o) red[threadIdx.x] += red[threadIdx.x + o];
    __syncthreads();
  }
  if (threadIdx.x == 0 && sq_partial) sq_partial[blockIdx.x] = red[0];
}
void launch_sgd(float* w, float* v, const float* g, long long n, float lr, float mu, float wd, const SgdSeg* segs_dev,
                int nseg, const int* block_seg_dev, const long long* block_start_dev, int nblocks, float* sq_partial,
                cudaStream_t st) {
  (void)n;
  (void)nseg;
  ProfScope ps(PC_SGD, st);
  sgd_kernel<<<nblocks, SGD_THREADS, 0, st>>>(w, v, g, lr, mu, wd, segs_dev, block_seg_dev, block_start_dev,
                                               sq_partial);
  CK(cudaGetLastError());
}

__global__ void shadow_pack_kernel(const float* __restrict__ w, const SgdSeg* __restrict__ segs) {
  const SgdSeg sg = segs[blockIdx.y];
  if (!sg.shadow) return;
  for (long long l = blockIdx.x * (long long)blockDim.x + threadIdx.x; l < sg.count; l += (long long)gridDim.x * blockDim.x) {
    const float x = w[sg.off + l];
    shadow_store(sg, l, &x, 1);
  }
}
void launch_shadow_pack(const float* w, const SgdSeg* segs_dev, int nseg, cudaStream_t st) {
  ProfScope ps(PC_SHADOW_PACK, st);
  shadow_pack_kernel<<<dim3(64, nseg), 256, 0, st>>>(w, segs_dev);
  CK(cudaGetLastError());
}

// ------------------------------------------------------------------------------------------------
// row gather by an index list with a device-side count (retraining batch assembly from the window pool)
__global__ void gather_rows_kernel(const uint4* __restrict__ src, const int32_t* __restrict__ idx, const int32_t* count,
                                   int n_static, long long row_vec, uint4* __restrict__ dst) {
  const int n = count ? min(*count, n_static) : n_static;
  const long long total = (long long)n * row_vec;
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < total; i += (long long)gridDim.x * blockDim.x) {
    const long long r = i / row_vec, c = i - r * row_vec;
    dst[i] = __ldg(src + (long long)idx[r] * row_vec + c);
  }
}
// one row per grid.y, 4 x 16 bytes per thread (no per-element division); rows past the device count return
__global__ void __launch_bounds__(256) gather_rows2d_kernel(const uint4* __restrict__ src, const int32_t* __restrict__ idx,
                                                            const int32_t* count, int n_static, long long row_vec,
                                                            uint4* __restrict__ dst) {
  const int r = blockIdx.y;
  const int n = count ? min(*count, n_static) : n_static;
  if (r >= n) return;
  const uint4* s = src + (long long)__ldg(idx + r) * row_vec;
  uint4* d = dst + (long long)r * row_vec;
  const long long c0 = (long long)blockIdx.x * 1024 + threadIdx.x;
  uint4 v[4];
#pragma unroll
  for (int u = 0; u < 4; ++u) {
    const long long c = c0 + u * 256;
    if (c < row_vec) v[u] = __ldg(s + c);
  }
#pragma unroll
  for (int u = 0; u < 4; ++u) {
    const long long c = c0 + u * 256;
    if (c < row_vec) d[c] = v[u];
  }
}
__global__ void gather_rows4_kernel(const uint32_t* __restrict__ src, const int32_t* __restrict__ idx, const int32_t* count,
                                    int n_static, long long row_words, uint32_t* __restrict__ dst) {
  const int n = count ? min(*count, n_static) : n_static;
  const long long total = (long long)n * row_words;
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < total; i += (long long)gridDim.x * blockDim.x) {
    const long long r = i / row_words, c = i - r * row_words;
    dst[i] = __ldg(src + (long long)idx[r] * row_words + c);
  }
}
void launch_gather_rows(const void* src, const int32_t* idx, const int32_t* count, int n_static, long long row_bytes,
                        void* dst, cudaStream_t st, int prof_class) {
  if (row_bytes % 4) throw ShapeError("gather_rows: row bytes must be a multiple of 4");
  const bool v16 = (row_bytes % 16) == 0;
  const long long total = (long long)n_static * (row_bytes / (v16 ? 16 : 4));
  const int blocks = (int)std::min<long long>((total + 255) / 256, 32LL * num_sms());
  if (blocks <= 0) return;
  ProfScope ps(prof_class, st);
  if (v16 && row_bytes >= 16 * 1024 && n_static <= 65535) {  // large rows: 2-D grid, one row per grid.y
    const long long rv = row_bytes / 16;
    dim3 g((unsigned)((rv + 1023) / 1024), (unsigned)n_static);
    gather_rows2d_kernel<<<g, 256, 0, st>>>((const uint4*)src, idx, count, n_static, rv, (uint4*)dst);
  } else if (v16)
    gather_rows_kernel<<<blocks, 256, 0, st>>>((const uint4*)src, idx, count, n_static, row_bytes / 16, (uint4*)dst);
  else
    gather_rows4_kernel<<<blocks, 256, 0, st>>>((const uint32_t*)src, idx, count, n_static, row_bytes / 4,
                                                (uint32_t*)dst);
  CK(cudaGetLastError());
}

}  // namespace adainf

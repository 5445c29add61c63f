// ShuffleNet pieces on the GPU (the paper's video-DAG classifier family, "TinyYOLOv3 -> MobileNetV2 /
// ShuffleNet"; NEXT-3 of SURVEY §8(f)).  What is NOT here is the point of the design:
//   * grouped 1x1 convs run on the tensor cores as ONE dense implicit GEMM over a block-diagonal weight (the
//     shadow holds zeros off the diagonal blocks; SgdSeg places each master weight in its block).  At g = 8 the
//     GEMM does 8x the algorithmic MACs, but a grouped 1x1 layer is HBM-bound even then (ShuffleNet stage 2:
//     384 -> 96 channels, 49 KB of MACs per 960 B of traffic), so the waste costs no time;
//   * the channel shuffle moves no data: it is a permutation of the producing conv's output channels, folded
//     into that conv's shadow rows and bias (pi(co) = (co mod C/g) * g + co div C/g), so the conv writes the
//     shuffled tensor directly; dgrad through the permuted dense weight is automatically the shuffled backward.
// The kernels below are the few HBM-bound leftovers: the permuted bias, the gather of the dense weight gradient
// back into the master layout, and the stride-2 unit's 3x3/2 average-pool shortcut + concat (fwd and bwd).
// Rounding points follow the oracle (DESIGN.md readings): pool sum fp32 in (kh, kw) order, / (kh*kw) IEEE, bf16;
// concat copies bf16 values (act applied to the shortcut part); backward shortcut term = bf16(fp32 window-sum of
// the masked concat gradient / (kh*kw)), added by the block input's dgrad epilogue like a projection's dgrad.
#include <algorithm>

#include "common.cuh"
#include "kernels.cuh"
#include "prof.h"

namespace adainf {

namespace {

int grid_for(long long total) { return (int)std::max<long long>(1, std::min<long long>((total + 255) / 256, 32LL * num_sms())); }

__global__ void permute_bias_kernel(const float* __restrict__ b, int Cout, int g, float* __restrict__ out) {
  const int co = blockIdx.x * blockDim.x + threadIdx.x;
  if (co >= Cout) return;
  const int Cg = Cout / g;
  out[(co % Cg) * g + co / Cg] = b[co];
}

// master dw[co][tap][ci] <- dense[pi(co)][tap][grp(co) * Cig + ci], db[co] <- dbs[pi(co)]
__global__ void grouped_wgrad_gather_kernel(const float* __restrict__ dense, const float* __restrict__ dbs, int Cout,
                                            int taps, int Cin, int groups, int shuf_g, float* __restrict__ dw,
                                            float* __restrict__ db) {
  const int Cig = Cin / groups, Cog = Cout / groups;
  const long long total = (long long)Cout * taps * Cig;
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < total; i += (long long)gridDim.x * blockDim.x) {
    const int ci = (int)(i % Cig);
    const long long r = i / Cig;
    const int tap = (int)(r % taps), co = (int)(r / taps);
    int row = co;
    if (shuf_g > 1) {
      const int Cs = Cout / shuf_g;
      row = (co % Cs) * shuf_g + co / Cs;
    }
    dw[i] = dense[((long long)row * taps + tap) * Cin + (co / Cog) * Cig + ci];
    if (db && tap == 0 && ci == 0) db[co] = dbs[row];
  }
}

__device__ __forceinline__ void ld8f(const bf16* p, float* v) {
  const uint4 r = __ldg((const uint4*)p);
  const bf16* h = (const bf16*)&r;
#pragma unroll
  for (int q = 0; q < 8; ++q) v[q] = __bfloat162float(h[q]);
}

__global__ void avgpool_fwd_kernel(const AvgPoolArgs a) {
  const int n_rows = a.count ? *a.count : a.n_static;
  const int CG = a.C >> 3;
  const long long total = (long long)n_rows * a.Ho * a.Wo * CG;
  const float div = (float)(a.K * a.K);
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
    for (int kh = 0; kh < a.K; ++kh) {
      const int ih = ho * a.s - a.p + kh;
      if (ih < 0 || ih >= a.H) continue;
      for (int kw = 0; kw < a.K; ++kw) {
        const int iw = wo * a.s - a.p + kw;
        if (iw < 0 || iw >= a.W) continue;
        float v[8];
        ld8f(a.x + ((src * a.H + ih) * a.W + iw) * a.C + cg * 8, v);
#pragma unroll
        for (int q = 0; q < 8; ++q) acc[q] = __fadd_rn(acc[q], v[q]);
      }
    }
    __align__(16) bf16 o[8];
#pragma unroll
    for (int q = 0; q < 8; ++q) o[q] = __float2bfloat16_rn(__fdiv_rn(acc[q], div));
    *(uint4*)(a.y + (((long long)n * a.Ho + ho) * a.Wo + wo) * a.C + cg * 8) = *(const uint4*)o;
  }
}

// Z[p][0:Cs] = bf16(act(S[p])), Z[p][Cs:Cs+Co] = Y[p]  (Y already act-applied and bf16 by its conv's epilogue)
__global__ void concat_fwd_kernel(const bf16* __restrict__ S, const bf16* __restrict__ Y, const int* count,
                                  int n_static, int HW, int Cs, int Co, int act, bf16* __restrict__ Z) {
  const int n_rows = count ? *count : n_static;
  const int CZ = (Cs + Co) >> 3;
  const long long total = (long long)n_rows * HW * CZ;
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < total; i += (long long)gridDim.x * blockDim.x) {
    const int cz = (int)(i % CZ);
    const long long p = i / CZ;
    uint4 v;
    if (cz * 8 < Cs) {
      float f[8];
      ld8f(S + p * Cs + cz * 8, f);
      __align__(16) bf16 o[8];
#pragma unroll
      for (int q = 0; q < 8; ++q) o[q] = __float2bfloat16_rn(act_apply(act, f[q]));
      v = *(const uint4*)o;
    } else {
      v = __ldg((const uint4*)(Y + p * Co + (cz * 8 - Cs)));
    }
    *(uint4*)(Z + p * (Cs + Co) + cz * 8) = v;
  }
}

// dY[p][c] = dZ[p][Cs + c]  (dZ: the consumer's stored gradient of Z, already masked by act'(Z) and bf16)
__global__ void concat_split_kernel(const bf16* __restrict__ dZ, int n, int HW, int Cs, int Co, bf16* __restrict__ dY) {
  const int CY = Co >> 3;
  const long long total = (long long)n * HW * CY;
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < total; i += (long long)gridDim.x * blockDim.x) {
    const int c = (int)(i % CY);
    const long long p = i / CY;
    *(uint4*)(dY + p * Co + c * 8) = __ldg((const uint4*)(dZ + p * (Cs + Co) + Cs + c * 8));
  }
}

// shortcut term of the block input: sc[n][ih][iw][c] = bf16(fp32 sum over the windows containing (ih, iw), in
// ascending (ho, wo) order, of dZ[n][ho][wo][c] / (K*K))
__global__ void avgpool_bwd_kernel(const bf16* __restrict__ dZ, int ldz, int n, int H, int W, int C, int K, int s,
                                   int p, int Ho, int Wo, bf16* __restrict__ sc) {
  const int CG = C >> 3;
  const long long total = (long long)n * H * W * CG;
  const float div = (float)(K * K);
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < total; i += (long long)gridDim.x * blockDim.x) {
    const int cg = (int)(i % CG);
    long long pix = i / CG;
    const int iw = (int)(pix % W);
    pix /= W;
    const int ih = (int)(pix % H);
    const long long b = pix / H;
    // windows ho with ho*s - p <= ih <= ho*s - p + K - 1
    const int ho0 = max(0, (ih + p - K + s) / s), ho1 = min(Ho - 1, (ih + p) / s);
    const int wo0 = max(0, (iw + p - K + s) / s), wo1 = min(Wo - 1, (iw + p) / s);
    float acc[8];
#pragma unroll
    for (int q = 0; q < 8; ++q) acc[q] = 0.f;
    for (int ho = ho0; ho <= ho1; ++ho)
      for (int wo = wo0; wo <= wo1; ++wo) {
        float v[8];
        ld8f(dZ + ((b * Ho + ho) * Wo + wo) * ldz + cg * 8, v);
#pragma unroll
        for (int q = 0; q < 8; ++q) acc[q] = __fadd_rn(acc[q], v[q]);
      }
    __align__(16) bf16 o[8];
#pragma unroll
    for (int q = 0; q < 8; ++q) o[q] = __float2bfloat16_rn(__fdiv_rn(acc[q], div));
    *(uint4*)(sc + ((b * H + ih) * W + iw) * C + cg * 8) = *(const uint4*)o;
  }
}

// ROUTE with two sources (TinyYOLOv3's second scale, NEXT-3): out[p] = [A(h / f, w / f), B(h, w)] along channels,
// A read through its nearest-upsampling factor f (the UPSAMPLE op is never materialised)
__global__ void route_concat_kernel(const bf16* __restrict__ A, int HA, int WA, int CA, int f, const bf16* __restrict__ Bt,
                                    int CB, const int* count, int n_static, int H, int W, bf16* __restrict__ out) {
  const int n_rows = count ? *count : n_static;
  const int CZ = (CA + CB) >> 3;
  const long long total = (long long)n_rows * H * W * CZ;
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < total; i += (long long)gridDim.x * blockDim.x) {
    const int cz = (int)(i % CZ);
    long long p = i / CZ;
    const int w = (int)(p % W);
    const long long q = p / W;
    const int h = (int)(q % H);
    const long long n = q / H;
    uint4 v;
    if (cz * 8 < CA) v = __ldg((const uint4*)(A + ((n * HA + h / f) * WA + w / f) * CA + cz * 8));
    else v = __ldg((const uint4*)(Bt + p * CB + (cz * 8 - CA)));
    *(uint4*)(out + p * (CA + CB) + cz * 8) = v;
  }
}

}  // namespace

void route_concat(const bf16* A, int HA, int WA, int CA, int f, const bf16* B, int CB, const int* count, int n_static,
                  int H, int W, bf16* out, cudaStream_t st) {
  const long long total = (long long)n_static * H * W * ((CA + CB) / 8);
  if (total <= 0) return;
  ProfScope ps(PC_SHUFFLE, st);
  route_concat_kernel<<<grid_for(total), 256, 0, st>>>(A, HA, WA, CA, f, B, CB, count, n_static, H, W, out);
  CK(cudaGetLastError());
}

void permute_bias(const float* b, int Cout, int g, float* out, cudaStream_t st) {
  ProfScope ps(PC_SHUFFLE, st);
  permute_bias_kernel<<<(Cout + 255) / 256, 256, 0, st>>>(b, Cout, g, out);
  CK(cudaGetLastError());
}

void grouped_wgrad_gather(const float* dense, const float* dbs, int Cout, int taps, int Cin, int groups, int shuf_g,
                          float* dw, float* db, cudaStream_t st) {
  ProfScope ps(PC_SHUFFLE, st);
  grouped_wgrad_gather_kernel<<<grid_for((long long)Cout * taps * (Cin / groups)), 256, 0, st>>>(
      dense, dbs, Cout, taps, Cin, groups, shuf_g, dw, db);
  CK(cudaGetLastError());
}

void avgpool_fwd(const AvgPoolArgs& a, cudaStream_t st) {
  const long long total = (long long)a.n_static * a.Ho * a.Wo * (a.C / 8);
  if (total <= 0) return;
  ProfScope ps(PC_SHUFFLE, st);
  avgpool_fwd_kernel<<<grid_for(total), 256, 0, st>>>(a);
  CK(cudaGetLastError());
}

void concat_fwd(const bf16* S, const bf16* Y, const int* count, int n_static, int HW, int Cs, int Co, int act, bf16* Z,
                cudaStream_t st) {
  const long long total = (long long)n_static * HW * ((Cs + Co) / 8);
  if (total <= 0) return;
  ProfScope ps(PC_SHUFFLE, st);
  concat_fwd_kernel<<<grid_for(total), 256, 0, st>>>(S, Y, count, n_static, HW, Cs, Co, act, Z);
  CK(cudaGetLastError());
}

void concat_bwd(const bf16* dZ, int n, int H, int W, int Cs, int Co, int K, int s, int p, int Ho, int Wo, bf16* dY,
                bf16* sc, cudaStream_t st) {
  ProfScope ps(PC_SHUFFLE, st, 2);
  concat_split_kernel<<<grid_for((long long)n * Ho * Wo * (Co / 8)), 256, 0, st>>>(dZ, n, Ho * Wo, Cs, Co, dY);
  avgpool_bwd_kernel<<<grid_for((long long)n * H * W * (Cs / 8)), 256, 0, st>>>(dZ, Cs + Co, n, H, W, Cs, K, s, p, Ho,
                                                                                 Wo, sc);
  CK(cudaGetLastError());
}

}  // namespace adainf

// First detector layer fused with its max-pool (inference): 3x3 stride-1 pad-1 conv of a <= 4-channel image
// (packed to 8 channels) into 16 outputs + bias + activation, then the 2x2/2 max-pool, on CUDA cores.
// At K = 27 and N = 16 the implicit GEMM spends its time moving 16-byte operand rows (the layer measured 15 ms at
// 512 frames of 416x416 through the tensor-core kernel, 280 GB/s); as a direct conv each thread owns one pooled pixel:
// it reads the 4x4 input patch once, accumulates the four conv outputs x 16 channels in fp32 in the fixed
// (kh, kw, c) order, rounds each conv output to bf16 after bias + activation (the oracle's storage point), and
// writes only the pooled row: the 416x416x16 conv tensor never reaches HBM.  Weights live in shared memory as fp32.
#include "common.cuh"
#include "kernels.cuh"
#include "prof.h"

namespace adainf {

namespace {

constexpr int CP_CO = 16;

__global__ void __launch_bounds__(256) conv_first_pool_kernel(ConvPoolArgs a) {
  __shared__ float4 ws[27 * CP_CO / 4];  // [kh][kw][c][co], c < 3 (cin_real <= 3 padded in K to 3 slots)
  __shared__ float bs[CP_CO];
  const int cr = a.cin_real;
  for (int i = threadIdx.x; i < 9 * 3 * CP_CO; i += blockDim.x) {
    const int co = i % CP_CO, r = i / CP_CO, c = r % 3, tap = r / 3;
    ((float*)ws)[i] = c < cr ? __bfloat162float(a.shadow[(long long)co * a.ldb + tap * a.cin_pad + c]) : 0.f;
  }
  if (threadIdx.x < CP_CO) bs[threadIdx.x] = a.bias[threadIdx.x];
  __syncthreads();
  const int n_rows = a.count ? *a.count : a.n_static;
  const int Hp = a.H / 2, Wp = a.W / 2;
  const long long total = (long long)n_rows * Hp * Wp;
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < total; i += (long long)gridDim.x * blockDim.x) {
    const int pw = (int)(i % Wp);
    const long long r = i / Wp;
    const int ph = (int)(r % Hp);
    const long long n = r / Hp;
    // 4x4 input patch rows 2ph-1 .. 2ph+2, cols 2pw-1 .. 2pw+2 (zero padding outside)
    float xin[4][4][3];
#pragma unroll
    for (int dy = 0; dy < 4; ++dy) {
      const int ih = 2 * ph - 1 + dy;
#pragma unroll
      for (int dx = 0; dx < 4; ++dx) {
        const int iw = 2 * pw - 1 + dx;
        const bool in = ih >= 0 && ih < a.H && iw >= 0 && iw < a.W;
        uint2 v = make_uint2(0u, 0u);
        if (in) v = __ldg((const uint2*)(a.x + ((n * a.H + ih) * a.W + iw) * a.cin_pad));
        const bf16* h = (const bf16*)&v;
#pragma unroll
        for (int c = 0; c < 3; ++c) xin[dy][dx][c] = __bfloat162float(h[c]);
      }
    }
    float best[CP_CO];
#pragma unroll
    for (int co = 0; co < CP_CO; ++co) best[co] = -INFINITY;
#pragma unroll
    for (int oy = 0; oy < 2; ++oy)
#pragma unroll
      for (int ox = 0; ox < 2; ++ox) {
        float acc[CP_CO];
#pragma unroll
        for (int co = 0; co < CP_CO; ++co) acc[co] = 0.f;
#pragma unroll
        for (int kh = 0; kh < 3; ++kh)
#pragma unroll
          for (int kw = 0; kw < 3; ++kw)
#pragma unroll
            for (int c = 0; c < 3; ++c) {
              const float xv = xin[oy + kh][ox + kw][c];
#pragma unroll
              for (int q = 0; q < CP_CO / 4; ++q) {
                const float4 w4 = ws[((kh * 3 + kw) * 3 + c) * (CP_CO / 4) + q];
                acc[4 * q] = fmaf(xv, w4.x, acc[4 * q]);
                acc[4 * q + 1] = fmaf(xv, w4.y, acc[4 * q + 1]);
                acc[4 * q + 2] = fmaf(xv, w4.z, acc[4 * q + 2]);
                acc[4 * q + 3] = fmaf(xv, w4.w, acc[4 * q + 3]);
              }
            }
#pragma unroll
        for (int co = 0; co < CP_CO; ++co) {
          const float y = __bfloat162float(__float2bfloat16_rn(act_apply(a.act, __fadd_rn(acc[co], bs[co]))));
          best[co] = fmaxf(best[co], y);
        }
      }
    __align__(16) bf16 o[CP_CO];
#pragma unroll
    for (int co = 0; co < CP_CO; ++co) o[co] = __float2bfloat16_rn(best[co]);
    uint4* dst = (uint4*)(a.y + (((n * Hp + ph) * Wp) + pw) * CP_CO);
    dst[0] = ((const uint4*)o)[0];
    dst[1] = ((const uint4*)o)[1];
  }
}

}  // namespace

bool conv_first_pool_ok(const ConvGeom& g, int cin_real, int pk, int ps, int pp) {
  return g.KH == 3 && g.KW == 3 && g.stride == 1 && g.pad == 1 && g.Cout == CP_CO && cin_real <= 3 &&
         (g.Cin == 4 || g.Cin == 8) && pk == 2 && ps == 2 && pp == 0 && g.H % 2 == 0 && g.W % 2 == 0;
}

void conv_first_pool(const ConvPoolArgs& a, cudaStream_t st) {
  const long long total = (long long)a.n_static * (a.H / 2) * (a.W / 2);
  if (total <= 0) return;
  const int grid = (int)std::min<long long>((total + 255) / 256, 16LL * num_sms());
  ProfScope ps(PC_CONV_FWD, st);
  conv_first_pool_kernel<<<grid, 256, 0, st>>>(a);
  CK(cudaGetLastError());
}

}  // namespace adainf

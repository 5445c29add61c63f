// 3x3 / stride 2 / pad 1 max-pool backward for one 2x2 input block and 8 channels, shared by the standalone
// kernel (kernels.cu) and the stem weight-gradient producer that consumes it in place (stem.cu), so both
// produce bit-identical dZ.  cw[w] / gw[w]: argmax codes (8 x uint8, ReLU mask folded in: 0xFF = no route)
// and pooled-output gradients (8 x bf16) of windows w00 = (bi, bj), w01 = (bi, bj+1), w10 = (bi+1, bj),
// w11 = (bi+1, bj+1) (out-of-range windows: code 0xFF, gradient 0).  Positions and their (window, code) pairs:
//   (0,0): w00 code 4     (0,1): w00 5, w01 3     (1,0): w00 7, w10 1     (1,1): w00 8, w01 6, w10 2, w11 0
// summed in window order (ho, then wo ascending).  out[p] = 8 bf16 of position p = (0,0), (0,1), (1,0), (1,1).
#pragma once
#include "common.cuh"

namespace adainf {

__device__ __forceinline__ void pool_bwd_k3s2_block(const uint2 (&cw)[4], const uint4 (&gw)[4], uint4 (&out)[4]) {
  __align__(16) bf16 o00[8], o01[8], o10[8], o11[8];
#pragma unroll
  for (int q = 0; q < 8; ++q) {
    const uint32_t c00 = ((const uint8_t*)&cw[0])[q], c01 = ((const uint8_t*)&cw[1])[q];
    const uint32_t c10 = ((const uint8_t*)&cw[2])[q], c11 = ((const uint8_t*)&cw[3])[q];
    const float g00 = __bfloat162float(((const bf16*)&gw[0])[q]), g01 = __bfloat162float(((const bf16*)&gw[1])[q]);
    const float g10 = __bfloat162float(((const bf16*)&gw[2])[q]), g11 = __bfloat162float(((const bf16*)&gw[3])[q]);
    const float a00 = c00 == 4 ? g00 : 0.f;
    const float a01 = __fadd_rn(c00 == 5 ? g00 : 0.f, c01 == 3 ? g01 : 0.f);
    const float a10 = __fadd_rn(c00 == 7 ? g00 : 0.f, c10 == 1 ? g10 : 0.f);
    const float a11 = __fadd_rn(__fadd_rn(__fadd_rn(c00 == 8 ? g00 : 0.f, c01 == 6 ? g01 : 0.f), c10 == 2 ? g10 : 0.f),
                                c11 == 0 ? g11 : 0.f);
    o00[q] = __float2bfloat16_rn(a00);
    o01[q] = __float2bfloat16_rn(a01);
    o10[q] = __float2bfloat16_rn(a10);
    o11[q] = __float2bfloat16_rn(a11);
  }
  out[0] = *(const uint4*)o00;
  out[1] = *(const uint4*)o01;
  out[2] = *(const uint4*)o10;
  out[3] = *(const uint4*)o11;
}

// loads of one block's four windows (codes + gradients) at pooled position (b, bi, bj), channel vector cv
__device__ __forceinline__ void pool_bwd_k3s2_load(const bf16* __restrict__ dT, const uint8_t* __restrict__ amax,
                                                   long long b, int bi, int bj, int cv, int C, int Ho, int Wo,
                                                   uint2 (&cw)[4], uint4 (&gw)[4]) {
#pragma unroll
  for (int wq = 0; wq < 4; ++wq) {
    const int ho = bi + (wq >> 1), wo = bj + (wq & 1);
    if (ho < Ho && wo < Wo) {
      const long long oi = ((b * Ho + ho) * Wo + wo) * C + cv * 8;
      cw[wq] = __ldg((const uint2*)(amax + oi));
      gw[wq] = __ldg((const uint4*)(dT + oi));
    } else {
      cw[wq] = make_uint2(0xFFFFFFFFu, 0xFFFFFFFFu);
      gw[wq] = make_uint4(0u, 0u, 0u, 0u);
    }
  }
}

}  // namespace adainf

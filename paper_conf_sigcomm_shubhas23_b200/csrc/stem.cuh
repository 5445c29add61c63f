// ResNet stem on sm_100a: 7x7/2 conv (pad 3, <= 4 input channels, 64 outputs) + bias + ReLU + 3x3/2 max-pool
// (pad 1), the first block of the paper's classifiers (ResNet-18 early-exit, P:93-95 / Fig. 4 models).
//
// Space-to-depth: the input is packed as S[n][H/2][W/2][16] with channel (bh*2 + bw)*4 + c = X[2i+bh][2j+bw][c],
// which turns the stride-2 7x7 conv into a stride-1 4x4 conv over 16 channels (taps (ah, aw) in -2..1, weight
// zero where 2*ah + bh + 3 or 2*aw + bw + 3 falls outside 0..6).  One 32-byte s2d pixel is one K=16 slice,
// so each tap is one tcgen05.mma (M=128 output columns of one row, N=64, K=16) and the 16 taps are row
// shifts of one TMA-loaded window (no swizzle: 16-byte core-matrix rows, two channel planes).
//
//   stem_fwd   : conv + bias + ReLU -> bf16 rows in shared memory -> 3x3/2 max-pool (+ first-argmax) in
//                the epilogue; only the pooled tensor (and argmax for training) reaches HBM.
//   stem_wgrad : dW[tap][ch][co] = sum_q S(q + tap)[ch] * dZ(q)[co], computed as
//                D[(tap pair, co)][ch] += dZ(q' - tap)^T * S(q'): the dZ rows sit in a ring of shared
//                memory slots (each loaded once), two taps of one row offset per M=128 MMA (N=16).
//                Bias gradient fused (column sums of the dZ rows).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "common.cuh"

namespace adainf {

// stem eligibility (model build): 7x7 stride 2 pad 3, cin <= 4, cout 64, even H and W, W/2 <= 125
bool stem_s2d_ok(int H, int W, int cin, int cout, int KH, int KW, int stride, int pad);

// x [n][H][W][cin] (rows through map / device count) -> S [n][H/2][W/2][16]
void launch_pack_s2d(const bf16* x, const int* map, const int* count, int n_static, int H, int W, int cin, bf16* s,
                     cudaStream_t st);
// shadow [64][ldb] (K = (kh*7 + kw)*4 + c) -> wprep [16 taps][2 planes][64 co][8 ch] (bf16)
void launch_stem_wprep(const bf16* shadow, int ldb, bf16* wprep, cudaStream_t st);

// fused conv + bias + ReLU + maxpool(3,2,1): s = S2D input (Hs = H/2 rows, Ws = W/2 cols), pooled
// [n][Hp][Wp][64] with Hp = (Hs - 1)/2 + 1, argmax (nullable) uint8 window index kh*3 + kw of the first max
void stem_fwd(const bf16* s, const int* count, int n_static, int Hs, int Ws, const bf16* wprep, const float* bias,
              bf16* pooled, uint8_t* argmax, cudaStream_t st);

// weight + bias gradient of the stem conv from dZ [n][Hs][Ws][64] (conv-output gradient, after the
// activation mask): dw [64][7][7][cin_real] fp32, db [64] fp32.  ws: workspace of stem_wgrad_ws_bytes().
size_t stem_wgrad_ws_bytes(int n);
void stem_wgrad(const bf16* s, const bf16* dz, int n, int Hs, int Ws, int cin_real, float* ws, size_t ws_bytes,
                float* dw, float* db, cudaStream_t st);
// same, with the stem's 3x3/2 max-pool backward fused in: dZ is built on chip from the pooled-output gradient
// pool_dT [n][Hp][Wp][64] and the forward's argmax codes (ReLU mask folded in), never written to HBM
void stem_wgrad_pooled(const bf16* s, const bf16* pool_dT, const uint8_t* pool_codes, int Hp, int Wp, int n, int Hs,
                       int Ws, int cin_real, float* ws, size_t ws_bytes, float* dw, float* db, cudaStream_t st);

}  // namespace adainf

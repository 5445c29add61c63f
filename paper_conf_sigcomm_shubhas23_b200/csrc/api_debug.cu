// Kernel-level entry points (include/adainf_debug.h) used by the per-kernel GPU parity tests.
#include <cstring>

#include "../../include/adainf_debug.h"
#include "api_common.h"
#include "runtime.h"
#include "kernels.cuh"
#include "stem.cuh"

using namespace adainf;

static ConvGeom geom(int H, int W, int C, int Co, int KH, int KW, int s, int p) {
  ConvGeom g;
  g.Cin = C;
  g.Cout = Co;
  g.KH = KH;
  g.KW = KW;
  g.stride = s;
  g.pad = p;
  g.H = H;
  g.W = W;
  g.Ho = (H + 2 * p - KH) / s + 1;
  g.Wo = (W + 2 * p - KW) / s + 1;
  return g;
}

extern "C" adainf_status adainf_dbg_conv_fwd(const void* x, int32_t n, int32_t H, int32_t W, int32_t C,
                                             const void* w, const float* b, int32_t Co, int32_t KH, int32_t KW,
                                             int32_t stride, int32_t pad, int32_t act, const void* res, void* out,
                                             int32_t out_f32, adainf_stream_t stream) {
  return guard([&] {
    if ((C % 8 && C != 4) || n <= 0 || KH * KW > 49) throw ShapeError("conv_fwd: C must be 4 or a multiple of 8");
    require_device();
    ConvGeom g = geom(H, W, C, Co, KH, KW, stride, pad);
    const int K = KH * KW * C, ldb = (K + 7) / 8 * 8;  // GEMM-ready rows are 16-byte aligned
    const bf16* wp = (const bf16*)w;
    bf16* tmp = nullptr;
    cudaStream_t st = (cudaStream_t)stream;
    if (ldb != K) {
      CK(cudaMallocAsync((void**)&tmp, (size_t)Co * ldb * 2, st));
      CK(cudaMemsetAsync(tmp, 0, (size_t)Co * ldb * 2, st));
      CK(cudaMemcpy2DAsync(tmp, ldb * 2, w, K * 2, K * 2, Co, cudaMemcpyDeviceToDevice, st));
      wp = tmp;
    }
    conv_fwd(g, (const bf16*)x, nullptr, nullptr, n, wp, ldb, b, (const bf16*)res, nullptr, act, out, out_f32 != 0, st);
    if (tmp) CK(cudaFreeAsync(tmp, st));
  });
}

extern "C" adainf_status adainf_dbg_conv3_pool(const void* x, int32_t n, int32_t H, int32_t W, int32_t C,
                                               int32_t cin_real, const void* w, const float* b, int32_t Co,
                                               int32_t act, int32_t first, void* y, adainf_stream_t stream) {
  return guard([&] {
    if (n <= 0) throw ShapeError("conv3_pool: n must be positive");
    require_device();
    ConvGeom g = geom(H, W, C, Co, 3, 3, 1, 1);
    if (!conv3_pool_ok(g, first != 0, cin_real, 2, 2, 0)) throw ShapeError("conv3_pool: unsupported geometry");
    cudaStream_t st = (cudaStream_t)stream;
    const int K = 9 * C, ldb = (K + 7) / 8 * 8;
    bf16* tmp = nullptr;  // GEMM-ready shadow rows (16-byte aligned) and the expanded weights
    bf16* wexp = nullptr;
    bf16* xs = nullptr;
    CK(cudaMallocAsync((void**)&tmp, (size_t)Co * ldb * 2, st));
    CK(cudaMemsetAsync(tmp, 0, (size_t)Co * ldb * 2, st));
    CK(cudaMemcpy2DAsync(tmp, ldb * 2, w, K * 2, K * 2, Co, cudaMemcpyDeviceToDevice, st));
    CK(cudaMallocAsync((void**)&wexp, conv3_pool_wexp_bytes(g, first != 0), st));
    const bf16* src = (const bf16*)x;
    if (first) {  // space-to-depth pack of the 4-channel input, as the model's ingest does
      CK(cudaMallocAsync((void**)&xs, (size_t)n * H * W * 4 * 2, st));
      launch_pack_s2d((const bf16*)x, nullptr, nullptr, n, H, W, 4, xs, st);
      src = xs;
    }
    conv3_pool(g, first != 0, src, nullptr, n, tmp, ldb, cin_real, b, act, wexp, (bf16*)y, st);
    CK(cudaFreeAsync(tmp, st));
    CK(cudaFreeAsync(wexp, st));
    if (xs) CK(cudaFreeAsync(xs, st));
  });
}

extern "C" adainf_status adainf_dbg_conv_dgrad(const void* dz, int32_t n, int32_t H, int32_t W, int32_t C,
                                               const void* w, int32_t Co, int32_t KH, int32_t KW, int32_t stride,
                                               int32_t pad, const float* bcast, const void* sc, const void* yact,
                                               int32_t mask_act, void* dx, adainf_stream_t stream) {
  return guard([&] {
    if (C % 8 || Co % 8 || n <= 0) throw ShapeError("conv_dgrad: C, Co must be multiples of 8");
    require_device();
    ConvGeom g = geom(H, W, C, Co, KH, KW, stride, pad);
    if (dgrad_sp_ok(g)) {  // the runtime's route for stride-2 3x3 layers (one sub-pixel GEMM)
      bf16* wsp = nullptr;
      CK(cudaMallocAsync((void**)&wsp, dgrad_sp_ws_bytes(g), (cudaStream_t)stream));
      conv_dgrad_sp(g, (const bf16*)dz, (const bf16*)w, KH * KW * C, wsp, n, bcast, (const bf16*)sc, false,
                    (const bf16*)yact, mask_act, (bf16*)dx, (cudaStream_t)stream);
      CK(cudaFreeAsync(wsp, (cudaStream_t)stream));
      return;
    }
    conv_dgrad(g, (const bf16*)dz, (const bf16*)w, KH * KW * C, n, bcast, (const bf16*)sc, (const bf16*)yact,
               mask_act, (bf16*)dx, (cudaStream_t)stream);
  });
}

extern "C" adainf_status adainf_dbg_conv_wgrad(const void* x, const void* dz, int32_t n, int32_t H, int32_t W,
                                               int32_t C, int32_t Co, int32_t KH, int32_t KW, int32_t stride,
                                               int32_t pad, float* dw, float* db, adainf_stream_t stream) {
  return guard([&] {
    if ((C % 8 && C != 4) || Co % 8 || n <= 0) throw ShapeError("conv_wgrad: C must be 4 or a multiple of 8, Co of 8");
    require_device();
    ConvGeom g = geom(H, W, C, Co, KH, KW, stride, pad);
    const size_t ws = wgrad_ws_bytes(g, n);
    float* buf = nullptr;
    CK(cudaMallocAsync((void**)&buf, ws, (cudaStream_t)stream));
    conv_wgrad(g, (const bf16*)x, (const bf16*)dz, n, C, buf, ws, dw, db, (cudaStream_t)stream);
    CK(cudaFreeAsync(buf, (cudaStream_t)stream));
  });
}

extern "C" adainf_status adainf_dbg_stem_fwd(const void* x, int32_t n, int32_t H, int32_t W, int32_t cin,
                                             const void* w, const float* b, void* pooled, uint8_t* argmax,
                                             adainf_stream_t stream) {
  return guard([&] {
    if (n <= 0 || !stem_s2d_ok(H, W, cin, 64, 7, 7, 2, 3)) throw ShapeError("stem_fwd: ineligible shape");
    require_device();
    cudaStream_t st = (cudaStream_t)stream;
    // GEMM-ready shadow [64][200] (K = (kh*7 + kw)*4 + c, zero-padded channels), then the per-tap layout
    bf16 *shadow = nullptr, *wprep = nullptr, *s = nullptr;
    CK(cudaMallocAsync((void**)&shadow, 64 * 200 * 2, st));
    CK(cudaMallocAsync((void**)&wprep, 16 * 2 * 64 * 8 * 2, st));
    CK(cudaMallocAsync((void**)&s, (size_t)n * H * W * 4 * 2, st));
    CK(cudaMemsetAsync(shadow, 0, 64 * 200 * 2, st));
    for (int co = 0; co < 64; ++co)  // 49 taps of cin channels -> 8-byte slots, rows of 200 elements
      CK(cudaMemcpy2DAsync(shadow + co * 200, 8, (const bf16*)w + (size_t)co * 49 * cin, cin * 2, cin * 2, 49,
                           cudaMemcpyDeviceToDevice, st));
    launch_pack_s2d((const bf16*)x, nullptr, nullptr, n, H, W, cin, s, st);
    launch_stem_wprep(shadow, 200, wprep, st);
    stem_fwd(s, nullptr, n, H / 2, W / 2, wprep, b, (bf16*)pooled, argmax, st);
    CK(cudaFreeAsync(s, st));
    CK(cudaFreeAsync(wprep, st));
    CK(cudaFreeAsync(shadow, st));
  });
}

extern "C" adainf_status adainf_dbg_stem_wgrad(const void* x, const void* dz, int32_t n, int32_t H, int32_t W,
                                               int32_t cin, float* dw, float* db, adainf_stream_t stream) {
  return guard([&] {
    if (n <= 0 || !stem_s2d_ok(H, W, cin, 64, 7, 7, 2, 3)) throw ShapeError("stem_wgrad: ineligible shape");
    require_device();
    cudaStream_t st = (cudaStream_t)stream;
    bf16* s = nullptr;
    float* ws = nullptr;
    const size_t wsb = stem_wgrad_ws_bytes(n);
    CK(cudaMallocAsync((void**)&s, (size_t)n * H * W * 4 * 2, st));
    CK(cudaMallocAsync((void**)&ws, wsb, st));
    launch_pack_s2d((const bf16*)x, nullptr, nullptr, n, H, W, cin, s, st);
    stem_wgrad(s, (const bf16*)dz, n, H / 2, W / 2, cin, ws, wsb, dw, db, st);
    CK(cudaFreeAsync(ws, st));
    CK(cudaFreeAsync(s, st));
  });
}

extern "C" adainf_status adainf_dbg_set_win_mode(int32_t mode) {
  return guard([&] { set_win_mode(mode); });
}


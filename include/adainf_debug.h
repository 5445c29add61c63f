/*
 * adainf_debug.h — kernel-level entry points of libadainf.so, used by the per-kernel GPU parity
 * tests (tests/test_gpu_kernels.py) and the bench's roofline leg.  Same conventions as adainf.h:
 * device pointers, caller-owned buffers, stream-ordered, status return, no CPU fallback.
 */
#ifndef ADAINF_DEBUG_H_
#define ADAINF_DEBUG_H_
#include "adainf.h"

#ifdef __cplusplus
extern "C" {
#endif

/* Implicit-GEMM conv forward on the tensor cores:
 * out[n][ho][wo][co] = act(sum x * w + b [+ res]) in bf16 (fp32 if out_f32).
 * x: device [n][H][W][C] bf16 (C multiple of 8); w: device bf16 [Co][KH][KW][C]; b: device fp32 [Co];
 * res: device bf16 [n][Ho][Wo][Co] or NULL. */
adainf_status adainf_dbg_conv_fwd(const void* x, int32_t n, int32_t H, int32_t W, int32_t C, const void* w,
                                  const float* b, int32_t Co, int32_t KH, int32_t KW, int32_t stride,
                                  int32_t pad, int32_t act, const void* res, void* out, int32_t out_f32,
                                  adainf_stream_t stream);
/* dgrad: dx[n][H][W][C] = bf16( (sum_{tap,co} dz * w) [+ bcast[n][c]] [+ sc] ) * act'(yact)
 * (conv transpose of the forward conv above; stride-s phases). */
adainf_status adainf_dbg_conv_dgrad(const void* dz, int32_t n, int32_t H, int32_t W, int32_t C, const void* w,
                                    int32_t Co, int32_t KH, int32_t KW, int32_t stride, int32_t pad,
                                    const float* bcast, const void* sc, const void* yact, int32_t mask_act,
                                    void* dx, adainf_stream_t stream);
/* wgrad: dw[co][kh][kw][c] = sum_{n,ho,wo} dz[n][ho][wo][co] * x[n][ho*s-p+kh][wo*s-p+kw][c] (fp32),
 * db[co] = sum dz (fp32, optional). Deterministic split-K. */
adainf_status adainf_dbg_conv_wgrad(const void* x, const void* dz, int32_t n, int32_t H, int32_t W, int32_t C,
                                    int32_t Co, int32_t KH, int32_t KW, int32_t stride, int32_t pad, float* dw,
                                    float* db, adainf_stream_t stream);

/* Conv kernel selection for A/B tests (process-wide, not thread-safe; tests restore 1):
 *   0 = generic cp.async gather kernels only
 *   1 = default routing (TMA window kernels for stride-1 3x3, TMA generic wgrad, cp.async elsewhere)
 *   2 = window kernel for every eligible stride-1 3x3 fwd/dgrad
 *   4 = cp.async warp-specialised window variant, no TMA
 *   5 = no TMA weight-gradient kernels (cp.async window for 64x64 3x3, else generic)
 *   6 = TMA generic weight gradient even where the window variant applies
 *   7 = TMA window weight gradient forced for every eligible shape (any width)
 *   8 = default routing, but models created while it is set keep the unfused stem (generic 7x7 conv +
 *       separate max-pool) instead of the space-to-depth stem kernels */
adainf_status adainf_dbg_set_win_mode(int32_t mode);

/* 3x3/1 pad-1 conv + bias + act + 2x2/2 max-pool in one tensor-core kernel (conv3pool.cu, the detector's few-channel
 * layers; C3, reading Q18):  x [n][H][W][C] bf16 (H, W even), w [Co][3][3][C] bf16, b [Co] fp32 ->
 * y [n][H/2][W/2][Co] bf16 = maxpool2x2(bf16(act(conv + b))).  first = 0: C in {16, 32}, Co in {32, 64, 96, 128};
 * first = 1: C <= 4 real channels given as 4 (space-to-depth packed internally), Co in {16, 32}.
 * ADAINF_ERR_SHAPE outside those. */
adainf_status adainf_dbg_conv3_pool(const void* x, int32_t n, int32_t H, int32_t W, int32_t C, int32_t cin_real,
                                    const void* w, const float* b, int32_t Co, int32_t act, int32_t first, void* y,
                                    adainf_stream_t stream);

/* ResNet stem (7x7/2 pad 3 conv, <= 4 input channels, 64 outputs, ReLU, then 3x3/2 pad 1 max-pool) through
 * the space-to-depth kernels (stem.cuh):
 *   stem_fwd  : x [n][H][W][cin] bf16 (H, W even, W/2 <= 125), w [64][7][7][cin] bf16, b [64] fp32 ->
 *               pooled [n][Hp][Wp][64] bf16 (Hp = (H/2 - 1)/2 + 1), argmax [n][Hp][Wp][64] uint8 (window
 *               index kh*3 + kw of the FIRST maximum in row-major order; nullable)
 *   stem_wgrad: x as above, dz [n][H/2][W/2][64] bf16 -> dw [64][7][7][cin] fp32, db [64] fp32 (nullable)
 * Device pointers; temporaries are allocated stream-ordered.  Errors: ADAINF_ERR_SHAPE for ineligible shapes. */
adainf_status adainf_dbg_stem_fwd(const void* x, int32_t n, int32_t H, int32_t W, int32_t cin, const void* w,
                                  const float* b, void* pooled, uint8_t* argmax, adainf_stream_t stream);
adainf_status adainf_dbg_stem_wgrad(const void* x, const void* dz, int32_t n, int32_t H, int32_t W, int32_t cin,
                                    float* dw, float* db, adainf_stream_t stream);

/* Device pointer of the routed-crop batch of DET_CROP edge `edge` of `app` (library-owned, valid until the app
 * is destroyed): [max_routed_per_dst][crop_h][crop_w][dst in_c] bf16, rows in route order, written by the last
 * adainf_infer_dag (rows past n_routed are stale).  For the stage-isolated crop parity test (reading Q20). */
adainf_status adainf_dbg_app_crops(adainf_app_t app, int32_t edge, const void** crops);
/* Layout of that batch: *s2d = 1 when the destination runs the space-to-depth ResNet stem and the crops were written
 * straight into its packed input, [rows][crop_h/2][crop_w/2][16] with channel (bh*2 + bw)*4 + c (c >= in_c zero);
 * 0 for the plain layout above. */
adainf_status adainf_dbg_app_crop_layout(adainf_app_t app, int32_t edge, int32_t* s2d);

/* Launch accounting and per-kernel-class timing (CUDA events on the launching stream).
 * adainf_launch_count: total kernels launched by the library since load (host-side counter).
 * adainf_prof_enable(1): bracket every launch class with events; adainf_prof_query (synchronizing)
 * returns per-class launch counts and summed device milliseconds since the last reset. */
typedef struct {
  const char* name;
  int64_t launches;
  double total_ms;
} adainf_prof_entry;
int64_t adainf_launch_count(void);
adainf_status adainf_prof_enable(int32_t on);
adainf_status adainf_prof_reset(void);
adainf_status adainf_prof_query(adainf_prof_entry* out, int32_t max_entries, int32_t* n_out);

#ifdef __cplusplus
}
#endif
#endif

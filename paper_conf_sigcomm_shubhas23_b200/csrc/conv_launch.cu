// Host-side launchers for the tcgen05 implicit-GEMM conv kernels (fwd / dgrad phases / wgrad split-K
// + deterministic reduction) and the bias-gradient column sums.
#include <algorithm>
#include <cstdio>
#include <stdexcept>

#include <cstdlib>

#include "conv_gemm.cuh"
#include "conv_win.cuh"
#include "conv_tma.cuh"
#include "prof.h"
#include "runtime.h"

namespace adainf {

static int g_num_sms = 0;
int num_sms() {
  if (!g_num_sms) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&g_num_sms, cudaDevAttrMultiProcessorCount, dev);
    if (g_num_sms <= 0) g_num_sms = 148;
  }
  return g_num_sms;
}

// persistent launch: one CTA per SM (or fewer when there are fewer tiles)
template <int MODE, int BN>
static void launch_t(const ConvArgs& a, long long max_tiles, cudaStream_t st) {
  dim3 grid((unsigned)std::max(1LL, std::min<long long>(max_tiles, num_sms())));
  using Cfg = ConvCfg<MODE, BN>;
  static bool attr = false;
  if (!attr) {
    CK(cudaFuncSetAttribute(conv_umma_kernel<MODE, BN>, cudaFuncAttributeMaxDynamicSharedMemorySize, Cfg::SMEM));
    attr = true;
  }
  ProfScope ps(MODE == MODE_FWD ? PC_CONV_FWD : (MODE == MODE_DGRAD ? PC_CONV_DGRAD : PC_CONV_WGRAD), st);
  conv_umma_kernel<MODE, BN><<<grid, NUM_THREADS, Cfg::SMEM, st>>>(a);
  CK(cudaGetLastError());
}

template <int MODE>
static void launch_bn(int BN, const ConvArgs& a, long long max_tiles, cudaStream_t st) {
  switch (BN) {
    case 32:
      if constexpr (MODE == MODE_FWD) { launch_t<MODE, 32>(a, max_tiles, st); return; }
      break;
    case 64: launch_t<MODE, 64>(a, max_tiles, st); return;
    case 128: launch_t<MODE, 128>(a, max_tiles, st); return;
    case 256: launch_t<MODE, 256>(a, max_tiles, st); return;
  }
  throw std::runtime_error("unsupported BN");
}

// ---- window kernel (stride-1 3x3 pad-1) ----
static int g_win_mode = -1;  // -1 unset, 0 disabled, 1 base-offset 0, 2 base-offset phase
int win_mode() {
  if (g_win_mode < 0) {
    const char* e = getenv("ADAINF_WIN");
    g_win_mode = e ? atoi(e) : 1;
  }
  return g_win_mode;
}
void set_win_mode(int m) { g_win_mode = m; }

static bool win_ok(const ConvGeom& g) {
  return win_mode() > 0 && g.KH == 3 && g.KW == 3 && g.stride == 1 && g.pad == 1 && g.Cin % 64 == 0 &&
         g.Cout % 64 == 0 && g.W <= 56 && g.H == g.Ho && g.W == g.Wo;
}

template <int BN>
static void launch_win_t(const WinArgs& w, long long max_tiles, cudaStream_t st) {
  using Cfg = WinCfg<BN>;
  static bool attr = false;
  if (!attr) {
    CK(cudaFuncSetAttribute(conv_win_kernel<BN>, cudaFuncAttributeMaxDynamicSharedMemorySize, Cfg::SMEM));
    attr = true;
  }
  dim3 grid((unsigned)std::max(1LL, std::min<long long>(max_tiles, num_sms())));
  ProfScope ps(w.dgrad ? PC_CONV_DGRAD : PC_CONV_FWD, st);
  conv_win_kernel<BN><<<grid, NUM_THREADS, Cfg::SMEM, st>>>(w);
  CK(cudaGetLastError());
}

// TMA weight-stationary 64x64 window conv (FWD: e0 = residual; DGRAD: e0 = shortcut grad, e1 = activation)
static void launch_ws_tma(const ConvArgs& c, bool dgrad, int nstatic, cudaStream_t st) {
  static WsTmaArgs a;  // host staging (copied into the launch parameters)
  a = WsTmaArgs{};
  const int H = c.Hs, W = c.Ws;
  int Wp = 1;
  while (Wp < W + 1) Wp <<= 1;
  const int R = std::max(1, 128 / Wp);
  a.H = H;
  a.W = W;
  a.Wp = Wp;
  a.R = R;
  a.tpi = (H + R - 1) / R;
  a.smap = c.src_map;
  a.count = c.count;
  a.n_static = nstatic;
  a.B = c.B;
  a.ldb = c.ldb;
  a.dgrad = dgrad;
  a.act = c.act;
  a.mask_act = c.mask_act;
  a.bias = c.bias;
  a.bcast = c.bcast;
  a.out = (bf16*)c.out;
  for (int kh = 0; kh < 3; ++kh)
    for (int kw = 0; kw < 3; ++kw) {
      a.tap_off[kh * 3 + kw] = dgrad ? 8 + (2 - kh) * Wp + (1 - kw) : 8 + kh * Wp + kw - 1;
      a.btap[kh * 3 + kw] = kh * 3 + kw;
    }
  a.win_map = make_tmap_nhwc(c.src, nstatic, H, W, 64, 64, Wp, R + 2);
  const bf16* e0 = dgrad ? c.sc : c.res;
  const bf16* e1 = dgrad && c.mask_act ? c.yact : nullptr;
  a.has_e0 = e0 != nullptr;
  a.has_e1 = e1 != nullptr;
  if (e0) a.e0_map = make_tmap_nhwc(e0, nstatic, H, W, 64, 64, Wp, R);
  if (e1) a.e1_map = make_tmap_nhwc(e1, nstatic, H, W, 64, 64, Wp, R);
  if (!dgrad && c.res_map && c.res_map != c.src_map) throw std::runtime_error("ws_tma: residual map differs");
  a.win_bytes = ((16 + (R + 2) * Wp) * 128 + 1023) / 1024 * 1024;
  const int fixed = 9 * 8192 + 2 * (a.has_e0 + a.has_e1) * 16384 + 1024 /*align*/ + 512 /*barriers*/;
  a.wstages = std::min(8, (227 * 1024 - fixed) / a.win_bytes);
  if (a.wstages < 2) throw std::runtime_error("ws_tma: shared memory");
  const int smem = a.wstages * a.win_bytes + fixed;
  static bool attr = false;
  if (!attr) {
    CK(cudaFuncSetAttribute(conv_ws_tma_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024));
    attr = true;
  }
  const long long tiles = (long long)nstatic * a.tpi;
  dim3 grid((unsigned)std::max(1LL, std::min<long long>(tiles, num_sms())));
  ProfScope ps(dgrad ? PC_CONV_DGRAD : PC_CONV_FWD, st);
  conv_ws_tma_kernel<<<grid, TMA_WS_THREADS, smem, st>>>(a);
  CK(cudaGetLastError());
}

// general TMA window conv (Cin multiple of 64, BN 128/256, W <= 28)
template <int BN>
static void launch_win_tma_t(WinTmaArgs& a, int nstatic, cudaStream_t st) {
  constexpr int B_BYTES = BN * 128;
  const int fixed = 1024 + 1024;
  const int budget = 227 * 1024 - fixed;
  a.wstages = 2;
  a.bstages = std::min(16, (budget - 2 * a.win_bytes) / B_BYTES);
  if (a.bstages < 3) {
    a.wstages = 1;
    a.bstages = std::min(16, (budget - a.win_bytes) / B_BYTES);
  }
  if (a.bstages < 2) throw std::runtime_error("win_tma: shared memory");
  const int smem = a.wstages * a.win_bytes + a.bstages * B_BYTES + fixed;
  static bool attr = false;
  if (!attr) {
    CK(cudaFuncSetAttribute(conv_win_tma_kernel<BN>, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024));
    attr = true;
  }
  const long long tiles = (long long)nstatic * a.tpi * ((a.Nout + BN - 1) / BN);
  dim3 grid((unsigned)std::max(1LL, std::min<long long>(tiles, num_sms())));
  ProfScope ps(a.dgrad ? PC_CONV_DGRAD : PC_CONV_FWD, st);
  conv_win_tma_kernel<BN><<<grid, NUM_THREADS, smem, st>>>(a);
  CK(cudaGetLastError());
}

static bool win_tma_ok(const ConvArgs& c, int nout) {
  return c.Cs % 64 == 0 && nout % 128 == 0 && c.Ws <= 28 && c.Ws >= 8 && win_mode() != 4;
}

static void launch_win_tma(const ConvArgs& c, bool dgrad, int nstatic, int nout, cudaStream_t st) {
  static WinTmaArgs a;
  a = WinTmaArgs{};
  const int H = c.Hs, W = c.Ws;
  int Wp = 1;
  while (Wp < W + 1) Wp <<= 1;
  const int R = std::max(1, 128 / Wp);
  a.H = H;
  a.W = W;
  a.Wp = Wp;
  a.R = R;
  a.tpi = (H + R - 1) / R;
  a.ncb = c.Cs / 64;
  a.Nout = nout;
  a.smap = c.src_map;
  a.count = c.count;
  a.n_static = nstatic;
  a.dgrad = dgrad;
  a.act = c.act;
  a.mask_act = c.mask_act;
  a.bias = c.bias;
  a.res = c.res;
  a.bcast = c.bcast;
  a.sc = c.sc;
  a.yact = c.yact;
  a.out = (bf16*)c.out;
  if (!dgrad && c.res && c.res_map != c.src_map) throw std::runtime_error("win_tma: residual map differs");
  for (int kh = 0; kh < 3; ++kh)
    for (int kw = 0; kw < 3; ++kw) {
      a.tap_off[kh * 3 + kw] = dgrad ? 8 + (2 - kh) * Wp + (1 - kw) : 8 + kh * Wp + kw - 1;
      a.btap[kh * 3 + kw] = kh * 3 + kw;
    }
  a.win_map = make_tmap_nhwc(c.src, nstatic, H, W, c.Cs, 64, Wp, R + 2);
  const int BN = nout >= 256 ? 256 : 128;
  // weights shadow rows: FWD [Cout = nout][ldb]; DGRAD [Cout = Cs][ldb] read MN-major
  const long long wrows = dgrad ? c.Cs : nout;
  if (!dgrad) a.b_map = make_tmap_2d(c.B, wrows, c.ldb, c.ldb, 64, BN);
  else a.b_map = make_tmap_2d(c.B, wrows, c.ldb, c.ldb, 64, 64);
  a.win_bytes = ((16 + (R + 2) * Wp) * 128 + 1023) / 1024 * 1024;
  if (BN == 256) launch_win_tma_t<256>(a, nstatic, st);
  else launch_win_tma_t<128>(a, nstatic, st);
}

static void launch_win(WinArgs& w, int nstatic, int nout, cudaStream_t st) {
  if (win_tma_ok(w.c, nout) && !(w.c.Cs == 64 && nout == 64)) {
    launch_win_tma(w.c, w.dgrad != 0, nstatic, nout, st);
    return;
  }
  if (w.c.Cs == 64 && nout == 64 && win_mode() != 4) {  // TMA weight-stationary (mode 4: cp.async variant)
    launch_ws_tma(w.c, w.dgrad != 0, nstatic, st);
    return;
  }
  if (w.c.Cs == 64 && nout == 64) {  // weight-stationary 64x64 variant (ResNet layer1)
    static bool attr = false;
    if (!attr) {
      CK(cudaFuncSetAttribute(conv_win_ws_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, WinWsCfg::SMEM));
      attr = true;
    }
    const long long Q = (long long)nstatic * (w.c.Hs + 1) * (w.c.Ws + 1);
    const long long tiles = (Q + BM - 1) / BM;
    dim3 grid((unsigned)std::max(1LL, std::min<long long>(tiles, num_sms())));
    ProfScope ps(w.dgrad ? PC_CONV_DGRAD : PC_CONV_FWD, st);
    conv_win_ws_kernel<<<grid, WS_THREADS, WinWsCfg::SMEM, st>>>(w);
    CK(cudaGetLastError());
    return;
  }
  const int BN = nout >= 256 ? 256 : (nout >= 128 ? 128 : 64);
  const long long Q = (long long)nstatic * (w.c.Hs + 1) * (w.c.Ws + 1);
  const long long tiles = ((Q + BM - 1) / BM) * ((nout + BN - 1) / BN);
  w.base_off = 0;  // the 128B swizzle follows absolute smem address bits: no phase in the descriptor
  switch (BN) {
    case 64: launch_win_t<64>(w, tiles, st); break;
    case 128: launch_win_t<128>(w, tiles, st); break;
    default: launch_win_t<256>(w, tiles, st); break;
  }
}

static int pick_bn(int nout, bool mn_major_b) {
  if (nout <= 32 && !mn_major_b) return 32;
  if (nout <= 64) return 64;
  if (nout <= 128) return 128;
  return 256;
}

static void check_extent(long long pixels) {
  if (pixels >= (1LL << 31) - (1LL << 20)) throw ShapeError("conv: more than 2^31 output positions");
}

void conv_fwd(const ConvGeom& g, const bf16* x, const int* x_map, const int* count, int n_static,
              const bf16* w, int ldb, const float* bias, const bf16* res, const int* res_map, int act, void* out,
              bool out_f32, cudaStream_t st) {
  check_extent((long long)n_static * (g.H + 1) * (g.W + 1));
  ConvArgs a{};
  a.src = x;
  a.src_map = x_map;
  a.Hs = g.H;
  a.Ws = g.W;
  a.Cs = g.Cin;
  a.count = count;
  a.n_static = n_static;
  a.Hg = g.Ho;
  a.Wg = g.Wo;
  a.sy = g.stride;
  a.sx = g.stride;
  a.ntaps = g.KH * g.KW;
  if (a.ntaps > MAX_TAPS) throw std::runtime_error("kernel too large");
  for (int kh = 0; kh < g.KH; ++kh)
    for (int kw = 0; kw < g.KW; ++kw) {
      a.ty[kh * g.KW + kw] = (int8_t)(kh - g.pad);
      a.tx[kh * g.KW + kw] = (int8_t)(kw - g.pad);
    }
  a.B = w;
  a.ldb = ldb;
  a.K = a.ntaps * g.Cin;
  a.Nout = g.Cout;
  a.out = out;
  a.out_f32 = out_f32;
  a.Ho = g.Ho;
  a.Wo = g.Wo;
  a.oys = a.oxs = 1;
  a.bias = bias;
  a.res = res;
  a.res_map = res_map;
  a.act = act;
  if (n_static <= 0) return;
  if (win_ok(g) && !out_f32 &&
      (win_mode() >= 2 || (g.Cin == 64 && g.Cout == 64) || (win_mode() != 4 && g.W <= 28 && g.W >= 8 && g.Cout % 128 == 0))) {
    // window kernel: weight-stationary 64x64 variant by default; the general window FWD measured slower
    WinArgs w{};
    w.c = a;
    w.dgrad = 0;
    for (int kh = 0; kh < 3; ++kh)
      for (int kw = 0; kw < 3; ++kw) {
        w.tap_off[kh * 3 + kw] = kh * (g.W + 1) + kw;
        w.btap[kh * 3 + kw] = kh * 3 + kw;
      }
    launch_win(w, n_static, g.Cout, st);
    return;
  }
  {
    static int expf = -1;
    if (expf < 0) {
      const char* e = getenv("ADAINF_EXP");
      expf = e ? atoi(e) : 0;
    }
    a.exp_flags = expf;
  }
  const int BN = pick_bn(g.Cout, false);
  const long long mt = ((long long)n_static * g.Ho * g.Wo + BM - 1) / BM;
  if (mt == 0) return;
  launch_bn<MODE_FWD>(BN, a, mt * ((g.Cout + BN - 1) / BN), st);
}

void conv_dgrad(const ConvGeom& g, const bf16* dz, const bf16* w, int ldb, int n, const float* bcast,
                const bf16* sc, const bf16* yact, int mask_act, bf16* dx, cudaStream_t st) {
  check_extent((long long)n * (g.H + 1) * (g.W + 1));
  // dX[y] = sum_{kh: (y + pad - kh) % s == 0} dZ[(y + pad - kh)/s] W[kh]; split by output phase (py,px)
  if (win_ok(g) && (g.H <= 14 || win_mode() >= 2 || (g.Cin == 64 && g.Cout == 64) || (g.W <= 28 && g.Cin % 128 == 0))) {
    // stride 1: one window launch with flipped taps (faster at H<=14; weight-stationary at 64x64)
    WinArgs wa{};
    ConvArgs& a = wa.c;
    a.src = dz;
    a.Hs = g.Ho;
    a.Ws = g.Wo;
    a.Cs = g.Cout;
    a.n_static = n;
    a.B = w;
    a.ldb = ldb;
    a.Nout = g.Cin;
    a.out = dx;
    a.Ho = g.H;
    a.Wo = g.W;
    a.bcast = bcast;
    a.sc = sc;
    a.yact = yact;
    a.mask_act = mask_act;
    wa.dgrad = 1;
    for (int kh = 0; kh < 3; ++kh)
      for (int kw = 0; kw < 3; ++kw) {
        wa.tap_off[kh * 3 + kw] = (2 - kh) * (g.W + 1) + (2 - kw);
        wa.btap[kh * 3 + kw] = kh * 3 + kw;
      }
    launch_win(wa, n, g.Cin, st);
    return;
  }
  const int s = g.stride;
  for (int py = 0; py < s; ++py)
    for (int px = 0; px < s; ++px) {
      ConvArgs a{};
      a.src = dz;
      a.Hs = g.Ho;
      a.Ws = g.Wo;
      a.Cs = g.Cout;
      a.n_static = n;
      a.Hg = (g.H - py + s - 1) / s;
      a.Wg = (g.W - px + s - 1) / s;
      if (a.Hg <= 0 || a.Wg <= 0) continue;
      a.sy = a.sx = 1;
      int nt = 0;
      for (int kh = 0; kh < g.KH; ++kh) {
        const int qy = py + g.pad - kh;
        if (((qy % s) + s) % s) continue;
        for (int kw = 0; kw < g.KW; ++kw) {
          const int qx = px + g.pad - kw;
          if (((qx % s) + s) % s) continue;
          a.ty[nt] = (int8_t)((qy - (((qy % s) + s) % s)) / s);
          a.tx[nt] = (int8_t)((qx - (((qx % s) + s) % s)) / s);
          a.btap[nt] = (int16_t)(kh * g.KW + kw);
          nt++;
        }
      }
      a.ntaps = nt;
      a.B = w;
      a.ldb = ldb;
      a.K = nt * g.Cout;
      a.Nout = g.Cin;
      a.out = dx;
      a.Ho = g.H;
      a.Wo = g.W;
      a.oys = s;
      a.oxs = s;
      a.oyo = py;
      a.oxo = px;
      a.bcast = bcast;
      a.sc = sc;
      a.yact = yact;
      a.mask_act = mask_act;
      const int BN = pick_bn(g.Cin, true);
      const long long mt = ((long long)n * a.Hg * a.Wg + BM - 1) / BM;
      launch_bn<MODE_DGRAD>(BN, a, mt * ((g.Cin + BN - 1) / BN), st);
    }
}

// partial [S][Kconv][Cout] -> dw [Cout][taps][cin_real] (fp32), summed over S in fixed order
__global__ void wgrad_reduce_kernel(const float* __restrict__ part, int S, int Kconv, int Cout, int cin_pad,
                                    int cin_real, float* __restrict__ dw) {
  __shared__ float tile[32][33];
  const int k0 = blockIdx.x * 32, c0 = blockIdx.y * 32;
  const int tx = threadIdx.x, ty = threadIdx.y;  // 32 x 8
  for (int r = ty; r < 32; r += 8) {
    const int k = k0 + r, co = c0 + tx;
    float acc = 0.f;
    if (k < Kconv && co < Cout)
      for (int s = 0; s < S; ++s) acc += part[((long long)s * Kconv + k) * Cout + co];
    tile[r][tx] = acc;
  }
  __syncthreads();
  for (int r = ty; r < 32; r += 8) {
    const int co = c0 + r, k = k0 + tx;
    if (k < Kconv && co < Cout) {
      const int tap = k / cin_pad, ci = k - tap * cin_pad;
      if (ci < cin_real) {
        const int ntaps = Kconv / cin_pad;
        dw[((long long)co * ntaps + tap) * cin_real + ci] = tile[tx][r];
      }
    }
  }
}

// column sums of dz [P][C] -> db[C], deterministic: each block reduces a contiguous row range with
// 128-bit loads (thread = 8-channel vector x row group), fixed-order smem reduction -> part[block][C];
// then a fixed-order sum over blocks.
constexpr int CS_THREADS = 256;
__global__ void __launch_bounds__(CS_THREADS) colsum_partial_kernel(const bf16* __restrict__ dz, long long P, int C,
                                                                     long long rows_per_block,
                                                                     float* __restrict__ part) {
  extern __shared__ float red[];  // [groups][C]
  const int CV = C / 8, groups = CS_THREADS / CV;
  const int v = threadIdx.x % CV, g = threadIdx.x / CV;
  const long long r0 = (long long)blockIdx.x * rows_per_block;
  const long long r1 = min(P, r0 + rows_per_block);
  float acc[8];
#pragma unroll
  for (int q = 0; q < 8; ++q) acc[q] = 0.f;
  if (g < groups)
    for (long long r = r0 + g; r < r1; r += groups) {
      const uint4 raw = __ldg((const uint4*)(dz + r * C + v * 8));
      const bf16* h = (const bf16*)&raw;
#pragma unroll
      for (int q = 0; q < 8; ++q) acc[q] += __bfloat162float(h[q]);
    }
  if (g < groups)
#pragma unroll
    for (int q = 0; q < 8; ++q) red[g * C + v * 8 + q] = acc[q];
  __syncthreads();
  for (int c = threadIdx.x; c < C; c += CS_THREADS) {
    float s = 0.f;
    for (int q = 0; q < groups; ++q) s += red[q * C + c];
    part[(long long)blockIdx.x * C + c] = s;
  }
}
__global__ void colsum_final_kernel(const float* __restrict__ part, int nb, int C, float* __restrict__ out) {
  const int c = blockIdx.x * blockDim.x + threadIdx.x;
  if (c >= C) return;
  float acc = 0.f;
  for (int b = 0; b < nb; ++b) acc += part[(long long)b * C + c];
  out[c] = acc;
}
static int colsum_blocks(long long P) { return (int)std::max(1LL, std::min<long long>((P + 63) / 64, 4LL * num_sms())); }

// split-K factor: one balanced wave of persistent CTAs (units = tiles * S <= #SMs), each unit a contiguous
// range of 64-pixel K-blocks; the fp32 partials are reduced in fixed order (deterministic)
static int wgrad_splits(int tiles, int nkb) {
  if (tiles >= num_sms()) return 1;
  return std::max(1, std::min(nkb, num_sms() / tiles));
}

size_t wgrad_ws_bytes(const ConvGeom& g, int n) {
  const long long npix = (long long)n * g.Ho * g.Wo;
  const int nkb = (int)((npix + BK - 1) / BK);
  const int Kconv = g.KH * g.KW * g.Cin;
  const int BN = pick_bn(g.Cout, true);
  const int tiles = ((Kconv + BM - 1) / BM) * ((g.Cout + BN - 1) / BN);
  int S = wgrad_splits(tiles, nkb);
  const int kbs = (nkb + S - 1) / S;
  S = (nkb + kbs - 1) / kbs;
  size_t need = (size_t)S * Kconv * g.Cout * sizeof(float) + (size_t)colsum_blocks(npix) * g.Cout * sizeof(float);
  if (g.KH == 3 && g.KW == 3 && g.stride == 1 && g.Cin == 64 && g.Cout == 64)  // window variant
    need = std::max(need, (size_t)num_sms() * 576 * 64 * 4 + (size_t)colsum_blocks(npix) * g.Cout * 4);
  return need;
}

static bool win_wgrad_ok(const ConvGeom& g) {
  return win_mode() > 0 && g.KH == 3 && g.KW == 3 && g.stride == 1 && g.pad == 1 && g.Cin == 64 && g.Cout == 64 &&
         g.W <= 56 && g.H == g.Ho && g.W == g.Wo;
}

template <int BN>
static void launch_wgrad_tma_t(WgTmaArgs& a, cudaStream_t st) {
  constexpr int STAGE = 16384 + BN * 128;
  a.stages = std::min(16, (225 * 1024 - 2048) / STAGE);
  const int smem = a.stages * STAGE + 2048;
  static bool attr = false;
  if (!attr) {
    CK(cudaFuncSetAttribute(conv_wgrad_tma_kernel<BN>, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024));
    attr = true;
  }
  const long long units = (long long)((a.Kconv + 127) / 128) * ((a.Cout + BN - 1) / BN) * a.splits;
  dim3 grid((unsigned)std::max(1LL, std::min<long long>(units, num_sms())));
  ProfScope ps(PC_CONV_WGRAD, st);
  conv_wgrad_tma_kernel<BN><<<grid, NUM_THREADS, smem, st>>>(a);
  CK(cudaGetLastError());
}

static bool wgrad_tma_ok(const ConvGeom& g) {
  return win_mode() != 4 && win_mode() != 5 && g.Cin % 64 == 0 && g.Cout % 64 == 0 && g.Wo <= 64 && g.stride <= 2;
}

void conv_wgrad(const ConvGeom& g, const bf16* x, const bf16* dz, int n, int cin_real, float* ws, size_t ws_bytes,
                float* dw, float* db, cudaStream_t st) {
  check_extent((long long)n * (g.H + 1) * (g.W + 1));
  if (wgrad_tma_ok(g)) {
    static WgTmaArgs a;
    a = WgTmaArgs{};
    int Wp = 8;
    while (Wp < g.Wo) Wp <<= 1;
    a.n = n;
    a.Ho = g.Ho;
    a.Wo = g.Wo;
    a.Wp = Wp;
    a.Rk = 64 / Wp;
    a.rg = (g.Ho + a.Rk - 1) / a.Rk;
    a.KW = g.KW;
    a.stride = g.stride;
    a.pad = g.pad;
    a.ncb = g.Cin / 64;
    a.Kconv = g.KH * g.KW * g.Cin;
    a.Cout = g.Cout;
    const int BN = g.Cout <= 64 ? 64 : (g.Cout <= 128 ? 128 : 256);
    const int nkb = n * a.rg;
    const int tiles = ((a.Kconv + 127) / 128) * ((g.Cout + BN - 1) / BN);
    int S = wgrad_splits(tiles, nkb);
    const int kbs = (nkb + S - 1) / S;
    S = (nkb + kbs - 1) / kbs;
    a.kb_per_split = kbs;
    a.splits = S;
    if ((size_t)S * a.Kconv * g.Cout * 4 + (size_t)colsum_blocks((long long)n * g.Ho * g.Wo) * g.Cout * 4 > ws_bytes)
      throw std::runtime_error("wgrad workspace too small (tma)");
    a.out = ws;
    a.x_map = make_tmap_nhwc(x, n, g.H, g.W, g.Cin, 64, Wp, a.Rk, g.stride);
    a.dz_map = make_tmap_nhwc(dz, n, g.Ho, g.Wo, g.Cout, 64, Wp, a.Rk, 1);
    if (BN == 64) launch_wgrad_tma_t<64>(a, st);
    else if (BN == 128) launch_wgrad_tma_t<128>(a, st);
    else launch_wgrad_tma_t<256>(a, st);
    {
      dim3 rg((a.Kconv + 31) / 32, (g.Cout + 31) / 32);
      ProfScope ps(PC_WGRAD_REDUCE, st);
      wgrad_reduce_kernel<<<rg, dim3(32, 8), 0, st>>>(ws, S, a.Kconv, g.Cout, g.Cin, cin_real, dw);
      CK(cudaGetLastError());
    }
    if (db) {
      const long long npix = (long long)n * g.Ho * g.Wo;
      float* part = ws + (size_t)S * a.Kconv * g.Cout;
      const int nb = colsum_blocks(npix);
      const long long rpb = (npix + nb - 1) / nb;
      const int groups = CS_THREADS / (g.Cout / 8);
      ProfScope ps(PC_BIAS_COLSUM, st, 2);
      colsum_partial_kernel<<<nb, CS_THREADS, (size_t)groups * g.Cout * 4, st>>>(dz, npix, g.Cout, rpb, part);
      colsum_final_kernel<<<(g.Cout + 127) / 128, 128, 0, st>>>(part, nb, g.Cout, db);
      CK(cudaGetLastError());
    }
    return;
  }
  if (win_wgrad_ok(g)) {
    // one K-range of 64-position blocks per persistent CTA; partials [S][576][64] reduced in fixed order
    const long long Q = (long long)n * (g.H + 1) * (g.W + 1);
    const int nkb = (int)((Q + 63) / 64);
    int S = std::min(num_sms(), nkb);
    const int kbs = (nkb + S - 1) / S;
    S = (nkb + kbs - 1) / kbs;
    if ((size_t)S * 576 * 64 * 4 + (size_t)colsum_blocks((long long)n * g.Ho * g.Wo) * g.Cout * 4 > ws_bytes)
      throw std::runtime_error("wgrad workspace too small (window)");
    WinArgs w{};
    w.c.src = x;
    w.c.Hs = g.H;
    w.c.Ws = g.W;
    w.c.Cs = 64;
    w.c.n_static = n;
    w.c.B = dz;
    w.c.Nout = 64;
    w.c.out = ws;
    w.c.kb_per_split = kbs;
    for (int kh = 0; kh < 3; ++kh)
      for (int kw = 0; kw < 3; ++kw) w.tap_off[kh * 3 + kw] = kh * (g.W + 1) + kw;
    static bool attr = false;
    if (!attr) {
      CK(cudaFuncSetAttribute(conv_win_wgrad_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, WinWgCfg::SMEM));
      attr = true;
    }
    {
      ProfScope ps(PC_CONV_WGRAD, st);
      conv_win_wgrad_kernel<<<S, NUM_THREADS, WinWgCfg::SMEM, st>>>(w);
      CK(cudaGetLastError());
    }
    {
      dim3 rg((576 + 31) / 32, 2);
      ProfScope ps(PC_WGRAD_REDUCE, st);
      wgrad_reduce_kernel<<<rg, dim3(32, 8), 0, st>>>(ws, S, 576, 64, 64, cin_real, dw);
      CK(cudaGetLastError());
    }
    if (db) {
      const long long npix = (long long)n * g.Ho * g.Wo;
      float* part = ws + (size_t)S * 576 * 64;
      const int nb = colsum_blocks(npix);
      const long long rpb = (npix + nb - 1) / nb;
      const int groups = CS_THREADS / (g.Cout / 8);
      ProfScope ps(PC_BIAS_COLSUM, st, 2);
      colsum_partial_kernel<<<nb, CS_THREADS, (size_t)groups * g.Cout * 4, st>>>(dz, npix, g.Cout, rpb, part);
      colsum_final_kernel<<<(g.Cout + 127) / 128, 128, 0, st>>>(part, nb, g.Cout, db);
      CK(cudaGetLastError());
    }
    return;
  }
  const long long npix = (long long)n * g.Ho * g.Wo;
  const int nkb = (int)((npix + BK - 1) / BK);
  const int Kconv = g.KH * g.KW * g.Cin;
  const int BN = pick_bn(g.Cout, true);
  const int tiles = ((Kconv + BM - 1) / BM) * ((g.Cout + BN - 1) / BN);
  int S = wgrad_splits(tiles, nkb);
  const int kbs = (nkb + S - 1) / S;
  S = (nkb + kbs - 1) / kbs;
  if (wgrad_ws_bytes(g, n) > ws_bytes) throw std::runtime_error("wgrad workspace too small");
  ConvArgs a{};
  a.src = x;
  a.Hs = g.H;
  a.Ws = g.W;
  a.Cs = g.Cin;
  a.n_static = n;
  a.Hg = g.Ho;
  a.Wg = g.Wo;
  a.sy = a.sx = g.stride;
  a.ntaps = g.KH * g.KW;
  for (int kh = 0; kh < g.KH; ++kh)
    for (int kw = 0; kw < g.KW; ++kw) {
      a.ty[kh * g.KW + kw] = (int8_t)(kh - g.pad);
      a.tx[kh * g.KW + kw] = (int8_t)(kw - g.pad);
    }
  a.B = dz;
  a.K = Kconv;
  a.Nout = g.Cout;
  a.out = ws;
  a.kb_per_split = kbs;
  a.splits = S;
  launch_bn<MODE_WGRAD>(BN, a, (long long)tiles * S, st);
  dim3 rg((Kconv + 31) / 32, (g.Cout + 31) / 32);
  {
  ProfScope ps(PC_WGRAD_REDUCE, st);
  wgrad_reduce_kernel<<<rg, dim3(32, 8), 0, st>>>(ws, S, Kconv, g.Cout, g.Cin, cin_real, dw);
  CK(cudaGetLastError());
  }
  if (db) {
    float* part = ws + (size_t)S * Kconv * g.Cout;
    const int nb = colsum_blocks(npix);
    const long long rpb = (npix + nb - 1) / nb;
    if (g.Cout % 8 || g.Cout / 8 > CS_THREADS) throw ShapeError("colsum: Cout must be a multiple of 8, <= 2048");
    const int groups = CS_THREADS / (g.Cout / 8);
    ProfScope ps(PC_BIAS_COLSUM, st, 2);
    colsum_partial_kernel<<<nb, CS_THREADS, (size_t)groups * g.Cout * 4, st>>>(dz, npix, g.Cout, rpb, part);
    colsum_final_kernel<<<(g.Cout + 127) / 128, 128, 0, st>>>(part, nb, g.Cout, db);
    CK(cudaGetLastError());
  }
}

}  // namespace adainf

#ifdef ADAINF_TIMING
// instrumented builds only (tools/build_timing.sh): per-CTA barrier-wait cycle counters of this TU's kernels
extern "C" int adainf_dbg_wait_cycles(unsigned long long* host_out /* 4096*8 */, int reset) {
  cudaDeviceSynchronize();
  cudaMemcpyFromSymbol(host_out, adainf::g_wait_cycles, sizeof(unsigned long long) * 4096 * 8);
  if (reset) {
    static unsigned long long z[4096][8];
    cudaMemcpyToSymbol(adainf::g_wait_cycles, z, sizeof(z));
  }
  return 0;
}
#endif

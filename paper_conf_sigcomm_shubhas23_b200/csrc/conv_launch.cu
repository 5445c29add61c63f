// Host-side launchers for the tcgen05 implicit-GEMM conv kernels (fwd / dgrad phases / wgrad split-K
// + deterministic reduction) and the bias-gradient column sums.
#include <algorithm>
#include <cstdio>
#include <stdexcept>

#include <cstdlib>

#include "conv_gemm.cuh"
#include "conv_win.cuh"
#include "conv_tma.cuh"
#include "conv_pair.cuh"
#include "conv_dualm.cuh"
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
template <int MODE, int BN, int EW>
static void launch_t_ew(const ConvArgs& a, long long max_tiles, cudaStream_t st) {
  dim3 grid((unsigned)std::max(1LL, std::min<long long>(max_tiles, num_sms())));
  using Cfg = ConvCfg<MODE, BN, EW>;
  static bool attr = false;
  if (!attr) {
    CK(cudaFuncSetAttribute(conv_umma_kernel<MODE, BN, EW>, cudaFuncAttributeMaxDynamicSharedMemorySize, Cfg::SMEM));
    attr = true;
  }
  ProfScope ps(MODE == MODE_FWD ? PC_CONV_FWD : (ModeTraits<MODE>::DG_EPI ? PC_CONV_DGRAD : PC_CONV_WGRAD), st);
  conv_umma_kernel<MODE, BN, EW><<<grid, gemm_threads(EW), Cfg::SMEM, st>>>(a);
  CK(cudaGetLastError());
}
// persistent launch: one CTA per SM (or fewer when there are fewer tiles).  Short-K forward tiles (<= 4
// K-blocks: the 1x1 projections) are epilogue-bound: they get two epilogue warps per TMEM lane quadrant.
template <int MODE, int BN>
static void launch_t(const ConvArgs& a, long long max_tiles, cudaStream_t st) {
  // (measured: the dgrad modes lose more to the 128-register cap of the wider CTA than they gain)
  const bool wide_epi = MODE == MODE_FWD && BN >= 64 && a.K <= 4 * BK;
  if constexpr (MODE == MODE_FWD && BN >= 64) {
    if (wide_epi) {
      launch_t_ew<MODE, BN, 2>(a, max_tiles, st);
      return;
    }
  }
  launch_t_ew<MODE, BN, 1>(a, max_tiles, st);
}

// ---- CTA-pair kernel (cta_group::2, M = 256 tiles) ----
// Default for the BN = 256 layers (ResNet layers 3-4 forward and stride-1 dgrad; BN = 128 goes to the dual-M
// kernel first): both CTAs' TMA loads complete on the leader's stage barrier (.cta_group::2), so per SM the
// weight operand's shared-memory reads, writes and L2 -> SM bytes halve with no forwarding hop.  1,024 images:
// layer-3 fwd 178 -> 156 us, dgrad 202 -> 181 us; layer-4 fwd 177 -> 155 us, dgrad 195 -> 173 us.
// ADAINF_PAIR=0 disables.
static int g_pair = -1;
static bool pair_on() {
  if (g_pair < 0) {
    const char* e = getenv("ADAINF_PAIR");
    g_pair = e ? atoi(e) : 1;
  }
  return g_pair != 0;
}
template <int MODE, int BN>
static void launch_pair_t(const ConvArgs& a, long long pair_tiles, cudaStream_t st) {
  using Cfg = PairCfg<MODE, BN>;
  static bool attr = false;
  if (!attr) {
    CK(cudaFuncSetAttribute(conv_pair_kernel<MODE, BN>, cudaFuncAttributeMaxDynamicSharedMemorySize, Cfg::SMEM));
    attr = true;
  }
  const long long pairs = std::max(1LL, std::min<long long>(pair_tiles, num_sms() / 2));
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)(2 * pairs));
  cfg.blockDim = dim3(NUM_THREADS);
  cfg.dynamicSmemBytes = Cfg::SMEM;
  cfg.stream = st;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeClusterDimension;
  at[0].val.clusterDim.x = 2;
  at[0].val.clusterDim.y = 1;
  at[0].val.clusterDim.z = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  ProfScope ps(MODE == MODE_FWD ? PC_CONV_FWD : PC_CONV_DGRAD, st);
  CK(cudaLaunchKernelEx(&cfg, conv_pair_kernel<MODE, BN>, a));
}
// pair launch when eligible: all-TMA operands, BN in {128, 256}; returns false otherwise
template <int MODE>
static bool try_launch_pair(int BN, const ConvArgs& a, long long npix_static, cudaStream_t st) {
  if (!pair_on() || !a.a_tma || !a.b_tma || (BN != 128 && BN != 256)) return false;
  const long long pt = ((npix_static + 2 * BM - 1) / (2 * BM)) * ((a.Nout + BN - 1) / BN);
  if (BN == 128) launch_pair_t<MODE, 128>(a, pt, st);
  else launch_pair_t<MODE, 256>(a, pt, st);
  return true;
}

// ---- dual-M kernel (two 128-row tiles share each weight tile; ADAINF_DUALM=0 disables) ----
static int g_dualm = -1;
static bool dualm_on() {
  if (g_dualm < 0) {
    const char* e = getenv("ADAINF_DUALM");
    g_dualm = e ? atoi(e) : 1;
  }
  return g_dualm != 0;
}
template <int MODE, int BN>
static void launch_dualm_t(const ConvArgs& a, long long tiles, cudaStream_t st) {
  using Cfg = DualMCfg<MODE, BN>;
  static bool attr = false;
  if (!attr) {
    CK(cudaFuncSetAttribute(conv_dualm_kernel<MODE, BN>, cudaFuncAttributeMaxDynamicSharedMemorySize, Cfg::SMEM));
    attr = true;
  }
  dim3 grid((unsigned)std::max(1LL, std::min<long long>(tiles, num_sms())));
  ProfScope ps(MODE == MODE_FWD ? PC_CONV_FWD : PC_CONV_DGRAD, st);
  conv_dualm_kernel<MODE, BN><<<grid, DUALM_THREADS, Cfg::SMEM, st>>>(a);
  CK(cudaGetLastError());
}
template <int MODE>
static bool try_launch_dualm(int BN, const ConvArgs& a, long long npix_static, cudaStream_t st) {
  if (!dualm_on() || !a.a_tma || !a.b_tma || (BN != 128 && BN != 256)) return false;
  // short-K (1x1) launches are bound by per-tile waits / commits: sharing them between two M tiles helps too
  // (layer-2 1x1/2 projection forward 137 -> 106 us); ADAINF_DUALM_SHORTK=0 restores the generic kernel
  if (a.K <= 4 * BK && getenv("ADAINF_DUALM_SHORTK") && atoi(getenv("ADAINF_DUALM_SHORTK")) == 0) return false;
  // BN = 256 (single-buffered accumulators, 2 smem stages) measured slower than the generic kernel: opt-in only
  if (BN == 256 && !(getenv("ADAINF_DUALM256") && atoi(getenv("ADAINF_DUALM256")) == 1)) return false;
  const long long tiles = ((npix_static + 2 * BM - 1) / (2 * BM)) * ((a.Nout + BN - 1) / BN);
  if (BN == 128) launch_dualm_t<MODE, 128>(a, tiles, st);
  else launch_dualm_t<MODE, 256>(a, tiles, st);
  return true;
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
  thread_local WsTmaArgs a;  // host staging (copied into the launch parameters); per thread: handles are independent
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
  // one box per image row when the padded pitch exceeds W (ADAINF_ROWBOX=0: one {64, Wp, R+2} box with
  // out-of-bounds columns)
  static int rowbox = -1;
  if (rowbox < 0) {
    const char* e = getenv("ADAINF_ROWBOX");
    rowbox = e ? atoi(e) : 1;
  }
  a.rowbox = rowbox && Wp > W && W % 8 == 0 && W <= 256;
  a.win_map = a.rowbox ? make_tmap_nhwc(c.src, nstatic, H, W, 64, 64, W, 1)
                       : make_tmap_nhwc(c.src, nstatic, H, W, 64, 64, Wp, R + 2);
  const bf16* e0 = dgrad ? c.sc : c.res;
  const bf16* e1 = dgrad && c.mask_act ? c.yact : nullptr;
  a.has_e0 = e0 != nullptr;
  a.has_e1 = e1 != nullptr;
  if (e0) a.e0_map = make_tmap_nhwc(e0, nstatic, H, W, 64, 64, Wp, R);
  if (e1) a.e1_map = make_tmap_nhwc(e1, nstatic, H, W, 64, 64, Wp, R);
  a.out_map = make_tmap_nhwc(c.out, nstatic, H, W, 64, 64, Wp, R);
  if (!dgrad && c.res_map && c.res_map != c.src_map) throw std::runtime_error("ws_tma: residual map differs");
  const int fixed = 9 * 8192 + 2 * std::max(1, a.has_e0 + a.has_e1) * 16384 + 1024 /*align*/ +
                    512 /*barriers*/;
  // tile pairs (unit mode) when two pair windows of 2R+2 rows fit next to the resident weights and the
  // epilogue staging (forward; the dgrad staging of two operands leaves room for one): ADAINF_WS_UNIT=0 disables
  static int unit_env = -1;
  if (unit_env < 0) {
    const char* e = getenv("ADAINF_WS_UNIT");
    unit_env = e ? atoi(e) : 1;
  }
  const int unit_bytes = ((16 + (2 * R + 2) * Wp) * 128 + 1023) / 1024 * 1024;
  a.unit = unit_env && a.rowbox && 227 * 1024 - fixed >= 2 * unit_bytes;
  a.upi = (a.tpi + 1) / 2;
  a.win_bytes = a.unit ? unit_bytes : ((16 + (R + 2) * Wp) * 128 + 1023) / 1024 * 1024;
  a.wstages = a.unit ? 2 : std::min(8, (227 * 1024 - fixed) / a.win_bytes);
  if (const char* e = getenv("ADAINF_WS_STAGES"))
    if (!a.unit) a.wstages = std::min(a.wstages, std::max(1, atoi(e)));
  if (a.wstages < 2) throw std::runtime_error("ws_tma: shared memory");
  const int smem = a.wstages * a.win_bytes + fixed;
  static bool attr = false;
  if (!attr) {
    CK(cudaFuncSetAttribute(conv_ws_tma_kernel<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024));
    CK(cudaFuncSetAttribute(conv_ws_tma_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024));
    attr = true;
  }
  const long long items = (long long)nstatic * (a.unit ? a.upi : a.tpi);
  dim3 grid((unsigned)std::max(1LL, std::min<long long>(items, num_sms())));
  ProfScope ps(dgrad ? PC_CONV_DGRAD : PC_CONV_FWD, st);
  if (a.unit) conv_ws_tma_kernel<true><<<grid, TMA_WS_THREADS, smem, st>>>(a);
  else conv_ws_tma_kernel<false><<<grid, TMA_WS_THREADS, smem, st>>>(a);
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
  thread_local WinTmaArgs a;
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

// TMA for the weight operand of the generic kernel (ADAINF_BTMA=0 restores the cp.async B path)
static int g_btma = -1;
static bool btma_on() {
  if (g_btma < 0) {
    const char* e = getenv("ADAINF_BTMA");
    g_btma = e ? atoi(e) : 1;
  }
  return g_btma != 0;
}

// TMA im2col for the A operand of the generic kernel (ADAINF_ATMA=0 restores the cp.async gather)
static int g_atma = -1;
static bool atma_on() {
  if (g_atma < 0) {
    const char* e = getenv("ADAINF_ATMA");
    g_atma = e ? atoi(e) : 1;
  }
  return g_atma != 0;
}
// Switch the A operand to im2col TMA loads when the gather is a plain strided window over a dense source:
// the base pixel of GEMM row (n, gy, gx) is (gy * s + lo, gx * s + lo) and every tap offset is >= 0 from it.
static void try_a_tma(ConvArgs& a) {
  if (!atma_on() || !a.b_tma || a.src_map || a.Cs % 64 != 0 || a.Hs != a.Ws || a.Hg != a.Wg || a.sy != a.sx ||
      a.sy > 8 || a.ntaps <= 0)
    return;
  int loy = 127, lox = 127;
  for (int t = 0; t < a.ntaps; ++t) loy = std::min(loy, (int)a.ty[t]), lox = std::min(lox, (int)a.tx[t]);
  if (loy != lox) return;
  const int lo = loy, up = lo + (a.Hg - 1) * a.sy - (a.Hs - 1);
  if (lo < -128 || up < -128 || up > 127) return;
  a.a_map = make_tmap_im2col(a.src, a.n_static, a.Hs, a.Ws, a.Cs, lo, up, a.sy, 64, BM);
  a.a_lo = lo;
  a.a_tma = 1;
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
  // the generic kernel with im2col TMA operands beats the window kernels except at 64x64 (BN = 64); the window
  // kernels still serve survivor-mapped sources (x_map), which im2col TMA cannot gather
  const bool gen_tma = atma_on() && btma_on() && !x_map && g.Cin % 64 == 0 && g.H == g.W;
  if (win_ok(g) && !out_f32 &&
      (win_mode() >= 2 || (g.Cin == 64 && g.Cout == 64) ||
       (!gen_tma && win_mode() != 4 && g.W <= 28 && g.W >= 8 && g.Cout % 128 == 0))) {
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
  int BN = pick_bn(g.Cout, false);
  const long long mt = ((long long)n_static * g.Ho * g.Wo + BM - 1) / BM;
  if (mt == 0) return;
  // small batches (early-exit survivors; the device-side count is at most n_static): narrower N tiles until the
  // full-batch tile count covers two waves, so a partial survivor set still spreads over the SMs
  static int narrow = -1;  // ADAINF_NARROW=0 keeps the full BN (tests use it to reach the wide-tile kernels)
  if (narrow < 0) {
    const char* e = getenv("ADAINF_NARROW");
    narrow = e ? atoi(e) : 1;
  }
  while (narrow && BN > 64 && mt * ((g.Cout + BN - 1) / BN) < 2 * num_sms()) BN /= 2;
  if (btma_on() && ldb % 8 == 0 && ((uintptr_t)w & 15) == 0) {
    a.b_tma = 1;
    a.b_map = make_tmap_2d(w, g.Cout, a.K, ldb, 64, BN);  // K-major [Cout][K]; k >= K and rows >= Cout read 0
    try_a_tma(a);
    if (try_launch_dualm<MODE_FWD>(BN, a, (long long)n_static * g.Ho * g.Wo, st)) return;
    if (a.a_tma && pair_on() && (BN == 128 || BN == 256) && a.K > 4 * BK) {
      a.b_map = make_tmap_2d(w, g.Cout, a.K, ldb, 64, BN / 2);  // each CTA of the pair loads half the N rows
      if (try_launch_pair<MODE_FWD>(BN, a, (long long)n_static * g.Ho * g.Wo, st)) return;
    }
  }
  launch_bn<MODE_FWD>(BN, a, mt * ((g.Cout + BN - 1) / BN), st);
}

void conv_dgrad(const ConvGeom& g, const bf16* dz, const bf16* w, int ldb, int n, const float* bcast,
                const bf16* sc, const bf16* yact, int mask_act, bf16* dx, cudaStream_t st) {
  check_extent((long long)n * (g.H + 1) * (g.W + 1));
  // dX[y] = sum_{kh: (y + pad - kh) % s == 0} dZ[(y + pad - kh)/s] W[kh]; split by output phase (py,px)
  // W < 8 (ResNet layer 4): the generic kernel with TMA weight boxes beats the cp.async window kernel
  const bool small_w_generic = g.W < 8 && btma_on() && g.Cout % 64 == 0 && g.Cin % 64 == 0 && win_mode() < 2;
  const bool gen_tma = atma_on() && btma_on() && g.Cout % 64 == 0 && g.Cin % 64 == 0 && g.H == g.W;
  if (win_ok(g) && !small_w_generic &&
      (win_mode() >= 2 || (g.Cin == 64 && g.Cout == 64) ||
       (!gen_tma && (g.H <= 14 || (g.W <= 28 && g.Cin % 128 == 0))))) {
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
      if (btma_on() && g.Cout % 64 == 0 && g.Cin % 64 == 0 && BN % 64 == 0 && ldb % 8 == 0 &&
          ((uintptr_t)w & 15) == 0) {
        a.b_tma = 1;
        a.b_map = make_tmap_2d(w, g.Cout, ldb, ldb, 64, 64);  // rows co, cols (tap, ci): MN-major boxes
        try_a_tma(a);
        if (s == 1 && try_launch_dualm<MODE_DGRAD>(BN, a, (long long)n * a.Hg * a.Wg, st)) continue;
        if (s == 1 && a.K > 4 * BK && try_launch_pair<MODE_DGRAD>(BN, a, (long long)n * a.Hg * a.Wg, st)) continue;
      }
      launch_bn<MODE_DGRAD>(BN, a, mt * ((g.Cin + BN - 1) / BN), st);
    }
}

// ---- stride-2 dgrad as one sub-pixel GEMM (see MODE_DGRAD_SP in conv_gemm.cuh) ----
bool dgrad_sp_ok(const ConvGeom& g) {
  return btma_on() && g.stride == 2 && g.KH == 3 && g.KW == 3 && g.pad == 1 && g.Cin % 64 == 0 &&
         g.Cout % 64 == 0 && g.H <= 2 * g.Ho && g.W <= 2 * g.Wo && getenv("ADAINF_NO_SP") == nullptr;
}
size_t dgrad_sp_ws_bytes(const ConvGeom& g) { return (size_t)4 * g.Cin * 4 * g.Cout * 2; }

// Bsp[(py,px,ci)][(a,b,co)] = W[co][kh = py+p-2a][kw = px+p-2b][ci], 0 where the tap does not exist.
// One thread per 8 consecutive output columns (8 co of one (a,b)): eight 2-byte gathers from the (L2-resident)
// shadow, one coalesced 16-byte store.
__global__ void sp_weight_kernel(const bf16* __restrict__ w, int ldb, int Cin, int Cout, int K, int pad,
                                 bf16* __restrict__ bsp) {
  const int K4 = 4 * Cout, KV = K4 / 8;
  const long long total = 4LL * Cin * KV;
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < total; i += (long long)gridDim.x * blockDim.x) {
    const int kv = (int)(i % KV);
    const long long r = i / KV;  // output row (ph, ci)
    const int ci = (int)(r % Cin), ph = (int)(r / Cin);
    const int kcol0 = kv * 8;
    const int ab = kcol0 / Cout, co0 = kcol0 - ab * Cout;
    const int py = ph >> 1, px = ph & 1, aa = ab >> 1, bb = ab & 1;
    const int kh = py + pad - 2 * aa, kw = px + pad - 2 * bb;
    __align__(16) bf16 h[8];
    const bool ok = kh >= 0 && kh < K && kw >= 0 && kw < K;
#pragma unroll
    for (int q = 0; q < 8; ++q)
      h[q] = ok ? w[(long long)(co0 + q) * ldb + (kh * K + kw) * Cin + ci] : __float2bfloat16_rn(0.f);
    *(uint4*)(bsp + r * K4 + kcol0) = *(const uint4*)h;
  }
}

void conv_dgrad_sp(const ConvGeom& g, const bf16* dz, const bf16* w, int ldb, bf16* wsp, int n, const float* bcast,
                   const bf16* sc, bool sc_compact, const bf16* yact, int mask_act, bf16* dx, cudaStream_t st) {
  if (!dgrad_sp_ok(g)) throw ShapeError("conv_dgrad_sp: unsupported geometry");
  check_extent((long long)n * (g.H + 1) * (g.W + 1));
  if (n <= 0) return;
  {
    ProfScope ps(PC_CONV_DGRAD_PREP, st);
    const long long total = 4LL * g.Cin * (4 * g.Cout / 8);
    const int blocks = (int)std::min<long long>((total + 255) / 256, 8LL * num_sms());
    sp_weight_kernel<<<blocks, 256, 0, st>>>(w, ldb, g.Cin, g.Cout, 3, g.pad, wsp);
    CK(cudaGetLastError());
  }
  thread_local ConvArgs a;
  a = ConvArgs{};
  a.src = dz;
  a.Hs = g.Ho;
  a.Ws = g.Wo;
  a.Cs = g.Cout;
  a.n_static = n;
  a.Hg = g.Ho;
  a.Wg = g.Wo;
  a.sy = a.sx = 1;
  a.ntaps = 4;
  for (int t = 0; t < 4; ++t) {
    a.ty[t] = (int8_t)(t >> 1);
    a.tx[t] = (int8_t)(t & 1);
  }
  a.B = wsp;
  a.ldb = 4 * g.Cout;
  a.K = 4 * g.Cout;
  a.Nout = 4 * g.Cin;
  a.out = dx;
  a.Ho = g.H;
  a.Wo = g.W;
  a.oys = a.oxs = 1;
  a.bcast = bcast;
  a.sc = sc;
  a.yact = yact;
  a.mask_act = mask_act;
  a.sp_cin = g.Cin;
  a.sp_sc_compact = sc_compact ? 1 : 0;
  if (const char* e = getenv("ADAINF_EXP")) a.exp_flags = atoi(e);  // experiments only
  a.b_tma = 1;
  try_a_tma(a);
  // CTA pair when the packed weights span several N tiles (layers 3-4: 4*Cin >= 512; each CTA streams half of
  // them per K-block): layer-4 sub-pixel dgrad 178 -> 158 us, layer 3 223 -> 221 us; layer 2 (one N tile,
  // epilogue-bound) is 3% slower as a pair and stays single
  if (a.a_tma && pair_on() && a.Nout >= 512) {
    a.b_map = make_tmap_2d(wsp, a.Nout, a.K, a.ldb, 64, 128);
    if (try_launch_pair<MODE_DGRAD_SP>(256, a, (long long)n * g.Ho * g.Wo, st)) return;
  }
  a.b_map = make_tmap_2d(wsp, a.Nout, a.K, a.ldb, 64, 256);
  const long long mt = ((long long)n * g.Ho * g.Wo + BM - 1) / BM;
  launch_t<MODE_DGRAD_SP, 256>(a, mt * ((a.Nout + 255) / 256), st);
}

// partial [S][Kconv][Cout] -> dw [Cout][taps][cin_real] (fp32), summed over S in fixed order
// stage 1 of the split-K reduction when there are many splits: group g sums splits [g*SG, (g+1)*SG) in
// order (float4 per thread); stage 2 (wgrad_reduce_kernel) sums the groups in order and transposes.
constexpr int WG_SG = 8;
__global__ void wgrad_reduce_groups_kernel(const float4* __restrict__ part, int S, long long n4,
                                           float4* __restrict__ out) {
  const long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n4) return;
  const int s0 = blockIdx.y * WG_SG, s1 = min(S, s0 + WG_SG);
  float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
  for (int s = s0; s < s1; ++s) {
    const float4 v = __ldg(part + (long long)s * n4 + i);
    acc.x += v.x;
    acc.y += v.y;
    acc.z += v.z;
    acc.w += v.w;
  }
  out[(long long)blockIdx.y * n4 + i] = acc;
}

__global__ void wgrad_reduce_kernel(const float* __restrict__ part, int S, int Kconv, int Cout, int cin_pad,
                                    int cin_real, float* __restrict__ dw) {
  __shared__ float tile[32][33];
  const int k0 = blockIdx.x * 32, c0 = blockIdx.y * 32;
  const int tx = threadIdx.x, ty = threadIdx.y;  // 32 x (8 or 32)
  const int ry = blockDim.y;
  for (int r = ty; r < 32; r += ry) {
    const int k = k0 + r, co = c0 + tx;
    float acc = 0.f;
    if (k < Kconv && co < Cout) {  // eight independent loads in flight, summed in ascending split order
      const float* pp = part + (long long)k * Cout + co;
      const long long sstride = (long long)Kconv * Cout;
      int s = 0;
      for (; s + 8 <= S; s += 8) {
        float v[8];
#pragma unroll
        for (int u = 0; u < 8; ++u) v[u] = __ldg(pp + (s + u) * sstride);
#pragma unroll
        for (int u = 0; u < 8; ++u) acc += v[u];
      }
      for (; s < S; ++s) acc += __ldg(pp + s * sstride);
    }
    tile[r][tx] = acc;
  }
  __syncthreads();
  for (int r = ty; r < 32; r += ry) {
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
// out[c] = sum over nb partial rows, deterministic: 8 row groups per channel (rows g, g+8, ... in order, eight
// loads in flight), then the 8 group sums in group order
__global__ void __launch_bounds__(256) colsum_final_kernel(const float* __restrict__ part, int nb, int C,
                                                           float* __restrict__ out) {
  __shared__ float red[8][33];
  const int cx = threadIdx.x & 31, gy = threadIdx.x >> 5;
  const int c = blockIdx.x * 32 + cx;
  float acc = 0.f;
  if (c < C) {
    int b = gy;
    for (; b + 56 < nb; b += 64) {
      float v[8];
#pragma unroll
      for (int u = 0; u < 8; ++u) v[u] = __ldg(part + (long long)(b + 8 * u) * C + c);
#pragma unroll
      for (int u = 0; u < 8; ++u) acc += v[u];
    }
    for (; b < nb; b += 8) acc += __ldg(part + (long long)b * C + c);
  }
  red[gy][cx] = acc;
  __syncthreads();
  if (gy == 0 && c < C) {
    float t = red[0][cx];
#pragma unroll
    for (int g = 1; g < 8; ++g) t += red[g][cx];
    out[c] = t;
  }
}
static int colsum_blocks(long long P) { return (int)std::max(1LL, std::min<long long>((P + 63) / 64, 4LL * num_sms())); }

// split-K factor: one balanced wave of persistent CTAs (units = tiles * S <= #SMs), each unit a contiguous
// range of 64-pixel K-blocks; the fp32 partials are reduced in fixed order (deterministic)
static int wgrad_splits(int tiles, int nkb) {
  if (tiles >= num_sms()) return 1;
  return std::max(1, std::min(nkb, num_sms() / tiles));
}

// Weight-gradient execution plan, shared by the workspace query and the launcher so both agree on the
// split-K factor.  Paths: TMA window (stride-1 3x3, 64-aligned channels), TMA generic (64-aligned
// channels, Wo <= 64), cp.async window (64x64 3x3, when TMA is disabled by the debug mode), generic.
enum WgPath { WG_GENERIC = 0, WG_WIN_CPASYNC = 1, WG_TMA = 2, WG_WIN_TMA = 3 };
struct WgPlan {
  WgPath path;
  int S, kbs, nkb, Kconv, tiles;
  int BN;          // WG_TMA / WG_GENERIC
  int Wp, R, rg;   // TMA paths
  int i2c;         // WG_TMA: K-blocks of 64 consecutive output pixels via im2col TMA
  int pm = 1;      // WG_TMA: 128-row M tiles per tile (2: two M tiles share each dZ K-block)
};

static bool win_wgrad_ok(const ConvGeom& g) {
  return win_mode() > 0 && g.KH == 3 && g.KW == 3 && g.stride == 1 && g.pad == 1 && g.Cin == 64 && g.Cout == 64 &&
         g.W <= 56 && g.H == g.Ho && g.W == g.Wo;
}
static bool tma_wgrad_allowed() { return win_mode() != 4 && win_mode() != 5; }
static bool win_tma_wgrad_ok(const ConvGeom& g) {
  return tma_wgrad_allowed() && win_mode() != 6 && g.KH == 3 && g.KW == 3 && g.stride == 1 && g.pad == 1 &&
         g.Cin % 64 == 0 && g.Cout % 64 == 0 && g.H == g.Ho && g.W == g.Wo && g.W <= 127 &&
         ((g.W >= 14 && g.Cout < 256) || win_mode() == 7);  // below 14 columns the padded window wastes too much;
  // from Cout = 256 the two-M-tile TMA GEMM (N = 256) beats the N = 64 window kernel (181 vs 263 us, layer 3)
}
static bool wgrad_tma_ok(const ConvGeom& g) {
  return tma_wgrad_allowed() && g.Cin % 64 == 0 && g.Cout % 64 == 0 && g.Wo <= 64 && g.stride <= 2;
}

// im2col TMA for the weight-gradient A operand (ADAINF_WG_I2C=0: padded-pitch boxes)
static bool wgrad_i2c_ok(const ConvGeom& g) {
  static int env = -1;
  if (env < 0) {
    const char* e = getenv("ADAINF_WG_I2C");
    env = e ? atoi(e) : 1;
  }
  const int lo = -g.pad, up = lo + (g.Ho - 1) * g.stride - (g.H - 1);
  return env && atma_on() && g.H == g.W && g.Ho == g.Wo && g.KH == g.KW && lo >= -128 && up >= -128 && up <= 127;
}

static void finish_splits(WgPlan& p) {
  p.S = wgrad_splits(p.tiles, p.nkb);
  p.kbs = (p.nkb + p.S - 1) / p.S;
  p.S = (p.nkb + p.kbs - 1) / p.kbs;
}

static int win_wg_stage_bytes(int Wp, int R) { return (16 + (R + 2) * Wp) * 128 + R * Wp * 128; }

static WgPlan plan_wgrad(const ConvGeom& g, int n) {
  WgPlan p{};
  p.Kconv = g.KH * g.KW * g.Cin;
  if (win_tma_wgrad_ok(g)) {
    p.path = WG_WIN_TMA;
    int Wp = 8;
    while (Wp < g.W + 1) Wp <<= 1;
    // R rows per K-block: K = R*Wp pixels a multiple of 16 and <= 256, >= 3 pipeline stages; least padded
    // rows (R * ceil(H/R)) first, then the largest K
    int bestR = 0;
    long long best_rows = 0;
    for (int R = 1; R * Wp <= 256; ++R) {
      if ((R * Wp) % 16) continue;
      if (3 * win_wg_stage_bytes(Wp, R) + 4096 > 225 * 1024) continue;
      const long long rows = (long long)R * ((g.H + R - 1) / R);
      if (!bestR || rows < best_rows || (rows == best_rows && R > bestR)) {
        bestR = R;
        best_rows = rows;
      }
    }
    if (bestR) {
      p.Wp = Wp;
      p.R = bestR;
      p.rg = (g.H + bestR - 1) / bestR;
      p.nkb = n * p.rg;
      p.tiles = (g.Cin / 64) * (g.Cout / 64);
      finish_splits(p);
      return p;
    }
  }
  if (wgrad_tma_ok(g)) {
    p.path = WG_TMA;
    int Wp = 8;
    while (Wp < g.Wo) Wp <<= 1;
    p.Wp = Wp;
    p.R = 64 / Wp;
    p.rg = (g.Ho + p.R - 1) / p.R;
    p.nkb = n * p.rg;
    if (wgrad_i2c_ok(g)) {  // K-blocks of 64 consecutive output pixels: no pitch padding
      p.i2c = 1;
      p.nkb = (int)(((long long)n * g.Ho * g.Wo + 63) / 64);
    }
    p.BN = g.Cout <= 64 ? 64 : (g.Cout <= 128 ? 128 : 256);
    {
      static int env_pm = -1;  // ADAINF_WG_PM=1 keeps one M tile per tile
      if (env_pm < 0) {
        const char* e = getenv("ADAINF_WG_PM");
        env_pm = e ? atoi(e) : 2;
      }
      p.pm = (env_pm == 2 && p.BN >= 128 && (p.Kconv + 127) / 128 >= 3) ? 2 : 1;  // 1x1 (<= 2 M tiles): 1
    }
    p.tiles = (((p.Kconv + 127) / 128 + p.pm - 1) / p.pm) * ((g.Cout + p.BN - 1) / p.BN);
    finish_splits(p);
    return p;
  }
  if (win_wgrad_ok(g)) {
    p.path = WG_WIN_CPASYNC;
    const long long Q = (long long)n * (g.H + 1) * (g.W + 1);
    p.nkb = (int)((Q + 63) / 64);
    p.tiles = 1;
    p.S = std::min(num_sms(), p.nkb);
    p.kbs = (p.nkb + p.S - 1) / p.S;
    p.S = (p.nkb + p.kbs - 1) / p.kbs;
    return p;
  }
  p.path = WG_GENERIC;
  const long long npix = (long long)n * g.Ho * g.Wo;
  p.nkb = (int)((npix + BK - 1) / BK);
  p.BN = pick_bn(g.Cout, true);
  p.tiles = ((p.Kconv + BM - 1) / BM) * ((g.Cout + p.BN - 1) / p.BN);
  finish_splits(p);
  return p;
}

// workspace: [S][Kconv][Cout] split partials, then column-sum partials [max(S, colsum blocks)][Cout], then
// the grouped partials [ceil(S / WG_SG)][Kconv][Cout] of the two-stage reduction
static size_t wgrad_ws_floats(const WgPlan& p, const ConvGeom& g, int n, size_t* cs_off, size_t* grp_off) {
  const long long npix = (long long)n * g.Ho * g.Wo;
  const size_t kc = (size_t)p.Kconv * g.Cout;
  const size_t a = (size_t)p.S * kc;
  const size_t b = (size_t)std::max(p.S * ((p.Kconv + 127) / 128), colsum_blocks(npix)) * g.Cout;
  const size_t grp = p.S > WG_SG ? (size_t)((p.S + WG_SG - 1) / WG_SG) * kc : 0;
  if (cs_off) *cs_off = a;
  if (grp_off) *grp_off = (a + b + 3) / 4 * 4;
  return (a + b + 3) / 4 * 4 + grp;
}

size_t wgrad_ws_bytes(const ConvGeom& g, int n) {
  const WgPlan p = plan_wgrad(g, n);
  return wgrad_ws_floats(p, g, n, nullptr, nullptr) * sizeof(float);
}

template <int BN, int PM>
static void launch_wgrad_tma_t(WgTmaArgs& a, cudaStream_t st) {
  constexpr int STAGE = PM * 16384 + BN * 128;
  a.stages = std::min(16, (225 * 1024 - 5120) / STAGE);
  const int smem = a.stages * STAGE + 2048 + 3072;
  static bool attr = false;
  if (!attr) {
    CK(cudaFuncSetAttribute(conv_wgrad_tma_kernel<BN, PM>, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024));
    attr = true;
  }
  const long long units =
      (long long)(((a.Kconv + 127) / 128 + PM - 1) / PM) * ((a.Cout + BN - 1) / BN) * a.splits;
  dim3 grid((unsigned)std::max(1LL, std::min<long long>(units, num_sms())));
  ProfScope ps(PC_CONV_WGRAD, st);
  conv_wgrad_tma_kernel<BN, PM><<<grid, NUM_THREADS, smem, st>>>(a);
  CK(cudaGetLastError());
}

void conv_wgrad(const ConvGeom& g, const bf16* x, const bf16* dz, int n, int cin_real, float* ws, size_t ws_bytes,
                float* dw, float* db, cudaStream_t st) {
  check_extent((long long)n * (g.H + 1) * (g.W + 1));
  const WgPlan p = plan_wgrad(g, n);
  const long long npix = (long long)n * g.Ho * g.Wo;
  size_t cs_off = 0, grp_off = 0;
  if (wgrad_ws_floats(p, g, n, &cs_off, &grp_off) * sizeof(float) > ws_bytes)
    throw std::runtime_error("wgrad workspace too small");
  float* cs_part = ws + cs_off;
  const bool fused_cs = db && (p.path == WG_WIN_TMA || p.path == WG_TMA);
  if (db && (g.Cout % 8 || g.Cout / 8 > CS_THREADS)) throw ShapeError("colsum: Cout must be a multiple of 8, <= 2048");
  const int S = p.S;

  if (p.path == WG_WIN_TMA) {
    thread_local WinWgTmaArgs a;
    a = WinWgTmaArgs{};
    a.n = n;
    a.H = g.H;
    a.Wp = p.Wp;
    a.R = p.R;
    a.rg = p.rg;
    a.ncb = g.Cin / 64;
    a.nnb = g.Cout / 64;
    a.Cin = g.Cin;
    a.Cout = g.Cout;
    a.kb_per_split = p.kbs;
    a.splits = S;
    a.out = ws;
    a.a_bytes = (16 + (p.R + 2) * p.Wp) * 128;
    a.cs_part = fused_cs ? cs_part : nullptr;
    const int stage = win_wg_stage_bytes(p.Wp, p.R);
    a.stages = std::min(8, (225 * 1024 - 7168) / stage);
    const int smem = a.stages * stage + 2048 + 1024 + 256 + 3072;
    a.x_map = make_tmap_nhwc(x, n, g.H, g.W, g.Cin, 64, p.Wp, p.R + 2);
    a.dz_map = make_tmap_nhwc(dz, n, g.H, g.W, g.Cout, 64, p.Wp, p.R);
    static bool attr = false;
    if (!attr) {
      CK(cudaFuncSetAttribute(conv_wgrad_win_tma_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024));
      attr = true;
    }
    const int units = p.tiles * S;
    ProfScope ps(PC_CONV_WGRAD, st);
    conv_wgrad_win_tma_kernel<<<std::max(1, std::min(units, num_sms())), NUM_THREADS, smem, st>>>(a);
    CK(cudaGetLastError());
  } else if (p.path == WG_TMA) {
    thread_local WgTmaArgs a;
    a = WgTmaArgs{};
    a.n = n;
    a.Ho = g.Ho;
    a.Wo = g.Wo;
    a.Wp = p.Wp;
    a.Rk = p.R;
    a.rg = p.rg;
    a.KW = g.KW;
    a.stride = g.stride;
    a.pad = g.pad;
    a.ncb = g.Cin / 64;
    a.Kconv = p.Kconv;
    a.Cout = g.Cout;
    a.kb_per_split = p.kbs;
    a.splits = S;
    a.out = ws;
    a.cs_part = fused_cs ? cs_part : nullptr;
    if (p.i2c) {
      a.i2c = 1;
      a.lo = -g.pad;
      a.n = p.nkb;  // K-blocks (rg = 1)
      a.rg = 1;
      a.x_map = make_tmap_im2col(x, n, g.H, g.W, g.Cin, -g.pad, -g.pad + (g.Ho - 1) * g.stride - (g.H - 1), g.stride,
                                 64, 64);
      a.dz_map = make_tmap_2d(dz, (long long)n * g.Ho * g.Wo, g.Cout, g.Cout, 64, 64);
    } else {
      a.x_map = make_tmap_nhwc(x, n, g.H, g.W, g.Cin, 64, p.Wp, p.R, g.stride);
      a.dz_map = make_tmap_nhwc(dz, n, g.Ho, g.Wo, g.Cout, 64, p.Wp, p.R, 1);
    }
    if (p.BN == 64) launch_wgrad_tma_t<64, 1>(a, st);
    else if (p.BN == 128) {
      if (p.pm == 2) launch_wgrad_tma_t<128, 2>(a, st);
      else launch_wgrad_tma_t<128, 1>(a, st);
    } else {
      if (p.pm == 2) launch_wgrad_tma_t<256, 2>(a, st);
      else launch_wgrad_tma_t<256, 1>(a, st);
    }
  } else if (p.path == WG_WIN_CPASYNC) {
    // one K-range of 64-position blocks per persistent CTA; partials [S][576][64] reduced in fixed order
    WinArgs w{};
    w.c.src = x;
    w.c.Hs = g.H;
    w.c.Ws = g.W;
    w.c.Cs = 64;
    w.c.n_static = n;
    w.c.B = dz;
    w.c.Nout = 64;
    w.c.out = ws;
    w.c.kb_per_split = p.kbs;
    for (int kh = 0; kh < 3; ++kh)
      for (int kw = 0; kw < 3; ++kw) w.tap_off[kh * 3 + kw] = kh * (g.W + 1) + kw;
    static bool attr = false;
    if (!attr) {
      CK(cudaFuncSetAttribute(conv_win_wgrad_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, WinWgCfg::SMEM));
      attr = true;
    }
    ProfScope ps(PC_CONV_WGRAD, st);
    conv_win_wgrad_kernel<<<S, NUM_THREADS, WinWgCfg::SMEM, st>>>(w);
    CK(cudaGetLastError());
  } else {
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
    a.K = p.Kconv;
    a.Nout = g.Cout;
    a.out = ws;
    a.kb_per_split = p.kbs;
    a.splits = S;
    launch_bn<MODE_WGRAD>(p.BN, a, (long long)p.tiles * S, st);
  }
  {
    ProfScope ps(PC_WGRAD_REDUCE, st, S > WG_SG ? 2 : 1);
    const float* src = ws;
    int S2 = S;
    if (S > WG_SG) {
      const long long n4 = (long long)p.Kconv * g.Cout / 4;  // Cout % 8 == 0
      const int G = (S + WG_SG - 1) / WG_SG;
      dim3 gg((unsigned)((n4 + 255) / 256), G);
      wgrad_reduce_groups_kernel<<<gg, 256, 0, st>>>((const float4*)ws, S, n4, (float4*)(ws + grp_off));
      src = ws + grp_off;
      S2 = G;
    }
    dim3 rg((p.Kconv + 31) / 32, (g.Cout + 31) / 32);
    // small weight tensors: one thread per element of the 32x32 tile (more loads in flight per SM)
    const dim3 rb(32, (long long)rg.x * rg.y < 2LL * num_sms() ? 32 : 8);
    wgrad_reduce_kernel<<<rg, rb, 0, st>>>(src, S2, p.Kconv, g.Cout, g.Cin, cin_real, dw);
    CK(cudaGetLastError());
  }
  if (db) {
    ProfScope ps(PC_BIAS_COLSUM, st, fused_cs ? 1 : 2);
    int nb = p.path == WG_TMA ? S * (((p.Kconv + 127) / 128 + p.pm - 1) / p.pm) : S;  // fused partial rows
    if (!fused_cs) {
      nb = colsum_blocks(npix);
      const long long rpb = (npix + nb - 1) / nb;
      const int groups = CS_THREADS / (g.Cout / 8);
      colsum_partial_kernel<<<nb, CS_THREADS, (size_t)groups * g.Cout * 4, st>>>(dz, npix, g.Cout, rpb, cs_part);
    }
    colsum_final_kernel<<<(g.Cout + 31) / 32, 256, 0, st>>>(cs_part, nb, g.Cout, db);
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

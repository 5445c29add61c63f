// 3x3 stride-1 conv + bias + act + 2x2/2 max-pool in ONE tensor-core kernel, for the few-channel early layers of
// the TinyYOLOv3-like detector (BASELINE config 3, reading Q18; P:29 / P:74 the video DAG's first model).  These
// layers carry most of the detector's bytes but little arithmetic (416x416x3 -> 16, 208x208x16 -> 32,
// 104x104x32 -> 64, 52x52x64 -> 128, each followed by a 2x2/2 pool): through the generic implicit GEMM they ran at
// 0.3-0.7 TB/s (K = 9 x 16 per output, per-K-block pipeline overhead) and wrote the full-resolution conv tensor only
// for the pool to read it back.  Here the conv output never reaches HBM: only the pooled tensor is written.
//
// Layout (as the stem kernel, stem.cu): the input is NHWC bf16 viewed as P planes of 16 channels; one TMA box per
// plane loads a window of RIN image rows x 136 positions (columns c0-1 .. c0+134, out-of-bounds -> zeros) with
// SWIZZLE_32B (32-byte rows = one K=16 slice per position).  Tap (dy, dx) of the 3x3 stencil is that window viewed
// (dy*136 + dx) rows further: one tcgen05.mma M=128 (output columns c0 .. c0+127) x N x K=16 per (tap, plane), the
// weights resident in shared memory (no-swizzle K-major core matrices).
//   ROWPAIR (Cin = 16P, P <= 2, Cout = N <= 128): a work item is two output rows (2rp, 2rp+1) of one 128-column
//     tile; two TMEM accumulators; the epilogue thread of column x takes the vertical max of the fp32 sums, then
//     the horizontal max with lane x^1 (shuffle), and even lanes add the bias, apply the act and round to bf16
//     (all non-decreasing, so this equals the oracle's pool of rounded conv outputs exactly).
//   S2D (first layer, <= 4 input channels): the input is space-to-depth packed (pack_s2d: 2x2 pixels x 4 ch = 16
//     channels per position), so the stride-1 3x3 conv over a 2x2 output block is a 3x3 conv on the s2d grid with
//     N = 4 sub-pixels x Cout (weights expanded, zero where the original tap falls outside 3x3); the 2x2 pool is
//     the max over the four sub-pixel column groups of one thread: no neighbour exchange (two s2d rows per item).
// Warp roles: warp 0 TMA producer, warp 1 MMA issuer, then NB groups of 4 epilogue warps (TMEM lane quadrant =
// warp % 4), one TMEM accumulator buffer each.
#include <algorithm>

#include "common.cuh"
#include "conv_gemm.cuh"
#include "kernels.cuh"
#include "prof.h"
#include "runtime.h"
#include "tma.cuh"

namespace adainf {

namespace {

constexpr int CP_POS = 136;          // window positions per row (c0-1 .. c0+134); 136 x 32 B = 17 swizzle atoms
constexpr int CP_ROW = CP_POS * 32;  // bytes of one plane row
constexpr int CP_SMEM_MAX = 225 * 1024;

// TMEM accumulator buffers = epilogue groups of 4 warps (group g finishes items it = g, g + NB, ...): the
// epilogue is a dependent chain per item (tcgen05.ld, bias, act, round, max, store), so items overlap across
// groups, not within one
template <int N, bool S2D>
constexpr int c3p_nbuf() {
  return (512 / (2 * N)) >= 4 ? 4 : 512 / (2 * N);
}
template <int N, bool S2D>
constexpr int c3p_threads() { return 64 + 128 * c3p_nbuf<N, S2D>(); }

template <int P, int N, bool S2D>
constexpr int c3p_wbytes() { return 9 * P * 2 * N * 16; }
template <int P, bool S2D>
constexpr int c3p_stage() { return P * 4 * CP_ROW; }
// window stages: as many as fit next to the resident weights (at most 12).  An item's MMAs take ~0.2-0.5 us and a
// window load ~1-2 us of latency, so the ring has to cover several items (measured: 4 stages left the first layer
// at 0.71 ms, TMA-latency bound)
template <int P, int N, bool S2D>
constexpr int c3p_stages() {
  return (CP_SMEM_MAX - 2048 - c3p_wbytes<P, N, S2D>()) / c3p_stage<P, S2D>() >= 12
             ? 12
             : (CP_SMEM_MAX - 2048 - c3p_wbytes<P, N, S2D>()) / c3p_stage<P, S2D>();
}

struct C3PArgs {
  CUtensorMap x_map;  // input [n][H][W][Cin] (S2D: [n][H][W][16] packed), box {16, 136, RIN, 1}, SWIZZLE_32B
  const bf16* wexp;   // [9][P][2][N][8] bf16 (no-swizzle K-major core matrices per (tap, plane))
  const float* bias;  // [Cout]
  const int* count;
  int n_static, H, W, Cout, act;
  int tiles;          // 128-column tiles per row
  bf16* y;            // pooled [n][H/2][W/2][Cout] (S2D: [n][H][W][Cout])
};

template <int P, int N, bool S2D>
__global__ void __launch_bounds__(c3p_threads<N, S2D>(), 1) conv3_pool_kernel(const __grid_constant__ C3PArgs a) {
  constexpr int RIN = 4;                     // window rows
  constexpr int NACC = 2;                    // accumulators per item: two output rows (S2D: of the s2d grid)
  constexpr int ACC_COLS = NACC * N;         // TMEM columns per item
  constexpr int NB = c3p_nbuf<N, S2D>();     // accumulator buffers = epilogue groups
  constexpr int TCOLS = NB * ACC_COLS <= 64 ? 64 : (NB * ACC_COLS <= 128 ? 128 : (NB * ACC_COLS <= 256 ? 256 : 512));
  constexpr int PLANE = RIN * CP_ROW;
  constexpr int STAGE = P * PLANE;
  constexpr int WBYTES = c3p_wbytes<P, N, S2D>();
  constexpr int CP_STAGES = c3p_stages<P, N, S2D>();
  static_assert(CP_STAGES >= 2, "conv3_pool: window stages do not fit");
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = smem_align1024(smem_raw);
  uint8_t* stages = smem;
  uint8_t* wsm = stages + CP_STAGES * STAGE;
  uint64_t* full = (uint64_t*)(wsm + WBYTES);
  uint64_t* empty = full + CP_STAGES;
  uint64_t* tfull = empty + CP_STAGES;
  uint64_t* tempty = tfull + NB;
  uint32_t* tmem_slot = (uint32_t*)(tempty + NB);
  float* s_bias = (float*)(tmem_slot + 4);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int nimg = a.count ? min(*a.count, a.n_static) : a.n_static;
  const int rows_out = (a.H + 1) / 2;  // items per tile column: row pairs
  const long long nitems = (long long)nimg * rows_out * a.tiles;
  if ((long long)blockIdx.x >= nitems) return;

  for (int i = threadIdx.x; i < WBYTES / 16; i += blockDim.x) ((uint4*)wsm)[i] = __ldg((const uint4*)a.wexp + i);
  for (int i = threadIdx.x; i < a.Cout; i += blockDim.x) s_bias[i] = a.bias[i];
  if (threadIdx.x == 0) {
    for (int s = 0; s < CP_STAGES; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], 1);
    }
    for (int b = 0; b < NB; ++b) {
      mbar_init(&tfull[b], 1);
      mbar_init(&tempty[b], 128);
    }
    fence_mbar_init();
    tma_prefetch_desc(&a.x_map);
  }
  if (warp == 1) tmem_alloc<TCOLS>(tmem_slot);
  fence_proxy_async_smem();
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  const uint32_t st_base = smem_u32(stages);

  if (warp == 0) {
    if (lane == 0) {
      int it = 0;
      for (long long u = blockIdx.x; u < nitems; u += gridDim.x, ++it) {
        const int tcol = (int)(u % a.tiles);
        const long long r = u / a.tiles;
        const int ro = (int)(r % rows_out), n = (int)(r / rows_out);
        const int s = it % CP_STAGES, ph = it / CP_STAGES;
        if (ph > 0) mbar_wait(&empty[s], (ph - 1) & 1);
        mbar_expect_tx(&full[s], STAGE);
        const int r_in0 = 2 * ro - 1;
#pragma unroll
        for (int p = 0; p < P; ++p)
          tma_load_4d(st_base + s * STAGE + p * PLANE, &a.x_map, &full[s], 16 * p, tcol * 128 - 1, r_in0, n);
      }
    }
  } else if (warp == 1) {
    constexpr uint32_t IDESC = make_idesc(128, N, 0, 0);
    const uint64_t bdesc0 = make_sdesc_plain(smem_u32(wsm), N * 16, 128);
    int it = 0;
    for (long long u = blockIdx.x; u < nitems; u += gridDim.x, ++it) {
      const int b = it % NB, ub = it / NB;
      if (ub > 0) mbar_wait(&tempty[b], (ub - 1) & 1);
      const int s = it % CP_STAGES, ph = it / CP_STAGES;
      mbar_wait(&full[s], ph & 1);
      tc_fence_after();
      if (elect_one()) {
        const uint64_t adesc0 = make_sdesc_sw32(st_base + s * STAGE, 16, 256);
#pragma unroll
        for (int acc = 0; acc < NACC; ++acc) {
#pragma unroll
          for (int t = 0; t < 9; ++t) {
#pragma unroll
            for (int p = 0; p < P; ++p) {
              // window row (acc + dy), position dx: (acc + t/3) * CP_POS + t%3 32-byte rows past the plane base
              const uint32_t a_off = (uint32_t)(p * PLANE + ((acc + t / 3) * CP_POS + t % 3) * 32);
              const uint32_t b_off = (uint32_t)((t * P + p) * 2 * N * 16);
              umma_bf16(tmem + (uint32_t)(b * ACC_COLS + acc * N), adesc0 + (uint64_t)(a_off >> 4),
                        bdesc0 + (uint64_t)(b_off >> 4), IDESC, (t | p) != 0);
            }
          }
        }
        umma_commit(&empty[s]);
        umma_commit(&tfull[b]);
      }
      __syncwarp();
    }
  } else {
    const int grp = (warp - 2) >> 2;  // epilogue group = TMEM buffer
    const int qd = warp & 3;
    const int x = qd * 32 + lane;  // output column within the tile (TMEM lane)
    const uint32_t lane_base = (uint32_t)(qd * 32) << 16;
    const int Hp = S2D ? a.H : a.H / 2, Wp = S2D ? a.W : a.W / 2;
    const int act = a.act;
    // bias + act + bf16 rounding of two fp32 accumulators into one bf16x2 (the oracle's storage point)
    auto rnd2 = [act](float u, float v, float bu, float bv) -> __nv_bfloat162 {
      return __floats2bfloat162_rn(act_apply(act, __fadd_rn(u, bu)), act_apply(act, __fadd_rn(v, bv)));
    };
    int it = grp, ub = 0;
    for (long long u = blockIdx.x + (long long)grp * gridDim.x; u < nitems; u += (long long)NB * gridDim.x, it += NB, ++ub) {
      const int tcol = (int)(u % a.tiles);
      const long long r = u / a.tiles;
      const int ro = (int)(r % rows_out), n = (int)(r / rows_out);
      const int col = tcol * 128 + x;
      const int b = grp;
      mbar_wait(&tfull[b], ub & 1);
      tc_fence_after();
      const uint32_t acc0 = tmem + (uint32_t)(b * ACC_COLS) + lane_base;
      // max-pool first: bias, act and bf16 rounding are all non-decreasing, so max_s bf16(act(v_s + b)) ==
      // bf16(act(max_s v_s + b)) exactly -- one epilogue per pooled value instead of four
      if constexpr (S2D) {
        // N = 4 sub-pixels x CO: pooled channel c = bf16(act(max_s acc[s*CO + c] + b[c])), rows 2ro and 2ro + 1
        constexpr int CO = N / 4;
        float mx[2][CO];
#pragma unroll
        for (int acc = 0; acc < 2; ++acc)
#pragma unroll
          for (int ch = 0; ch < N / 32; ++ch) {
            float v[32];
            tmem_ld32(acc0 + (uint32_t)(acc * N + ch * 32), v);
#pragma unroll
            for (int i = 0; i < 32; ++i) {
              const int c = (ch * 32 + i) % CO, sub = (ch * 32 + i) / CO;
              mx[acc][c] = sub == 0 ? v[i] : fmaxf(mx[acc][c], v[i]);
            }
          }
        tc_fence_before();
        mbar_arrive(&tempty[b]);
#pragma unroll
        for (int acc = 0; acc < 2; ++acc) {
          const int row = 2 * ro + acc;
          if (col < a.W && row < a.H) {
            __align__(16) __nv_bfloat162 y[CO / 2];
#pragma unroll
            for (int c = 0; c < CO; c += 2) y[c / 2] = rnd2(mx[acc][c], mx[acc][c + 1], s_bias[c], s_bias[c + 1]);
            uint4* o = (uint4*)(a.y + (((long long)n * Hp + row) * Wp + col) * CO);
#pragma unroll
            for (int c = 0; c < CO / 8; ++c) o[c] = ((const uint4*)y)[c];
          }
        }
      } else {
        // rows 2ro and 2ro+1: vertical max in the thread, horizontal max with lane x^1, even lanes finish + store
#pragma unroll
        for (int ch = 0; ch < N / 32; ++ch) {
          float v0[32], v1[32];
          tmem_ld32(acc0 + (uint32_t)(ch * 32), v0);
          tmem_ld32(acc0 + (uint32_t)(N + ch * 32), v1);
          if (ch == N / 32 - 1) {
            tc_fence_before();
            mbar_arrive(&tempty[b]);
          }
#pragma unroll
          for (int i = 0; i < 32; ++i) {
            const float m = fmaxf(v0[i], v1[i]);
            v0[i] = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, 1));
          }
          if (!(x & 1) && col < a.W) {
            __align__(16) __nv_bfloat162 y[16];
#pragma unroll
            for (int i = 0; i < 32; i += 2) y[i / 2] = rnd2(v0[i], v0[i + 1], s_bias[ch * 32 + i], s_bias[ch * 32 + i + 1]);
            uint4* o = (uint4*)(a.y + (((long long)n * Hp + ro) * Wp + col / 2) * a.Cout + ch * 32);
#pragma unroll
            for (int c = 0; c < 4; ++c) o[c] = ((const uint4*)y)[c];
          }
        }
      }
    }
  }

  tc_fence_before();
  __syncthreads();
  if (warp == 1) {
    tc_fence_after();
    tmem_dealloc<TCOLS>(tmem);
  }
}

template <int P, int N, bool S2D>
constexpr int c3p_smem() {
  return 1024 + c3p_stages<P, N, S2D>() * c3p_stage<P, S2D>() + c3p_wbytes<P, N, S2D>() + 1024;
}

// shadow [Cout][ldb] (K = tap * Cin + c) -> wexp [9][P][2][N][8]
__global__ void c3p_wprep_rows_kernel(const bf16* __restrict__ shadow, int ldb, int Cin, int Cout,
                                      bf16* __restrict__ w) {
  const int P = Cin / 16;
  const int total = 9 * P * 2 * Cout * 8;
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < total; i += gridDim.x * blockDim.x) {
    const int j = i & 7;
    int r = i >> 3;
    const int co = r % Cout;
    r /= Cout;
    const int q = r & 1, tp = r >> 1;
    const int p = tp % P, t = tp / P;
    w[i] = shadow[(long long)co * ldb + t * Cin + p * 16 + q * 8 + j];
  }
}
// first layer on the s2d grid: s2d tap (ah, aw) in -1..1, s2d channel ch = (bh*2 + bw)*4 + c, output column
// j = (oh*2 + ow) * Cout + co; original tap kh = 2ah + bh - oh + 1, kw = 2aw + bw - ow + 1 (zero outside 0..2 or
// for c >= cin_real); shadow K = (kh*3 + kw) * cin_pad + c
__global__ void c3p_wprep_s2d_kernel(const bf16* __restrict__ shadow, int ldb, int cin_real, int cin_pad, int Cout,
                                     bf16* __restrict__ w) {
  const int N = 4 * Cout;
  const int total = 9 * 2 * N * 8;
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < total; i += gridDim.x * blockDim.x) {
    const int jj = i & 7;
    int r = i >> 3;
    const int jcol = r % N;
    r /= N;
    const int q = r & 1, t = r >> 1;
    const int ah = t / 3 - 1, aw = t % 3 - 1;
    const int ch = q * 8 + jj;
    const int bh = ch >> 3, bw = (ch >> 2) & 1, c = ch & 3;
    const int sub = jcol / Cout, co = jcol % Cout;
    const int oh = sub >> 1, ow = sub & 1;
    const int kh = 2 * ah + bh - oh + 1, kw = 2 * aw + bw - ow + 1;
    bf16 v = __float2bfloat16_rn(0.f);
    if (kh >= 0 && kh < 3 && kw >= 0 && kw < 3 && c < cin_real) v = shadow[(long long)co * ldb + (kh * 3 + kw) * cin_pad + c];
    w[i] = v;
  }
}

template <int P, int N, bool S2D>
void launch_c3p(const C3PArgs& a, long long nitems, cudaStream_t st) {
  constexpr int smem = c3p_smem<P, N, S2D>();
  static bool attr = false;
  if (!attr) {
    CK(cudaFuncSetAttribute(conv3_pool_kernel<P, N, S2D>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
    attr = true;
  }
  const int grid = (int)std::min<long long>(nitems, num_sms());
  conv3_pool_kernel<P, N, S2D><<<grid, c3p_threads<N, S2D>(), smem, st>>>(a);
}

}  // namespace

bool conv3_pool_ok(const ConvGeom& g, bool first, int cin_real, int pk, int ps, int pp) {
  if (g.KH != 3 || g.KW != 3 || g.stride != 1 || g.pad != 1 || pk != 2 || ps != 2 || pp != 0) return false;
  if (g.H % 2 || g.W % 2 || g.H < 2 || g.W < 2) return false;
  if (first) return cin_real <= 4 && g.Cin == 4 && (g.Cout == 16 || g.Cout == 32);
  return (g.Cin == 16 || g.Cin == 32) && (g.Cout == 32 || g.Cout == 64 || g.Cout == 96 || g.Cout == 128);
}

size_t conv3_pool_wexp_bytes(const ConvGeom& g, bool first) {
  return first ? (size_t)9 * 2 * 4 * g.Cout * 8 * 2 : (size_t)9 * (g.Cin / 16) * 2 * g.Cout * 8 * 2;
}

void conv3_pool(const ConvGeom& g, bool first, const bf16* x, const int* count, int n_static, const bf16* shadow,
                int ldb, int cin_real, const float* bias, int act, bf16* wexp, bf16* y, cudaStream_t st) {
  if (n_static <= 0) return;
  thread_local C3PArgs a;
  a = C3PArgs{};
  a.wexp = wexp;
  a.bias = bias;
  a.count = count;
  a.n_static = n_static;
  a.Cout = g.Cout;
  a.act = act;
  ProfScope ps(PC_CONV_FWD, st, 2);
  if (first) {
    // s2d grid: H/2 x W/2 positions of 16 channels
    const int Hs = g.H / 2, Ws = g.W / 2;
    a.x_map = make_tmap_nhwc_swz(x, n_static, Hs, Ws, 16, 16, CP_POS, 4, 32);
    a.H = Hs;
    a.W = Ws;
    a.tiles = (Ws + 127) / 128;
    a.y = y;
    c3p_wprep_s2d_kernel<<<64, 256, 0, st>>>(shadow, ldb, cin_real, g.Cin, g.Cout, wexp);
    const long long nitems = (long long)n_static * ((Hs + 1) / 2) * a.tiles;
    if (g.Cout == 16) launch_c3p<1, 64, true>(a, nitems, st);
    else launch_c3p<1, 128, true>(a, nitems, st);
  } else {
    a.x_map = make_tmap_nhwc_swz(x, n_static, g.H, g.W, g.Cin, 16, CP_POS, 4, 32);
    a.H = g.H;
    a.W = g.W;
    a.tiles = (g.W + 127) / 128;
    a.y = y;
    c3p_wprep_rows_kernel<<<64, 256, 0, st>>>(shadow, ldb, g.Cin, g.Cout, wexp);
    const long long nitems = (long long)n_static * (g.H / 2) * a.tiles;
    const int P = g.Cin / 16;
#define C3P_CASE(PP, NN) \
  if (P == PP && g.Cout == NN) { launch_c3p<PP, NN, false>(a, nitems, st); CK(cudaGetLastError()); return; }
    C3P_CASE(1, 32) C3P_CASE(1, 64) C3P_CASE(1, 96) C3P_CASE(1, 128)
    C3P_CASE(2, 32) C3P_CASE(2, 64) C3P_CASE(2, 96) C3P_CASE(2, 128)
#undef C3P_CASE
    throw ShapeError("conv3_pool: unsupported channels");
  }
  CK(cudaGetLastError());
}

}  // namespace adainf

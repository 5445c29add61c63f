// Window implicit GEMM for stride-1, pad-1, 3x3 convolutions (FWD and DGRAD), tcgen05 + TMEM.
//
// Output positions are enumerated on a "padded flattened" grid: per image (H+1) rows x (W+1) columns,
// q = (n*(H+1) + h)*(W+1) + w, where row h = H and column w = W are zero padding (their outputs are
// computed and discarded).  With this enumeration every tap (dy, dx) of a 3x3 stencil is a CONSTANT
// shift of q: source q' = q + dy*(W+1) + dx.  A 128-row output tile therefore needs one window of
// L = 128 + 2*(W+1) + 2 source rows per 64-channel block, loaded ONCE, and the A operand of each of the
// 9 taps is the same window viewed at a row offset (UMMA descriptor start + 128 B * offset, with the
// 128B-swizzle phase carried in the descriptor's base-offset field).  This cuts the im2col re-reads of
// the generic gather (9x per input row) to ~(1 + 2(W+1)/128)x.
//
//   FWD   D[q][co] = sum_{cb,tap} Win_cb[q + off(tap)][c] * W[co][tap][cb*64+c]     B K-major
//   DGRAD D[q][ci] = sum_{cb,tap} Win_cb[q + off(tap)][co] * W[cb*64+co][tap][ci]  B MN-major (flipped taps)
//
// Warp roles as in conv_gemm.cuh: 4 producer warps (cp.async), 1 MMA warp, 4 epilogue warps; persistent
// CTAs over tiles; double-buffered TMEM accumulators.
#pragma once
#include "conv_gemm.cuh"

namespace adainf {

struct WinArgs {
  ConvArgs c;        // src/src_map/Hs/Ws/Cs, count/n_static, B/ldb/Nout, epilogue fields (Ho=Hs, Wo=Ws)
  int dgrad;
  int tap_off[9];    // window row offset of each tap: (dy+1)*(W+1) + (dx+1)
  int btap[9];       // forward tap index feeding B (DGRAD: flipped)
  int base_off;      // 1: carry the start row's swizzle phase in the descriptor base-offset field
};

constexpr int WIN_MAX_L = 128 + 2 * 57 + 2;  // W <= 56

template <int BN>
struct WinCfg {
  static constexpr int WIN_BYTES = ((WIN_MAX_L + 7) / 8) * 1024;  // rows padded to whole 1024-B atoms
  static constexpr int WSTAGES = 2;
  static constexpr int B_BYTES = BN * 64 * 2;
  static constexpr int BSTAGES = (196 * 1024 - WSTAGES * WIN_BYTES) / B_BYTES > 8
                                     ? 8
                                     : (196 * 1024 - WSTAGES * WIN_BYTES) / B_BYTES;
  static constexpr int SMEM = WSTAGES * WIN_BYTES + BSTAGES * B_BYTES + 1024 + 512;
  static constexpr int ACC_COLS = BN;
  static constexpr int TMEM_COLS = 2 * BN;
};

// descriptor for a K-major SW128 operand whose first row sits `row` rows into a 1024-B aligned region
__device__ __forceinline__ uint64_t make_sdesc_rows(uint32_t region, int row, int kk, int base_off) {
  const uint32_t addr = region + (uint32_t)row * 128u + (uint32_t)kk * 32u;
  uint64_t d = make_sdesc(addr, 16, 1024);
  if (base_off) d |= (uint64_t)((addr >> 7) & 7u) << 49;  // swizzle phase of the start row (base offset)
  return d;
}

template <int BN>
__global__ void __launch_bounds__(NUM_THREADS, 1) conv_win_kernel(const WinArgs w) {
  using Cfg = WinCfg<BN>;
  const ConvArgs& a = w.c;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = smem_align1024(smem_raw);
  uint8_t* win_base = smem;
  uint8_t* b_base = smem + Cfg::WSTAGES * Cfg::WIN_BYTES;
  uint64_t* bars = (uint64_t*)(b_base + Cfg::BSTAGES * Cfg::B_BYTES);
  uint64_t* wfull = bars;                       // [WSTAGES]
  uint64_t* wempty = wfull + Cfg::WSTAGES;      // [WSTAGES]
  uint64_t* bfull = wempty + Cfg::WSTAGES;      // [BSTAGES]
  uint64_t* bempty = bfull + Cfg::BSTAGES;      // [BSTAGES]
  uint64_t* tfull = bempty + Cfg::BSTAGES;      // [2]
  uint64_t* tempty = tfull + 2;                 // [2]
  uint32_t* tmem_slot = (uint32_t*)(tempty + 2);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int H = a.Hs, W = a.Ws, Wp = W + 1, Hp = H + 1;
  const int nsamp = a.count ? *a.count : a.n_static;
  const long long Qimg = (long long)Hp * Wp;
  const long long Q = (long long)nsamp * Qimg;
  const int nt = (a.Nout + BN - 1) / BN;
  const int mt = (int)((Q + BM - 1) / BM);
  const int ntile = mt * nt;
  const int ncb = a.Cs / 64;
  const int L = BM + 2 * Wp + 2;
  if ((int)blockIdx.x >= ntile) return;

  if (threadIdx.x == 0) {
    for (int s = 0; s < Cfg::WSTAGES; ++s) {
      mbar_init(&wfull[s], 128);
      mbar_init(&wempty[s], 1);
    }
    for (int s = 0; s < Cfg::BSTAGES; ++s) {
      mbar_init(&bfull[s], 128);
      mbar_init(&bempty[s], 1);
    }
    for (int b = 0; b < 2; ++b) {
      mbar_init(&tfull[b], 1);
      mbar_init(&tempty[b], 128);
    }
    fence_mbar_init();
  }
  if (warp == 4) tmem_alloc<Cfg::TMEM_COLS>(tmem_slot);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  const uint32_t wsm = smem_u32(win_base), bsm = smem_u32(b_base);

  if (warp < 4) {
    // ================= producers =================
    const int t = threadIdx.x;
    const int j = t & 7;
    int wit = 0, bit = 0;
    for (int tile = blockIdx.x; tile < ntile; tile += gridDim.x) {
      const int n0 = (tile % nt) * BN;
      const long long q0 = (long long)(tile / nt) * BM;
      // decode this thread's window rows once per tile (same for every channel block)
      constexpr int RPT = (WIN_MAX_L + 15) / 16;
      int rb[RPT];  // source pixel index (n*H + h)*W + x, or -1 for zero rows
#pragma unroll
      for (int i = 0; i < RPT; ++i) {
        const int r = (t >> 3) + 16 * i;
        const long long qs = q0 - Wp - 1 + r;
        rb[i] = -1;
        if (r < L && qs >= 0 && qs < Q) {
          const int qi = (int)qs;
          const int n = qi / (int)Qimg;
          const int rem = qi - n * (int)Qimg;
          const int h = rem / Wp, x = rem - h * Wp;
          if (h < H && x < W) {
            const int sn = a.src_map ? __ldg(a.src_map + n) : n;
            rb[i] = (sn * H + h) * W + x;
          }
        }
      }
      for (int cb = 0; cb < ncb; ++cb) {
        // ---- window rows [q0 - Wp - 1, q0 - Wp - 1 + L) of channel block cb ----
        {
          const int s = wit % Cfg::WSTAGES, u = wit / Cfg::WSTAGES;
          if (u > 0) mbar_wait(&wempty[s], (u - 1) & 1);
          const uint32_t sw = wsm + s * Cfg::WIN_BYTES;
#pragma unroll
          for (int i = 0; i < RPT; ++i) {
            const int r = (t >> 3) + 16 * i;
            if (r < L) {
              const bool v = rb[i] >= 0;
              cp_async16(sw + kmaj_off(r, j), v ? a.src + ((long long)rb[i] * a.Cs + cb * 64 + j * 8) : a.src, v);
            }
          }
          cp_async_arrive_noinc(&wfull[s]);
          ++wit;
        }
        // ---- 9 B tiles (one per tap) ----
        for (int tp = 0; tp < 9; ++tp) {
          const int s = bit % Cfg::BSTAGES, u = bit / Cfg::BSTAGES;
          if (u > 0) mbar_wait(&bempty[s], (u - 1) & 1);
          const uint32_t sb = bsm + s * Cfg::B_BYTES;
          if (!w.dgrad) {
            // W [Nout][9*Cs] K-major: rows co, 64 columns of tap tp, channel block cb
#pragma unroll
            const bf16* wb = a.B + (long long)w.btap[tp] * a.Cs + cb * 64;
            for (int idx = t; idx < BN * 8; idx += 128) {
              const int r = idx >> 3, jj = idx & 7;
              const bool v = (n0 + r) < a.Nout;
              const bf16* g = v ? wb + ((long long)(n0 + r) * a.ldb + jj * 8) : a.B;
              cp_async16(sb + kmaj_off(r, jj), g, v);
            }
          } else {
            // DGRAD: B MN-major [64 co rows][BN ci] = W[cb*64 + r][btap][n0 + ci]
            constexpr int CH = BN / 8;
            const bf16* wb = a.B + (long long)(cb * 64) * a.ldb + (long long)w.btap[tp] * a.Nout + n0;
#pragma unroll
            for (int idx = t; idx < 64 * CH; idx += 128) {
              const int r = idx / CH, jj = idx % CH;
              const bool v = (n0 + jj * 8) < a.Nout;
              const bf16* g = v ? wb + (long long)r * a.ldb + jj * 8 : a.B;
              cp_async16(sb + mnmaj_off(r, jj), g, v);
            }
          }
          cp_async_arrive_noinc(&bfull[s]);
          ++bit;
        }
      }
    }
  } else if (warp == 4) {
    // ================= MMA issuer =================
    const uint32_t IDESC = make_idesc(BM, BN, 0, w.dgrad ? 1 : 0);
    int wit = 0, bit = 0, lt = 0;
    for (int tile = blockIdx.x; tile < ntile; tile += gridDim.x, ++lt) {
      const int b = lt & 1, ub = lt >> 1;
      if (ub > 0) mbar_wait(&tempty[b], (ub - 1) & 1);
      tc_fence_after();
      const uint32_t dacc = tmem + (uint32_t)(b * Cfg::ACC_COLS);
      for (int cb = 0; cb < ncb; ++cb) {
        const int ws = wit % Cfg::WSTAGES, wu = wit / Cfg::WSTAGES;
        mbar_wait(&wfull[ws], wu & 1);
        const uint32_t sw = wsm + ws * Cfg::WIN_BYTES;
        for (int tp = 0; tp < 9; ++tp) {
          const int s = bit % Cfg::BSTAGES, u = bit / Cfg::BSTAGES;
          mbar_wait(&bfull[s], u & 1);
          fence_proxy_async_smem();
          tc_fence_after();
          if (elect_one()) {
            const uint32_t sb = bsm + s * Cfg::B_BYTES;
#pragma unroll
            for (int kk = 0; kk < 4; ++kk) {
              const uint64_t ad = make_sdesc_rows(sw, w.tap_off[tp], kk, w.base_off);
              const uint64_t bd = w.dgrad ? make_sdesc(sb + kk * 2048, 8192, 1024) : make_sdesc(sb + kk * 32, 16, 1024);
              umma_bf16(dacc, ad, bd, IDESC, (cb | tp | kk) != 0);
            }
            umma_commit(&bempty[s]);
            if (tp == 8) {
              umma_commit(&wempty[ws]);
              if (cb == ncb - 1) umma_commit(&tfull[b]);
            }
          }
          __syncwarp();
          ++bit;
        }
        ++wit;
      }
    }
  } else {
    // ================= epilogue =================
    const int qd = warp & 3;
    const int row = qd * 32 + lane;
    int lt = 0;
    for (int tile = blockIdx.x; tile < ntile; tile += gridDim.x, ++lt) {
      const int n0 = (tile % nt) * BN;
      const long long q = (long long)(tile / nt) * BM + row;
      const int b = lt & 1, ub = lt >> 1;
      mbar_wait(&tfull[b], ub & 1);
      tc_fence_after();
      const uint32_t trow = tmem + (uint32_t)(b * Cfg::ACC_COLS) + ((uint32_t)(qd * 32) << 16);
      bool rv = q < Q;
      int n = 0, h = 0, x = 0;
      if (rv) {
        n = (int)(q / Qimg);
        const int rem = (int)(q - (long long)n * Qimg);
        h = rem / Wp;
        x = rem - h * Wp;
        rv = h < H && x < W;
      }
      const long long orow = ((long long)n * H + h) * W + x;
      long long rrow = orow;
      if (!w.dgrad && a.res && rv) rrow = ((long long)(a.res_map ? __ldg(a.res_map + n) : n) * H + h) * W + x;
#pragma unroll 1
      for (int c0 = 0; c0 < BN; c0 += 32) {
        float v[32];
        tmem_ld32(trow + c0, v);
        if (c0 + 32 >= BN) {
          tc_fence_before();
          mbar_arrive(&tempty[b]);
        }
        const int cbase = n0 + c0;
        if (!rv || cbase >= a.Nout) continue;
        // Nout is a multiple of 64 on this path: full 32-column vectors
        if (!w.dgrad) {
#pragma unroll
          for (int i = 0; i < 32; ++i) v[i] = __fadd_rn(v[i], __ldg(a.bias + cbase + i));
          if (a.res) {
#pragma unroll
            for (int i = 0; i < 32; i += 8) {
              float r8[8];
              ld_bf16x8(a.res + rrow * a.Nout + cbase + i, r8);
#pragma unroll
              for (int qq = 0; qq < 8; ++qq) v[i + qq] = __fadd_rn(v[i + qq], r8[qq]);
            }
          }
#pragma unroll
          for (int i = 0; i < 32; ++i) v[i] = act_apply(a.act, v[i]);
        } else {
          if (a.bcast) {
#pragma unroll
            for (int i = 0; i < 32; i += 4) {
              const float4 bb = __ldg((const float4*)(a.bcast + (long long)n * a.Nout + cbase + i));
              v[i] = __fadd_rn(v[i], bb.x);
              v[i + 1] = __fadd_rn(v[i + 1], bb.y);
              v[i + 2] = __fadd_rn(v[i + 2], bb.z);
              v[i + 3] = __fadd_rn(v[i + 3], bb.w);
            }
          }
          if (a.sc) {
#pragma unroll
            for (int i = 0; i < 32; i += 8) {
              float r8[8];
              ld_bf16x8(a.sc + orow * a.Nout + cbase + i, r8);
#pragma unroll
              for (int qq = 0; qq < 8; ++qq) v[i + qq] = __fadd_rn(v[i + qq], r8[qq]);
            }
          }
          if (a.mask_act) {
#pragma unroll
            for (int i = 0; i < 32; i += 8) {
              float y8[8];
              ld_bf16x8(a.yact + orow * a.Nout + cbase + i, y8);
#pragma unroll
              for (int qq = 0; qq < 8; ++qq) v[i + qq] = __fmul_rn(v[i + qq], act_grad(a.mask_act, y8[qq]));
            }
          }
        }
        bf16* o = (bf16*)a.out + orow * a.Nout + cbase;
#pragma unroll
        for (int i = 0; i < 32; i += 8) st_bf16x8(o + i, v + i);
      }
    }
  }

  tc_fence_before();
  __syncthreads();
  if (warp == 4) {
    tc_fence_after();
    tmem_dealloc<Cfg::TMEM_COLS>(tmem);
  }
}

}  // namespace adainf

namespace adainf {

// ------------------------------------------------------------------------------------------------
// Weight-stationary variant for 64-channel 3x3 layers (ResNet layer1: Cin = Cout = 64): all 9 tap tiles
// of B (9 x 64 x 64 bf16 = 72 KB) are loaded into shared memory ONCE per persistent CTA, so the only
// per-tile traffic is the input window (~31 KB at 56x56) instead of 9 im2col A tiles + 9 B tiles
// (216 KB) in the gather kernel.
struct WinWsCfg {
  static constexpr int WIN_BYTES = ((WIN_MAX_L + 7) / 8) * 1024;
  static constexpr int WSTAGES = 2;
  static constexpr int B_BYTES = 64 * 64 * 2;
  static constexpr int STAGE_E = 2 * 128 * 256;  // epilogue staging: 2 groups x 128 rows x (2 x 128 B)
  static constexpr int SMEM = WSTAGES * WIN_BYTES + 9 * B_BYTES + STAGE_E + 1024 + 512;
  static constexpr int ACC_COLS = 64;
  static constexpr int TMEM_COLS = 128;
};

constexpr int WS_THREADS = 416;  // 4 producer warps, 1 MMA warp, 2 x 4 epilogue warps (alternate tiles)

__global__ void __launch_bounds__(WS_THREADS, 1) conv_win_ws_kernel(const WinArgs w) {
  using Cfg = WinWsCfg;
  const ConvArgs& a = w.c;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = smem_align1024(smem_raw);
  uint8_t* win_base = smem;
  uint8_t* b_base = smem + Cfg::WSTAGES * Cfg::WIN_BYTES;
  uint8_t* e_base = b_base + 9 * Cfg::B_BYTES;
  uint64_t* bars = (uint64_t*)(e_base + Cfg::STAGE_E);
  uint64_t* wfull = bars;
  uint64_t* wempty = wfull + Cfg::WSTAGES;
  uint64_t* bready = wempty + Cfg::WSTAGES;
  uint64_t* tfull = bready + 1;
  uint64_t* tempty = tfull + 2;
  uint32_t* tmem_slot = (uint32_t*)(tempty + 2);
  float* s_bias = (float*)(tmem_slot + 4);  // 64 floats (FWD bias, staged once per CTA)

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int H = a.Hs, W = a.Ws, Wp = W + 1, Hp = H + 1;
  const int nsamp = a.count ? *a.count : a.n_static;
  const int Qimg = Hp * Wp;
  const long long Q = (long long)nsamp * Qimg;
  const int ntile = (int)((Q + BM - 1) / BM);
  const int L = BM + 2 * Wp + 2;
  if ((int)blockIdx.x >= ntile) return;
  if (threadIdx.x < 64) s_bias[threadIdx.x] = (!w.dgrad && a.bias) ? a.bias[threadIdx.x] : 0.f;

  if (threadIdx.x == 0) {
    for (int s = 0; s < Cfg::WSTAGES; ++s) {
      mbar_init(&wfull[s], 128);
      mbar_init(&wempty[s], 1);
    }
    mbar_init(bready, 128);
    for (int b = 0; b < 2; ++b) {
      mbar_init(&tfull[b], 1);
      mbar_init(&tempty[b], 128);
    }
    fence_mbar_init();
  }
  if (warp == 4) tmem_alloc<Cfg::TMEM_COLS>(tmem_slot);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  const uint32_t wsm = smem_u32(win_base), bsm = smem_u32(b_base);

  if (warp < 4) {
    const int t = threadIdx.x;
    const int j = t & 7;
    // ---- resident B: 9 tap tiles ----
    for (int tp = 0; tp < 9; ++tp) {
      const uint32_t sb = bsm + tp * Cfg::B_BYTES;
      if (!w.dgrad) {
        const bf16* wb = a.B + (long long)w.btap[tp] * 64;
#pragma unroll
        for (int idx = t; idx < 64 * 8; idx += 128) {
          const int r = idx >> 3, jj = idx & 7;
          cp_async16(sb + kmaj_off(r, jj), wb + (long long)r * a.ldb + jj * 8, true);
        }
      } else {
        const bf16* wb = a.B + (long long)w.btap[tp] * 64;
#pragma unroll
        for (int idx = t; idx < 64 * 8; idx += 128) {
          const int r = idx >> 3, jj = idx & 7;
          cp_async16(sb + mnmaj_off(r, jj), wb + (long long)r * a.ldb + jj * 8, true);
        }
      }
    }
    cp_async_arrive_noinc(bready);
    // ---- windows ----
    constexpr int RPT = (WIN_MAX_L + 15) / 16;
    int wit = 0;
    for (int tile = blockIdx.x; tile < ntile; tile += gridDim.x, ++wit) {
      const long long q0 = (long long)tile * BM;
      const int s = wit % Cfg::WSTAGES, u = wit / Cfg::WSTAGES;
      // decode the first row of this thread once, then step by 16 rows with carries
      long long qs = q0 - Wp - 1 + (t >> 3);
      int n = 0, h = 0, x = 0;
      if (qs >= 0) {
        n = (int)(qs / Qimg);
        const int rem = (int)(qs - (long long)n * Qimg);
        h = rem / Wp;
        x = rem - h * Wp;
      }
      if (u > 0) TIMED_WAIT(0, mbar_wait(&wempty[s], (u - 1) & 1));
      const uint32_t sw = wsm + s * Cfg::WIN_BYTES;
#ifdef ADAINF_TIMING
      const long long _ti0 = clock64();
#endif
#pragma unroll
      for (int i = 0; i < RPT; ++i) {
        const int r = (t >> 3) + 16 * i;
        if (r < L) {
          const bool v = qs >= 0 && qs < Q && h < H && x < W;
          const bf16* g = a.src;
          if (v) {
            const int sn = a.src_map ? __ldg(a.src_map + n) : n;
            g = a.src + ((long long)((sn * H + h) * W + x) * 64 + j * 8);
          }
          cp_async16(sw + kmaj_off(r, j), g, v);
        }
        // advance 16 rows
        qs += 16;
        if (qs >= 0) {
          if (qs < 16) {  // crossed from negative: decode afresh
            n = 0;
            h = (int)qs / Wp;
            x = (int)qs - h * Wp;
          } else {
            x += 16;
            while (x >= Wp) {  // Wp may be < 16 (small maps): possibly several carries
              x -= Wp;
              if (++h >= Hp) {
                h = 0;
                ++n;
              }
            }
          }
        }
      }
      cp_async_arrive_noinc(&wfull[s]);
#ifdef ADAINF_TIMING
      if ((threadIdx.x & 31) == 0) atomicAdd(&g_wait_cycles[blockIdx.x & 4095][4], (unsigned long long)(clock64() - _ti0));
#endif
    }
  } else if (warp == 4) {
    const uint32_t IDESC = make_idesc(BM, 64, 0, w.dgrad ? 1 : 0);
    mbar_wait(bready, 0);
    int wit = 0;
    for (int tile = blockIdx.x; tile < ntile; tile += gridDim.x, ++wit) {
      const int b = wit & 1, ub = wit >> 1;
      if (ub > 0) TIMED_WAIT(1, mbar_wait(&tempty[b], (ub - 1) & 1));
      tc_fence_after();
      const uint32_t dacc = tmem + (uint32_t)(b * Cfg::ACC_COLS);
      const int s = wit % Cfg::WSTAGES, u = wit / Cfg::WSTAGES;
      TIMED_WAIT(2, mbar_wait(&wfull[s], u & 1));
      fence_proxy_async_smem();
      tc_fence_after();
      if (elect_one()) {
        const uint32_t sw = wsm + s * Cfg::WIN_BYTES;
#pragma unroll 1
        for (int tp = 0; tp < 9; ++tp) {
          const uint32_t sb = bsm + tp * Cfg::B_BYTES;
#pragma unroll
          for (int kk = 0; kk < 4; ++kk) {
            const uint64_t ad = make_sdesc_rows(sw, w.tap_off[tp], kk, 0);
            const uint64_t bd = w.dgrad ? make_sdesc(sb + kk * 2048, 8192, 1024) : make_sdesc(sb + kk * 32, 16, 1024);
            umma_bf16(dacc, ad, bd, IDESC, (tp | kk) != 0);
          }
        }
        umma_commit(&wempty[s]);
        umma_commit(&tfull[b]);
      }
      __syncwarp();
    }
  } else {
    const int grp = (warp - 5) >> 2;  // 0: even local tiles (accumulator 0), 1: odd (accumulator 1)
    const int qd = warp & 3;
    const int row = qd * 32 + lane;
    int lt = grp;
    for (int tile = blockIdx.x + grp * gridDim.x; tile < ntile; tile += 2 * gridDim.x, lt += 2) {
      const long long q = (long long)tile * BM + row;
      const int b = grp, ub = lt >> 1;
      bool rv = q < Q;
      int n = 0, h = 0, x = 0;
      if (rv) {
        n = (int)(q / Qimg);
        const int rem = (int)(q - (long long)n * Qimg);
        h = rem / Wp;
        x = rem - h * Wp;
        rv = h < H && x < W;
      }
      const long long orow = ((long long)n * H + h) * W + x;
      long long rrow = orow;
      if (!w.dgrad && a.res && rv) rrow = ((long long)(a.res_map ? __ldg(a.res_map + n) : n) * H + h) * W + x;
      // stage this row's epilogue operands (residual / shortcut-gradient, stored activation) into shared
      // memory with cp.async before waiting for the accumulator (hides the global-load latency)
      const bf16* p0 = nullptr;
      const bf16* p1 = nullptr;
      if (rv) {
        if (!w.dgrad) p0 = a.res ? a.res + rrow * 64 : nullptr;
        else {
          p0 = a.sc ? a.sc + orow * 64 : nullptr;
          p1 = a.mask_act ? a.yact + orow * 64 : nullptr;
        }
      }
      const uint32_t est = smem_u32(e_base) + (uint32_t)((grp * 128 + row) * 256);
      if (p0)
#pragma unroll
        for (int i = 0; i < 8; ++i) cp_async16(est + i * 16, p0 + i * 8, true);
      if (p1)
#pragma unroll
        for (int i = 0; i < 8; ++i) cp_async16(est + 128 + i * 16, p1 + i * 8, true);
      asm volatile("cp.async.commit_group;" ::: "memory");
      TIMED_WAIT(3, mbar_wait(&tfull[b], ub & 1));
      tc_fence_after();
      const uint32_t trow = tmem + (uint32_t)(b * Cfg::ACC_COLS) + ((uint32_t)(qd * 32) << 16);
      float v[64];
      tmem_ld32(trow, v);
      tmem_ld32(trow + 32, v + 32);
      tc_fence_before();
      mbar_arrive(&tempty[b]);
      asm volatile("cp.async.wait_all;" ::: "memory");
      if (!rv) continue;
      const uint8_t* es = e_base + (grp * 128 + row) * 256;
      if (!w.dgrad) {
#pragma unroll
        for (int i = 0; i < 64; ++i) v[i] = __fadd_rn(v[i], s_bias[i]);
        if (p0) {
#pragma unroll
          for (int i = 0; i < 8; ++i) {
            const uint4 e = *(const uint4*)(es + i * 16);
            const bf16* hh = (const bf16*)&e;
#pragma unroll
            for (int qq = 0; qq < 8; ++qq) v[i * 8 + qq] = __fadd_rn(v[i * 8 + qq], __bfloat162float(hh[qq]));
          }
        }
#pragma unroll
        for (int i = 0; i < 64; ++i) v[i] = act_apply(a.act, v[i]);
      } else {
        if (a.bcast) {
#pragma unroll
          for (int i = 0; i < 64; i += 4) {
            const float4 bb = __ldg((const float4*)(a.bcast + (long long)n * 64 + i));
            v[i] = __fadd_rn(v[i], bb.x);
            v[i + 1] = __fadd_rn(v[i + 1], bb.y);
            v[i + 2] = __fadd_rn(v[i + 2], bb.z);
            v[i + 3] = __fadd_rn(v[i + 3], bb.w);
          }
        }
        if (p0) {
#pragma unroll
          for (int i = 0; i < 8; ++i) {
            const uint4 e = *(const uint4*)(es + i * 16);
            const bf16* hh = (const bf16*)&e;
#pragma unroll
            for (int qq = 0; qq < 8; ++qq) v[i * 8 + qq] = __fadd_rn(v[i * 8 + qq], __bfloat162float(hh[qq]));
          }
        }
        if (p1) {
#pragma unroll
          for (int i = 0; i < 8; ++i) {
            const uint4 e = *(const uint4*)(es + 128 + i * 16);
            const bf16* hh = (const bf16*)&e;
#pragma unroll
            for (int qq = 0; qq < 8; ++qq)
              v[i * 8 + qq] = __fmul_rn(v[i * 8 + qq], act_grad(a.mask_act, __bfloat162float(hh[qq])));
          }
        }
      }
      bf16* o = (bf16*)a.out + orow * 64;
#pragma unroll
      for (int i = 0; i < 64; i += 8) st_bf16x8(o + i, v + i);
    }
  }

  tc_fence_before();
  __syncthreads();
  if (warp == 4) {
    tc_fence_after();
    tmem_dealloc<Cfg::TMEM_COLS>(tmem);
  }
}

}  // namespace adainf

namespace adainf {

// ------------------------------------------------------------------------------------------------
// Window WGRAD for 64-channel stride-1 3x3 layers (ResNet layer1):
//   dW[(tap, ci)][co] = sum_q X[q + off(tap)][ci] * dZ[q][co]    (q on the padded flattened grid)
// Per 64-position K-block the CTA loads ONE window of X rows (64 + 2(W+1) + 2) and the 64 dZ rows; the
// A operand of tap pair (t, t+1) is the window viewed MN-major at row offset off(t) with the second MN
// atom LBO = (off(t+1) - off(t)) rows away (tap 8 pairs with a zero atom).  Five TMEM accumulators
// (5 x 64 columns) cover all 576 kconv rows, so each K-block's operands are used by 20 MMAs.  Each CTA
// reduces a contiguous range of K-blocks into fp32 partials [split][576][64] (fixed-order reduction
// afterwards: deterministic).
struct WinWgCfg {
  static constexpr int WROWS = 64 + 2 * 57 + 2;                       // <= W 56
  static constexpr int WIN_BYTES = ((WROWS + 7) / 8) * 1024;            // 23 KB
  static constexpr int B_BYTES = 64 * 64 * 2;                           // dZ block, MN-major
  static constexpr int STAGE_BYTES = WIN_BYTES + B_BYTES;
  static constexpr int STAGES = 5;
  static constexpr int ZERO_BYTES = 2048;                               // zero MN atom for tap 8
  static constexpr int SMEM = STAGES * STAGE_BYTES + ZERO_BYTES + 1024 + 256;
  static constexpr int TMEM_COLS = 512;                                 // 5 x 64 used
};

__global__ void __launch_bounds__(NUM_THREADS, 1) conv_win_wgrad_kernel(const WinArgs w) {
  using Cfg = WinWgCfg;
  const ConvArgs& a = w.c;  // src = X (Cs = 64), B = dZ (Nout = 64), out = partial, kb_per_split
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = smem_align1024(smem_raw);
  uint8_t* zero = smem + Cfg::STAGES * Cfg::STAGE_BYTES;
  uint64_t* full = (uint64_t*)(zero + Cfg::ZERO_BYTES);
  uint64_t* empty = full + Cfg::STAGES;
  uint64_t* tfull = empty + Cfg::STAGES;
  uint32_t* tmem_slot = (uint32_t*)(tfull + 1);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int H = a.Hs, W = a.Ws, Wp = W + 1, Hp = H + 1;
  const int nsamp = a.n_static;
  const int Qimg = Hp * Wp;
  const int Q = nsamp * Qimg;
  const int nkb = (Q + 63) / 64;
  const int kb0 = blockIdx.x * a.kb_per_split;
  const int kb1 = min(kb0 + a.kb_per_split, nkb);
  const int L = 64 + 2 * Wp + 2;

  for (int i = threadIdx.x; i < Cfg::ZERO_BYTES / 16; i += blockDim.x) ((uint4*)zero)[i] = make_uint4(0, 0, 0, 0);
  if (threadIdx.x == 0) {
    for (int s = 0; s < Cfg::STAGES; ++s) {
      mbar_init(&full[s], 128);
      mbar_init(&empty[s], 1);
    }
    mbar_init(tfull, 1);
    fence_mbar_init();
  }
  if (warp == 4) tmem_alloc<Cfg::TMEM_COLS>(tmem_slot);
  fence_proxy_async_smem();
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  const uint32_t sbase = smem_u32(smem);

  if (warp < 4) {
    const int t = threadIdx.x, j = t & 7;
    constexpr int RPT = (Cfg::WROWS + 15) / 16;
    int it = 0;
    for (int kb = kb0; kb < kb1; ++kb, ++it) {
      const int s = it % Cfg::STAGES, u = it / Cfg::STAGES;
      if (u > 0) mbar_wait(&empty[s], (u - 1) & 1);
      const uint32_t sw = sbase + s * Cfg::STAGE_BYTES;
      const uint32_t sb = sw + Cfg::WIN_BYTES;
      const int q0 = kb * 64;  // Q < 2^31 (asserted on the host)
      // X window rows [q0 - Wp - 1, q0 - Wp - 1 + L): decode the first row, then step 16 with carries
      {
        int qs = q0 - Wp - 1 + (t >> 3);
        int n = 0, h = 0, x = 0;
        if (qs >= 0) {
          n = qs / Qimg;
          const int rem = qs - n * Qimg;
          h = rem / Wp;
          x = rem - h * Wp;
        }
#pragma unroll
        for (int i = 0; i < RPT; ++i) {
          const int r = (t >> 3) + 16 * i;
          if (r < L) {
            const bool v = qs >= 0 && qs < Q && h < H && x < W;
            const bf16* g = v ? a.src + ((long long)((n * H + h) * W + x) * 64 + j * 8) : a.src;
            cp_async16(sw + kmaj_off(r, j), g, v);
          }
          qs += 16;
          if (qs >= 0) {
            if (qs < 16) {
              n = 0;
              h = qs / Wp;
              x = qs - h * Wp;
            } else {
              x += 16;
              while (x >= Wp) {
                x -= Wp;
                if (++h >= Hp) {
                  h = 0;
                  ++n;
                }
              }
            }
          }
        }
      }
      // dZ rows q0 .. q0+63 (zero at padding positions)
      {
        int q = q0 + (t >> 3);
        int n = q / Qimg;
        const int rem = q - n * Qimg;
        int h = rem / Wp, x = rem - h * Wp;
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          const int r = (t >> 3) + 16 * i;
          const bool v = q < Q && h < H && x < W;
          const bf16* g = v ? a.B + ((long long)((n * H + h) * W + x) * 64 + j * 8) : a.B;
          cp_async16(sb + kmaj_off(r, j), g, v);  // == MN-major layout for a single 64-wide atom
          q += 16;
          x += 16;
          while (x >= Wp) {
            x -= Wp;
            if (++h >= Hp) {
              h = 0;
              ++n;
            }
          }
        }
      }
      cp_async_arrive_noinc(&full[s]);
    }
  } else if (warp == 4) {
    const uint32_t IDESC = make_idesc(BM, 64, 1, 1);
    const uint32_t zaddr = smem_u32(zero);
    int it = 0;
    for (int kb = kb0; kb < kb1; ++kb, ++it) {
      const int s = it % Cfg::STAGES, u = it / Cfg::STAGES;
      mbar_wait(&full[s], u & 1);
      fence_proxy_async_smem();
      tc_fence_after();
      if (elect_one()) {
        const uint32_t sw = sbase + s * Cfg::STAGE_BYTES;
        const uint32_t sb = sw + Cfg::WIN_BYTES;
#pragma unroll
        for (int p = 0; p < 5; ++p) {
          const int t0 = 2 * p;
#pragma unroll
          for (int kk = 0; kk < 4; ++kk) {
            const uint32_t a0 = sw + (uint32_t)(w.tap_off[t0] + kk * 16) * 128u;
            const uint32_t a1 = (t0 + 1 < 9) ? sw + (uint32_t)(w.tap_off[t0 + 1] + kk * 16) * 128u : zaddr;
            const uint64_t ad = make_sdesc(a0, a1 - a0, 1024);
            const uint64_t bd = make_sdesc(sb + kk * 2048, 8192, 1024);
            umma_bf16(tmem + (uint32_t)(p * 64), ad, bd, IDESC, (it | kk) != 0);
          }
        }
        umma_commit(&empty[s]);
      }
      __syncwarp();
    }
    if (lane == 0) {
      if (kb1 > kb0) umma_commit(tfull);
      else mbar_arrive(tfull);
    }
    __syncwarp();
  } else {
    const int qd = warp & 3;
    const int row = qd * 32 + lane;
    mbar_wait(tfull, 0);
    tc_fence_after();
    const uint32_t trow = tmem + ((uint32_t)(qd * 32) << 16);
    for (int p = 0; p < 5; ++p) {
      const int kconv = p * 128 + row;
      float* outp = (float*)a.out + ((long long)blockIdx.x * 576 + kconv) * 64;
#pragma unroll 1
      for (int c0 = 0; c0 < 64; c0 += 32) {
        float v[32];
        if (kb1 > kb0) tmem_ld32(trow + p * 64 + c0, v);
        else
#pragma unroll
          for (int i = 0; i < 32; ++i) v[i] = 0.f;
        if (kconv < 576)
#pragma unroll
          for (int i = 0; i < 32; i += 4) *(float4*)(outp + c0 + i) = make_float4(v[i], v[i + 1], v[i + 2], v[i + 3]);
      }
    }
  }

  tc_fence_before();
  __syncthreads();
  if (warp == 4) {
    tc_fence_after();
    tmem_dealloc<Cfg::TMEM_COLS>(tmem);
  }
}

}  // namespace adainf

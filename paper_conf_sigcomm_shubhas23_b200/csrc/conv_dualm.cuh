// Dual-M implicit-GEMM conv for FWD / stride-1 DGRAD with all-TMA operands and BN = 128 (ResNet layer 2):
// each tile is 256 GEMM rows (two 128-row im2col A loads) x 128 columns sharing ONE weight tile per K-block,
// accumulated in two TMEM accumulators (double-buffered: 4 x 128 columns).  Measured: the generic kernel is
// bound by TMA/L2 -> SM bytes per K-block (~45-50 B/cycle/SM); sharing the weight tile between two M tiles
// moves 48 KB instead of 64 KB per 256 x 128 x 64 block.  8 epilogue warps: warps 5-8 drain the first
// accumulator, warps 9-12 the second (one warp per TMEM lane quadrant each).
#pragma once
#include "conv_gemm.cuh"

namespace adainf {

constexpr int DUALM_THREADS = 416;

// BN = 128: accumulators double-buffered (4 x 128 TMEM columns); BN = 256 (layers 3-4): single-buffered
// (2 x 256 columns), the epilogue of a tile is short next to its 36+ K-blocks of MMAs
template <int MODE, int BN_>
struct DualMCfg {
  static constexpr int BN = BN_;
  static constexpr int NBUF = BN == 128 ? 2 : 1;
  static constexpr int A_BYTES = 2 * BM * BK * 2;  // two 128-row tiles
  static constexpr int B_BYTES = BN * BK * 2;
  static constexpr int STAGE_BYTES = A_BYTES + B_BYTES;
  static constexpr int EPI_BYTES = 8 * 8192;
  static constexpr int BIAS_BYTES = MODE == MODE_FWD ? 4096 : 0;
  static constexpr int STAGES_FIT = (222 * 1024 - EPI_BYTES - BIAS_BYTES - 1536) / STAGE_BYTES;
  static constexpr int STAGES = STAGES_FIT > 8 ? 8 : STAGES_FIT;
  static constexpr int SMEM = STAGES * STAGE_BYTES + 1024 + 512 + EPI_BYTES + BIAS_BYTES;
};

template <int MODE, int BN_>
__global__ void __launch_bounds__(DUALM_THREADS, 1) conv_dualm_kernel(const __grid_constant__ ConvArgs a) {
  static_assert(MODE == MODE_FWD || MODE == MODE_DGRAD, "dual-M kernel: FWD / DGRAD");
  using Cfg = DualMCfg<MODE, BN_>;
  constexpr int NBUF = Cfg::NBUF;
  constexpr int BN = Cfg::BN;
  constexpr int STAGES = Cfg::STAGES;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = smem_align1024(smem_raw);
  uint64_t* full = (uint64_t*)(smem + STAGES * Cfg::STAGE_BYTES);
  uint64_t* empty = full + 8;
  uint64_t* tfull = empty + 8;   // [2]
  uint64_t* tempty = tfull + 2;  // [2]
  uint32_t* tmem_slot = (uint32_t*)(tempty + 2);
  uint8_t* epi_smem = smem + STAGES * Cfg::STAGE_BYTES + 512;
  float* bias_s = nullptr;
  if (MODE == MODE_FWD && a.bias && a.Nout <= 1024) {
    bias_s = (float*)(epi_smem + Cfg::EPI_BYTES);
    for (int i = threadIdx.x; i < a.Nout; i += DUALM_THREADS) bias_s[i] = __ldg(a.bias + i);
  }

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int nsamp = a.count ? *a.count : a.n_static;
  const int HWg = a.Hg * a.Wg;
  const long long npix = (long long)nsamp * HWg;
  const int nt = (a.Nout + BN - 1) / BN;
  const int mt2 = (int)((npix + 2 * BM - 1) / (2 * BM));
  const int ntile = mt2 * nt;
  const int nkb = (a.K + BK - 1) / BK;
  if ((int)blockIdx.x >= ntile) return;

  if (threadIdx.x == 0) {
    for (int s = 0; s < STAGES; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], 1);
    }
    for (int b = 0; b < 2; ++b) {
      mbar_init(&tfull[b], 1);
      mbar_init(&tempty[b], 256);
    }
    fence_mbar_init();
  }
  if (warp == 4) tmem_alloc<2 * BN * NBUF>(tmem_slot);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  const uint32_t smem_base = smem_u32(smem);

  if (warp == 0) {
    if (lane == 0) {
      int it = 0;
      for (int tile = blockIdx.x; tile < ntile; tile += gridDim.x) {
        const int nb = tile % nt, mb = tile / nt;
        const int n0 = nb * BN;
        int bw[2], bh[2], ni[2];
        for (int h = 0; h < 2; ++h) {
          long long m0 = (long long)mb * 2 * BM + h * BM;
          if (m0 >= npix) m0 = 0;  // second half wholly past the batch: load (unused) rows from the start
          ni[h] = (int)(m0 / HWg);
          const int pix = (int)m0 - ni[h] * HWg;
          const int gy = pix / a.Wg, gx = pix - gy * a.Wg;
          bw[h] = gx * a.sx + a.a_lo;
          bh[h] = gy * a.sy + a.a_lo;
        }
        int tap = 0, c = 0;
        for (int kb = 0; kb < nkb; ++kb, ++it) {
          const int s = it % STAGES, u = it / STAGES;
          if (u > 0) mbar_wait(&empty[s], (u - 1) & 1);
          const uint32_t sa = smem_base + s * Cfg::STAGE_BYTES, sb = sa + Cfg::A_BYTES;
          mbar_expect_tx(&full[s], (uint32_t)Cfg::STAGE_BYTES);
#pragma unroll
          for (int h = 0; h < 2; ++h)
            tma_load_im2col_4d(sa + h * (BM * BK * 2), &a.a_map, &full[s], c, bw[h], bh[h], ni[h],
                               (uint16_t)(a.tx[tap] - a.a_lo), (uint16_t)(a.ty[tap] - a.a_lo));
          if (MODE == MODE_FWD) {
            tma_load_2d(sb, &a.b_map, &full[s], kb * BK, n0);
          } else {
#pragma unroll
            for (int b = 0; b < BN / 64; ++b)
              tma_load_2d(sb + b * 8192, &a.b_map, &full[s], a.btap[tap] * a.Nout + n0 + b * 64, c);
          }
          c += BK;
          if (c >= a.Cs) c = 0, ++tap;
        }
      }
    }
  } else if (warp == 4) {
    constexpr uint32_t IDESC = make_idesc(BM, BN, 0, MODE == MODE_FWD ? 0 : 1);
    int it = 0, lt = 0;
    for (int tile = blockIdx.x; tile < ntile; tile += gridDim.x, ++lt) {
      const int b = NBUF == 2 ? (lt & 1) : 0, ub = NBUF == 2 ? (lt >> 1) : lt;
      if (ub > 0) mbar_wait(&tempty[b], (ub - 1) & 1);
      tc_fence_after();
      const uint32_t dacc = tmem + (uint32_t)(b * 2 * BN);
      for (int kb = 0; kb < nkb; ++kb, ++it) {
        const int s = it % STAGES, u = it / STAGES;
        mbar_wait(&full[s], u & 1);
        tc_fence_after();
        if (elect_one()) {
          const uint32_t sa = smem_base + s * Cfg::STAGE_BYTES, sb = sa + Cfg::A_BYTES;
          const uint64_t a0 = make_sdesc(sa, 16, 1024), a1 = make_sdesc(sa + BM * BK * 2, 16, 1024);
          const uint64_t bd0 = MODE == MODE_FWD ? make_sdesc(sb, 16, 1024) : make_sdesc(sb, 8192, 1024);
          constexpr uint32_t B_KK = MODE == MODE_FWD ? 2u : 128u;
#pragma unroll
          for (int kk = 0; kk < BK / 16; ++kk) {
            // both M tiles multiply the same weight slice: the second reads it from the B collector
            umma_bf16_ws_fill(dacc, a0 + 2u * kk, bd0 + kk * B_KK, IDESC, (kb | kk) != 0);
            umma_bf16_ws_lastuse(dacc + BN, a1 + 2u * kk, bd0 + kk * B_KK, IDESC, (kb | kk) != 0);
          }
          umma_commit(&empty[s]);
          if (kb == nkb - 1) umma_commit(&tfull[b]);
        }
        __syncwarp();
      }
    }
  } else if (warp >= 5) {
    const int q = warp & 3;
    const int half = (warp - 5) >> 2;  // which 128-row half of the tile this warp drains
    const int row = q * 32 + lane;
    int lt = 0;
    for (int tile = blockIdx.x; tile < ntile; tile += gridDim.x, ++lt) {
      const int nb = tile % nt, mb = tile / nt;
      TileInfo ti;
      ti.m0 = (long long)mb * 2 * BM + half * BM;
      ti.n0 = nb * BN;
      ti.kb0 = 0;
      ti.kb1 = nkb;
      ti.z = 0;
      const int b = NBUF == 2 ? (lt & 1) : 0, ub = NBUF == 2 ? (lt >> 1) : lt;
      const uint32_t trow = tmem + (uint32_t)(b * 2 * BN + half * BN) + ((uint32_t)(q * 32) << 16);
      const long long m = ti.m0 + row;
      const bool rv = m < npix;
      long long orow = 0, rrow = 0;
      int n = 0;
      if (rv) {
        n = (int)m / HWg;
        const int pix = (int)m - n * HWg;
        const int gy = pix / a.Wg, gx = pix - gy * a.Wg;
        orow = ((long long)n * a.Ho + gy * a.oys + a.oyo) * a.Wo + gx * a.oxs + a.oxo;
        if (MODE == MODE_FWD && a.res) {
          const int rn = a.res_map ? __ldg(a.res_map + n) : n;
          rrow = (long long)rn * a.Ho * a.Wo + (orow - (long long)n * a.Ho * a.Wo);
        }
      }
      epilogue_coalesced<MODE, BN, 1>(a, ti, trow, &tfull[b], ub & 1, &tempty[b], nkb, m, rv, n, orow, rrow, HWg,
                                      epi_smem + (warp - 5) * 8192, lane, bias_s, 0);
    }
  }

  tc_fence_before();
  __syncthreads();
  if (warp == 4) {
    tc_fence_after();
    tmem_dealloc<2 * BN * NBUF>(tmem);
  }
}

}  // namespace adainf

// CTA-pair (cta_group::2) implicit-GEMM conv for FWD / stride-1 DGRAD with all-TMA operands (SURVEY §8(a)
// a2, a9).  A cluster of two CTAs on neighbouring SMs computes 256-row tiles: CTA r loads GEMM rows
// [256t + 128r, +128) of A (im2col TMA) and HALF of the weight tile (N columns [r*BN/2, (r+1)*BN/2)) into the
// same shared-memory offsets; the leader issues tcgen05.mma.cta_group::2 with M = 256, which reads A from
// each CTA's own shared memory and the two B halves from both, and accumulates each CTA's 128 rows in its
// own TMEM.  Per SM this halves the weight operand's shared-memory reads and writes and its L2 -> SM
// traffic, which bound the single-CTA kernel at N <= 128 (ResNet layer 2).
//
// Synchronisation (validated with tools/exp_2cta.cu):
//   full[s]   the LEADER's barrier, two arrivals per stage: each CTA's producer arms it with its own bytes
//             (remote arrive.expect_tx from the peer) and issues its TMA loads with .cta_group::2, so both
//             halves complete their transaction bytes on it directly (no forwarding hop through the peer)
//   empty[s]  tcgen05.commit.cta_group::2 multicast to both CTAs (each producer reuses its own stage)
//   tfull[b]  same multicast commit at the tile's last K-block (each epilogue reads its own TMEM lanes)
//   tempty[b] leader-side, 256 arrivals: both CTAs' epilogue threads (the peer's arrive remotely)
// TMEM is allocated with cta_group::2 (same columns in both CTAs).
#pragma once
#include "conv_gemm.cuh"

namespace adainf {

template <int MODE, int BN>
struct PairCfg {
  static constexpr int A_BYTES = BM * BK * 2;
  static constexpr int B_BYTES = (BN / 2) * BK * 2;  // this CTA's half of the weight tile
  static constexpr int STAGE_BYTES = A_BYTES + B_BYTES;
  // the sub-pixel dgrad's epilogue double-buffers its two staged operands per warp
  static constexpr int EPI_BYTES = MODE == MODE_DGRAD_SP ? 4 * 16384 : 4 * 8192;
  static constexpr int BIAS_BYTES = MODE == MODE_FWD ? 4096 : 0;
  static constexpr int STAGES_FIT = (220 * 1024 - EPI_BYTES - BIAS_BYTES - 1280) / STAGE_BYTES;
  static constexpr int STAGES = STAGES_FIT > 8 ? 8 : STAGES_FIT;
  static constexpr int SMEM = STAGES * STAGE_BYTES + 1024 + 512 + EPI_BYTES + BIAS_BYTES;
  static constexpr int TMEM_COLS = 2 * BN;
};

template <int MODE, int BN>
__global__ void __launch_bounds__(NUM_THREADS, 1) conv_pair_kernel(const __grid_constant__ ConvArgs a) {
  static_assert(MODE == MODE_FWD || MODE == MODE_DGRAD || MODE == MODE_DGRAD_SP, "pair kernel: FWD / DGRAD / SP");
  constexpr bool B_KMAJ = MODE != MODE_DGRAD;  // FWD and the sub-pixel dgrad: K-major weight rows
  static_assert(BN == 128 || BN == 256, "pair kernel: BN 128 / 256");
  using Cfg = PairCfg<MODE, BN>;
  constexpr int STAGES = Cfg::STAGES;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = smem_align1024(smem_raw);
  uint64_t* full = (uint64_t*)(smem + STAGES * Cfg::STAGE_BYTES);
  uint64_t* empty = full + 8;
  uint64_t* tfull = empty + 8;  // [2]
  uint64_t* tempty = tfull + 2;  // [2] (leader)
  uint32_t* tmem_slot = (uint32_t*)(tempty + 2);
  uint8_t* epi_smem = smem + STAGES * Cfg::STAGE_BYTES + 512;
  float* bias_s = nullptr;
  if (MODE == MODE_FWD && a.bias && a.Nout <= 1024) {
    bias_s = (float*)(epi_smem + Cfg::EPI_BYTES);
    for (int i = threadIdx.x; i < a.Nout; i += NUM_THREADS) bias_s[i] = __ldg(a.bias + i);
  }

  const uint32_t rank = cluster_ctarank();
  const int pair = blockIdx.x >> 1, npairs = gridDim.x >> 1;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int nsamp = a.count ? *a.count : a.n_static;
  const int HWg = a.Hg * a.Wg;
  const long long npix = (long long)nsamp * HWg;
  const int nt = (a.Nout + BN - 1) / BN;
  const int mt2 = (int)((npix + 2 * BM - 1) / (2 * BM));
  const int ntile = mt2 * nt;
  const int nkb = (a.K + BK - 1) / BK;
  if (pair >= ntile) return;  // both CTAs of the pair leave together

  if (threadIdx.x == 0) {
    for (int s = 0; s < STAGES; ++s) {
      mbar_init(&full[s], 2);
      mbar_init(&empty[s], 1);
    }
    for (int b = 0; b < 2; ++b) {
      mbar_init(&tfull[b], 1);
      mbar_init(&tempty[b], 2 * 128);
    }
    fence_mbar_init();
  }
  if (warp == 4) {
    asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)),
                 "n"(Cfg::TMEM_COLS));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;");
  }
  tc_fence_before();
  cluster_sync_all();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  const uint32_t smem_base = smem_u32(smem);

  auto tile_rows = [&](int tile, long long& m0, int& n0) {
    const int nb = tile % nt, mb = tile / nt;
    m0 = (long long)mb * 2 * BM + rank * BM;
    n0 = nb * BN;
  };

  if (warp == 0) {
    if (lane == 0) {
      // ---- producer: im2col A (own 128 rows) + this CTA's half of the weight tile, per K-block ----
      int it = 0;
      for (int tile = pair; tile < ntile; tile += npairs) {
        long long m0;
        int n0;
        tile_rows(tile, m0, n0);
        const long long mm = m0 < npix ? m0 : 0;  // a peer tile wholly past the batch loads (unused) rows 0..
        const int n0i = (int)(mm / HWg);
        const int pix = (int)mm - n0i * HWg;
        const int gy = pix / a.Wg, gx = pix - gy * a.Wg;
        const int bw = gx * a.sx + a.a_lo, bh = gy * a.sy + a.a_lo;
        int tap = 0, c = 0;
        for (int kb = 0; kb < nkb; ++kb, ++it) {
          const int s = it % STAGES, u = it / STAGES;
          if (u > 0) mbar_wait(&empty[s], (u - 1) & 1);
          const uint32_t sa = smem_base + s * Cfg::STAGE_BYTES, sb = sa + Cfg::A_BYTES;
          const uint32_t fbar = mapa_rank(smem_u32(&full[s]), 0);  // the leader's stage barrier
          mbar_expect_tx_cluster(fbar, (uint32_t)Cfg::STAGE_BYTES);
          tma_load_im2col_4d_cg2(sa, &a.a_map, fbar, c, bw, bh, n0i, (uint16_t)(a.tx[tap] - a.a_lo),
                                 (uint16_t)(a.ty[tap] - a.a_lo));
          if (B_KMAJ) {
            tma_load_2d_cg2(sb, &a.b_map, fbar, kb * BK, n0 + (int)rank * (BN / 2));  // box {64 K, BN/2 rows}
          } else {
#pragma unroll
            for (int b = 0; b < BN / 128; ++b)
              tma_load_2d_cg2(sb + b * 8192, &a.b_map, fbar,
                              a.btap[tap] * a.Nout + n0 + (int)rank * (BN / 2) + b * 64, c);
          }
          c += BK;
          if (c >= a.Cs) c = 0, ++tap;
        }
      }
    }
  } else if (warp == 4) {
    if (rank == 1) {
      // peer: its stages complete on the leader's barriers; nothing to issue
    } else {
      // ---- leader: tcgen05.mma.cta_group::2, M = 256 ----
      constexpr uint32_t IDESC = make_idesc(2 * BM, BN, 0, B_KMAJ ? 0 : 1);
      int it = 0, lt = 0;
      for (int tile = pair; tile < ntile; tile += npairs, ++lt) {
        const int b = lt & 1, ub = lt >> 1;
        if (ub > 0) mbar_wait(&tempty[b], (ub - 1) & 1);
        tc_fence_after();
        const uint32_t dacc = tmem + (uint32_t)(b * BN);
        for (int kb = 0; kb < nkb; ++kb, ++it) {
          const int s = it % STAGES, u = it / STAGES;
          mbar_wait(&full[s], u & 1);
          tc_fence_after();
          if (elect_one()) {
            const uint32_t sa = smem_base + s * Cfg::STAGE_BYTES, sb = sa + Cfg::A_BYTES;
            const uint64_t ad0 = make_sdesc(sa, 16, 1024);
            const uint64_t bd0 = B_KMAJ ? make_sdesc(sb, 16, 1024) : make_sdesc(sb, 8192, 1024);
            constexpr uint32_t B_KK = B_KMAJ ? 2u : 128u;
#pragma unroll
            for (int kk = 0; kk < BK / 16; ++kk) {
              asm volatile(
                  "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                  "tcgen05.mma.cta_group::2.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(dacc),
                  "l"(ad0 + 2u * kk), "l"(bd0 + kk * B_KK), "r"(IDESC), "r"((uint32_t)((kb | kk) != 0))
                  : "memory");
            }
            asm volatile(
                "tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;" ::"r"(
                    smem_u32(&empty[s])),
                "h"((uint16_t)3)
                : "memory");
            if (kb == nkb - 1)
              asm volatile(
                  "tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], "
                  "%1;" ::"r"(smem_u32(&tfull[b])),
                  "h"((uint16_t)3)
                  : "memory");
          }
          __syncwarp();
        }
      }
    }
  } else if (warp >= 5) {
    // ---- epilogue: this CTA's 128 rows of each pair tile (same code as the single-CTA kernel) ----
    const int q = warp & 3;
    const int row = q * 32 + lane;
    const uint32_t remote_tempty = rank ? mapa_rank(smem_u32(tempty), 0) : 0u;
    int lt = 0;
    for (int tile = pair; tile < ntile; tile += npairs, ++lt) {
      long long m0;
      int n0;
      tile_rows(tile, m0, n0);
      TileInfo ti;
      ti.m0 = m0;
      ti.n0 = n0;
      ti.kb0 = 0;
      ti.kb1 = nkb;
      ti.z = 0;
      const int b = lt & 1, ub = lt >> 1;
      const uint32_t trow = tmem + (uint32_t)(b * BN) + ((uint32_t)(q * 32) << 16);
      const long long m = m0 + row;
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
      epilogue_coalesced<MODE, BN, 1>(a, ti, trow, &tfull[b], ub & 1,
                                      rank ? nullptr : &tempty[b], nkb, m, rv, n, orow, rrow, HWg,
                                      epi_smem + q * (Cfg::EPI_BYTES / 4), lane, bias_s, 0,
                                      rank ? remote_tempty + (uint32_t)(b * 8) : 0u);
    }
  }

  tc_fence_before();
  cluster_sync_all();
  if (warp == 4) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(tmem), "n"(Cfg::TMEM_COLS));
  }
}

}  // namespace adainf

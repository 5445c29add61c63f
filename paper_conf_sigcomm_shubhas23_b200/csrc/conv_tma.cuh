// Weight-stationary window conv for 64-channel stride-1 3x3 layers (ResNet layer1), operands moved by
// TMA (cp.async.bulk.tensor) instead of per-thread cp.async.
//
// Why TMA: the cp.async gather keeps only a bounded number of 16-byte requests in flight per SM, so for
// DRAM-resident activations it delivered ~3-5 B/cycle/SM (producers spent 75% of their time issuing);
// one bulk tensor copy per window moves 32 KB with a single instruction and an mbarrier transaction count.
//
// Tiling: a tile is R = 128 / Wp consecutive image rows of ONE image on a padded row pitch Wp (power of
// two >= W+1, the columns x >= W are the zero padding the TMA box reads out of bounds).  The window of a
// tile is the TMA box {64 ch, Wp px, R+2 rows} starting at row h0-1 (row -1 / H are out of bounds ->
// zeros), so every tap (dy, dx) of the 3x3 stencil is the window viewed at row offset 8 + (dy+1)Wp + dx
// (8 zero rows lead the box in shared memory).  B (9 tap tiles, 72 KB) stays resident in shared memory;
// the epilogue operands (residual / shortcut-gradient / stored activation) are staged by TMA too.
#pragma once
#include "conv_gemm.cuh"
#include "tma.cuh"
#include "colsum_tile.cuh"

namespace adainf {

struct WsTmaArgs {
  CUtensorMap win_map;  // source activations, box {64, Wp, R+2, 1}
  CUtensorMap e0_map;   // FWD: residual; DGRAD: shortcut gradient   (box {64, Wp, R, 1})
  CUtensorMap e1_map;   // DGRAD: stored activation for the act' mask (box {64, Wp, R, 1})
  CUtensorMap out_map;  // output (box {64, Wp, R, 1}): the epilogue stages each tile in shared memory, one TMA store
  const int* smap;      // optional sample map for the window / residual (inference stages)
  const int* count;
  int n_static;
  int H, W, Wp, R, tpi;  // tiles per image = ceil(H / R)
  const bf16* B;
  int ldb;
  int tap_off[9], btap[9];
  int dgrad, has_e0, has_e1, act, mask_act;
  const float* bias;
  const float* bcast;
  bf16* out;
  int wstages, win_bytes;
  int rowbox;  // 1: the window is R+2 boxes {64, W, 1, 1} (one per image row, no out-of-bounds columns); the
               // pad columns W..Wp-1 of every row slot are zeroed once and never written by the TMA
  int unit;    // 1: work items are PAIRS of vertically adjacent tiles sharing one 2R+2-row window; their MMAs
               // alternate between the two accumulators and share each B slice through the weight-stationary
               // collector, one commit per pair (wstages == 2, the window stage doubles as the accumulator pair)
  int upi;     // unit mode: tile pairs per image = ceil(tpi / 2)
};

constexpr int TMA_WS_THREADS = 416;  // warp 0 TMA producer (+ warps 1-3 help load B), warp 4 MMA, 8 epilogue warps

template <bool UNIT>
__global__ void __launch_bounds__(TMA_WS_THREADS, 1) conv_ws_tma_kernel(const __grid_constant__ WsTmaArgs a) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = smem_align1024(smem_raw);
  const int WS = a.wstages;
  uint8_t* win = smem;
  uint8_t* bres = win + WS * a.win_bytes;               // 9 x 8 KB
  const int ntens = a.has_e0 + a.has_e1;
  const int nstg = ntens > 0 ? ntens : 1;                // the output is staged in the first buffer
  uint8_t* stg = bres + 9 * 8192;                        // [2 groups][nstg tensors][16 KB]
  uint64_t* bars = (uint64_t*)(stg + 2 * nstg * 16384);
  uint64_t* wfull = bars;          // [WS]
  uint64_t* wempty = wfull + 8;    // [WS]
  uint64_t* tfull = wempty + 8;    // [2]
  uint64_t* tempty = tfull + 2;    // [2]
  uint64_t* efull = tempty + 2;    // [2]
  uint64_t* bready = efull + 2;
  uint32_t* tmem_slot = (uint32_t*)(bready + 1);
  float* s_bias = (float*)(tmem_slot + 4);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int nsamp = a.count ? *a.count : a.n_static;
  // work items: tiles, or (unit mode) pairs of vertically adjacent tiles of one image
  const int nitem = nsamp * (UNIT ? a.upi : a.tpi);
  if ((int)blockIdx.x >= nitem) return;
  const int Wp = a.Wp, R = a.R, H = a.H, W = a.W;
  const int WR = UNIT ? 2 * R + 2 : R + 2;  // window rows per item

  // zero the 8 lead / 8 trail rows of every window buffer (the TMA never writes them)
  for (int i = threadIdx.x; i < WS * 2 * 64; i += blockDim.x) {
    const int s = i / 128, k = i % 128;
    const int rows = 8 + WR * Wp;
    uint4* p = (uint4*)(win + s * a.win_bytes + (k < 64 ? k * 16 : rows * 128 + (k - 64) * 16));
    *p = make_uint4(0, 0, 0, 0);
  }
  if (a.rowbox) {
    const int padc = Wp - W, per_stage = WR * padc * 8;
    for (int i = threadIdx.x; i < WS * per_stage; i += blockDim.x) {
      const int s = i / per_stage, k = i - s * per_stage;
      const int j = k / (padc * 8), rem = k - j * (padc * 8);
      const int x = W + rem / 8, c = rem % 8;
      *(uint4*)(win + s * a.win_bytes + 1024 + (j * Wp + x) * 128 + c * 16) = make_uint4(0, 0, 0, 0);
    }
  }
  if (threadIdx.x < 64) s_bias[threadIdx.x] = (!a.dgrad && a.bias) ? a.bias[threadIdx.x] : 0.f;
  if (threadIdx.x == 0) {
    for (int s = 0; s < WS; ++s) {
      mbar_init(&wfull[s], 1);
      mbar_init(&wempty[s], 1);
    }
    for (int b = 0; b < 2; ++b) {
      mbar_init(&tfull[b], 1);
      mbar_init(&tempty[b], UNIT ? 256 : 128);
      mbar_init(&efull[b], 1);
    }
    mbar_init(bready, 128);
    fence_mbar_init();
    tma_prefetch_desc(&a.win_map);
  }
  if (warp == 4) tmem_alloc<UNIT ? 256 : 128>(tmem_slot);
  fence_proxy_async_smem();
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  const uint32_t wsm = smem_u32(win), bsm = smem_u32(bres), ssm = smem_u32(stg);
  const uint32_t box_bytes = 64u * 2u * Wp * (R + 2);
  const uint32_t ebox_bytes = 64u * 2u * Wp * R;

  if (warp < 4) {
    // ---- resident B (once per CTA, cp.async by all 128 producer threads) ----
    const int t = threadIdx.x;
    for (int tp = 0; tp < 9; ++tp) {
      const uint32_t sb = bsm + tp * 8192;
      const bf16* wb = a.B + (long long)a.btap[tp] * 64;
#pragma unroll
      for (int idx = t; idx < 64 * 8; idx += 128) {
        const int r = idx >> 3, jj = idx & 7;
        const uint32_t off = a.dgrad ? mnmaj_off(r, jj) : kmaj_off(r, jj);
        cp_async16(sb + off, wb + (long long)r * a.ldb + jj * 8, true);
      }
    }
    cp_async_arrive_noinc(bready);
    // ---- windows: one TMA box per tile, issued by one thread ----
    if (warp == 0 && lane == 0) {
      int it = 0;
      const int per = UNIT ? a.upi : a.tpi;
      for (int item = blockIdx.x; item < nitem; item += gridDim.x, ++it) {
        const int n = item / per, h0 = (item - n * per) * (UNIT ? 2 * R : R);
        const int sn = a.smap ? __ldg(a.smap + n) : n;
        const int s = it % WS, u = it / WS;
        // unit mode: the pair's commit (tfull) also frees its window stage (wstages == 2)
        if (u > 0) TIMED_WAIT(0, mbar_wait(UNIT ? &tfull[s] : &wempty[s], (u - 1) & 1));
        if (a.rowbox) {
          mbar_expect_tx(&wfull[s], 64u * 2u * W * WR);
          for (int j = 0; j < WR; ++j)
            tma_load_4d(wsm + s * a.win_bytes + 1024 + j * Wp * 128, &a.win_map, &wfull[s], 0, 0, h0 - 1 + j, sn);
        } else {
          mbar_expect_tx(&wfull[s], box_bytes);
          tma_load_4d(wsm + s * a.win_bytes + 1024, &a.win_map, &wfull[s], 0, 0, h0 - 1, sn);
        }
      }
    }
  } else if (warp == 4) {
    // ---- MMA issuer ----
    const uint32_t IDESC = make_idesc(BM, 64, 0, a.dgrad ? 1 : 0);
    // descriptors are linear in the start address (16-byte units, < 2^14): build the bases once and add
    // per-(tap, k-step) offsets, so the single issuing thread spends ~3 uniform ops per MMA instead of ~18
    const uint64_t b_base = a.dgrad ? make_sdesc(bsm, 8192, 1024) : make_sdesc(bsm, 16, 1024);
    const uint32_t b_kk = a.dgrad ? 128u : 2u;
    uint32_t toff[9];
#pragma unroll
    for (int tp = 0; tp < 9; ++tp) toff[tp] = (uint32_t)a.tap_off[tp] * 8u;
    mbar_wait(bready, 0);
    fence_proxy_async_smem();
#ifdef ADAINF_TIMING
    const long long t_mma0 = clock64();
#endif
    int it = 0;
    const uint32_t unit_off = (uint32_t)(R * Wp * 8);  // second tile of a pair: R rows further (16-byte units)
    for (int item = blockIdx.x; item < nitem; item += gridDim.x, ++it) {
      const int b = it & 1, ub = it >> 1;
      if (ub > 0) TIMED_WAIT(1, mbar_wait(&tempty[b], (ub - 1) & 1));
      const int s = it % WS, u = it / WS;
      TIMED_WAIT(2, mbar_wait(&wfull[s], u & 1));
      tc_fence_after();
      if (elect_one()) {
        const uint32_t sw = wsm + s * a.win_bytes;
        const uint64_t a_base = make_sdesc(sw, 16, 1024);
        if constexpr (UNIT) {
          const uint32_t d0 = tmem + (uint32_t)(b * 128);
#pragma unroll
          for (int tp = 0; tp < 9; ++tp) {
#pragma unroll
            for (int kk = 0; kk < 4; ++kk) {
              const uint64_t bd = b_base + (uint32_t)(tp * 512 + kk * b_kk);
              const uint32_t acc = (tp | kk) != 0;
              umma_bf16_ws_fill(d0, a_base + (toff[tp] + 2u * kk), bd, IDESC, acc);
              umma_bf16_ws_lastuse(d0 + 64u, a_base + (toff[tp] + 2u * kk + unit_off), bd, IDESC, acc);
            }
          }
          umma_commit(&tfull[b]);
        } else {
          const uint32_t dacc = tmem + (uint32_t)(b * 64);
#pragma unroll
          for (int tp = 0; tp < 9; ++tp) {
#pragma unroll
            for (int kk = 0; kk < 4; ++kk)
              umma_bf16(dacc, a_base + (toff[tp] + 2u * kk), b_base + (uint32_t)(tp * 512 + kk * b_kk), IDESC,
                        (tp | kk) != 0);
          }
          umma_commit(&wempty[s]);
          umma_commit(&tfull[b]);
        }
      }
      __syncwarp();
    }
#ifdef ADAINF_TIMING
    if (lane == 0) atomicAdd(&g_wait_cycles[blockIdx.x & 4095][7], (unsigned long long)(clock64() - t_mma0));
#endif
  } else {
    // ---- epilogue: 2 groups of 4 warps, group g handles this CTA's local tiles g, g+2, ... ----
    const int grp = (warp - 5) >> 2;
    const int qd = warp & 3;
    const int row = qd * 32 + lane;  // output position p within the tile
    const bool leader = (warp == 5 + 4 * grp) && lane == 0;
    const uint32_t sg = ssm + grp * nstg * 16384;
    // tile mode: group g takes this CTA's items g, g+2, ...; unit mode: group g takes tile g of every pair
    int lt = UNIT ? 0 : grp, use = 0;
    for (int item = blockIdx.x + (UNIT ? 0 : grp * gridDim.x); item < nitem;
         item += (UNIT ? 1 : 2) * gridDim.x, lt += (UNIT ? 1 : 2), ++use) {
      const int per = UNIT ? a.upi : a.tpi;
      const int n = item / per, h0 = (item - n * per) * (UNIT ? 2 * R : R) + (UNIT ? grp * R : 0);
      const int h = h0 + row / Wp, x = row % Wp;
      const bool rv = h < H && x < W;
      const long long orow = ((long long)n * H + h) * W + x;
      if (ntens && leader) {  // stage the epilogue operands of this tile once the previous output store has read
        tma_store_wait_read();  // the buffer
        mbar_expect_tx(&efull[grp], ntens * ebox_bytes);
        const int sn = (!a.dgrad && a.smap) ? __ldg(a.smap + n) : n;
        if (a.has_e0) tma_load_4d(sg, &a.e0_map, &efull[grp], 0, 0, h0, sn);
        if (a.has_e1) tma_load_4d(sg + a.has_e0 * 16384, &a.e1_map, &efull[grp], 0, 0, h0, n);
      }
      const int b = UNIT ? (lt & 1) : grp, ub = lt >> 1;
      TIMED_WAIT(3, mbar_wait(&tfull[b], ub & 1));
      tc_fence_after();
      const uint32_t trow = tmem + (uint32_t)(UNIT ? b * 128 + grp * 64 : b * 64) + ((uint32_t)(qd * 32) << 16);
      float v[64];
      tmem_ld32(trow, v);
      tmem_ld32(trow + 32, v + 32);
      tc_fence_before();
      mbar_arrive(&tempty[b]);
      if (ntens) TIMED_WAIT(4, mbar_wait(&efull[grp], use & 1));
      uint8_t* e0 = stg + (grp * nstg) * 16384 + row * 128;
      const uint8_t* e1 = e0 + a.has_e0 * 16384;
      if (rv) {
        if (!a.dgrad) {
#pragma unroll
          for (int i = 0; i < 64; ++i) v[i] = __fadd_rn(v[i], s_bias[i]);
          if (a.has_e0) {
#pragma unroll
            for (int i = 0; i < 8; ++i) {
              const uint4 e = *(const uint4*)(e0 + ((i ^ (row & 7)) << 4));
              const bf16* hh = (const bf16*)&e;
#pragma unroll
              for (int qq = 0; qq < 8; ++qq) v[i * 8 + qq] = __fadd_rn(v[i * 8 + qq], __bfloat162float(hh[qq]));
            }
          }
          act_vec<64>(a.act, v);
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
          if (a.has_e0) {
#pragma unroll
            for (int i = 0; i < 8; ++i) {
              const uint4 e = *(const uint4*)(e0 + ((i ^ (row & 7)) << 4));
              const bf16* hh = (const bf16*)&e;
#pragma unroll
              for (int qq = 0; qq < 8; ++qq) v[i * 8 + qq] = __fadd_rn(v[i * 8 + qq], __bfloat162float(hh[qq]));
            }
          }
          if (a.has_e1) {
            if (a.mask_act == 1) {  // ReLU' as a select (the kind tested once per row)
#pragma unroll
              for (int i = 0; i < 8; ++i) {
                const uint4 e = *(const uint4*)(e1 + ((i ^ (row & 7)) << 4));
                const bf16* hh = (const bf16*)&e;
#pragma unroll
                for (int qq = 0; qq < 8; ++qq)
                  v[i * 8 + qq] = __fmul_rn(v[i * 8 + qq], __bfloat162float(hh[qq]) > 0.f ? 1.f : 0.f);
              }
            } else {
#pragma unroll
              for (int i = 0; i < 8; ++i) {
                const uint4 e = *(const uint4*)(e1 + ((i ^ (row & 7)) << 4));
                const bf16* hh = (const bf16*)&e;
#pragma unroll
                for (int qq = 0; qq < 8; ++qq)
                  v[i * 8 + qq] = __fmul_rn(v[i * 8 + qq], act_grad(a.mask_act, __bfloat162float(hh[qq])));
              }
            }
          }
        }
      }
      // the output row goes into the staging buffer (over this row's own residual / shortcut bytes, same 128B
      // swizzle as the TMA map), then one TMA store per tile: 16-byte shared stores instead of 128-byte-strided
      // global ones (32 L1 wavefronts per warp store), and no global store latency in the epilogue
      if (!ntens) {  // dedicated buffer: the previous tile's store must have read it
        if (leader) tma_store_wait_read();
        TIMED_WAIT(5, asm volatile("bar.sync %0, 128;" ::"r"(1 + grp) : "memory"));
      }
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        uint4 q;
        q.x = pack_bf16x2(v[i * 8 + 0], v[i * 8 + 1]);
        q.y = pack_bf16x2(v[i * 8 + 2], v[i * 8 + 3]);
        q.z = pack_bf16x2(v[i * 8 + 4], v[i * 8 + 5]);
        q.w = pack_bf16x2(v[i * 8 + 6], v[i * 8 + 7]);
        *(uint4*)(e0 + ((i ^ (row & 7)) << 4)) = q;
      }
      fence_proxy_async_smem();
      TIMED_WAIT(6, asm volatile("bar.sync %0, 128;" ::"r"(1 + grp) : "memory"));
      if (leader) {
        tma_store_4d(&a.out_map, sg, 0, 0, h0, n);
        tma_store_commit();
      }
      (void)orow;
      (void)rv;
    }
    if (leader) tma_store_wait_all();
  }

  tc_fence_before();
  __syncthreads();
  if (warp == 4) {
    tc_fence_after();
    tmem_dealloc<UNIT ? 256 : 128>(tmem);
  }
}

}  // namespace adainf

namespace adainf {

// ------------------------------------------------------------------------------------------------
// General TMA window conv for stride-1 3x3 layers with Cin = 64*ncb and BN in {128, 256} (ResNet layers
// 2-3): per tile and 64-channel block, one window box {64, Wp, R+2, 1} and nine B boxes (FWD: K-major
// {64 K, BN co} from the [Cout][9*Cin] shadow; DGRAD: MN-major, BN/64 boxes {64 ci, 64 co} per tap), all
// issued by one thread and completed on mbarrier transaction counts.  Epilogue as in conv_gemm.cuh
// (4 warps, double-buffered TMEM accumulators, 128-bit global loads / stores).
struct WinTmaArgs {
  CUtensorMap win_map;  // source activations, box {64, Wp, R+2, 1}
  CUtensorMap b_map;    // weights shadow [Cout][ldb] (2-D): FWD box {64, BN}; DGRAD box {64, 64}
  const int* smap;
  const int* count;
  int n_static;
  int H, W, Wp, R, tpi, ncb, Nout;
  int tap_off[9], btap[9];
  int dgrad, act, mask_act;
  const float* bias;
  const bf16* res;
  const float* bcast;
  const bf16* sc;
  const bf16* yact;
  bf16* out;
  int wstages, bstages, win_bytes;
};

template <int BN>
__global__ void __launch_bounds__(NUM_THREADS, 1) conv_win_tma_kernel(const __grid_constant__ WinTmaArgs a) {
  constexpr int B_BYTES = BN * 128;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = smem_align1024(smem_raw);
  const int WS = a.wstages, BS = a.bstages;
  uint8_t* win = smem;
  uint8_t* bb = win + WS * a.win_bytes;
  uint64_t* bars = (uint64_t*)(bb + BS * B_BYTES);
  uint64_t* wfull = bars;
  uint64_t* wempty = wfull + 8;
  uint64_t* bfull = wempty + 8;
  uint64_t* bempty = bfull + 16;
  uint64_t* tfull = bempty + 16;
  uint64_t* tempty = tfull + 2;
  uint32_t* tmem_slot = (uint32_t*)(tempty + 2);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int nsamp = a.count ? *a.count : a.n_static;
  const int nt = (a.Nout + BN - 1) / BN;
  const int ntile = nsamp * a.tpi * nt;
  if ((int)blockIdx.x >= ntile) return;
  const int Wp = a.Wp, R = a.R, H = a.H, W = a.W;

  for (int i = threadIdx.x; i < WS * 2 * 64; i += blockDim.x) {
    const int s = i / 128, k = i % 128;
    const int rows = 8 + (R + 2) * Wp;
    *(uint4*)(win + s * a.win_bytes + (k < 64 ? k * 16 : rows * 128 + (k - 64) * 16)) = make_uint4(0, 0, 0, 0);
  }
  if (threadIdx.x == 0) {
    for (int s = 0; s < WS; ++s) {
      mbar_init(&wfull[s], 1);
      mbar_init(&wempty[s], 1);
    }
    for (int s = 0; s < BS; ++s) {
      mbar_init(&bfull[s], 1);
      mbar_init(&bempty[s], 1);
    }
    for (int b = 0; b < 2; ++b) {
      mbar_init(&tfull[b], 1);
      mbar_init(&tempty[b], 128);
    }
    fence_mbar_init();
    tma_prefetch_desc(&a.win_map);
    tma_prefetch_desc(&a.b_map);
  }
  if (warp == 4) tmem_alloc<2 * BN>(tmem_slot);
  fence_proxy_async_smem();
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  const uint32_t wsm = smem_u32(win), bsm = smem_u32(bb);
  const uint32_t box_bytes = 64u * 2u * Wp * (R + 2);

  if (warp == 0) {
    if (lane == 0) {
      int wit = 0, bit = 0;
      for (int tile = blockIdx.x; tile < ntile; tile += gridDim.x) {
        const int nb = tile % nt, r = tile / nt;
        const int n = r / a.tpi, h0 = (r - n * a.tpi) * R;
        const int n0 = nb * BN;
        const int sn = a.smap ? __ldg(a.smap + n) : n;
        for (int cb = 0; cb < a.ncb; ++cb, ++wit) {
          const int s = wit % WS, u = wit / WS;
          if (u > 0) mbar_wait(&wempty[s], (u - 1) & 1);
          mbar_expect_tx(&wfull[s], box_bytes);
          tma_load_4d(wsm + s * a.win_bytes + 1024, &a.win_map, &wfull[s], cb * 64, 0, h0 - 1, sn);
          for (int tp = 0; tp < 9; ++tp, ++bit) {
            const int bs = bit % BS, bu = bit / BS;
            if (bu > 0) mbar_wait(&bempty[bs], (bu - 1) & 1);
            mbar_expect_tx(&bfull[bs], B_BYTES);
            const uint32_t dst = bsm + bs * B_BYTES;
            if (!a.dgrad) {
              // K-major: rows co = n0.., columns btap*Cin + cb*64 ..
              tma_load_2d(dst, &a.b_map, &bfull[bs], a.btap[tp] * a.ncb * 64 + cb * 64, n0);
            } else {
              // MN-major: atom j = ci block n0 + 64j, rows co = cb*64 .. +64
#pragma unroll
              for (int j = 0; j < BN / 64; ++j)
                tma_load_2d(dst + j * 8192, &a.b_map, &bfull[bs], a.btap[tp] * a.Nout + n0 + j * 64, cb * 64);
            }
          }
        }
      }
    }
  } else if (warp == 4) {
    const uint32_t IDESC = make_idesc(BM, BN, 0, a.dgrad ? 1 : 0);
    int wit = 0, bit = 0, lt = 0;
    for (int tile = blockIdx.x; tile < ntile; tile += gridDim.x, ++lt) {
      const int b = lt & 1, ub = lt >> 1;
      if (ub > 0) mbar_wait(&tempty[b], (ub - 1) & 1);
      tc_fence_after();
      const uint32_t dacc = tmem + (uint32_t)(b * BN);
      for (int cb = 0; cb < a.ncb; ++cb, ++wit) {
        const int s = wit % WS, u = wit / WS;
        mbar_wait(&wfull[s], u & 1);
        const uint32_t sw = wsm + s * a.win_bytes;
        for (int tp = 0; tp < 9; ++tp, ++bit) {
          const int bs = bit % BS, bu = bit / BS;
          mbar_wait(&bfull[bs], bu & 1);
          tc_fence_after();
          if (elect_one()) {
            const uint32_t sb = bsm + bs * B_BYTES;
            const uint64_t ad0 = make_sdesc(sw + (uint32_t)a.tap_off[tp] * 128u, 16, 1024);
            const uint64_t bd0 = a.dgrad ? make_sdesc(sb, 8192, 1024) : make_sdesc(sb, 16, 1024);
            const uint32_t bkk = a.dgrad ? 128u : 2u;
#pragma unroll
            for (int kk = 0; kk < 4; ++kk) umma_bf16(dacc, ad0 + 2u * kk, bd0 + kk * bkk, IDESC, (cb | tp | kk) != 0);
            umma_commit(&bempty[bs]);
            if (tp == 8) {
              umma_commit(&wempty[s]);
              if (cb == a.ncb - 1) umma_commit(&tfull[b]);
            }
          }
          __syncwarp();
        }
      }
    }
  } else if (warp >= 5) {
    const int qd = warp & 3;
    const int row = qd * 32 + lane;
    int lt = 0;
    for (int tile = blockIdx.x; tile < ntile; tile += gridDim.x, ++lt) {
      const int nb = tile % nt, r = tile / nt;
      const int n = r / a.tpi, h0 = (r - n * a.tpi) * R;
      const int n0 = nb * BN;
      const int h = h0 + row / Wp, x = row % Wp;
      const bool rv = h < H && x < W;
      const long long orow = ((long long)n * H + h) * W + x;
      long long rrow = orow;
      if (!a.dgrad && a.res && rv && a.smap) rrow = ((long long)__ldg(a.smap + n) * H + h) * W + x;
      const int b = lt & 1, ub = lt >> 1;
      mbar_wait(&tfull[b], ub & 1);
      tc_fence_after();
      const uint32_t trow = tmem + (uint32_t)(b * BN) + ((uint32_t)(qd * 32) << 16);
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
        if (!a.dgrad) {
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
              const float4 q4 = __ldg((const float4*)(a.bcast + (long long)n * a.Nout + cbase + i));
              v[i] = __fadd_rn(v[i], q4.x);
              v[i + 1] = __fadd_rn(v[i + 1], q4.y);
              v[i + 2] = __fadd_rn(v[i + 2], q4.z);
              v[i + 3] = __fadd_rn(v[i + 3], q4.w);
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
        bf16* o = a.out + orow * a.Nout + cbase;
#pragma unroll
        for (int i = 0; i < 32; i += 8) st_bf16x8(o + i, v + i);
      }
    }
  }

  tc_fence_before();
  __syncthreads();
  if (warp == 4) {
    tc_fence_after();
    tmem_dealloc<2 * BN>(tmem);
  }
}

}  // namespace adainf

namespace adainf {


// ------------------------------------------------------------------------------------------------
// TMA weight-gradient GEMM for convs with Cin % 64 == 0 (any kernel size / stride / pad):
//   dW[(tap, ci)][co] = sum_{positions} X[s*oh + kh - p][s*ow + kw - p][ci] * dZ[oh][ow][co]
// K-blocks are R_k = 64 / Wp output rows of one image on a padded pitch Wp (power of two >= Wo).  Per
// K-block and M tile (128 kconv = two (tap, 64-ci) atoms) the A atoms are TMA boxes {64 ci, Wp, R_k}
// of X started at the tap's offset (element stride s; out-of-bounds -> 0) and the B atoms are boxes
// {64 co, Wp, R_k} of dZ (positions x >= Wo are out of bounds -> 0, so they contribute nothing).  Both
// land directly in the MN-major 128B-swizzled UMMA layout.  Split-K units write fp32 partials.
struct WgTmaArgs {
  CUtensorMap x_map;    // X [N][H][W][Cin], box {64, Wp, R_k} with element stride s
  CUtensorMap dz_map;   // dZ [N][Ho][Wo][Cout], box {64, Wp, R_k}
  int n, Ho, Wo, Wp, Rk, rg;  // rg = row groups per image = ceil(Ho / Rk)
  int KW, stride, pad, ncb;   // ncb = Cin / 64
  int Kconv, Cout;
  int kb_per_split, splits;
  float* out;           // partials [split][Kconv][Cout]
  float* cs_part;       // bias-gradient partials [split][Cout] (nullptr: not fused)
  int stages;
  // i2c = 1: K-blocks are 64 consecutive output pixels (no pitch padding): x_map is an im2col map (64 pixels x
  // 64 channels per load, base pixel = output position * stride + lo, tap offsets (kw, kh)), dz_map a 2-D map
  // over dZ as [n*Ho*Wo][Cout] with box {64 co, 64 pixels}; n = #K-blocks and rg = 1 so nkb = n * rg
  int i2c, lo;
};

// PM = M tiles (128 kconv rows each) per tile: PM = 2 shares each dZ (B) K-block between two M tiles (fewer TMA
// bytes per MAC; 8 MMAs per full-barrier wait / commit); accumulators double-buffered when they fit in TMEM.
template <int BN, int PM = 1>
__global__ void __launch_bounds__(NUM_THREADS, 1) conv_wgrad_tma_kernel(const __grid_constant__ WgTmaArgs a) {
  constexpr int A_BYTES = PM * 16384, B_BYTES = BN * 128, STAGE = A_BYTES + B_BYTES;
  constexpr int NBUF = 2 * PM * BN <= 512 ? 2 : 1;  // accumulator buffers
  constexpr int TCOLS = PM * BN * NBUF;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = smem_align1024(smem_raw);
  const int ST = a.stages;
  uint64_t* full = (uint64_t*)(smem + ST * STAGE);
  uint64_t* empty = full + 16;
  uint64_t* tfull = empty + 16;
  uint64_t* tempty = tfull + 2;
  uint32_t* tmem_slot = (uint32_t*)(tempty + 2);
  float* cs_red = (float*)((uint8_t*)full + 512);  // [NPH][BN] column-sum combine scratch (3 KB)

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int mt1 = (a.Kconv + 127) / 128;        // 128-row M tiles
  const int mt = (mt1 + PM - 1) / PM, nt = (a.Cout + BN - 1) / BN;
  const int ntile = mt * nt * a.splits;
  const int nkb = a.n * a.rg;
  if ((int)blockIdx.x >= ntile) return;
  if (threadIdx.x == 0) {
    for (int s = 0; s < ST; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], a.cs_part ? 4 : 1);  // MMA commit (+ one arrive per column-sum warp)
    }
    for (int b = 0; b < 2; ++b) {
      mbar_init(&tfull[b], 1);
      mbar_init(&tempty[b], 128);
    }
    fence_mbar_init();
    tma_prefetch_desc(&a.x_map);
    tma_prefetch_desc(&a.dz_map);
  }
  if (warp == 4) tmem_alloc<TCOLS>(tmem_slot);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  const uint32_t sbase = smem_u32(smem);

  if (warp == 0) {
    if (lane == 0) {
      int it = 0;
      for (int tile = blockIdx.x; tile < ntile; tile += gridDim.x) {
        const int nb = tile % nt, r = tile / nt, m = r % mt, z = r / mt;
        const int kb0 = z * a.kb_per_split, kb1 = min(kb0 + a.kb_per_split, nkb);
        // the 2*PM A atoms of this tile: (tap, ci block) = divmod(m*2*PM + i, ncb)
        int ax[2 * PM], ay[2 * PM], ac[2 * PM];
        bool av[2 * PM];
        for (int i = 0; i < 2 * PM; ++i) {
          const int at = m * 2 * PM + i;
          const int tap = at / a.ncb, cb = at - tap * a.ncb;
          av[i] = at * 64 < a.Kconv;
          ac[i] = cb * 64;
          ax[i] = (tap % a.KW) - a.pad;
          ay[i] = (tap / a.KW) - a.pad;
        }
        int nA = 0;
        for (int i = 0; i < 2 * PM; ++i) nA += av[i] ? 1 : 0;
        for (int kb = kb0; kb < kb1; ++kb, ++it) {
          const int s = it % ST, u = it / ST;
          if (u > 0) mbar_wait(&empty[s], (u - 1) & 1);
          const uint32_t sa = sbase + s * STAGE, sb = sa + A_BYTES;
          mbar_expect_tx(&full[s], nA * 8192 + (BN / 64) * 8192);
          if (a.i2c) {
            const int p0 = kb * 64, HWo = a.Ho * a.Wo;
            const int n0 = p0 / HWo, rem = p0 - n0 * HWo;
            const int oy = rem / a.Wo, ox = rem - oy * a.Wo;
            const int bw = ox * a.stride + a.lo, bh = oy * a.stride + a.lo;
            for (int i = 0; i < nA; ++i)
              tma_load_im2col_4d(sa + i * 8192, &a.x_map, &full[s], ac[i], bw, bh, n0, (uint16_t)(ax[i] - a.lo),
                                 (uint16_t)(ay[i] - a.lo));
#pragma unroll
            for (int j = 0; j < BN / 64; ++j) tma_load_2d(sb + j * 8192, &a.dz_map, &full[s], nb * BN + j * 64, p0);
            continue;
          }
          const int img = kb / a.rg, h0 = (kb - img * a.rg) * a.Rk;
          for (int i = 0; i < nA; ++i)
            tma_load_4d(sa + i * 8192, &a.x_map, &full[s], ac[i], ax[i], h0 * a.stride + ay[i], img);
#pragma unroll
          for (int j = 0; j < BN / 64; ++j) tma_load_4d(sb + j * 8192, &a.dz_map, &full[s], nb * BN + j * 64, 0, h0, img);
        }
      }
    }
  } else if (warp == 4) {
    constexpr uint32_t IDESC = make_idesc(BM, BN, 1, 1);
    int it = 0, lt = 0;
    for (int tile = blockIdx.x; tile < ntile; tile += gridDim.x, ++lt) {
      const int r = tile / nt, m = r % mt, z = r / mt;
      const int kb0 = z * a.kb_per_split, kb1 = min(kb0 + a.kb_per_split, nkb);
      const int b = NBUF == 2 ? (lt & 1) : 0, ub = NBUF == 2 ? (lt >> 1) : lt;
      if (ub > 0) mbar_wait(&tempty[b], (ub - 1) & 1);
      tc_fence_after();
      const uint32_t dacc = tmem + (uint32_t)(b * PM * BN);
      const bool second = PM == 2 && (m * 2 + 1) < mt1;  // the second M tile exists
      for (int kb = kb0; kb < kb1; ++kb, ++it) {
        const int s = it % ST, u = it / ST;
        mbar_wait(&full[s], u & 1);
        tc_fence_after();
        if (elect_one()) {
          const uint32_t sa = sbase + s * STAGE, sb = sa + A_BYTES;
          const uint64_t ad0 = make_sdesc(sa, 8192, 1024), bd0 = make_sdesc(sb, 8192, 1024);
#pragma unroll
          for (int kk = 0; kk < 4; ++kk) {
            umma_bf16(dacc, ad0 + kk * 128u, bd0 + kk * 128u, IDESC, (kb != kb0 || kk != 0));
            if (PM == 2 && second)  // A atoms 2, 3 (16 KB further): the second M tile
              umma_bf16(dacc + BN, ad0 + (16384u >> 4) + kk * 128u, bd0 + kk * 128u, IDESC, (kb != kb0 || kk != 0));
          }
          umma_commit(&empty[s]);
          if (kb == kb1 - 1) umma_commit(&tfull[b]);
        }
        __syncwarp();
      }
      if (kb1 <= kb0 && lane == 0) mbar_arrive(&tfull[b]);
      __syncwarp();
    }
  } else if (warp >= 1 && warp <= 3) {
    if (a.cs_part) {
      // fused bias gradient: the mt tiles of one (co block, split) see the same dZ K-blocks; tile m sums the
      // K-blocks with kb % mt == m into partial row z * mt + m
      TileColsum<BN> cs;
      const int t = threadIdx.x - 32;
      cs.init(t);
      int it = 0;
      for (int tile = blockIdx.x; tile < ntile; tile += gridDim.x) {
        const int nb = tile % nt, r = tile / nt, m = r % mt, z = r / mt;
        const int kb0 = z * a.kb_per_split, kb1 = min(kb0 + a.kb_per_split, nkb);
        cs.zero();
        for (int kb = kb0; kb < kb1; ++kb, ++it) {
          const int s = it % ST, u = it / ST;
          mbar_wait(&full[s], u & 1);
          if (kb % mt == m) cs.add(smem + s * STAGE + A_BYTES, 64);
          __syncwarp();
          if (lane == 0) mbar_arrive(&empty[s]);
        }
        cs.finish(cs_red, a.cs_part + ((long long)z * mt + m) * a.Cout + nb * BN, a.Cout - nb * BN, t);
      }
    }
  } else if (warp >= 5) {
    const int qd = warp & 3;
    const int row = qd * 32 + lane;
    int lt = 0;
    for (int tile = blockIdx.x; tile < ntile; tile += gridDim.x, ++lt) {
      const int nb = tile % nt, r = tile / nt, m = r % mt, z = r / mt;
      const int kb0 = z * a.kb_per_split, kb1 = min(kb0 + a.kb_per_split, nkb);
      const int b = NBUF == 2 ? (lt & 1) : 0, ub = NBUF == 2 ? (lt >> 1) : lt;
      mbar_wait(&tfull[b], ub & 1);
      tc_fence_after();
#pragma unroll 1
      for (int h = 0; h < PM; ++h) {
        const uint32_t trow = tmem + (uint32_t)(b * PM * BN + h * BN) + ((uint32_t)(qd * 32) << 16);
        const int kc = (m * PM + h) * 128 + row;
        float* outp = a.out + ((long long)z * a.Kconv + kc) * a.Cout + nb * BN;
#pragma unroll 1
        for (int c0 = 0; c0 < BN; c0 += 32) {
          float v[32];
          const bool live = kb1 > kb0 && (h == 0 || (m * PM + h) < mt1);
          if (live) tmem_ld32(trow + c0, v);
          else
#pragma unroll
            for (int i = 0; i < 32; ++i) v[i] = 0.f;
          if (h == PM - 1 && c0 + 32 >= BN) {
            tc_fence_before();
            mbar_arrive(&tempty[b]);
          }
          if (kc < a.Kconv && nb * BN + c0 < a.Cout)
#pragma unroll
            for (int i = 0; i < 32; i += 4) *(float4*)(outp + c0 + i) = make_float4(v[i], v[i + 1], v[i + 2], v[i + 3]);
        }
      }
    }
  }

  tc_fence_before();
  __syncthreads();
  if (warp == 4) {
    tc_fence_after();
    tmem_dealloc<TCOLS>(tmem);
  }
}

// ---- window weight gradient (stride-1 3x3, pad 1), TMA-fed --------------------------------------------
// dW[tap][ci][co] = sum_pix X(pix + tap) * dZ(pix).  K = output pixels of R rows of one image on a padded
// grid of Wp (>= W+1) columns; the X window (R+2 rows, 8 zero rows before and after) serves all nine taps
// as row-shifted MN-major A operands, so each dZ tile is loaded once for 9 taps.  M = (tap pair, 64 ci):
// five TMEM accumulators of 128 x 64 (the tenth slot reads a zero atom), N = 64 co.
struct WinWgTmaArgs {
  CUtensorMap x_map;    // X [N][H][W][Cin], box {64, Wp, R+2, 1}
  CUtensorMap dz_map;   // dZ [N][H][W][Cout], box {64, Wp, R, 1}
  int n, H, Wp, R, rg;  // rg = ceil(H / R) row groups per image
  int ncb, nnb, Cin, Cout;
  int kb_per_split, splits;
  float* out;           // partials [split][9*Cin][Cout]
  float* cs_part;       // bias-gradient partials [split][Cout] (nullptr: not fused)
  int stages, a_bytes;  // a_bytes = (16 + (R+2)*Wp) * 128
};

__global__ void __launch_bounds__(NUM_THREADS, 1) conv_wgrad_win_tma_kernel(const __grid_constant__ WinWgTmaArgs a) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = smem_align1024(smem_raw);
  const int ST = a.stages, Wp = a.Wp, R = a.R;
  const int b_bytes = R * Wp * 128;
  const int stage_bytes = a.a_bytes + b_bytes;
  uint8_t* zero = smem + ST * stage_bytes;
  uint64_t* full = (uint64_t*)(zero + 2048);
  uint64_t* empty = full + 8;
  uint64_t* tfull = empty + 8;
  uint64_t* tempty = tfull + 1;
  uint32_t* tmem_slot = (uint32_t*)(tempty + 1);
  float* cs_red = (float*)(zero + 2048 + 256);  // [12][64] column-sum combine scratch (3 KB)

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int tiles = a.ncb * a.nnb;
  const int nunit = tiles * a.splits;
  const int nkb = a.n * a.rg;
  if ((int)blockIdx.x >= nunit) return;
  // zero: 8 lead + 8 trail rows of every A stage, and the zero atom
  const int wrows = 8 + (R + 2) * Wp;
  for (int i = threadIdx.x; i < ST * 128 + 128; i += blockDim.x) {
    const int s = i / 128, k = i % 128;
    uint8_t* d = s < ST ? smem + s * stage_bytes + (k < 64 ? k * 16 : wrows * 128 + (k - 64) * 16) : zero + k * 16;
    *(uint4*)d = make_uint4(0, 0, 0, 0);
  }
  if (threadIdx.x == 0) {
    for (int s = 0; s < ST; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], a.cs_part ? 4 : 1);  // MMA commit (+ one arrive per column-sum warp)
    }
    mbar_init(tfull, 1);
    mbar_init(tempty, 128);
    fence_mbar_init();
    tma_prefetch_desc(&a.x_map);
    tma_prefetch_desc(&a.dz_map);
  }
  if (warp == 4) tmem_alloc<512>(tmem_slot);
  fence_proxy_async_smem();
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  const uint32_t sbase = smem_u32(smem);

  if (warp == 0) {
    if (lane == 0) {
      const uint32_t xbytes = 64u * 2u * Wp * (R + 2), zbytes = (uint32_t)b_bytes;
      int it = 0;
      for (int u = blockIdx.x; u < nunit; u += gridDim.x) {
        const int t = u % tiles, z = u / tiles;
        const int cb = t % a.ncb, nb = t / a.ncb;
        const int kb0 = z * a.kb_per_split, kb1 = min(kb0 + a.kb_per_split, nkb);
        for (int kb = kb0; kb < kb1; ++kb, ++it) {
          const int s = it % ST, ph = it / ST;
          if (ph > 0) mbar_wait(&empty[s], (ph - 1) & 1);
          const int img = kb / a.rg, h0 = (kb - img * a.rg) * R;
          const uint32_t sa = sbase + s * stage_bytes;
          mbar_expect_tx(&full[s], xbytes + zbytes);
          tma_load_4d(sa + 1024, &a.x_map, &full[s], cb * 64, 0, h0 - 1, img);
          tma_load_4d(sa + a.a_bytes, &a.dz_map, &full[s], nb * 64, 0, h0, img);
        }
      }
    }
  } else if (warp == 4) {
    constexpr uint32_t IDESC = make_idesc(BM, 64, 1, 1);
    const uint32_t zaddr = smem_u32(zero);
    const int ksteps = R * Wp / 16;
    int off[10];
#pragma unroll
    for (int tp = 0; tp < 9; ++tp) off[tp] = (8 + (tp / 3) * Wp + (tp % 3) - 1) * 128;
    int it = 0, lt = 0;
    for (int u = blockIdx.x; u < nunit; u += gridDim.x, ++lt) {
      const int z = u / tiles;
      const int kb0 = z * a.kb_per_split, kb1 = min(kb0 + a.kb_per_split, nkb);
      if (lt > 0) mbar_wait(tempty, (lt - 1) & 1);
      tc_fence_after();
      for (int kb = kb0; kb < kb1; ++kb, ++it) {
        const int s = it % ST, ph = it / ST;
        mbar_wait(&full[s], ph & 1);
        tc_fence_after();
        if (elect_one()) {
          const uint32_t sa = sbase + s * stage_bytes, sb = sa + a.a_bytes;
          // descriptors for K-step 0; each further K-step (16 pixel rows = 2048 B) adds 128 to the address field
          uint64_t da[5];
#pragma unroll
          for (int p = 0; p < 5; ++p) {
            const uint32_t a0 = sa + off[2 * p];
            const uint32_t a1 = p < 4 ? sa + off[2 * p + 1] : zaddr;
            da[p] = make_sdesc(a0, a1 - a0, 1024);
          }
          const uint64_t db0 = make_sdesc(sb, 8192, 1024);
          const uint32_t acc0 = kb != kb0;
          // the five tap-pair MMAs of a K-step share B (the dZ slice): read it once into the weight-stationary
          // collector (fill / use / lastuse)
          umma_bf16_ws_fill(tmem, da[0], db0, IDESC, acc0);
#pragma unroll
          for (int p = 1; p < 4; ++p) umma_bf16_ws_use(tmem + (uint32_t)(p * 64), da[p], db0, IDESC, acc0);
          umma_bf16_ws_lastuse(tmem + 256u, da[4], db0, IDESC, acc0);
          for (int kk = 1; kk < ksteps; ++kk) {
            const uint64_t inc = (uint64_t)(kk * 128);
            umma_bf16_ws_fill(tmem, da[0] + inc, db0 + inc, IDESC, 1u);
#pragma unroll
            for (int p = 1; p < 4; ++p) umma_bf16_ws_use(tmem + (uint32_t)(p * 64), da[p] + inc, db0 + inc, IDESC, 1u);
            // the tenth atom (zero) stays in place: LBO shrinks by the same 2048 B per K-step
            umma_bf16_ws_lastuse(tmem + 256u, da[4] + inc - ((uint64_t)(kk * 128) << 16), db0 + inc, IDESC, 1u);
          }
          umma_commit(&empty[s]);
          if (kb == kb1 - 1) umma_commit(tfull);
        }
        __syncwarp();
      }
      if (kb1 <= kb0 && lane == 0) mbar_arrive(tfull);
      __syncwarp();
    }
  } else if (warp >= 1 && warp <= 3) {
    if (a.cs_part) {
      // fused bias gradient: tiles with cb == 0 see every (pixel, co) of their co block exactly once
      TileColsum<64> cs;
      const int t = threadIdx.x - 32;
      cs.init(t);
      int it = 0;
      for (int u = blockIdx.x; u < nunit; u += gridDim.x) {
        const int tl = u % tiles, z = u / tiles;
        const int cb = tl % a.ncb, nb = tl / a.ncb;
        const int kb0 = z * a.kb_per_split, kb1 = min(kb0 + a.kb_per_split, nkb);
        cs.zero();
        for (int kb = kb0; kb < kb1; ++kb, ++it) {
          const int s = it % ST, ph = it / ST;
          mbar_wait(&full[s], ph & 1);
          if (cb == 0) cs.add(smem + s * stage_bytes + a.a_bytes, R * Wp);
          __syncwarp();
          if (lane == 0) mbar_arrive(&empty[s]);
        }
        if (cb == 0) cs.finish(cs_red, a.cs_part + (long long)z * a.Cout + nb * 64, 64, t);
      }
    }
  } else if (warp >= 5) {
    const int qd = warp & 3;
    const int row = qd * 32 + lane;
    const int Kconv = 9 * a.Cin;
    int lt = 0;
    for (int u = blockIdx.x; u < nunit; u += gridDim.x, ++lt) {
      const int t = u % tiles, z = u / tiles;
      const int cb = t % a.ncb, nb = t / a.ncb;
      const int kb0 = z * a.kb_per_split, kb1 = min(kb0 + a.kb_per_split, nkb);
      mbar_wait(tfull, lt & 1);
      tc_fence_after();
      const uint32_t trow = tmem + ((uint32_t)(qd * 32) << 16);
#pragma unroll 1
      for (int p = 0; p < 5; ++p) {
        const int tap = 2 * p + (row >> 6);
        const int kc = tap * a.Cin + cb * 64 + (row & 63);
        float* outp = a.out + ((long long)z * Kconv + kc) * a.Cout + nb * 64;
#pragma unroll 1
        for (int c0 = 0; c0 < 64; c0 += 32) {
          float v[32];
          if (kb1 > kb0) tmem_ld32(trow + p * 64 + c0, v);
          else
#pragma unroll
            for (int i = 0; i < 32; ++i) v[i] = 0.f;
          if (tap < 9)
#pragma unroll
            for (int i = 0; i < 32; i += 4) *(float4*)(outp + c0 + i) = make_float4(v[i], v[i + 1], v[i + 2], v[i + 3]);
        }
      }
      tc_fence_before();
      mbar_arrive(tempty);
    }
  }

  tc_fence_before();
  __syncthreads();
  if (warp == 4) {
    tc_fence_after();
    tmem_dealloc<512>(tmem);
  }
}

}  // namespace adainf

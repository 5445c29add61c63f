// Implicit-GEMM convolution on the 5th-gen tensor cores (tcgen05.mma kind::f16, fp32 accumulator in
// TMEM), one kernel template for the three contractions of the hot path:
//
//   FWD   D[pix][co]   = sum_{tap,ci} X[gather(pix,tap)][ci] * W[co][tap][ci]        A K-major, B K-major
//   DGRAD D[pix'][ci]  = sum_{tap',co} dZ[gather(pix',tap')][co] * W[co][tap(tap')][ci]  A K-major, B MN-major
//   WGRAD D[kconv][co] = sum_{pix} X[gather(pix,tap(kconv))][ci(kconv)] * dZ[pix][co]   A MN-major, B MN-major
//
// "Run one layer for all requests of the batch at once" is inherent: M spans every pixel of
// every sample of the (compacted) batch.  Operands are gathered by 4 producer warps with 16-byte
// cp.async (zero-fill for padding / out-of-range taps / rows beyond the device-side sample count) into
// 128B-swizzled UMMA tiles; one elected thread of warp 4 issues the MMAs; the producer warps then run
// the fused epilogue (TMEM -> registers -> bias / residual / activation / gradient masks -> HBM).
#pragma once
#include "common.cuh"

namespace adainf {

enum { MODE_FWD = 0, MODE_DGRAD = 1, MODE_WGRAD = 2 };
constexpr int MAX_TAPS = 49;

struct ConvArgs {
  // ---- gather source (A for FWD/DGRAD, im2col A for WGRAD) ----
  const bf16* src;      // NHWC [*][Hs][Ws][Cs]
  const int* src_map;   // optional: dense sample n -> source sample
  int Hs, Ws, Cs;
  // ---- pixel space (rows for FWD/DGRAD, reduction for WGRAD) ----
  const int* count;     // device sample count (nullptr -> n_static)
  int n_static;
  int Hg, Wg, sy, sx;
  int ntaps;
  int8_t ty[MAX_TAPS], tx[MAX_TAPS];
  // ---- B operand ----
  const bf16* B;        // FWD: W [Nout][ldb]; DGRAD: W [Cout][ldb] (fwd layout); WGRAD: dZ [pix][Nout]
  int ldb;
  int16_t btap[MAX_TAPS];  // DGRAD: forward tap index of phase tap t'
  int K;                // FWD: ntaps*Cs, DGRAD: ntaps*Cs (Cs = Cout), WGRAD: M extent = ntaps*Cs (kconv)
  int Nout;
  // ---- epilogue ----
  void* out;            // FWD/DGRAD: NHWC [*][Ho][Wo][Nout]; WGRAD: fp32 partial [split][Kconv][Nout]
  int out_f32;
  int Ho, Wo, oys, oxs, oyo, oxo;
  const float* bias;    // FWD
  const bf16* res;      // FWD residual (same geometry as out)
  const int* res_map;
  int act;              // FWD activation
  const float* bcast;   // DGRAD: + bcast[n][ch] (exit-head GAP gradient, pre-scaled by 1/HW)
  const bf16* sc;       // DGRAD: + shortcut gradient (same geometry as out)
  const bf16* yact;     // DGRAD: stored activation for the act' mask
  int mask_act;         // DGRAD: activation whose derivative masks (0 = none)
  int kb_per_split;     // WGRAD split-K (in 64-pixel blocks)
};

constexpr int BM = 128, BK = 64;
constexpr int NUM_THREADS = 160;  // warps 0-3 producers + epilogue, warp 4 MMA issuer / TMEM owner

template <int MODE, int BN>
struct ConvCfg {
  static constexpr int STAGES = BN >= 256 ? 4 : (BN >= 128 ? 3 : 4);
  static constexpr int A_BYTES = BM * BK * 2;
  static constexpr int B_BYTES = BN * BK * 2;
  static constexpr int STAGE_BYTES = A_BYTES + B_BYTES;
  static constexpr int SMEM = STAGES * STAGE_BYTES + 1024 /*align*/ + 256 /*barriers*/;
  static constexpr int TMEM_COLS = BN < 32 ? 32 : BN;
};

// 128B-swizzle offsets inside a tile (bytes).
// K-major tile [rows][64 elems]: row r, 16B chunk j.
__device__ __forceinline__ uint32_t kmaj_off(int r, int j) {
  return (uint32_t)((r >> 3) * 1024 + (r & 7) * 128 + ((j ^ (r & 7)) << 4));
}
// MN-major tile [K=64 rows][MN elems]: K row r, MN 16B chunk j (8 elems), atoms of 64 MN elems.
__device__ __forceinline__ uint32_t mnmaj_off(int r, int j) {
  return (uint32_t)((j >> 3) * 8192 + (r >> 3) * 1024 + (r & 7) * 128 + (((j & 7) ^ (r & 7)) << 4));
}

template <int MODE, int BN>
__global__ void __launch_bounds__(NUM_THREADS, 1) conv_umma_kernel(const ConvArgs a) {
  using Cfg = ConvCfg<MODE, BN>;
  static_assert(MODE == MODE_FWD || BN >= 64, "MN-major SW128 B tiles need >= 64 columns");
  constexpr int STAGES = Cfg::STAGES;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  uint64_t* full = (uint64_t*)(smem + STAGES * Cfg::STAGE_BYTES);
  uint64_t* empty = full + STAGES;
  uint64_t* tfull = empty + STAGES;
  uint32_t* tmem_slot = (uint32_t*)(tfull + 1);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int nsamp = a.count ? *a.count : a.n_static;
  const int HWg = a.Hg * a.Wg;
  const long long npix = (long long)nsamp * HWg;

  // tile coordinates
  long long m0;
  int n0, kb0, kb1;
  const int nkb_total = (MODE == MODE_WGRAD) ? (int)((npix + BK - 1) / BK) : (a.K + BK - 1) / BK;
  if (MODE == MODE_WGRAD) {
    m0 = (long long)blockIdx.x * BM;  // kconv
    n0 = blockIdx.y * BN;             // co
    kb0 = blockIdx.z * a.kb_per_split;
    kb1 = min(kb0 + a.kb_per_split, nkb_total);
    if (m0 >= a.K) return;
  } else {
    m0 = (long long)blockIdx.x * BM;  // pixel
    n0 = blockIdx.y * BN;
    kb0 = 0;
    kb1 = nkb_total;
    if (m0 >= npix) return;           // rows beyond the device-side count: nothing to do
  }
  const int nkb = max(kb1 - kb0, 0);

  if (threadIdx.x == 0) {
    for (int s = 0; s < STAGES; ++s) {
      mbar_init(&full[s], 128);
      mbar_init(&empty[s], 1);
    }
    mbar_init(tfull, 1);
    fence_mbar_init();
  }
  if (warp == 4) tmem_alloc<Cfg::TMEM_COLS>(tmem_slot);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  const uint32_t smem_base = smem_u32(smem);

  if (warp < 4) {
    // ================= producers =================
    const int t = threadIdx.x;  // 0..127
    if (MODE != MODE_WGRAD) {
      // A: 128 rows (pixels) x 8 chunks; thread -> chunk t&7, rows (t>>3)+16*i
      const int j = t & 7;
      long long rowbase[8];
      int iy0[8], ix0[8];
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        const long long m = m0 + (t >> 3) + 16 * i;
        if (m < npix) {
          const int n = (int)(m / HWg);
          const int pix = (int)(m - (long long)n * HWg);
          const int gy = pix / a.Wg, gx = pix - (pix / a.Wg) * a.Wg;
          const int sn = a.src_map ? a.src_map[n] : n;
          rowbase[i] = (long long)sn * a.Hs * a.Ws;
          iy0[i] = gy * a.sy;
          ix0[i] = gx * a.sx;
        } else {
          rowbase[i] = -1;
          iy0[i] = 0;
          ix0[i] = 0;
        }
      }
      for (int kbi = 0; kbi < nkb; ++kbi) {
        const int s = kbi % STAGES, u = kbi / STAGES;
        if (u > 0) mbar_wait(&empty[s], (u - 1) & 1);
        const uint32_t sa = smem_base + s * Cfg::STAGE_BYTES;
        const uint32_t sb = sa + Cfg::A_BYTES;
        const int k = (kb0 + kbi) * BK + j * 8;
        const int tap = k / a.Cs;
        const int c = k - tap * a.Cs;
        const bool kval = k < a.K;
        const int dy = kval ? a.ty[tap] : 0, dx = kval ? a.tx[tap] : 0;
#pragma unroll
        for (int i = 0; i < 8; ++i) {
          const int r = (t >> 3) + 16 * i;
          const int iy = iy0[i] + dy, ix = ix0[i] + dx;
          const bool v = kval && rowbase[i] >= 0 && iy >= 0 && iy < a.Hs && ix >= 0 && ix < a.Ws;
          const bf16* g = v ? a.src + ((rowbase[i] + (long long)iy * a.Ws + ix) * a.Cs + c) : a.src;
          cp_async16(sa + kmaj_off(r, j), g, v);
        }
        // B
        if (MODE == MODE_FWD) {
          // W [Nout][ldb] K-major: BN rows x 8 chunks
          for (int idx = t; idx < BN * 8; idx += 128) {
            const int r = idx >> 3, jj = idx & 7;
            const int kk = (kb0 + kbi) * BK + jj * 8;
            const bool v = (n0 + r) < a.Nout && kk < a.K;
            const bf16* g = v ? a.B + ((long long)(n0 + r) * a.ldb + kk) : a.B;
            cp_async16(sb + kmaj_off(r, jj), g, v);
          }
        } else {
          // DGRAD: B MN-major [K=64 (tap',co) rows][BN ci]: element (k=(t',co), n=ci) = W[co][btap[t']][ci]
          constexpr int CH = BN / 8;
          for (int idx = t; idx < 64 * CH; idx += 128) {
            const int r = idx / CH, jj = idx - (idx / CH) * CH;
            const int kk = (kb0 + kbi) * BK + r;
            const int tp = kk / a.Cs;
            const int co = kk - tp * a.Cs;
            const int ci = n0 + jj * 8;
            const bool v = kk < a.K && ci < a.Nout;
            const bf16* g = v ? a.B + ((long long)co * a.ldb + (long long)a.btap[tp] * a.Nout + ci) : a.B;
            cp_async16(sb + mnmaj_off(r, jj), g, v);
          }
        }
        cp_async_arrive_noinc(&full[s]);
      }
    } else {
      // WGRAD: A MN-major [K=64 pixels][128 kconv]; thread -> kconv chunk j = t&15, pixels (t>>4)+8*i
      const int j = t & 15;
      const int kc = (int)m0 + j * 8;
      const bool mval = kc < a.K;
      const int tap = mval ? kc / a.Cs : 0;
      const int c = kc - tap * a.Cs;
      const int dy = a.ty[tap], dx = a.tx[tap];
      for (int kbi = 0; kbi < nkb; ++kbi) {
        const int s = kbi % STAGES, u = kbi / STAGES;
        if (u > 0) mbar_wait(&empty[s], (u - 1) & 1);
        const uint32_t sa = smem_base + s * Cfg::STAGE_BYTES;
        const uint32_t sb = sa + Cfg::A_BYTES;
        const long long p0 = (long long)(kb0 + kbi) * BK;
#pragma unroll
        for (int i = 0; i < 8; ++i) {
          const int r = (t >> 4) + 8 * i;
          const long long p = p0 + r;
          bool v = mval && p < npix;
          const bf16* g = a.src;
          if (v) {
            const int n = (int)(p / HWg);
            const int pix = (int)(p - (long long)n * HWg);
            const int gy = pix / a.Wg, gx = pix - (pix / a.Wg) * a.Wg;
            const int iy = gy * a.sy + dy, ix = gx * a.sx + dx;
            v = iy >= 0 && iy < a.Hs && ix >= 0 && ix < a.Ws;
            const int sn = a.src_map ? a.src_map[n] : n;
            if (v) g = a.src + ((((long long)sn * a.Hs + iy) * a.Ws + ix) * a.Cs + c);
          }
          cp_async16(sa + mnmaj_off(r, j), g, v);
        }
        // B: dZ [pix][Nout] MN-major [64 pixels][BN co]
        constexpr int CH = BN / 8;
        for (int idx = t; idx < 64 * CH; idx += 128) {
          const int r = idx / CH, jj = idx - (idx / CH) * CH;
          const long long p = p0 + r;
          const bool v = p < npix && (n0 + jj * 8) < a.Nout;
          const bf16* g = v ? a.B + (p * a.Nout + n0 + jj * 8) : a.B;
          cp_async16(sb + mnmaj_off(r, jj), g, v);
        }
        cp_async_arrive_noinc(&full[s]);
      }
    }

    // ================= epilogue =================
    mbar_wait(tfull, 0);
    tc_fence_after();
    const int row = warp * 32 + lane;
    const long long m = m0 + row;
    const uint32_t trow = tmem + ((uint32_t)(warp * 32) << 16);
    if (MODE == MODE_WGRAD) {
      float* outp = (float*)a.out + ((long long)blockIdx.z * a.K + m) * a.Nout + n0;
      for (int c0 = 0; c0 < BN; c0 += 32) {
        float v[32];
        if (nkb > 0) tmem_ld32(trow + c0, v);  // whole warp (.sync.aligned), stores predicated below
        else
#pragma unroll
          for (int i = 0; i < 32; ++i) v[i] = 0.f;
        if (m >= a.K) continue;
        if (n0 + c0 + 32 <= a.Nout && (a.Nout & 3) == 0) {
#pragma unroll
          for (int i = 0; i < 32; i += 4)
            *(float4*)(outp + c0 + i) = make_float4(v[i], v[i + 1], v[i + 2], v[i + 3]);
        } else {
          for (int i = 0; i < 32; ++i)
            if (n0 + c0 + i < a.Nout) outp[c0 + i] = v[i];
        }
      }
    } else {
      const bool rv = m < npix;
      long long orow = 0;
      int n = 0;
      if (rv) {
        n = (int)(m / HWg);
        const int pix = (int)(m - (long long)n * HWg);
        const int gy = pix / a.Wg, gx = pix - (pix / a.Wg) * a.Wg;
        orow = ((long long)n * a.Ho + gy * a.oys + a.oyo) * a.Wo + gx * a.oxs + a.oxo;
      }
      for (int c0 = 0; c0 < BN; c0 += 32) {
        float v[32];
        if (nkb > 0) tmem_ld32(trow + c0, v);
        else
#pragma unroll
          for (int i = 0; i < 32; ++i) v[i] = 0.f;
        if (!rv) continue;
        const int cb = n0 + c0;
        if (cb >= a.Nout) continue;
        const bool full32 = (cb + 32 <= a.Nout) && ((a.Nout & 7) == 0);
        if (MODE == MODE_FWD) {
          long long rrow = 0;
          if (a.res) {
            const long long pix_o = orow - (long long)n * a.Ho * a.Wo;
            const int rn = a.res_map ? a.res_map[n] : n;
            rrow = (long long)rn * a.Ho * a.Wo + pix_o;
          }
#pragma unroll
          for (int i = 0; i < 32; ++i) {
            const int ch = cb + i;
            if (!full32 && ch >= a.Nout) break;
            float x = __fadd_rn(v[i], a.bias[ch]);
            if (a.res) x = __fadd_rn(x, __bfloat162float(a.res[rrow * a.Nout + ch]));
            v[i] = act_apply(a.act, x);
          }
          if (a.out_f32) {
            float* o = (float*)a.out + orow * a.Nout + cb;
            for (int i = 0; i < 32; ++i)
              if (cb + i < a.Nout) o[i] = v[i];
          } else {
            bf16* o = (bf16*)a.out + orow * a.Nout + cb;
            if (full32) {
#pragma unroll
              for (int i = 0; i < 32; i += 8) {
                __align__(16) bf16 h[8];
#pragma unroll
                for (int q = 0; q < 8; ++q) h[q] = __float2bfloat16_rn(v[i + q]);
                *(uint4*)(o + i) = *(uint4*)h;
              }
            } else {
              for (int i = 0; i < 32; ++i)
                if (cb + i < a.Nout) o[i] = __float2bfloat16_rn(v[i]);
            }
          }
        } else {  // DGRAD epilogue: + bcast + shortcut, x act'(y), -> bf16
          bf16* o = (bf16*)a.out + orow * a.Nout + cb;
          for (int i = 0; i < 32; ++i) {
            const int ch = cb + i;
            if (ch >= a.Nout) break;
            float x = v[i];
            if (a.bcast) x = __fadd_rn(x, a.bcast[(long long)n * a.Nout + ch]);
            if (a.sc) x = __fadd_rn(x, __bfloat162float(a.sc[orow * a.Nout + ch]));
            if (a.mask_act) x = __fmul_rn(x, act_grad(a.mask_act, __bfloat162float(a.yact[orow * a.Nout + ch])));
            o[i] = __float2bfloat16_rn(x);
          }
        }
      }
    }
  } else if (warp == 4) {
    // ================= MMA issuer =================
    if (nkb > 0) {
      constexpr uint32_t IDESC = make_idesc(BM, BN, MODE == MODE_WGRAD ? 1 : 0, MODE == MODE_FWD ? 0 : 1);
      for (int kbi = 0; kbi < nkb; ++kbi) {
        const int s = kbi % STAGES, u = kbi / STAGES;
        mbar_wait(&full[s], u & 1);
        fence_proxy_async_smem();
        tc_fence_after();
        if (lane == 0) {
          const uint32_t sa = smem_base + s * Cfg::STAGE_BYTES;
          const uint32_t sb = sa + Cfg::A_BYTES;
#pragma unroll
          for (int kk = 0; kk < BK / 16; ++kk) {
            uint64_t ad, bd;
            if (MODE == MODE_WGRAD) ad = make_sdesc(sa + kk * 2048, 8192, 1024);
            else ad = make_sdesc(sa + kk * 32, 16, 1024);
            if (MODE == MODE_FWD) bd = make_sdesc(sb + kk * 32, 16, 1024);
            else bd = make_sdesc(sb + kk * 2048, 8192, 1024);
            umma_bf16(tmem, ad, bd, IDESC, (kbi | kk) != 0);
          }
          umma_commit(&empty[s]);
          if (kbi == nkb - 1) umma_commit(tfull);
        }
        __syncwarp();
      }
    } else if (lane == 0) {
      mbar_arrive(tfull);
    }
    __syncwarp();
  }

  tc_fence_before();
  __syncthreads();
  if (warp == 4) {
    tc_fence_after();
    tmem_dealloc<Cfg::TMEM_COLS>(tmem);
  }
}

}  // namespace adainf

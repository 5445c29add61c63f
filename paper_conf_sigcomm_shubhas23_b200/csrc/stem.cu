// ResNet stem kernels (see stem.cuh for the space-to-depth formulation).
#include <algorithm>
#include <cmath>

#include "colsum_tile.cuh"
#include "conv_gemm.cuh"
#include "pool_bwd.cuh"
#include "prof.h"
#include "runtime.h"
#include "stem.cuh"
#include "tma.cuh"

namespace adainf {

bool stem_s2d_ok(int H, int W, int cin, int cout, int KH, int KW, int stride, int pad) {
  return KH == 7 && KW == 7 && stride == 2 && pad == 3 && cin >= 1 && cin <= 4 && cout == 64 && H % 2 == 0 &&
         W % 2 == 0 && W / 2 <= 125 && H >= 4 && W >= 4;
}

// ---- packing -----------------------------------------------------------------------------------------
__global__ void pack_s2d_kernel(const bf16* __restrict__ x, const int* __restrict__ map, const int* count,
                                int n_static, int H, int W, int cin, bf16* __restrict__ s) {
  const int n_rows = count ? *count : n_static;
  const int Hs = H / 2, Ws = W / 2;
  const long long total = (long long)n_rows * Hs * Ws;
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < total; i += (long long)gridDim.x * blockDim.x) {
    const long long n = i / (Hs * Ws);
    const int rem = (int)(i - n * Hs * Ws);
    const int si = rem / Ws, sj = rem - si * Ws;
    const long long src = map ? map[n] : n;
    if (src < 0) {  // sanitised row (retrain_step_rows: past the device count / out of range): zero input
      uint4* o = (uint4*)(s + i * 16);
      o[0] = make_uint4(0, 0, 0, 0);
      o[1] = make_uint4(0, 0, 0, 0);
      continue;
    }
    if (cin == 3) {
      // the two pixels of one input row are 12 contiguous, 4-byte aligned bytes (W even): three 32-bit loads
      // per row; channel 3 of each pixel is the zero pad
      uint4 o2[2];
#pragma unroll
      for (int bh = 0; bh < 2; ++bh) {
        const uint32_t* pw = (const uint32_t*)(x + ((src * H + 2 * si + bh) * W + 2 * sj) * 3);
        const uint32_t w0 = __ldg(pw), w1 = __ldg(pw + 1), w2 = __ldg(pw + 2);
        o2[bh] = make_uint4(w0, w1 & 0xFFFFu, (w1 >> 16) | (w2 << 16), w2 >> 16);
      }
      uint4* o = (uint4*)(s + i * 16);
      o[0] = o2[0];
      o[1] = o2[1];
      continue;
    }
    __align__(16) bf16 v[16];
#pragma unroll
    for (int bh = 0; bh < 2; ++bh)
#pragma unroll
      for (int bw = 0; bw < 2; ++bw) {
        const bf16* px = x + ((src * H + 2 * si + bh) * W + 2 * sj + bw) * cin;
#pragma unroll
        for (int c = 0; c < 4; ++c) v[(bh * 2 + bw) * 4 + c] = c < cin ? px[c] : __float2bfloat16_rn(0.f);
      }
    uint4* o = (uint4*)(s + i * 16);
    o[0] = ((const uint4*)v)[0];
    o[1] = ((const uint4*)v)[1];
  }
}

void launch_pack_s2d(const bf16* x, const int* map, const int* count, int n_static, int H, int W, int cin, bf16* s,
                     cudaStream_t st) {
  const long long total = (long long)n_static * (H / 2) * (W / 2);
  const int blocks = (int)std::min<long long>((total + 255) / 256, 16LL * num_sms());
  if (blocks <= 0) return;
  ProfScope ps(PC_PACK, st);
  pack_s2d_kernel<<<blocks, 256, 0, st>>>(x, map, count, n_static, H, W, cin, s);
  CK(cudaGetLastError());
}

// wprep[t][p][co][j]: tap t = (ah+2)*4 + (aw+2), s2d channel ch = p*8 + j = (bh*2 + bw)*4 + c
__global__ void stem_wprep_kernel(const bf16* __restrict__ shadow, int ldb, bf16* __restrict__ wprep) {
  const int idx = blockIdx.x * blockDim.x + threadIdx.x;
  if (idx >= 16 * 2 * 64 * 8) return;
  const int j = idx & 7, co = (idx >> 3) & 63, p = (idx >> 9) & 1, t = idx >> 10;
  const int ch = p * 8 + j;
  const int bh = ch >> 3, bw = (ch >> 2) & 1, c = ch & 3;
  const int kh = 2 * (t / 4 - 2) + bh + 3, kw = 2 * (t % 4 - 2) + bw + 3;
  bf16 v = __float2bfloat16_rn(0.f);
  if (kh >= 0 && kh < 7 && kw >= 0 && kw < 7) v = shadow[(long long)co * ldb + (kh * 7 + kw) * 4 + c];
  wprep[idx] = v;
}

void launch_stem_wprep(const bf16* shadow, int ldb, bf16* wprep, cudaStream_t st) {
  ProfScope ps(PC_STEM_AUX, st);
  stem_wprep_kernel<<<64, 256, 0, st>>>(shadow, ldb, wprep);
  CK(cudaGetLastError());
}

// pick a row-band split of the images so that units fill whole waves of #SMs; `halo` rows are
// recomputed / reloaded per band
static void pick_bands(int n, int rows, int halo, int* bands, int* band_rows) {
  const int G = num_sms();
  double best = -1;
  *bands = 1;
  *band_rows = rows;
  for (int b = 1; b <= 16 && b <= rows; ++b) {
    const int br = (rows + b - 1) / b;
    const int nb = (rows + br - 1) / br;
    const long long units = (long long)n * nb;
    const long long waves = (units + G - 1) / G;
    const double eff = (double)units / (double)(waves * G) * (double)rows / (double)(rows + (nb - 1) * halo);
    if (eff > best + 1e-9) {
      best = eff;
      *bands = nb;
      *band_rows = br;
    }
  }
}

// =====================================================================================================
// forward: conv + bias + ReLU + max-pool(3, 2, 1)
// =====================================================================================================
constexpr int SF_THREADS = 416;  // warp 0 TMA, warp 4 MMA, warps 5..12 epilogue (two per TMEM lane quadrant)
constexpr int SLOTS = 128;       // padded columns of one output row = the M tile
// window: 4 s2d rows x 128 positions x 32 B (SWIZZLE_32B: 16-byte chunk ^= row bit 2), + 8 trail rows
constexpr int SF_STAGE = ((4 * SLOTS + 8) * 32 + 1023) / 1024 * 1024;
constexpr int SF_STAGES = 6;
constexpr int SF_W_BYTES = 16 * 2048;
constexpr int SF_RING = 4;  // conv-row ring: bf16 [SLOTS][64], 16-byte chunk k of column x at k ^ (x & 7)
constexpr int SF_SMEM = 1024 + SF_W_BYTES + SF_STAGES * SF_STAGE + SF_RING * SLOTS * 128 + 256;

struct StemFwdArgs {
  CUtensorMap s_map;  // S2D [n][Hs][Ws][16], box {16, 128, 4, 1}, 32B swizzle
  const bf16* wprep;
  const float* bias;
  const int* count;
  int n_static, Hs, Ws, Hp, Wp, bands, band_rows;
  bf16* pooled;
  uint8_t* argmax;
};

struct StemUnit {
  int img, po0, po1, r0, r1;
};
__device__ __forceinline__ StemUnit stem_unit(const StemFwdArgs& a, int u) {
  StemUnit s;
  s.img = u / a.bands;
  const int band = u - s.img * a.bands;
  s.po0 = band * a.band_rows;
  s.po1 = min(a.Hp, s.po0 + a.band_rows);
  s.r0 = max(0, 2 * s.po0 - 1);
  s.r1 = min(a.Hs - 1, 2 * (s.po1 - 1) + 1);
  return s;
}

__global__ void __launch_bounds__(SF_THREADS, 1) stem_fwd_kernel(const __grid_constant__ StemFwdArgs a) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = smem_align1024(smem_raw);
  uint8_t* wsm = smem;
  uint8_t* stages = wsm + SF_W_BYTES;
  uint8_t* ring = stages + SF_STAGES * SF_STAGE;
  uint64_t* full = (uint64_t*)(ring + SF_RING * SLOTS * 128);
  uint64_t* empty = full + SF_STAGES;
  uint64_t* tfull = empty + SF_STAGES;
  uint64_t* tempty = tfull + 2;
  uint32_t* tmem_slot = (uint32_t*)(tempty + 2);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int nimg = a.count ? min(*a.count, a.n_static) : a.n_static;
  const int nunits = nimg * a.bands;
  if ((int)blockIdx.x >= nunits) return;

  // resident weights (written by the generic proxy, read by the tensor core: proxy fence below)
  for (int i = threadIdx.x; i < SF_W_BYTES / 16; i += blockDim.x)
    ((uint4*)wsm)[i] = __ldg((const uint4*)a.wprep + i);
  if (threadIdx.x == 0) {
    for (int s = 0; s < SF_STAGES; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], 1);
    }
    for (int b = 0; b < 2; ++b) {
      mbar_init(&tfull[b], 1);
      mbar_init(&tempty[b], 256);
    }
    fence_mbar_init();
    tma_prefetch_desc(&a.s_map);
  }
  if (warp == 4) tmem_alloc<128>(tmem_slot);
  fence_proxy_async_smem();
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  const uint32_t st_base = smem_u32(stages);

  if (warp == 0) {
    if (lane == 0) {
      int it = 0;
      for (int u = blockIdx.x; u < nunits; u += gridDim.x) {
        const StemUnit su = stem_unit(a, u);
        for (int r = su.r0; r <= su.r1; ++r, ++it) {
          const int s = it % SF_STAGES, ph = it / SF_STAGES;
          if (ph > 0) mbar_wait(&empty[s], (ph - 1) & 1);
          mbar_expect_tx(&full[s], 4 * SLOTS * 32);
          tma_load_4d(st_base + s * SF_STAGE, &a.s_map, &full[s], 0, -2, r - 2, su.img);
        }
      }
    }
  } else if (warp == 4) {
    constexpr uint32_t IDESC = make_idesc(128, 64, 0, 0);
    const uint64_t bdesc0 = make_sdesc_plain(smem_u32(wsm), 1024, 128);
    int it = 0;
    for (int u = blockIdx.x; u < nunits; u += gridDim.x) {
      const StemUnit su = stem_unit(a, u);
      for (int r = su.r0; r <= su.r1; ++r, ++it) {
        const int b = it & 1, ub = it >> 1;
        if (ub > 0) mbar_wait(&tempty[b], (ub - 1) & 1);
        const int s = it % SF_STAGES, ph = it / SF_STAGES;
        mbar_wait(&full[s], ph & 1);
        tc_fence_after();
        if (elect_one()) {
          // K-major SWIZZLE_32B: one 32-byte row (16 channels = K) per position, 8-row groups 256 B apart;
          // tap (ah, aw) = the window shifted by (ah+2)*128 + (aw+2) rows (swizzle follows address bits)
          const uint64_t adesc0 = make_sdesc_sw32(st_base + s * SF_STAGE, 16, 256);
#pragma unroll
          for (int t = 0; t < 16; ++t) {
            const uint32_t row_off = (uint32_t)((t >> 2) * SLOTS + (t & 3));
            umma_bf16(tmem + (uint32_t)(b * 64), adesc0 + (uint64_t)(row_off * 2), bdesc0 + (uint64_t)(t * 128), IDESC,
                      t > 0);
          }
          umma_commit(&empty[s]);
          umma_commit(&tfull[b]);
        }
        __syncwarp();
      }
    }
  } else if (warp >= 5) {
    const int e = warp - 5, qd = warp & 3, half = e >> 2;
    const int x = qd * 32 + lane;
    const int t = threadIdx.x - 160;  // 0..255
    float bz[32];
#pragma unroll
    for (int i = 0; i < 32; ++i) bz[i] = __ldg(a.bias + half * 32 + i);
    int it = 0;
    for (int u = blockIdx.x; u < nunits; u += gridDim.x) {
      const StemUnit su = stem_unit(a, u);
      for (int r = su.r0; r <= su.r1; ++r, ++it) {
        const int b = it & 1, ub = it >> 1;
        mbar_wait(&tfull[b], ub & 1);
        tc_fence_after();
        float v[32];
        tmem_ld32(tmem + (uint32_t)(b * 64 + half * 32) + ((uint32_t)(qd * 32) << 16), v);
        tc_fence_before();
        mbar_arrive(&tempty[b]);
        if (x < a.Ws) {
          uint8_t* rowp = ring + (r & 3) * SLOTS * 128 + x * 128;
#pragma unroll
          for (int j = 0; j < 4; ++j) {
            __align__(16) __nv_bfloat162 o[4];
#pragma unroll
            for (int q = 0; q < 4; ++q) {
              const float y0 = act_apply(1, v[j * 8 + 2 * q] + bz[j * 8 + 2 * q]);
              const float y1 = act_apply(1, v[j * 8 + 2 * q + 1] + bz[j * 8 + 2 * q + 1]);
              o[q] = __floats2bfloat162_rn(y0, y1);
            }
            const int k = half * 4 + j;
            *(uint4*)(rowp + ((k ^ (x & 7)) << 4)) = *(const uint4*)o;
          }
        }
        asm volatile("bar.sync 2, 256;" ::: "memory");
        // pooled row whose last input row is r
        int po = -1;
        if (r & 1) po = (r - 1) >> 1;
        else if (r == a.Hs - 1) po = r >> 1;
        if (po < su.po0 || po >= su.po1) continue;
        for (int item = t; item < a.Wp * 8; item += 256) {
          const int pw = item >> 3, k = item & 7;
          // the 3x3 window (bf16x2 x 4 per position; -inf outside the conv output)
          uint4 wv[9];
#pragma unroll
          for (int kh = 0; kh < 3; ++kh) {
            const int rr = 2 * po - 1 + kh;
            const uint8_t* slot = ring + (rr & 3) * SLOTS * 128;
#pragma unroll
            for (int kw = 0; kw < 3; ++kw) {
              const int cc = 2 * pw - 1 + kw;
              wv[kh * 3 + kw] = (rr >= 0 && rr < a.Hs && cc >= 0 && cc < a.Ws)
                                    ? *(const uint4*)(slot + cc * 128 + ((k ^ (cc & 7)) << 4))
                                    : make_uint4(0xFF80FF80u, 0xFF80FF80u, 0xFF80FF80u, 0xFF80FF80u);
            }
          }
          __nv_bfloat162 best[4];
#pragma unroll
          for (int q = 0; q < 4; ++q) best[q] = ((const __nv_bfloat162*)&wv[0])[q];
#pragma unroll
          for (int p = 1; p < 9; ++p)
#pragma unroll
            for (int q = 0; q < 4; ++q) best[q] = __hmax2(best[q], ((const __nv_bfloat162*)&wv[p])[q]);
          const long long oi = (((long long)su.img * a.Hp + po) * a.Wp + pw) * 64 + k * 8;
          *(uint4*)(a.pooled + oi) = *(const uint4*)best;
          if (a.argmax) {
            // FIRST maximal position in row-major window order: scan backwards, the last match written wins
            uint32_t arg[2] = {0u, 0u};
#pragma unroll
            for (int p = 8; p >= 0; --p) {
              const uint32_t kk = 0x01010101u * (uint32_t)p;
#pragma unroll
              for (int w = 0; w < 2; ++w) {
                const uint32_t m0 = __heq2_mask(((const __nv_bfloat162*)&wv[p])[2 * w], best[2 * w]);
                const uint32_t m1 = __heq2_mask(((const __nv_bfloat162*)&wv[p])[2 * w + 1], best[2 * w + 1]);
                const uint32_t pm = __byte_perm(m0, m1, 0x6420);  // one byte per channel
                arg[w] = (arg[w] & ~pm) | (kk & pm);
              }
            }
            // ReLU producer: a window whose max is 0 routes no gradient -> AMAX_MASKED (0xFF) code
#pragma unroll
            for (int w = 0; w < 2; ++w) {
              const __nv_bfloat162 z2 = __float2bfloat162_rn(0.f);
              const uint32_t z0 = __heq2_mask(best[2 * w], z2), z1 = __heq2_mask(best[2 * w + 1], z2);
              arg[w] |= __byte_perm(z0, z1, 0x6420);
            }
            *(uint2*)(a.argmax + oi) = make_uint2(arg[0], arg[1]);
          }
        }
      }
    }
  }

  tc_fence_before();
  __syncthreads();
  if (warp == 4) {
    tc_fence_after();
    tmem_dealloc<128>(tmem);
  }
}

void stem_fwd(const bf16* s, const int* count, int n_static, int Hs, int Ws, const bf16* wprep, const float* bias,
              bf16* pooled, uint8_t* argmax, cudaStream_t st) {
  if (n_static <= 0) return;
  if (Ws > 125) throw ShapeError("stem: width/2 must be <= 125");
  thread_local StemFwdArgs a;
  a = StemFwdArgs{};
  a.s_map = make_tmap_nhwc_swz(s, n_static, Hs, Ws, 16, 16, SLOTS, 4, 32);
  a.wprep = wprep;
  a.bias = bias;
  a.count = count;
  a.n_static = n_static;
  a.Hs = Hs;
  a.Ws = Ws;
  a.Hp = (Hs - 1) / 2 + 1;
  a.Wp = (Ws - 1) / 2 + 1;
  pick_bands(n_static, a.Hp, 1, &a.bands, &a.band_rows);
  a.pooled = pooled;
  a.argmax = argmax;
  static bool attr = false;
  if (!attr) {
    CK(cudaFuncSetAttribute(stem_fwd_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, SF_SMEM));
    attr = true;
  }
  const int units = n_static * a.bands;
  ProfScope ps(PC_STEM_FWD, st);
  stem_fwd_kernel<<<std::min(units, num_sms()), SF_THREADS, SF_SMEM, st>>>(a);
  CK(cudaGetLastError());
}

// =====================================================================================================
// weight gradient
// =====================================================================================================
constexpr int SW_THREADS = 288;  // warp 0 TMA, warps 1-3 bias column sums, warp 4 MMA, warps 5-8 epilogue
constexpr int SW_DZ_STAGE = 2 * SLOTS * 128;  // dZ rows i, i+1: 128 positions x 64 co each, 128B swizzle
constexpr int SW_ND = 3;                      // dZ row-pair stages
constexpr int SW_S_SLOT = SLOTS * 32;         // one S row: 128 positions (cols -2..125) x 16 ch, 32B swizzle
constexpr int SW_NS = 16;                     // S row ring
// fused pool backward: pooled rows (bi, bi+1) of dT (bf16) and codes (u8), box width 64 >= Wp + 1
constexpr int SW_PT_BYTES = 2 * 64 * 64 * 2, SW_PC_BYTES = 2 * 64 * 64, SW_PSTAGE = SW_PT_BYTES + SW_PC_BYTES;
constexpr int SW_NP = 2;
constexpr int SW_BUILDERS = 224;  // warps 1-3 and 5-8 build dZ (fused mode)
constexpr int SW_SMEM = 1024 + SW_ND * SW_DZ_STAGE + SW_NS * SW_S_SLOT + 1024 + SW_NP * SW_PSTAGE + 512 + 3072;

// dW[ah][aw][ch][co] = sum_q dZ(i, q)[co] * S(i + ah, q + aw)[ch], output rows taken in pairs (i, i+1):
// A = the two dZ rows (M = 2 x 64 co, MN-major, atoms 16 KB apart), B = one S row rho = i - 2 + o shifted
// by aw = -2..1 (N = 4 x 16 ch: MN-major SWIZZLE_32B atoms one 32-byte position apart), K = 16 positions.
// Accumulator o (64 TMEM columns) collects tap ah = o - 2 in its top half (row i) and ah = o - 3 in its
// bottom half (row i + 1); the finish kernel adds the two halves of each tap.
struct StemWgArgs {
  CUtensorMap s_map;   // S2D [n][Hs][Ws][16], box {16, 128, 1, 1}, 32B swizzle
  CUtensorMap dz_map;  // dZ [n][Hs][Ws][64], box {64, 128, 2, 1}, 128B swizzle
  int n, Hs, Ws, bands, band_rows;  // band_rows even
  float* part;     // [gridDim.x][2][256][64]
  float* cs_part;  // [gridDim.x][64] or nullptr
  // fused max-pool backward (pool_dT != nullptr): dZ is never materialised; warps 5-8 build each dZ row pair
  // in shared memory from the pooled-output gradient [n][Hp][Wp][64] and the argmax codes (pool_bwd.cuh),
  // in the layout the dZ TMA box would have produced
  const bf16* pool_dT;
  const uint8_t* pool_codes;
  int Hp, Wp;
  CUtensorMap pt_map;  // dT [n][Hp][Wp][64] bf16, box {64, 64, 2, 1}
  CUtensorMap pc_map;  // codes [n][Hp][Wp][64] u8, box {64, 64, 2, 1}
};

__global__ void __launch_bounds__(SW_THREADS, 1) stem_wgrad_kernel(const __grid_constant__ StemWgArgs a) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = smem_align1024(smem_raw);
  uint8_t* dzst = smem;
  uint8_t* sring = dzst + SW_ND * SW_DZ_STAGE;
  uint8_t* guard = sring + SW_NS * SW_S_SLOT;  // finite rows read past the last S slot (invalid positions only)
  uint8_t* pring = guard + 1024;  // [SW_NP][dT rows | code rows] (fused pool backward)
  uint64_t* dz_full = (uint64_t*)(pring + SW_NP * SW_PSTAGE);
  uint64_t* dz_empty = dz_full + SW_ND;
  uint64_t* s_full = dz_empty + SW_ND;
  uint64_t* s_empty = s_full + SW_NS;
  uint64_t* tfull = s_empty + SW_NS;
  uint64_t* p_full = tfull + 1;   // [SW_NP]
  uint64_t* p_empty = p_full + SW_NP;
  uint32_t* tmem_slot = (uint32_t*)(p_empty + SW_NP);
  float* cs_red = (float*)((uint8_t*)dz_full + 512);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int nunits = a.n * a.bands;
  // zero the S ring and the guard: B rows past the end of a slot (positions >= 125, where dZ is zero) read
  // the next slot, which must hold finite values even before its first load (0 * NaN = NaN)
  for (int i = threadIdx.x; i < (SW_NS * SW_S_SLOT + 1024) / 16; i += blockDim.x)
    ((uint4*)sring)[i] = make_uint4(0, 0, 0, 0);
  if (a.pool_dT) {  // columns >= Ws of both rows of every dZ stage stay zero (never written by the builders)
    const int padc = SLOTS - a.Ws, per = 2 * padc * 8;
    for (int i = threadIdx.x; i < SW_ND * per; i += blockDim.x) {
      const int st = i / per, k = i - st * per;
      const int r = k / (padc * 8), rem = k - r * (padc * 8);
      const int x = a.Ws + rem / 8, j = rem % 8;
      *(uint4*)(dzst + st * SW_DZ_STAGE + (r * SLOTS + x) * 128 + ((j ^ (x & 7)) << 4)) = make_uint4(0, 0, 0, 0);
    }
  }
  if (threadIdx.x == 0) {
    for (int s = 0; s < SW_ND; ++s) {
      mbar_init(&dz_full[s], a.pool_dT ? SW_BUILDERS : 1);  // TMA transaction, or the dZ-building threads
      // MMA commit (+ one arrive per column-sum warp; the builders sum the columns themselves in fused mode)
      mbar_init(&dz_empty[s], (a.cs_part && !a.pool_dT) ? 4 : 1);
    }
    for (int s = 0; s < SW_NS; ++s) {
      mbar_init(&s_full[s], 1);
      mbar_init(&s_empty[s], 1);
    }
    mbar_init(tfull, 1);
    for (int s = 0; s < SW_NP; ++s) {
      mbar_init(&p_full[s], 1);
      mbar_init(&p_empty[s], SW_BUILDERS);
    }
    fence_mbar_init();
    tma_prefetch_desc(&a.s_map);
    tma_prefetch_desc(&a.dz_map);
  }
  if (warp == 4) tmem_alloc<512>(tmem_slot);
  fence_proxy_async_smem();
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  const uint32_t dz_u = smem_u32(dzst), s_u = smem_u32(sring);

  auto unit_rows = [&](int u, int& img, int& i0, int& i1) {
    img = u / a.bands;
    i0 = (u - img * a.bands) * a.band_rows;
    i1 = min(a.Hs, i0 + a.band_rows);  // pairs (i, i+1) for i = i0, i0+2, ..; i+1 may be Hs (zero rows)
  };

  // ---- fused pool backward: warps 1-3 and 5-8 build each dZ row pair (2x2 blocks (i/2, bj), 8 channels per
  // item, two items per thread) from the staged pooled rows, sum its columns for the bias gradient, and hand it
  // to the MMA warp; the column partials are reduced in fixed order once all MMAs are done ----
  auto build_dz = [&]() {
    const int t = warp < 4 ? threadIdx.x - 32 : threadIdx.x - 64;  // 0..223
    const int j = t & 7;                                             // channel chunk (same for both items)
    const int BW = (a.Ws + 1) / 2, nitems = BW * 8;
    float csum[8];
#pragma unroll
    for (int q = 0; q < 8; ++q) csum[q] = 0.f;
    int P = 0;
    for (int u = blockIdx.x; u < nunits; u += gridDim.x) {
      int img, i0, i1;
      unit_rows(u, img, i0, i1);
      for (int i = i0; i < i1; i += 2, ++P) {
        const int st = P % SW_ND, ph = P / SW_ND;
        const int ps = P % SW_NP;
        mbar_wait(&p_full[ps], (P / SW_NP) & 1);
        const uint8_t* pt = pring + ps * SW_PSTAGE;
        const uint8_t* pc = pt + SW_PT_BYTES;
        uint4 ob[2][4];
#pragma unroll
        for (int q = 0; q < 2; ++q) {
          const int item = t + SW_BUILDERS * q;
          if (item >= nitems) continue;
          const int bj = item >> 3;
          uint2 cw[4];
          uint4 gw[4];
#pragma unroll
          for (int wq = 0; wq < 4; ++wq) {  // rows bi, bi+1 of the box; columns >= Wp / rows >= Hp read 0
            const int r = wq >> 1, c = bj + (wq & 1);
            cw[wq] = *(const uint2*)(pc + (r * 64 + c) * 64 + j * 8);
            gw[wq] = *(const uint4*)(pt + (r * 64 + c) * 128 + j * 16);
          }
          pool_bwd_k3s2_block(cw, gw, ob[q]);
        }
        mbar_arrive(&p_empty[ps]);
        if (ph > 0) mbar_wait(&dz_empty[st], (ph - 1) & 1);
        uint8_t* base = dzst + st * SW_DZ_STAGE;
        const uint4 z = make_uint4(0u, 0u, 0u, 0u);
#pragma unroll
        for (int q = 0; q < 2; ++q) {
          const int item = t + SW_BUILDERS * q;
          if (item >= nitems) continue;
          const int bj = item >> 3;
#pragma unroll
          for (int p = 0; p < 4; ++p) {
            const int r = p >> 1, x = 2 * bj + (p & 1);
            if (x >= a.Ws) continue;  // pad columns: zeroed once
            const uint4 v = i + r < a.Hs ? ob[q][p] : z;
            *(uint4*)(base + (r * SLOTS + x) * 128 + ((j ^ (x & 7)) << 4)) = v;
            const bf16* h = (const bf16*)&v;
#pragma unroll
            for (int c = 0; c < 8; ++c) csum[c] += __bfloat162float(h[c]);
          }
        }
        fence_proxy_async_smem();  // generic-proxy writes -> visible to the tensor core
        mbar_arrive(&dz_full[st]);
      }
    }
    if (a.cs_part) {
      // all MMAs done -> the dZ stages are free scratch: [224 threads][8] partials, summed per channel in
      // thread order
      mbar_wait(tfull, 0);
      float* red = (float*)dzst;
#pragma unroll
      for (int c = 0; c < 8; ++c) red[t * 8 + c] = csum[c];
      asm volatile("bar.sync 3, %0;" ::"n"(SW_BUILDERS) : "memory");
      if (t < 64) {
        const int jj = t >> 3, c = t & 7;
        float acc = 0.f;
        for (int tt = jj; tt < SW_BUILDERS; tt += 8) acc += red[tt * 8 + c];
        a.cs_part[(long long)blockIdx.x * 64 + t] = acc;
      }
      asm volatile("bar.sync 3, %0;" ::"n"(SW_BUILDERS) : "memory");
    }
  };

  if (warp == 0) {
    if (lane == 0) {
      int L = 0, P = 0;  // S rows loaded, dZ pairs loaded
      for (int u = blockIdx.x; u < nunits; u += gridDim.x) {
        int img, i0, i1;
        unit_rows(u, img, i0, i1);
        int nr = i0 - 2;  // next S row
        for (int i = i0; i < i1; i += 2, ++P) {
          for (; nr <= i + 2; ++nr, ++L) {
            const int slot = L % SW_NS, ph = L / SW_NS;
            if (ph > 0) mbar_wait(&s_empty[slot], (ph - 1) & 1);
            mbar_expect_tx(&s_full[slot], SW_S_SLOT);
            tma_load_4d(s_u + slot * SW_S_SLOT, &a.s_map, &s_full[slot], 0, -2, nr, img);
          }
          if (a.pool_dT) {  // dZ pairs are built on chip: stage their pooled rows bi, bi+1 instead
            const int ps = P % SW_NP, pph = P / SW_NP;
            if (pph > 0) mbar_wait(&p_empty[ps], (pph - 1) & 1);
            mbar_expect_tx(&p_full[ps], SW_PSTAGE);
            const uint32_t pd = smem_u32(pring + ps * SW_PSTAGE);
            tma_load_4d(pd, &a.pt_map, &p_full[ps], 0, 0, i >> 1, img);
            tma_load_4d(pd + SW_PT_BYTES, &a.pc_map, &p_full[ps], 0, 0, i >> 1, img);
            continue;
          }
          const int st = P % SW_ND, ph = P / SW_ND;
          if (ph > 0) mbar_wait(&dz_empty[st], (ph - 1) & 1);
          mbar_expect_tx(&dz_full[st], SW_DZ_STAGE);
          tma_load_4d(dz_u + st * SW_DZ_STAGE, &a.dz_map, &dz_full[st], 0, 0, i, img);
        }
      }
    }
  } else if (warp >= 1 && warp <= 3 && a.pool_dT) {
    build_dz();
  } else if (warp >= 1 && warp <= 3) {
    if (a.cs_part) {
      TileColsum<64> cs;
      const int t = threadIdx.x - 32;
      cs.init(t);
      cs.zero();
      int P = 0;
      for (int u = blockIdx.x; u < nunits; u += gridDim.x) {
        int img, i0, i1;
        unit_rows(u, img, i0, i1);
        for (int i = i0; i < i1; i += 2, ++P) {
          const int st = P % SW_ND;
          mbar_wait(&dz_full[st], (P / SW_ND) & 1);
          cs.add(dzst + st * SW_DZ_STAGE, 2 * SLOTS);  // rows >= Hs and columns >= Ws are zero-filled
          __syncwarp();
          if (lane == 0) mbar_arrive(&dz_empty[st]);
        }
      }
      cs.finish(cs_red, a.cs_part + (long long)blockIdx.x * 64, 64, t);
    }
  } else if (warp == 4) {
    constexpr uint32_t IDESC = make_idesc(128, 64, 1, 1);
    int L = 0, P = 0;
    bool first = true;
    for (int u = blockIdx.x; u < nunits; u += gridDim.x) {
      int img, i0, i1;
      unit_rows(u, img, i0, i1);
      const int Lb = L;  // load index of S row i0 - 2
      for (int i = i0; i < i1; i += 2, ++P) {
        // S rows up to i + 2 (load index Lb + (i + 2) - (i0 - 2))
        for (int q = (i == i0 ? 0 : 3); q <= 4; ++q) {
          const int Lx = Lb + (i - i0) + q;
          mbar_wait(&s_full[Lx % SW_NS], (Lx / SW_NS) & 1);
        }
        const int st = P % SW_ND;
        mbar_wait(&dz_full[st], (P / SW_ND) & 1);
        tc_fence_after();
        if (elect_one()) {
          const uint64_t adesc0 = make_sdesc(dz_u + st * SW_DZ_STAGE, SLOTS * 128, 1024);
          uint64_t bdesc[5];
#pragma unroll
          for (int o = 0; o < 5; ++o)
            bdesc[o] = make_sdesc_sw32(s_u + ((Lb + (i - i0) + o) % SW_NS) * SW_S_SLOT, 32, 256);
#pragma unroll 1
          for (int kk = 0; kk < 8; ++kk) {
            // the five MMAs of a K-step share A (the dZ row pair): read it once into the A collector
            const uint64_t ad = adesc0 + (uint64_t)(kk * 128);
            const uint32_t acc = (!first || kk > 0) ? 1u : 0u;
            umma_bf16_acoll<0>(tmem, ad, bdesc[0] + (uint64_t)(kk * 32), IDESC, acc);
#pragma unroll
            for (int o = 1; o < 4; ++o)
              umma_bf16_acoll<1>(tmem + (uint32_t)(o * 64), ad, bdesc[o] + (uint64_t)(kk * 32), IDESC, acc);
            umma_bf16_acoll<2>(tmem + 256u, ad, bdesc[4] + (uint64_t)(kk * 32), IDESC, acc);
          }
          umma_commit(&dz_empty[st]);
          // S rows i - 2, i - 1 are not used by the next pair; the unit's last pair releases all five
          const int nrel = (i + 2 >= i1) ? 5 : 2;
          for (int q = 0; q < nrel; ++q) umma_commit(&s_empty[(Lb + (i - i0) + q) % SW_NS]);
        }
        __syncwarp();
        first = false;
      }
      L = Lb + ((i1 - i0 + 1) / 2) * 2 + 3;  // S rows i0-2 .. (last pair start)+2
    }
    if (elect_one()) {
      if (!first) umma_commit(tfull);
      else mbar_arrive(tfull);
    }
    __syncwarp();
  } else if (warp >= 5) {
    if (a.pool_dT) build_dz();
    const int qd = warp & 3;
    const int m = qd * 32 + lane;
    const int half = m >> 6, co = m & 63;
    mbar_wait(tfull, 0);
    tc_fence_after();
    float* P = a.part + ((long long)blockIdx.x * 2 + half) * 256 * 64;
#pragma unroll 1
    for (int o = 0; o < 5; ++o) {
      const int ah = o - 2 - half;
      const bool valid = ah >= -2 && ah <= 1;
#pragma unroll 1
      for (int c0 = 0; c0 < 64; c0 += 32) {
        float v[32];
        tmem_ld32(tmem + (uint32_t)(o * 64 + c0) + ((uint32_t)(qd * 32) << 16), v);
        if (!valid) continue;
#pragma unroll
        for (int j = 0; j < 32; ++j) {
          const int n = c0 + j, aw = (n >> 4) - 2, ch = n & 15;
          const int tap = (ah + 2) * 4 + (aw + 2);
          P[(tap * 16 + ch) * 64 + co] = v[j];
        }
      }
    }
    // each half writes all 16 taps (top: accumulators 0..3, bottom: 1..4); the finish kernel adds them
  }

  tc_fence_before();
  __syncthreads();
  if (warp == 4) {
    tc_fence_after();
    tmem_dealloc<512>(tmem);
  }
}

// sum the per-CTA partials (both row halves) in fixed order and scatter (tap, s2d channel) back to
// dw [64][7][7][cin]
// 8 partial-row groups per output (groups g, g+8, ... summed in order, eight loads in flight), combined in group
// order through shared memory: 256 threads = 32 outputs x 8 groups
__global__ void __launch_bounds__(256) stem_wgrad_finish_kernel(const float* __restrict__ part, int G, int cin,
                                                                float* __restrict__ dw) {
  __shared__ float red[8][33];
  const int ox = threadIdx.x & 31, gy = threadIdx.x >> 5;
  const int idx = blockIdx.x * 32 + ox;  // < 256 * 64 (grid = 512 blocks)
  const int co = idx & 63, k = idx >> 6;
  float acc = 0.f;
  const int NG = 2 * G;
  int g = gy;
  for (; g + 56 < NG; g += 64) {
    float v[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) v[u] = __ldg(part + ((long long)(g + 8 * u) * 256 + k) * 64 + co);
#pragma unroll
    for (int u = 0; u < 8; ++u) acc += v[u];
  }
  for (; g < NG; g += 8) acc += __ldg(part + ((long long)g * 256 + k) * 64 + co);
  red[gy][ox] = acc;
  __syncthreads();
  if (gy != 0) return;
  float t = red[0][ox];
#pragma unroll
  for (int q = 1; q < 8; ++q) t += red[q][ox];
  const int tap = k >> 4, ch = k & 15;
  const int bh = ch >> 3, bw = (ch >> 2) & 1, c = ch & 3;
  const int kh = 2 * (tap / 4 - 2) + bh + 3, kw = 2 * (tap % 4 - 2) + bw + 3;
  if (kh >= 0 && kh < 7 && kw >= 0 && kw < 7 && c < cin) dw[((co * 7 + kh) * 7 + kw) * cin + c] = t;
}
__global__ void stem_colsum_final_kernel(const float* __restrict__ part, int G, float* __restrict__ db) {
  const int c = threadIdx.x;
  float acc = 0.f;
  int g = 0;
  for (; g + 8 <= G; g += 8) {
    float v[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) v[u] = __ldg(part + (g + u) * 64 + c);
#pragma unroll
    for (int u = 0; u < 8; ++u) acc += v[u];
  }
  for (; g < G; ++g) acc += __ldg(part + g * 64 + c);
  db[c] = acc;
}

size_t stem_wgrad_ws_bytes(int n) {
  (void)n;
  return (size_t)num_sms() * (2 * 256 * 64 + 64) * sizeof(float);
}

static void stem_wgrad_impl(const bf16* s, const bf16* dz, const bf16* pool_dT, const uint8_t* pool_codes, int Hp,
                            int Wp, int n, int Hs, int Ws, int cin_real, float* ws, size_t ws_bytes, float* dw, float* db,
                            cudaStream_t st);
void stem_wgrad(const bf16* s, const bf16* dz, int n, int Hs, int Ws, int cin_real, float* ws, size_t ws_bytes,
                float* dw, float* db, cudaStream_t st) {
  stem_wgrad_impl(s, dz, nullptr, nullptr, 0, 0, n, Hs, Ws, cin_real, ws, ws_bytes, dw, db, st);
}
void stem_wgrad_pooled(const bf16* s, const bf16* pool_dT, const uint8_t* pool_codes, int Hp, int Wp, int n, int Hs,
                       int Ws, int cin_real, float* ws, size_t ws_bytes, float* dw, float* db, cudaStream_t st) {
  if (Hp != (Hs - 1) / 2 + 1 || Wp != (Ws - 1) / 2 + 1) throw ShapeError("stem_wgrad_pooled: pool geometry");
  stem_wgrad_impl(s, nullptr, pool_dT, pool_codes, Hp, Wp, n, Hs, Ws, cin_real, ws, ws_bytes, dw, db, st);
}
static void stem_wgrad_impl(const bf16* s, const bf16* dz, const bf16* pool_dT, const uint8_t* pool_codes, int Hp,
                            int Wp, int n, int Hs, int Ws, int cin_real, float* ws, size_t ws_bytes, float* dw, float* db,
                            cudaStream_t st) {
  if (n <= 0) return;
  if (Ws > 125) throw ShapeError("stem: width/2 must be <= 125");
  if (ws_bytes < stem_wgrad_ws_bytes(n)) throw std::runtime_error("stem wgrad workspace too small");
  thread_local StemWgArgs a;
  a = StemWgArgs{};
  a.s_map = make_tmap_nhwc_swz(s, n, Hs, Ws, 16, 16, SLOTS, 1, 32);
  if (pool_dT) {
    a.pool_dT = pool_dT;
    a.pool_codes = pool_codes;
    a.Hp = Hp;
    a.Wp = Wp;
    if (Wp + 1 > 64) throw ShapeError("stem_wgrad_pooled: pooled width must be < 64");
    a.pt_map = make_tmap_nhwc_plain(pool_dT, n, Hp, Wp, 64, 64, 64, 2);  // row-major [2][64][64] in smem
    a.pc_map = make_tmap_nhwc_u8(pool_codes, n, Hp, Wp, 64, 64, 64, 2);
  } else {
    a.dz_map = make_tmap_nhwc(dz, n, Hs, Ws, 64, 64, SLOTS, 2);
  }
  a.n = n;
  a.Hs = Hs;
  a.Ws = Ws;
  // bands of an even number of rows (row pairs never straddle two units)
  const int pairs = (Hs + 1) / 2;
  int bands, bpairs;
  pick_bands(n, pairs, 2, &bands, &bpairs);
  a.bands = bands;
  a.band_rows = 2 * bpairs;
  const int G = std::min(n * a.bands, num_sms());
  a.part = ws;
  a.cs_part = db ? ws + (size_t)G * 2 * 256 * 64 : nullptr;
  static bool attr = false;
  if (!attr) {
    CK(cudaFuncSetAttribute(stem_wgrad_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, SW_SMEM));
    attr = true;
  }
  {
    ProfScope ps(PC_STEM_WGRAD, st);
    stem_wgrad_kernel<<<G, SW_THREADS, SW_SMEM, st>>>(a);
    CK(cudaGetLastError());
  }
  ProfScope ps(PC_STEM_AUX, st, db ? 2 : 1);
  stem_wgrad_finish_kernel<<<256 * 64 / 32, 256, 0, st>>>(ws, G, cin_real, dw);
  if (db) stem_colsum_final_kernel<<<1, 64, 0, st>>>(a.cs_part, G, db);
  CK(cudaGetLastError());
}

}  // namespace adainf

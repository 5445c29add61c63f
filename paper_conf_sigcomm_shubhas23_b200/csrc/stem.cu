// ResNet stem kernels (see stem.cuh for the space-to-depth formulation).
#include <algorithm>
#include <cmath>

#include "colsum_tile.cuh"
#include "conv_gemm.cuh"
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
constexpr int SF_PLANE = (4 * SLOTS + 8) * 16;  // 4 window rows x 128 positions x 16 B (+ 8 trail rows)
constexpr int SF_STAGE = 2 * SF_PLANE;
constexpr int SF_STAGES = 6;
constexpr int SF_W_BYTES = 16 * 2048;
constexpr int SF_RING = 4;  // conv-row ring: bf16 [SLOTS][64], 16-byte chunk k of column x at k ^ (x & 7)
constexpr int SF_SMEM = 1024 + SF_W_BYTES + SF_STAGES * SF_STAGE + SF_RING * SLOTS * 128 + 256;

struct StemFwdArgs {
  CUtensorMap s_map;  // S2D [n][Hs][Ws][16], box {8, 128, 4, 1}, no swizzle
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
  uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
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
          mbar_expect_tx(&full[s], 2 * 4 * SLOTS * 16);
          const uint32_t dst = st_base + s * SF_STAGE;
          tma_load_4d(dst, &a.s_map, &full[s], 0, -2, r - 2, su.img);
          tma_load_4d(dst + SF_PLANE, &a.s_map, &full[s], 8, -2, r - 2, su.img);
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
          const uint64_t adesc0 = make_sdesc_plain(st_base + s * SF_STAGE, SF_PLANE, 128);
#pragma unroll
          for (int t = 0; t < 16; ++t) {
            const uint32_t row_off = (uint32_t)((t >> 2) * SLOTS + (t & 3));  // window row of tap (ah, aw)
            umma_bf16(tmem + (uint32_t)(b * 64), adesc0 + row_off, bdesc0 + (uint64_t)(t * 128), IDESC, t > 0);
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
          float best[8];
          uint32_t arg[2] = {0u, 0u};
#pragma unroll
          for (int q = 0; q < 8; ++q) best[q] = -INFINITY;
#pragma unroll
          for (int kh = 0; kh < 3; ++kh) {
            const int rr = 2 * po - 1 + kh;
            if (rr < 0 || rr >= a.Hs) continue;
            const uint8_t* slot = ring + (rr & 3) * SLOTS * 128;
#pragma unroll
            for (int kw = 0; kw < 3; ++kw) {
              const int cc = 2 * pw - 1 + kw;
              if (cc < 0 || cc >= a.Ws) continue;
              const uint4 raw = *(const uint4*)(slot + cc * 128 + ((k ^ (cc & 7)) << 4));
              const __nv_bfloat162* h = (const __nv_bfloat162*)&raw;
#pragma unroll
              for (int q = 0; q < 4; ++q) {
                const float2 f = __bfloat1622float2(h[q]);
                // strict: the FIRST maximal element in row-major window order (as maxpool_fwd_kernel)
                if (f.x > best[2 * q]) {
                  best[2 * q] = f.x;
                  const int sh = ((2 * q) & 3) * 8;
                  arg[q >> 1] = (arg[q >> 1] & ~(0xFFu << sh)) | ((uint32_t)(kh * 3 + kw) << sh);
                }
                if (f.y > best[2 * q + 1]) {
                  best[2 * q + 1] = f.y;
                  const int sh = ((2 * q + 1) & 3) * 8;
                  arg[q >> 1] = (arg[q >> 1] & ~(0xFFu << sh)) | ((uint32_t)(kh * 3 + kw) << sh);
                }
              }
            }
          }
          __align__(16) __nv_bfloat162 o[4];
#pragma unroll
          for (int q = 0; q < 4; ++q) o[q] = __floats2bfloat162_rn(best[2 * q], best[2 * q + 1]);
          const long long oi = (((long long)su.img * a.Hp + po) * a.Wp + pw) * 64 + k * 8;
          *(uint4*)(a.pooled + oi) = *(const uint4*)o;
          if (a.argmax) *(uint2*)(a.argmax + oi) = make_uint2(arg[0], arg[1]);
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
  static StemFwdArgs a;
  a = StemFwdArgs{};
  a.s_map = make_tmap_nhwc_plain(s, n_static, Hs, Ws, 16, 8, SLOTS, 4);
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
constexpr int SW_NS = 8;         // dZ ring slots: 128 positions (col -1 .. 126) x 64 co, 128B swizzle
constexpr int SW_SS = 8;         // S stages: two planes of 128 positions x 8 channels
constexpr int SW_SLOT = SLOTS * 128;
constexpr int SW_SSTAGE = 2 * SLOTS * 16;
constexpr int SW_SMEM = 1024 + SW_NS * SW_SLOT + 1024 + SW_SS * SW_SSTAGE + 256 + 3072;

struct StemWgArgs {
  CUtensorMap s_map;   // S2D [n][Hs][Ws][16], box {8, 128, 1, 1}, no swizzle
  CUtensorMap dz_map;  // dZ [n][Hs][Ws][64], box {64, 128, 1, 1}, 128B swizzle
  int n, Hs, Ws, bands, band_rows;
  float* part;     // [gridDim.x][256][64]
  float* cs_part;  // [gridDim.x][64] or nullptr
};

__global__ void __launch_bounds__(SW_THREADS, 1) stem_wgrad_kernel(const __grid_constant__ StemWgArgs a) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  uint8_t* ring = smem;
  uint8_t* guard = ring + SW_NS * SW_SLOT;  // zero rows read (for invalid positions only) past the last slot
  uint8_t* sst = guard + 1024;
  uint64_t* dz_full = (uint64_t*)(sst + SW_SS * SW_SSTAGE);
  uint64_t* dz_empty = dz_full + SW_NS;
  uint64_t* s_full = dz_empty + SW_NS;
  uint64_t* s_empty = s_full + SW_SS;
  uint64_t* tfull = s_empty + SW_SS;
  uint32_t* tmem_slot = (uint32_t*)(tfull + 1);
  float* cs_red = (float*)((uint8_t*)dz_full + 256);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int nunits = a.n * a.bands;
  for (int i = threadIdx.x; i < 1024 / 16; i += blockDim.x) ((uint4*)guard)[i] = make_uint4(0, 0, 0, 0);
  if (threadIdx.x == 0) {
    for (int s = 0; s < SW_NS; ++s) {
      mbar_init(&dz_full[s], 1);
      mbar_init(&dz_empty[s], a.cs_part ? 4 : 1);  // MMA commit (+ one arrive per column-sum warp)
    }
    for (int s = 0; s < SW_SS; ++s) {
      mbar_init(&s_full[s], 1);
      mbar_init(&s_empty[s], 1);
    }
    mbar_init(tfull, 1);
    fence_mbar_init();
    tma_prefetch_desc(&a.s_map);
    tma_prefetch_desc(&a.dz_map);
  }
  if (warp == 4) tmem_alloc<128>(tmem_slot);
  fence_proxy_async_smem();
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  const uint32_t ring_u = smem_u32(ring), sst_u = smem_u32(sst);

  auto unit_rows = [&](int u, int& img, int& i0, int& i1) {
    img = u / a.bands;
    i0 = (u - img * a.bands) * a.band_rows;
    i1 = min(a.Hs, i0 + a.band_rows);
  };

  if (warp == 0) {
    if (lane == 0) {
      int L = 0, it = 0;
      for (int u = blockIdx.x; u < nunits; u += gridDim.x) {
        int img, i0, i1;
        unit_rows(u, img, i0, i1);
        int nd = i0 - 1;
        for (int i = i0; i < i1; ++i, ++it) {
          for (; nd <= i + 2; ++nd, ++L) {
            const int slot = L % SW_NS, ph = L / SW_NS;
            if (ph > 0) mbar_wait(&dz_empty[slot], (ph - 1) & 1);
            mbar_expect_tx(&dz_full[slot], SW_SLOT);
            tma_load_4d(ring_u + slot * SW_SLOT, &a.dz_map, &dz_full[slot], 0, -1, nd, img);
          }
          const int s = it % SW_SS, ph = it / SW_SS;
          if (ph > 0) mbar_wait(&s_empty[s], (ph - 1) & 1);
          mbar_expect_tx(&s_full[s], SW_SSTAGE);
          tma_load_4d(sst_u + s * SW_SSTAGE, &a.s_map, &s_full[s], 0, 0, i, img);
          tma_load_4d(sst_u + s * SW_SSTAGE + SLOTS * 16, &a.s_map, &s_full[s], 8, 0, i, img);
        }
      }
    }
  } else if (warp >= 1 && warp <= 3) {
    if (a.cs_part) {
      TileColsum<64> cs;
      const int t = threadIdx.x - 32;
      cs.init(t);
      cs.zero();
      int L = 0;
      for (int u = blockIdx.x; u < nunits; u += gridDim.x) {
        int img, i0, i1;
        unit_rows(u, img, i0, i1);
        for (int rho = i0 - 1; rho <= i1 + 1; ++rho, ++L) {
          const int slot = L % SW_NS;
          mbar_wait(&dz_full[slot], (L / SW_NS) & 1);
          if (rho >= i0 && rho < i1) cs.add(ring + slot * SW_SLOT, SLOTS);
          __syncwarp();
          if (lane == 0) mbar_arrive(&dz_empty[slot]);
        }
      }
      cs.finish(cs_red, a.cs_part + (long long)blockIdx.x * 64, 64, t);
    }
  } else if (warp == 4) {
    constexpr uint32_t IDESC = make_idesc(128, 16, 1, 1);
    int L = 0, it = 0;
    bool first = true;
    for (int u = blockIdx.x; u < nunits; u += gridDim.x) {
      int img, i0, i1;
      unit_rows(u, img, i0, i1);
      const int Lb = L;
      for (int i = i0; i < i1; ++i, ++it) {
        for (int q = (i == i0 ? 0 : 3); q <= 3; ++q) {
          const int Lx = Lb + (i - i0) + q;
          mbar_wait(&dz_full[Lx % SW_NS], (Lx / SW_NS) & 1);
        }
        const int s = it % SW_SS;
        mbar_wait(&s_full[s], (it / SW_SS) & 1);
        tc_fence_after();
        if (elect_one()) {
          // MN-major, no swizzle: LBO = K-direction stride of 8-row groups, SBO = N-direction (plane) stride
          const uint64_t bdesc0 = make_sdesc_plain(sst_u + s * SW_SSTAGE, 128, SLOTS * 16);
#pragma unroll
          for (int ah = -2; ah <= 1; ++ah) {
            const int Lr = Lb + (i - ah) - (i0 - 1);  // load index of dZ row i - ah
            const uint32_t base = ring_u + (Lr % SW_NS) * SW_SLOT;
#pragma unroll
            for (int pr = 0; pr < 2; ++pr) {
              // atoms: aw = 1 - 2*pr (row offset 2*pr), aw = -2*pr (row offset 2*pr + 1); LBO = one row
              const uint64_t adesc0 = make_sdesc(base + pr * 256, 128, 1024);
              const uint32_t acc = (uint32_t)(((ah + 2) * 2 + pr) * 16);
#pragma unroll
              for (int kk = 0; kk < 8; ++kk)
                umma_bf16(tmem + acc, adesc0 + (uint64_t)(kk * 128), bdesc0 + (uint64_t)(kk * 16), IDESC,
                          (!first || kk > 0) ? 1u : 0u);
            }
          }
          umma_commit(&s_empty[s]);
          umma_commit(&dz_empty[(Lb + (i - i0)) % SW_NS]);  // dZ row i - 1: no later use
          if (i == i1 - 1)
            for (int q = 1; q <= 3; ++q) umma_commit(&dz_empty[(Lb + (i - i0) + q) % SW_NS]);
        }
        __syncwarp();
        first = false;
      }
      L = Lb + (i1 - i0 + 3);
    }
    if (elect_one()) {
      if (!first) umma_commit(tfull);
      else mbar_arrive(tfull);
    }
    __syncwarp();
  } else if (warp >= 5) {
    const int qd = warp & 3;
    const int m = qd * 32 + lane;
    const int atom = m >> 6, co = m & 63;
    const bool any = (int)blockIdx.x < nunits;
    mbar_wait(tfull, 0);
    tc_fence_after();
    float* P = a.part + (long long)blockIdx.x * 256 * 64;
#pragma unroll 1
    for (int c0 = 0; c0 < 8; c0 += 2) {
      float v[32];
      if (any) tmem_ld32(tmem + (uint32_t)(c0 * 16) + ((uint32_t)(qd * 32) << 16), v);
      else
#pragma unroll
        for (int i = 0; i < 32; ++i) v[i] = 0.f;
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const int accn = c0 + h;
        const int ah = (accn >> 1) - 2, pr = accn & 1;
        const int aw = 1 - 2 * pr - atom;
        const int tap = (ah + 2) * 4 + (aw + 2);
#pragma unroll
        for (int ch = 0; ch < 16; ++ch) P[(tap * 16 + ch) * 64 + co] = v[h * 16 + ch];
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

// sum the per-CTA partials in fixed order and scatter (tap, s2d channel) back to dw [64][7][7][cin]
__global__ void stem_wgrad_finish_kernel(const float* __restrict__ part, int G, int cin, float* __restrict__ dw) {
  const int idx = blockIdx.x * blockDim.x + threadIdx.x;
  if (idx >= 256 * 64) return;
  const int co = idx & 63, k = idx >> 6;
  float acc = 0.f;
  for (int g = 0; g < G; ++g) acc += __ldg(part + ((long long)g * 256 + k) * 64 + co);
  const int t = k >> 4, ch = k & 15;
  const int bh = ch >> 3, bw = (ch >> 2) & 1, c = ch & 3;
  const int kh = 2 * (t / 4 - 2) + bh + 3, kw = 2 * (t % 4 - 2) + bw + 3;
  if (kh >= 0 && kh < 7 && kw >= 0 && kw < 7 && c < cin) dw[((co * 7 + kh) * 7 + kw) * cin + c] = acc;
}
__global__ void stem_colsum_final_kernel(const float* __restrict__ part, int G, float* __restrict__ db) {
  const int c = threadIdx.x;
  float acc = 0.f;
  for (int g = 0; g < G; ++g) acc += part[g * 64 + c];
  db[c] = acc;
}

size_t stem_wgrad_ws_bytes(int n) {
  (void)n;
  return (size_t)num_sms() * (256 * 64 + 64) * sizeof(float);
}

void stem_wgrad(const bf16* s, const bf16* dz, int n, int Hs, int Ws, int cin_real, float* ws, size_t ws_bytes,
                float* dw, float* db, cudaStream_t st) {
  if (n <= 0) return;
  if (Ws > 125) throw ShapeError("stem: width/2 must be <= 125");
  if (ws_bytes < stem_wgrad_ws_bytes(n)) throw std::runtime_error("stem wgrad workspace too small");
  static StemWgArgs a;
  a = StemWgArgs{};
  a.s_map = make_tmap_nhwc_plain(s, n, Hs, Ws, 16, 8, SLOTS, 1);
  a.dz_map = make_tmap_nhwc(dz, n, Hs, Ws, 64, 64, SLOTS, 1);
  a.n = n;
  a.Hs = Hs;
  a.Ws = Ws;
  pick_bands(n, Hs, 3, &a.bands, &a.band_rows);
  const int G = std::min(n * a.bands, num_sms());
  a.part = ws;
  a.cs_part = db ? ws + (size_t)G * 256 * 64 : nullptr;
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
  stem_wgrad_finish_kernel<<<64, 256, 0, st>>>(ws, G, cin_real, dw);
  if (db) stem_colsum_final_kernel<<<1, 64, 0, st>>>(a.cs_part, G, db);
  CK(cudaGetLastError());
}

}  // namespace adainf

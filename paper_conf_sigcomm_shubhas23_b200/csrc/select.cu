// Retraining-sample selection ("Cosine distance of the feature vector of every
// new sample with the mean feature vector of the old training samples ... after PCA", P:239 R_j^i
// samples, P:243 never reuse samples used by other jobs).
//
//   1. projection Y = X W on the tensor cores (the implicit-GEMM kernel as a 1x1 conv, fp32 out)
//   2. d_i = min_r (1 - cos(y_i, mu_r)), mu = ref W; excluded -> key 0; key = bits(d) + 1 (d >= 0)
//   3. exact top-k: 4-pass MSB radix select on the 32-bit keys (integer histograms) -> threshold T and
//      the number of ties at T to take; ties go to the lower index (reading Q15)
//   4. stable emit of the selected indices in ascending order (block counts -> scan -> emit)
#include <cfloat>

#include "api_common.h"
#include "common.cuh"
#include "model.h"
#include "prof.h"
#include "tma.cuh"

namespace adainf {

// Selection preparation in ONE launch (separate launches cost a few microseconds of latency each): blocks [0, nt)
// transpose W -> Wt; the remaining blocks project the reference rows, mu[r][p] = sum_d ref[r][d] * W[d][p] in fp32,
// one warp per (r, p), lanes stride d, fixed xor-tree combine.  The norms ||mu_r|| follow in ref_norm_kernel or,
// on the fused path, at the start of every select_fused CTA (same arithmetic).
__global__ void __launch_bounds__(256) select_prep_kernel(const float* __restrict__ ref, const bf16* __restrict__ W,
                                                          int D, int P, int M, int nt, bf16* __restrict__ Wt,
                                                          float* __restrict__ mu) {
  if ((int)blockIdx.x < nt) {
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i < D * P) {
      const int d = i / P, p = i - d * P;
      Wt[(long long)p * D + d] = W[i];
    }
    return;
  }
  const int gw = ((blockIdx.x - nt) * blockDim.x + threadIdx.x) >> 5, lane = threadIdx.x & 31;
  if (gw >= M * P) return;
  const int r = gw / P, p = gw - r * P;
  float a = 0.f;
  if (W) {
#pragma unroll 4
    for (int d = lane; d < D; d += 32) a = fmaf(ref[(long long)r * D + d], __bfloat162float(W[(long long)d * P + p]), a);
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) a += __shfl_xor_sync(0xffffffffu, a, o);
  } else {
    a = ref[(long long)r * D + p];
  }
  if (lane == 0) mu[(long long)r * P + p] = a;
}
// ||mu_r|| of one reference row: lanes stride p, fixed xor-tree combine (one warp)
__device__ __forceinline__ float ref_norm_warp(const float* mu_r, int P, int lane) {
  float sq = 0.f;
  for (int p = lane; p < P; p += 32) sq = fmaf(mu_r[p], mu_r[p], sq);
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) sq += __shfl_xor_sync(0xffffffffu, sq, o);
  return sqrtf(sq);
}
__global__ void ref_norm_kernel(const float* __restrict__ mu, int P, int M, float* __restrict__ mun) {
  const int r = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, lane = threadIdx.x & 31;
  if (r >= M) return;
  const float v = ref_norm_warp(mu + (long long)r * P, P, lane);
  if (lane == 0) mun[r] = v;
}

// one warp per row: cosine distance to every reference row, min; key
template <bool FROM_BF16>
__global__ void cosine_key_kernel(const void* __restrict__ Yv, long long N, int P, const float* __restrict__ mu,
                                  const float* __restrict__ mun, int M, const uint8_t* __restrict__ exclude,
                                  uint32_t* __restrict__ keys, float* __restrict__ dist_all) {
  const long long row = (blockIdx.x * (long long)blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  if (row >= N) return;
  float y[8];
  int ny = 0;
  float nn = 0.f;
  for (int p = lane; p < P; p += 32) {
    const float v = FROM_BF16 ? __bfloat162float(((const bf16*)Yv)[row * P + p]) : ((const float*)Yv)[row * P + p];
    y[ny++] = v;
    nn = fmaf(v, v, nn);
  }
  for (int o = 16; o > 0; o >>= 1) nn += __shfl_xor_sync(0xffffffffu, nn, o);
  const float yn = sqrtf(nn);
  float best = FLT_MAX;
  for (int r = 0; r < M; ++r) {
    float dot = 0.f;
    int q = 0;
    for (int p = lane; p < P; p += 32) dot = fmaf(y[q++], mu[(long long)r * P + p], dot);
    for (int o = 16; o > 0; o >>= 1) dot += __shfl_xor_sync(0xffffffffu, dot, o);
    const float cs = dot / fmaxf(yn * mun[r], 1e-12f);
    best = fminf(best, 1.0f - cs);
  }
  if (lane == 0) {
    const bool ex = exclude && exclude[row];
    const float d = fmaxf(best, 0.f);
    keys[row] = ex ? 0u : (__float_as_uint(d) + 1u);
    if (dist_all) dist_all[row] = ex ? -1.f : d;
  }
}

// many reference rows (M > 4, the GEMM-shaped variant of reading Q14): one warp per candidate row, the row's
// projected vector staged in shared memory, lanes stride the reference rows (each lane a full P-length dot in
// fixed order), min-reduced over lanes
template <bool FROM_BF16>
__global__ void __launch_bounds__(256) cosine_key_multi_kernel(const void* __restrict__ Yv, long long N, int P,
                                                               const float* __restrict__ mu,
                                                               const float* __restrict__ mun, int M,
                                                               const uint8_t* __restrict__ exclude,
                                                               uint32_t* __restrict__ keys, float* __restrict__ dist_all) {
  __shared__ float ys[8][256];
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const long long row = (blockIdx.x * (long long)blockDim.x + threadIdx.x) >> 5;
  if (row >= N) return;
  float nn = 0.f;
  for (int p = lane; p < P; p += 32) {
    const float v = FROM_BF16 ? __bfloat162float(((const bf16*)Yv)[row * P + p]) : ((const float*)Yv)[row * P + p];
    ys[w][p] = v;
    nn = fmaf(v, v, nn);
  }
  for (int o = 16; o > 0; o >>= 1) nn += __shfl_xor_sync(0xffffffffu, nn, o);
  __syncwarp();
  const float yn = sqrtf(nn);
  float best = FLT_MAX;
  for (int r = lane; r < M; r += 32) {
    const float* m = mu + (long long)r * P;
    float dot = 0.f;
    for (int p = 0; p < P; p += 4) {
      const float4 q = __ldg((const float4*)(m + p));
      dot = fmaf(ys[w][p], q.x, dot);
      dot = fmaf(ys[w][p + 1], q.y, dot);
      dot = fmaf(ys[w][p + 2], q.z, dot);
      dot = fmaf(ys[w][p + 3], q.w, dot);
    }
    const float cs = dot / fmaxf(yn * mun[r], 1e-12f);
    best = fminf(best, 1.0f - cs);
  }
  for (int o = 16; o > 0; o >>= 1) best = fminf(best, __shfl_xor_sync(0xffffffffu, best, o));
  if (lane == 0) {
    const bool ex = exclude && exclude[row];
    const float d = fmaxf(best, 0.f);
    keys[row] = ex ? 0u : (__float_as_uint(d) + 1u);
    if (dist_all) dist_all[row] = ex ? -1.f : d;
  }
}

// ---- fused projection + cosine key (one pass over X, no fp32 Y round trip) ---------------------------------
// Persistent, one CTA per SM: W^T [P][D] resident in shared memory (TMA, 128B swizzle, 64-column chunks), X streamed
// in 128-row x 64-column TMA boxes through a stage ring, Y tile = X W on the tensor cores (tcgen05.mma M=128,
// N=P, K=16; fp32 accumulators in TMEM, double-buffered), epilogue: one thread per row reads its P values from TMEM
// and computes ||y||, y.mu_r, d = max(0, min_r 1 - cos) and the key, in the row's own fixed order.
constexpr int SELF_THREADS = 192;  // warp 0 TMA, warp 1 MMA, warps 2-5 epilogue (TMEM lane quadrants 2,3,0,1)
constexpr int SELF_STAGES = 6;
constexpr int SELF_STAGE_BYTES = 128 * 128;  // 128 rows x 64 bf16 columns

struct SelFusedArgs {
  CUtensorMap x_map;  // X [N][D] bf16, box {64, 128}
  CUtensorMap w_map;  // W^T [P][D] bf16, box {64, P}
  long long N;
  int D, M;
  const float* mu;   // [M][P]
  const float* mun;  // [M]
  const uint8_t* exclude;
  uint32_t* keys;
  float* dist_all;
};

template <int NC>
__device__ __forceinline__ void tmem_ld_cols(uint32_t taddr, float* v) {
  if constexpr (NC == 16) {
    uint32_t r[16];
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
        : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
          "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
        : "r"(taddr));
    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
    for (int i = 0; i < 16; ++i) v[i] = __uint_as_float(r[i]);
  } else {
    tmem_ld32(taddr, v);
  }
}

template <int P>
__global__ void __launch_bounds__(SELF_THREADS, 1) select_fused_kernel(const __grid_constant__ SelFusedArgs a) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = smem_align1024(smem_raw);
  const int nkb = a.D / 64;
  uint8_t* wsm = smem;                                  // nkb chunks of [P][64] bf16 (P * 128 bytes each)
  uint8_t* xst = wsm + (size_t)nkb * P * 128;           // stage ring
  float* mus = (float*)(xst + SELF_STAGES * SELF_STAGE_BYTES);  // [M][P] then mun[M]
  uint64_t* full = (uint64_t*)(mus + 4 * P + 4);
  uint64_t* empty = full + SELF_STAGES;
  uint64_t* wbar = empty + SELF_STAGES;
  uint64_t* tfull = wbar + 1;
  uint64_t* tempty = tfull + 2;
  uint32_t* tmem_slot = (uint32_t*)(tempty + 2);
  constexpr int ACC = P;
  constexpr int TCOLS = 2 * P < 32 ? 32 : 2 * P;

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const long long ntiles = (a.N + 127) / 128;
  for (int i = threadIdx.x; i < a.M * P; i += blockDim.x) mus[i] = a.mu[i];
  __syncthreads();
  if ((threadIdx.x >> 5) < a.M) {  // ||mu_r||: warp r (M <= 4)
    const float v = ref_norm_warp(mus + (threadIdx.x >> 5) * P, P, threadIdx.x & 31);
    if ((threadIdx.x & 31) == 0) mus[4 * P + (threadIdx.x >> 5)] = v;
  }
  if (threadIdx.x == 0) {
    for (int s = 0; s < SELF_STAGES; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], 1);
    }
    mbar_init(wbar, 1);
    for (int b = 0; b < 2; ++b) {
      mbar_init(&tfull[b], 1);
      mbar_init(&tempty[b], 128);
    }
    fence_mbar_init();
    tma_prefetch_desc(&a.x_map);
    tma_prefetch_desc(&a.w_map);
  }
  if (warp == 1) tmem_alloc<TCOLS>(tmem_slot);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;

  if (warp == 0) {
    if (lane == 0) {
      mbar_expect_tx(wbar, (uint32_t)(nkb * P * 128));
      for (int kb = 0; kb < nkb; ++kb) tma_load_2d(smem_u32(wsm + (size_t)kb * P * 128), &a.w_map, wbar, kb * 64, 0);
      int it = 0;
      for (long long t = blockIdx.x; t < ntiles; t += gridDim.x)
        for (int kb = 0; kb < nkb; ++kb, ++it) {
          const int s = it % SELF_STAGES, ph = it / SELF_STAGES;
          if (ph > 0) mbar_wait(&empty[s], (ph - 1) & 1);
          mbar_expect_tx(&full[s], SELF_STAGE_BYTES);
          tma_load_2d(smem_u32(xst + s * SELF_STAGE_BYTES), &a.x_map, &full[s], kb * 64, (int)(t * 128));
        }
    }
  } else if (warp == 1) {
    constexpr uint32_t IDESC = make_idesc(128, P, 0, 0);
    mbar_wait(wbar, 0);
    int it = 0, lt = 0;
    for (long long t = blockIdx.x; t < ntiles; t += gridDim.x, ++lt) {
      const int b = lt & 1, ub = lt >> 1;
      if (ub > 0) mbar_wait(&tempty[b], (ub - 1) & 1);
      tc_fence_after();
      for (int kb = 0; kb < nkb; ++kb, ++it) {
        const int s = it % SELF_STAGES, u = it / SELF_STAGES;
        mbar_wait(&full[s], u & 1);
        tc_fence_after();
        if (elect_one()) {
          const uint64_t ad0 = make_sdesc(smem_u32(xst + s * SELF_STAGE_BYTES), 16, 1024);
          const uint64_t bd0 = make_sdesc(smem_u32(wsm + (size_t)kb * P * 128), 16, 1024);
#pragma unroll
          for (int kk = 0; kk < 4; ++kk)
            umma_bf16(tmem + (uint32_t)(b * ACC), ad0 + kk * 2, bd0 + kk * 2, IDESC, (kb | kk) != 0);
          umma_commit(&empty[s]);
          if (kb == nkb - 1) umma_commit(&tfull[b]);
        }
        __syncwarp();
      }
    }
  } else {
    const int q = warp & 3;
    const float* mun = mus + 4 * P;
    int lt = 0;
    for (long long t = blockIdx.x; t < ntiles; t += gridDim.x, ++lt) {
      const int b = lt & 1, ub = lt >> 1;
      mbar_wait(&tfull[b], ub & 1);
      tc_fence_after();
      const uint32_t trow = tmem + (uint32_t)(b * ACC) + ((uint32_t)(q * 32) << 16);
      float nn = 0.f, dot[4] = {0.f, 0.f, 0.f, 0.f};
      constexpr int CH = P < 32 ? P : 32;
#pragma unroll 1
      for (int c0 = 0; c0 < P; c0 += CH) {
        float v[CH];
        tmem_ld_cols<CH>(trow + (uint32_t)c0, v);
#pragma unroll
        for (int i = 0; i < CH; ++i) {
          nn = fmaf(v[i], v[i], nn);
#pragma unroll
          for (int r = 0; r < 4; ++r)
            if (r < a.M) dot[r] = fmaf(v[i], mus[r * P + c0 + i], dot[r]);
        }
      }
      tc_fence_before();
      mbar_arrive(&tempty[b]);
      const long long row = t * 128 + q * 32 + lane;
      if (row < a.N) {
        const float yn = sqrtf(nn);
        float best = FLT_MAX;
#pragma unroll
        for (int r = 0; r < 4; ++r)
          if (r < a.M) best = fminf(best, 1.0f - dot[r] / fmaxf(yn * mun[r], 1e-12f));
        const bool ex = a.exclude && a.exclude[row];
        const float d = fmaxf(best, 0.f);
        a.keys[row] = ex ? 0u : (__float_as_uint(d) + 1u);
        if (a.dist_all) a.dist_all[row] = ex ? -1.f : d;
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

static bool select_fused_ok(int D, int P, int M) {
  return D % 64 == 0 && (P == 16 || P == 32 || P == 64 || P == 128 || P == 256) && M <= 4 && (long long)D * P * 2 <= 98304;
}

static size_t select_fused_smem(int D, int P) {
  return 1024 + (size_t)D * P * 2 + SELF_STAGES * SELF_STAGE_BYTES + (4 * P + 4) * 4 + 256;
}

template <int P>
static void launch_select_fused_p(const SelFusedArgs& a, int D, cudaStream_t st) {
  const size_t sm = select_fused_smem(D, P);
  static bool attr = false;
  if (!attr) {
    CK(cudaFuncSetAttribute(select_fused_kernel<P>, cudaFuncAttributeMaxDynamicSharedMemorySize, 232448));
    attr = true;
  }
  const long long ntiles = (a.N + 127) / 128;
  const int grid = (int)std::min<long long>(ntiles, num_sms());
  select_fused_kernel<P><<<grid, SELF_THREADS, sm, st>>>(a);
  CK(cudaGetLastError());
}

static void launch_select_fused(const bf16* X, const bf16* Wt, long long N, int D, int P, int M, const float* mu,
                                const float* mun, const uint8_t* exclude, uint32_t* keys, float* dist_all,
                                cudaStream_t st) {
  thread_local SelFusedArgs a;
  a = SelFusedArgs{};
  a.x_map = make_tmap_2d(X, N, D, D, 64, 128);
  a.w_map = make_tmap_2d(Wt, P, D, D, 64, P);
  a.N = N;
  a.D = D;
  a.M = M;
  a.mu = mu;
  a.mun = mun;
  a.exclude = exclude;
  a.keys = keys;
  a.dist_all = dist_all;
  ProfScope ps(PC_SELECT_PROJ, st);
  switch (P) {
    case 16: launch_select_fused_p<16>(a, D, st); break;
    case 32: launch_select_fused_p<32>(a, D, st); break;
    case 64: launch_select_fused_p<64>(a, D, st); break;
    case 128: launch_select_fused_p<128>(a, D, st); break;
    default: launch_select_fused_p<256>(a, D, st); break;
  }
}

// ---- radix select state: [0] prefix, [1] k remaining, [2] pass, hist[256] ----
struct RadixState {
  uint32_t prefix;
  uint32_t krem;
  uint32_t hist[256];
  uint32_t T;
  uint32_t need_eq;
  uint32_t n_eligible;
  uint32_t ticket;  // blocks of the current pass done (the last one runs the digit pick)
};

__global__ void radix_init_kernel(RadixState* s, int k) {
  if (threadIdx.x == 0) {
    s->prefix = 0;
    s->krem = (uint32_t)k;
    s->n_eligible = 0;
    s->ticket = 0;
  }
  s->hist[threadIdx.x] = 0;
}

__device__ void radix_pick_block(RadixState* s, int shift, int last);

__global__ void __launch_bounds__(256) radix_hist_kernel(const uint32_t* __restrict__ keys, long long N,
                                                         RadixState* s, int shift, uint32_t mask_hi,
                                                         int count_eligible, int last_pass) {
  __shared__ uint32_t h[256];
  __shared__ uint32_t elig;
  h[threadIdx.x] = 0;
  if (threadIdx.x == 0) elig = 0;
  __syncthreads();
  const uint32_t prefix = s->prefix;
  uint32_t e = 0;
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < N; i += (long long)gridDim.x * blockDim.x) {
    const uint32_t key = keys[i];
    if (count_eligible && key) e++;
    if ((key & mask_hi) == prefix) atomicAdd(&h[(key >> shift) & 255u], 1u);
  }
  if (count_eligible) atomicAdd(&elig, e);
  __syncthreads();
  if (h[threadIdx.x]) atomicAdd(&s->hist[threadIdx.x], h[threadIdx.x]);
  if (count_eligible && threadIdx.x == 0) atomicAdd(&s->n_eligible, elig);
  // the last block to finish this pass picks the digit (threadfence-reduction pattern)
  __shared__ bool is_last;
  __threadfence();
  __syncthreads();
  if (threadIdx.x == 0) is_last = atomicAdd(&s->ticket, 1u) == gridDim.x - 1;
  __syncthreads();
  if (is_last) {
    __threadfence();
    radix_pick_block(s, shift, last_pass);
  }
}

// 256 threads: suffix counts of the histogram (digit 255 down), the digit d where the running count reaches krem;
// run by the last block of each histogram pass (no separate launch)
__device__ void radix_pick_block(RadixState* s, int shift, int last) {
  __shared__ uint32_t suf[256];  // suf[d] = count of digits > d
  __shared__ int s_d;
  __shared__ uint32_t wsum[8];
  const int t = threadIdx.x, lane = t & 31, w = t >> 5;
  const int d = 255 - t;  // thread t handles digit 255 - t (descending)
  const uint32_t c = __ldcg(&s->hist[d]);
  uint32_t x = c;  // inclusive scan over t (i.e. over descending digits)
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) wsum[w] = x;
  __syncthreads();
  uint32_t off = 0;
  for (int q = 0; q < w; ++q) off += wsum[q];
  const uint32_t incl = off + x, excl = incl - c;
  suf[d] = excl;
  if (t == 0) s_d = 0;  // fewer keys than k with this prefix (only when k > #keys): take everything
  __syncthreads();
  const uint32_t krem = s->krem;
  if (excl < krem && incl >= krem) s_d = d;  // exactly one digit satisfies this (counts are non-negative)
  __syncthreads();
  if (t == 0) {
    const int dd = s_d;
    s->prefix |= ((uint32_t)dd << shift);
    s->krem = krem - suf[dd];
    if (last) {
      s->T = s->prefix;
      s->need_eq = s->krem;
    }
    s->ticket = 0;
  }
  s->hist[t] = 0;
}

constexpr int EMIT_THREADS = 1024;

__device__ void emit_scan_warp(int nb, const RadixState* s, const int* blk, int* __restrict__ offs,
                               int32_t* out_count, int k);

// per-block counts of (key > T) and (key == T); the last block to finish runs the scan
__global__ void emit_count_kernel(const uint32_t* __restrict__ keys, long long N, RadixState* s,
                                  int* __restrict__ blk, int* __restrict__ offs, int32_t* out_count, int k) {
  __shared__ int sg, se;
  if (threadIdx.x == 0) sg = se = 0;
  __syncthreads();
  const uint32_t T = s->T;
  const long long i = blockIdx.x * (long long)EMIT_THREADS + threadIdx.x;
  int g = 0, e = 0;
  if (i < N) {
    const uint32_t k = keys[i];
    if (T == 0) g = k > 0;
    else {
      g = k > T;
      e = k == T;
    }
  }
  const int wg = __popc(__ballot_sync(0xffffffffu, g)), we = __popc(__ballot_sync(0xffffffffu, e));
  if ((threadIdx.x & 31) == 0) {
    atomicAdd(&sg, wg);
    atomicAdd(&se, we);
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    blk[2 * blockIdx.x] = sg;
    blk[2 * blockIdx.x + 1] = se;
  }
  __shared__ bool is_last;
  __threadfence();
  __syncthreads();
  if (threadIdx.x == 0) is_last = atomicAdd(&s->ticket, 1u) == gridDim.x - 1;
  __syncthreads();
  if (is_last && threadIdx.x < 32) {
    __threadfence();
    emit_scan_warp((int)gridDim.x, s, blk, offs, out_count, k);
    if (threadIdx.x == 0) s->ticket = 0;
  }
}
// exclusive scans: eq prefix per block, then take_b = g_b + clamp(need - eqpre_b, 0, e_b) and its prefix; one warp,
// run by the last block of emit_count_kernel (no separate launch)
__device__ void emit_scan_warp(int nb, const RadixState* s, const int* blk, int* __restrict__ offs,
                               int32_t* out_count, int k) {
  const int lane = threadIdx.x & 31;
  const int need = (int)s->need_eq;
  int run_eq = 0, run_take = 0;
  for (int b0 = 0; b0 < nb; b0 += 32) {
    const int b = b0 + lane;
    const int g = b < nb ? __ldcg(blk + 2 * b) : 0, e = b < nb ? __ldcg(blk + 2 * b + 1) : 0;
    int xe = e;
    for (int o = 1; o < 32; o <<= 1) {
      const int u = __shfl_up_sync(0xffffffffu, xe, o);
      if (lane >= o) xe += u;
    }
    const int eqpre = run_eq + xe - e;
    const int take = g + max(0, min(need - eqpre, e));
    int xt = take;
    for (int o = 1; o < 32; o <<= 1) {
      const int u = __shfl_up_sync(0xffffffffu, xt, o);
      if (lane >= o) xt += u;
    }
    if (b < nb) {
      offs[2 * b] = run_take + xt - take;  // output offset
      offs[2 * b + 1] = eqpre;             // ties before this block
    }
    run_eq += __shfl_sync(0xffffffffu, xe, 31);
    run_take += __shfl_sync(0xffffffffu, xt, 31);
  }
  if (lane == 0) *out_count = min(run_take, k);
}
__global__ void emit_write_kernel(const uint32_t* __restrict__ keys, long long N, const RadixState* s,
                                  const int* __restrict__ offs, int32_t* __restrict__ out_idx,
                                  float* __restrict__ out_dist, int k) {
  __shared__ int wt[EMIT_THREADS / 32], we_[EMIT_THREADS / 32];
  const uint32_t T = s->T;
  const int need = (int)s->need_eq;
  const long long i = blockIdx.x * (long long)EMIT_THREADS + threadIdx.x;
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  uint32_t key = i < N ? keys[i] : 0u;
  const bool g = (T == 0) ? key > 0 : key > T;
  const bool e = (T != 0) && key == T;
  const unsigned be = __ballot_sync(0xffffffffu, e);
  if (lane == 0) we_[w] = __popc(be);
  __syncthreads();
  int eqrank = offs[2 * blockIdx.x + 1] + __popc(be & ((1u << lane) - 1u));
  for (int q = 0; q < w; ++q) eqrank += we_[q];
  const bool take = g || (e && eqrank < need);
  const unsigned bt = __ballot_sync(0xffffffffu, take);
  if (lane == 0) wt[w] = __popc(bt);
  __syncthreads();
  if (take) {
    int o = offs[2 * blockIdx.x] + __popc(bt & ((1u << lane) - 1u));
    for (int q = 0; q < w; ++q) o += wt[q];
    if (o < k) {
      out_idx[o] = (int32_t)i;
      if (out_dist) out_dist[o] = __uint_as_float(key - 1u);
    }
  }
}

// Single-CTA exact top-k for small pools (N <= 1,024 x 32): every thread holds 32 consecutive keys in registers (one
// read of the keys), the four 8-bit MSB radix passes run on the registers (warp-aggregated shared histograms, the digit
// picked by a 256-thread suffix scan), and the ascending stable emit (ties -> lower position) needs two block-wide
// exclusive scans: ties before each thread, then outputs before each thread. One launch.
constexpr int TOPK1_THREADS = 1024, TOPK1_KPT = 32;
constexpr long long TOPK1_MAX_N = (long long)TOPK1_THREADS * TOPK1_KPT;

// exclusive scan of one value per thread over a 1,024-thread block; ws: 33 words of shared memory
__device__ __forceinline__ uint32_t scan1024(uint32_t v, uint32_t* ws, uint32_t& total) {
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  uint32_t x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) ws[w] = x;
  __syncthreads();
  if (w == 0) {
    const uint32_t y = ws[lane];
    uint32_t z = y;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t u = __shfl_up_sync(0xffffffffu, z, o);
      if (lane >= o) z += u;
    }
    ws[lane] = z - y;
    if (lane == 31) ws[32] = z;
  }
  __syncthreads();
  const uint32_t r = ws[w] + x - v;
  total = ws[32];
  __syncthreads();
  return r;
}

__global__ void __launch_bounds__(TOPK1_THREADS, 1) topk_single_kernel(const uint32_t* __restrict__ keys, int N,
                                                                       int k, int32_t* __restrict__ out_idx,
                                                                       float* __restrict__ out_dist,
                                                                       int32_t* __restrict__ out_count) {
  __shared__ uint32_t hist[256];
  __shared__ uint32_t ws[33];
  __shared__ int s_d;
  __shared__ uint32_t s_cum, s_tot;
  const int t = threadIdx.x, lane = t & 31, w = t >> 5;
  const int kpt = (N + TOPK1_THREADS - 1) / TOPK1_THREADS;  // keys per thread (<= 32): every thread busy
  const int base = t * kpt;
  const int nv = max(0, min(kpt, N - base));  // this thread's valid keys
  uint32_t kv[TOPK1_KPT];
#pragma unroll
  for (int j = 0; j < TOPK1_KPT; ++j) kv[j] = j < nv ? __ldg(keys + base + j) : 0u;
  uint32_t prefix = 0, krem = (uint32_t)min(k, N);
#pragma unroll 1
  for (int pass = 0; pass < 4; ++pass) {
    const int shift = 24 - 8 * pass;
    const uint32_t mask_hi = pass == 0 ? 0u : (0xFFFFFFFFu << (32 - 8 * pass));
    if (t < 256) hist[t] = 0;
    if (t == 0) s_d = -1;
    __syncthreads();
    // run-length aggregation over the thread's consecutive keys (the distance keys share their top bytes, so a
    // pass-0 thread issues one atomic), then shared-memory atomics
    uint32_t run_d = 0, run_c = 0;
#pragma unroll
    for (int j = 0; j < TOPK1_KPT; ++j) {
      if (j < nv && (kv[j] & mask_hi) == prefix) {
        const uint32_t dig = (kv[j] >> shift) & 255u;
        if (run_c && dig != run_d) {
          atomicAdd(&hist[run_d], run_c);
          run_c = 0;
        }
        run_d = dig;
        ++run_c;
      }
    }
    if (run_c) atomicAdd(&hist[run_d], run_c);
    __syncthreads();
    uint32_t c = 0, x = 0;
    if (t < 256) {  // thread t: digit 255 - t (descending), inclusive scan = keys with digit >= 255 - t
      c = x = hist[255 - t];
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
        if (lane >= o) x += y;
      }
      if (lane == 31) ws[w] = x;
    }
    __syncthreads();
    if (t < 256) {
      uint32_t off = 0;
      for (int q = 0; q < w; ++q) off += ws[q];
      const uint32_t incl = off + x, excl = incl - c;
      if (excl < krem && incl >= krem) {  // exactly one digit
        s_d = 255 - t;
        s_cum = excl;
      }
      if (t == 255) s_tot = incl;
    }
    __syncthreads();
    const int d = s_d;
    prefix |= (uint32_t)(d >= 0 ? d : 0) << shift;
    krem -= d >= 0 ? s_cum : s_tot;
    __syncthreads();
  }
  const uint32_t T = prefix, need = krem;
  uint32_t e_cnt = 0;
#pragma unroll
  for (int j = 0; j < TOPK1_KPT; ++j) e_cnt += (T != 0 && kv[j] == T) ? 1u : 0u;  // padding keys are 0
  uint32_t tot;
  uint32_t er = scan1024(e_cnt, ws, tot);  // ties before this thread's keys
  uint32_t take_mask = 0, take_cnt = 0;
#pragma unroll
  for (int j = 0; j < TOPK1_KPT; ++j) {
    const bool g = T == 0 ? kv[j] > 0u : kv[j] > T;
    const bool e = T != 0 && kv[j] == T;
    const bool tk = g || (e && er < need);
    er += e ? 1u : 0u;
    take_mask |= (tk ? 1u : 0u) << j;
    take_cnt += tk ? 1u : 0u;
  }
  uint32_t o = scan1024(take_cnt, ws, tot);  // outputs before this thread's keys
#pragma unroll
  for (int j = 0; j < TOPK1_KPT; ++j) {
    if ((take_mask >> j) & 1u) {
      if (o < (uint32_t)k) {
        out_idx[o] = base + j;
        if (out_dist) out_dist[o] = __uint_as_float(kv[j] - 1u);
      }
      ++o;
    }
  }
  if (t == 0) *out_count = (int32_t)min(tot, (uint32_t)k);
}

// exact top-k of 32-bit keys (0 = not eligible), ties -> lower position, emitted in ascending position order
static void topk_emit(const uint32_t* keys, long long N, int k, RadixState* rs, int* blk, int* offs, int32_t* out_idx,
                      float* out_dist, int32_t* out_count, cudaStream_t st) {
  const long long nb = (N + EMIT_THREADS - 1) / EMIT_THREADS;
  const int k_eff = (int)std::min<long long>(k, N);  // the k-th largest must exist
  // single CTA wins below ~24k keys (measured: 27 vs 37 us at 16,384; 45 vs 39 us at 32,768)
  if (N <= std::min<long long>(24576, TOPK1_MAX_N) && !getenv("ADAINF_TOPK_MULTI")) {
    ProfScope ps_topk(PC_SELECT_TOPK, st, 1);
    topk_single_kernel<<<1, TOPK1_THREADS, 0, st>>>(keys, (int)N, k, out_idx, out_dist, out_count);
    CK(cudaGetLastError());
    return;
  }
  ProfScope ps_topk(PC_SELECT_TOPK, st, 7);
  radix_init_kernel<<<1, 256, 0, st>>>(rs, k_eff);
  const int hb = (int)std::min<long long>((N + 1023) / 1024, 4LL * num_sms());
  for (int pass = 0; pass < 4; ++pass) {
    const int shift = 24 - 8 * pass;
    const uint32_t mask_hi = pass == 0 ? 0u : (0xFFFFFFFFu << (32 - 8 * pass));
    radix_hist_kernel<<<hb, 256, 0, st>>>(keys, N, rs, shift, mask_hi, pass == 0, pass == 3);
  }
  emit_count_kernel<<<(unsigned)nb, EMIT_THREADS, 0, st>>>(keys, N, rs, blk, offs, out_count, k);
  emit_write_kernel<<<(unsigned)nb, EMIT_THREADS, 0, st>>>(keys, N, rs, offs, out_idx, out_dist, k);
  CK(cudaGetLastError());
}

struct SelectWs {
  size_t bytes(long long N, int P, int M) const {
    const long long nb = (N + EMIT_THREADS - 1) / EMIT_THREADS;
    return (size_t)N * P * 4 + (size_t)P * 1024 * 2 + (size_t)M * P * 4 + M * 4 + sizeof(RadixState) + N * 4 +
           nb * 16 + (size_t)P * 4 + 4096;
  }
};

void select_retrain(const adainf_select_in& in, int k, int32_t* out_idx, float* out_dist, int32_t* out_count,
                    float* dist_all, cudaStream_t st) {
  const long long N = in.N;
  const int D = in.D, P = in.W_bf16 ? in.P : in.D, M = in.M;
  if (N <= 0 || N > (1LL << 31) - 1 || D <= 0 || D % 8 || D > 1024 || P <= 0 || P > 256 || P % 16 || M <= 0 ||
      M > 4096 || k <= 0)
    throw ShapeError("select: N in 1..2^31, D multiple of 8 <= 1024, P multiple of 16 <= 256, M in 1..4096, k > 0");
  if (!in.X_bf16 || !in.ref) throw InvalidError("select: X and ref are required");
  SelectWs sw;
  void* wsp = nullptr;
  const size_t wsb = sw.bytes(N, P, M);
  CK(cudaMallocAsync(&wsp, wsb, st));
  char* w = (char*)wsp;
  auto take = [&](size_t b) {
    char* p = w;
    w += (b + 255) / 256 * 256;
    return p;
  };
  static int fused_env = -1;
  if (fused_env < 0) {
    const char* e = getenv("ADAINF_SELECT_FUSED");
    fused_env = e ? atoi(e) : 1;
  }
  const bool fused = in.W_bf16 && fused_env && select_fused_ok(D, P, M);
  float* Y = (in.W_bf16 && !fused) ? (float*)take((size_t)N * P * 4) : nullptr;
  bf16* Wt = in.W_bf16 ? (bf16*)take((size_t)P * D * 2) : nullptr;
  float* mu = (float*)take((size_t)M * P * 4);
  float* mun = (float*)take((size_t)M * 4);
  float* zb = (float*)take((size_t)P * 4);
  RadixState* rs = (RadixState*)take(sizeof(RadixState));
  uint32_t* keys = (uint32_t*)take((size_t)N * 4);
  const long long nb = (N + EMIT_THREADS - 1) / EMIT_THREADS;
  int* blk = (int*)take((size_t)nb * 8);
  int* offs = (int*)take((size_t)nb * 8);
  {
    ProfScope ps(PC_SELECT_PROJ, st);
    const int nt = in.W_bf16 ? (D * P + 255) / 256 : 0;
    select_prep_kernel<<<nt + (M * P * 32 + 255) / 256, 256, 0, st>>>(in.ref, (const bf16*)in.W_bf16, D, P, M, nt, Wt,
                                                                       mu);
    if (!fused) ref_norm_kernel<<<(M * 32 + 255) / 256, 256, 0, st>>>(mu, P, M, mun);
    CK(cudaGetLastError());
  }
  if (fused) {
    launch_select_fused((const bf16*)in.X_bf16, Wt, N, D, P, M, mu, mun, in.exclude, keys, dist_all, st);
  } else if (in.W_bf16) {
    CK(cudaMemsetAsync(zb, 0, (size_t)P * 4, st));
    ConvGeom g{};
    g.Cin = D;
    g.Cout = P;
    g.KH = g.KW = 1;
    g.stride = 1;
    g.pad = 0;
    g.H = g.W = g.Ho = g.Wo = 1;
    // Y [N][P] fp32 = X [N][D] . W [D][P] on the tensor cores
    conv_fwd(g, (const bf16*)in.X_bf16, nullptr, nullptr, (int)N, Wt, D, zb, nullptr, nullptr, 0, Y, true, st);
    ProfScope ps(PC_SELECT_COSINE, st);
    if (M > 4)
      cosine_key_multi_kernel<false><<<(unsigned)((N * 32 + 255) / 256), 256, 0, st>>>(Y, N, P, mu, mun, M,
                                                                                      in.exclude, keys, dist_all);
    else
      cosine_key_kernel<false><<<(unsigned)((N * 32 + 255) / 256), 256, 0, st>>>(Y, N, P, mu, mun, M, in.exclude,
                                                                                keys, dist_all);
  } else {
    ProfScope ps(PC_SELECT_COSINE, st);
    if (M > 4)
      cosine_key_multi_kernel<true><<<(unsigned)((N * 32 + 255) / 256), 256, 0, st>>>(in.X_bf16, N, P, mu, mun, M,
                                                                                     in.exclude, keys, dist_all);
    else
      cosine_key_kernel<true><<<(unsigned)((N * 32 + 255) / 256), 256, 0, st>>>(in.X_bf16, N, P, mu, mun, M,
                                                                               in.exclude, keys, dist_all);
  }
  topk_emit(keys, N, k, rs, blk, offs, out_idx, out_dist, out_count, st);
  CK(cudaFreeAsync(wsp, st));
}

// K12: merge of per-shard top-k lists into the global top-k.  Candidate block b (one per shard,
// block_len entries, the first block_count[b] valid) holds local indices i -> global index i * idx_mul + b *
// block_off, with their distances; the keys are scattered into a dense key array over the global index space so
// the same radix select + ascending emit applies (ties -> lower GLOBAL index, reading Q15).
__global__ void merge_scatter_kernel(const float* __restrict__ dist, const int32_t* __restrict__ idx,
                                     const int32_t* __restrict__ block_count, int n_blocks, int block_len,
                                     long long idx_mul, long long block_off, long long n_total,
                                     uint32_t* __restrict__ keys) {
  const long long t = blockIdx.x * (long long)blockDim.x + threadIdx.x;
  if (t >= (long long)n_blocks * block_len) return;
  const int b = (int)(t / block_len), j = (int)(t - (long long)b * block_len);
  const int cnt = block_count ? min(block_count[b], block_len) : block_len;
  if (j >= cnt) return;
  const float d = dist[t];
  const long long g = (long long)idx[t] * idx_mul + b * block_off;
  if (g < 0 || g >= n_total || !(d >= 0.f)) return;
  keys[g] = __float_as_uint(d) + 1u;
}

void select_merge(const float* dist, const int32_t* idx, const int32_t* block_count, int n_blocks, int block_len,
                  long long idx_mul, long long block_off, long long n_total, int k, int32_t* out_idx, float* out_dist,
                  int32_t* out_count, cudaStream_t st) {
  if (n_blocks <= 0 || block_len <= 0 || n_total <= 0 || n_total > (1LL << 31) - 1 || k <= 0 || idx_mul <= 0 ||
      block_off < 0)
    throw ShapeError("select_merge: bad sizes");
  if (!dist || !idx) throw InvalidError("select_merge: dist and idx are required");
  const long long nb = (n_total + EMIT_THREADS - 1) / EMIT_THREADS;
  const size_t bytes = (size_t)n_total * 4 + 256 + sizeof(RadixState) + 256 + (size_t)nb * 16 + 512;
  void* wsp = nullptr;
  CK(cudaMallocAsync(&wsp, bytes, st));
  char* w = (char*)wsp;
  auto take = [&](size_t b) {
    char* p = w;
    w += (b + 255) / 256 * 256;
    return p;
  };
  uint32_t* keys = (uint32_t*)take((size_t)n_total * 4);
  RadixState* rs = (RadixState*)take(sizeof(RadixState));
  int* blk = (int*)take((size_t)nb * 8);
  int* offs = (int*)take((size_t)nb * 8);
  CK(cudaMemsetAsync(keys, 0, (size_t)n_total * 4, st));
  {
    ProfScope ps(PC_SELECT_COSINE, st);
    const long long n = (long long)n_blocks * block_len;
    merge_scatter_kernel<<<(unsigned)((n + 255) / 256), 256, 0, st>>>(dist, idx, block_count, n_blocks, block_len,
                                                                     idx_mul, block_off, n_total, keys);
  }
  topk_emit(keys, n_total, k, rs, blk, offs, out_idx, out_dist, out_count, st);
  CK(cudaFreeAsync(wsp, st));
}

}  // namespace adainf

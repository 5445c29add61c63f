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

namespace adainf {

__global__ void transpose_w_kernel(const bf16* __restrict__ W, int D, int P, bf16* __restrict__ Wt) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= D * P) return;
  const int d = i / P, p = i - d * P;
  Wt[(long long)p * D + d] = W[i];
}

// mu[r][p] = sum_d ref[r][d] * W[d][p]  (fp32); mun[r] = ||mu_r||
__global__ void project_ref_kernel(const float* __restrict__ ref, const bf16* __restrict__ W, int D, int P, int M,
                                   float* __restrict__ mu, float* __restrict__ mun) {
  const int r = blockIdx.x;
  __shared__ float red[256];
  float sq = 0.f;
  for (int p = threadIdx.x; p < P; p += blockDim.x) {
    float a = 0.f;
    if (W)
      for (int d = 0; d < D; ++d) a = fmaf(ref[(long long)r * D + d], __bfloat162float(W[(long long)d * P + p]), a);
    else
      a = ref[(long long)r * D + p];
    mu[(long long)r * P + p] = a;
    sq = fmaf(a, a, sq);
  }
  red[threadIdx.x] = sq;
  __syncthreads();
  for (int o = blockDim.x / 2; o > 0; o >>= 1) {
    if (threadIdx.x < o) red[threadIdx.x] += red[threadIdx.x + o];
    __syncthreads();
  }
  if (threadIdx.x == 0) mun[r] = sqrtf(red[0]);
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

// ---- radix select state: [0] prefix, [1] k remaining, [2] pass, hist[256] ----
struct RadixState {
  uint32_t prefix;
  uint32_t krem;
  uint32_t hist[256];
  uint32_t T;
  uint32_t need_eq;
  uint32_t n_eligible;
};

__global__ void radix_init_kernel(RadixState* s, int k) {
  if (threadIdx.x == 0) {
    s->prefix = 0;
    s->krem = (uint32_t)k;
    s->n_eligible = 0;
  }
  s->hist[threadIdx.x] = 0;
}

__global__ void radix_hist_kernel(const uint32_t* __restrict__ keys, long long N, RadixState* s, int shift,
                                  uint32_t mask_hi, int count_eligible) {
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
}

__global__ void radix_pick_kernel(RadixState* s, int shift, int last) {
  // single warp: find the digit d (from 255 down) where the cumulative count reaches krem
  if (threadIdx.x != 0) return;
  uint32_t krem = s->krem;
  uint32_t cum = 0;
  int d = 255;
  for (; d >= 0; --d) {
    const uint32_t c = s->hist[d];
    if (cum + c >= krem) break;
    cum += c;
  }
  if (d < 0) d = 0;  // fewer keys than k with this prefix (only when k > #keys): take everything
  s->prefix |= ((uint32_t)d << shift);
  s->krem = krem - cum;
  for (int q = 0; q < 256; ++q) s->hist[q] = 0;
  if (last) {
    s->T = s->prefix;
    s->need_eq = s->krem;
  }
}

constexpr int EMIT_THREADS = 1024;

// per-block counts of (key > T) and (key == T)
__global__ void emit_count_kernel(const uint32_t* __restrict__ keys, long long N, const RadixState* s,
                                  int* __restrict__ blk) {
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
}
// exclusive scans: eq prefix per block, then take_b = g_b + clamp(need - eqpre_b, 0, e_b) and its prefix
__global__ void emit_scan_kernel(int nb, const RadixState* s, int* __restrict__ blk, int* __restrict__ offs,
                                 int32_t* out_count, int k) {
  const int lane = threadIdx.x;
  const int need = (int)s->need_eq;
  int run_eq = 0, run_take = 0;
  for (int b0 = 0; b0 < nb; b0 += 32) {
    const int b = b0 + lane;
    const int g = b < nb ? blk[2 * b] : 0, e = b < nb ? blk[2 * b + 1] : 0;
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

// exact top-k of 32-bit keys (0 = not eligible), ties -> lower position, emitted in ascending position order
static void topk_emit(const uint32_t* keys, long long N, int k, RadixState* rs, int* blk, int* offs, int32_t* out_idx,
                      float* out_dist, int32_t* out_count, cudaStream_t st) {
  const long long nb = (N + EMIT_THREADS - 1) / EMIT_THREADS;
  const int k_eff = (int)std::min<long long>(k, N);  // the k-th largest must exist
  ProfScope ps_topk(PC_SELECT_TOPK, st, 12);
  radix_init_kernel<<<1, 256, 0, st>>>(rs, k_eff);
  const int hb = (int)std::min<long long>((N + 1023) / 1024, 4LL * num_sms());
  for (int pass = 0; pass < 4; ++pass) {
    const int shift = 24 - 8 * pass;
    const uint32_t mask_hi = pass == 0 ? 0u : (0xFFFFFFFFu << (32 - 8 * pass));
    radix_hist_kernel<<<hb, 256, 0, st>>>(keys, N, rs, shift, mask_hi, pass == 0);
    radix_pick_kernel<<<1, 32, 0, st>>>(rs, shift, pass == 3);
  }
  emit_count_kernel<<<(unsigned)nb, EMIT_THREADS, 0, st>>>(keys, N, rs, blk);
  emit_scan_kernel<<<1, 32, 0, st>>>((int)nb, rs, blk, offs, out_count, k);
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
  float* Y = in.W_bf16 ? (float*)take((size_t)N * P * 4) : nullptr;
  bf16* Wt = in.W_bf16 ? (bf16*)take((size_t)P * D * 2) : nullptr;
  float* mu = (float*)take((size_t)M * P * 4);
  float* mun = (float*)take((size_t)M * 4);
  float* zb = (float*)take((size_t)P * 4);
  RadixState* rs = (RadixState*)take(sizeof(RadixState));
  uint32_t* keys = (uint32_t*)take((size_t)N * 4);
  const long long nb = (N + EMIT_THREADS - 1) / EMIT_THREADS;
  int* blk = (int*)take((size_t)nb * 8);
  int* offs = (int*)take((size_t)nb * 8);
  { ProfScope ps(PC_SELECT_PROJ, st);
  project_ref_kernel<<<M, 256, 0, st>>>(in.ref, (const bf16*)in.W_bf16, D, P, M, mu, mun); }
  if (in.W_bf16) {
    { ProfScope ps(PC_SELECT_PROJ, st);
    transpose_w_kernel<<<(D * P + 255) / 256, 256, 0, st>>>((const bf16*)in.W_bf16, D, P, Wt); }
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
  RadixState* unused = nullptr;
  (void)unused;
  topk_emit(keys, n_total, k, rs, blk, offs, out_idx, out_dist, out_count, st);
  CK(cudaFreeAsync(wsp, st));
}

}  // namespace adainf

// Microbenchmark (not product code): what does a tile boundary cost an N = 64 tcgen05 MMA stream?  One thread
// per SM issues `per` M=128 N=64 K=16 MMAs per tile into accumulator (t % NACC); every tile commits to its own
// mbarrier (ring of 8) `ncommit` times; every `group` tiles the issuer waits for the commit of tile (t - lag)
// (lag >= group: an old, normally completed phase).  Prints cycles per MMA.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I paper_conf_sigcomm_shubhas23_b200/csrc \
//   tools/exp_commit.cu -o /tmp/exp_commit
#include <cstdio>
#include <vector>
#include "common.cuh"

using namespace adainf;

struct Offs {
  int toff[9];  // runtime tap offsets (16-byte units), as the window kernels pass them
};

// STYLE 0: descriptor offsets are compile-time constants; STYLE 1: per-tap runtime offsets from the kernel
// parameters (the layer-1 window kernel's pattern: base + toff[tap] + 2 * kk)
template <int PER, int STYLE>
__global__ void __launch_bounds__(128, 1) rate(int tiles, int nacc, int ncommit, int group, int lag,
                                               const __grid_constant__ Offs o, long long* cycles) {
  __shared__ __align__(1024) uint8_t sA[20480];
  __shared__ __align__(1024) uint8_t sB[12288];
  __shared__ uint64_t bar[8], bar2[8], fin2[8], fin;
  __shared__ uint32_t tmem_slot;
  const int warp = threadIdx.x >> 5;
  for (int i = threadIdx.x; i < 20480 / 16; i += 128) ((uint4*)sA)[i] = make_uint4(0, 0, 0, 0);
  for (int i = threadIdx.x; i < 12288 / 16; i += 128) ((uint4*)sB)[i] = make_uint4(0, 0, 0, 0);
  if (threadIdx.x == 0) {
    for (int q = 0; q < 8; ++q) mbar_init(&bar[q], 1), mbar_init(&bar2[q], 1), mbar_init(&fin2[q], 1);
    mbar_init(&fin, 1);
    fence_mbar_init();
  }
  if (warp == 0) tmem_alloc<512>(&tmem_slot);
  fence_proxy_async_smem();
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = tmem_slot;
  if (warp == 0) {
    constexpr uint32_t IDESC = make_idesc(128, 64, 0, 0);
    const uint64_t ad = make_sdesc(smem_u32(sA), 16, 1024), bd = make_sdesc(smem_u32(sB), 16, 1024);
    uint32_t toff[9];
#pragma unroll
    for (int tp = 0; tp < 9; ++tp) toff[tp] = (uint32_t)o.toff[tp];
    const long long t0 = clock64();
    for (int t = 0; t < tiles; ++t) {
      if (group > 0 && t % group == 0 && t >= lag) {
        const int q = t - lag;
        mbar_wait(&bar[q & 7], (q >> 3) & 1);
      }
      if (elect_one()) {
        const uint32_t d = tmem + (uint32_t)((t % nacc) * 64);
        if (STYLE == 6 || STYLE == 7) {
          // tap-shifted views (start offsets of 1..3 x 128 B, not 1024-aligned): STYLE 6 MN-major A with two
          // M atoms at a tap-pair distance (the weight-gradient window kernel), STYLE 7 K-major A (layer-1 fwd)
          constexpr uint32_t ID2 = make_idesc(128, 64, STYLE == 6 ? 1 : 0, 0);
#pragma unroll
          for (int i = 0; i < PER; ++i) {
            const uint32_t sh = (uint32_t)((i / 4) % 3) * 8u;  // 0, 128, 256 B
            const uint64_t am = STYLE == 6 ? make_sdesc(smem_u32(sA) + sh * 16u, 1152, 1024) + (uint32_t)((i % 4) * 128)
                                           : make_sdesc(smem_u32(sA) + sh * 16u, 16, 1024) + (uint32_t)(2 * (i % 4));
            umma_bf16(d, am, bd + (uint32_t)(2 * (i % 4)), ID2, i > 0);
          }
        } else if (STYLE == 4 || STYLE == 5) {
          // MN-major A (STYLE 4) / MN-major A and B (STYLE 5): SW128 atoms of 64 MN elements x 8 K rows; one
          // K = 16 step = 16 rows of 128 B = +2 KB (128 descriptor units); two 64-row M atoms 8 KB apart
          constexpr uint32_t ID2 = make_idesc(128, 64, 1, STYLE == 5 ? 1 : 0);
          const uint64_t am = make_sdesc(smem_u32(sA), 8192, 1024), bm = STYLE == 5 ? make_sdesc(smem_u32(sB), 8192, 1024) : bd;
#pragma unroll
          for (int i = 0; i < PER; ++i) {
            const uint32_t ko = (uint32_t)((i % 4) * 128);
            umma_bf16(d, am + ko, STYLE == 5 ? bm + ko : bm + (uint32_t)(2 * (i % 4)), ID2, i > 0);
          }
        } else if (STYLE >= 2) {
          // two tiles per unit, MMAs alternating between their accumulators (same B for each pair); STYLE 3
          // keeps the pair's B in the weight-stationary collector (fill / lastuse)
          const uint32_t d0 = tmem + (uint32_t)((t % 2) * 128);
#pragma unroll
          for (int i = 0; i < PER; ++i) {
            const int j = i / 2;
            const uint32_t aoff = (uint32_t)(((j / 4) % 4) * 64 + 2 * (j % 4) + (i & 1) * 16);
            const uint64_t bdesc = bd + (uint32_t)((j / 4) % 4 * 128 + 2 * (j % 4)) / 4;
            const uint32_t dd = d0 + (uint32_t)((i & 1) * 64);
            const uint32_t acc = i >= 2;
            if (STYLE == 2) {
              umma_bf16(dd, ad + aoff, bdesc, IDESC, acc);
            } else if ((i & 1) == 0) {
              asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\n"
                           "tcgen05.mma.ws.cta_group::1.kind::f16.collector::b0::fill [%0], %1, %2, %3, p;\n}\n" ::"r"(dd),
                           "l"(ad + aoff), "l"(bdesc), "r"(IDESC), "r"(acc));
            } else {
              asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\n"
                           "tcgen05.mma.ws.cta_group::1.kind::f16.collector::b0::lastuse [%0], %1, %2, %3, p;\n}\n" ::"r"(dd),
                           "l"(ad + aoff), "l"(bdesc), "r"(IDESC), "r"(acc));
            }
          }
        } else {
#pragma unroll
        for (int i = 0; i < PER; ++i) {
          const uint32_t aoff = STYLE == 0 ? (uint32_t)(((i / 4) % 4) * 64 + 2 * (i % 4))
                                           : toff[(i / 4) % 9] + 2u * (i % 4);
          umma_bf16(d, ad + aoff, bd + (uint32_t)((i / 4) % 4 * 128 + 2 * (i % 4)) / 4, IDESC, i > 0);
        }
        }
        if (ncommit >= 3) umma_commit(&fin2[t & 7]);
        if (ncommit >= 2) umma_commit(&bar2[t & 7]);
        if (ncommit >= 1) umma_commit(&bar[t & 7]);
      }
      __syncwarp();
    }
    if (elect_one()) umma_commit(&fin);
    __syncwarp();
    mbar_wait(&fin, 0);
    if (threadIdx.x == 0) cycles[blockIdx.x] = clock64() - t0;
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 0) {
    tc_fence_after();
    tmem_dealloc<512>(tmem);
  }
}

int main() {
  long long* cyc;
  cudaMalloc(&cyc, 8 * 148);
  Offs o;
  for (int tp = 0; tp < 9; ++tp) o.toff[tp] = ((tp % 3) * 8 + (tp / 3) * 64) % 192;  // within the 16 KB tile
  struct Cfg { int per, style, nacc, ncommit, group, lag; const char* what; };
  const Cfg cfgs[] = {
      {36, 0, 2, 0, 0, 0, "36/tile const descs: no commit, no wait"},
      {36, 0, 2, 1, 0, 0, "36/tile const descs: 1 commit, no wait"},
      {36, 0, 2, 2, 0, 0, "36/tile const descs: 2 commits, no wait"},
      {36, 0, 2, 1, 1, 2, "36/tile const descs: 1 commit, wait t-2"},
      {36, 0, 2, 2, 1, 2, "36/tile const descs: 2 commits, wait t-2"},
      {36, 1, 2, 2, 1, 2, "36/tile runtime tap offsets: 2 commits, wait t-2 (layer-1 kernel)"},
      {36, 1, 2, 1, 1, 2, "36/tile runtime tap offsets: 1 commit, wait t-2"},
      {36, 1, 4, 1, 2, 4, "36/tile runtime tap offsets: 1 commit, wait t-4 every 2nd"},
      {72, 0, 2, 1, 1, 2, "72/tile const descs: 1 commit, wait t-2"},
      {144, 6, 2, 0, 0, 0, "144/tile MN-major A, tap-shifted starts, atoms 1152 B apart"},
      {144, 7, 2, 0, 0, 0, "144/tile K-major A, tap-shifted starts"},
      {36, 4, 2, 0, 0, 0, "36/tile MN-major A, no commit, no wait"},
      {36, 5, 2, 0, 0, 0, "36/tile MN-major A and B, no commit, no wait"},
      {144, 0, 2, 0, 0, 0, "144/tile K-major, no commit"},
      {144, 4, 2, 0, 0, 0, "144/tile MN-major A, no commit"},
      {144, 5, 2, 0, 0, 0, "144/tile MN-major A and B, no commit"},
      {72, 2, 2, 1, 1, 2, "2-tile unit (72 MMAs alternating 2 accs): 1 commit, wait u-2"},
      {72, 3, 2, 1, 1, 2, "2-tile unit + B collector (ws fill/lastuse): 1 commit, wait u-2"},
      {72, 2, 2, 3, 1, 2, "2-tile unit: 3 commits, wait u-2"},
      {32, 2, 2, 1, 1, 2, "stem 2-row unit (32 MMAs alternating): 1 commit, wait u-2"},
      {32, 3, 2, 1, 1, 2, "stem 2-row unit + B collector: 1 commit, wait u-2"},
      {16, 0, 2, 1, 1, 2, "16/tile const descs (stem row): 1 commit, wait t-2"},
      {16, 0, 4, 1, 1, 4, "16/tile const descs: 1 commit, wait t-4"},
      {16, 0, 2, 2, 1, 2, "16/tile const descs: 2 commits, wait t-2"},
  };
  for (const Cfg& c : cfgs) {
    const int tiles = 144000 / c.per;
    if (c.per == 36 && c.style == 0) rate<36, 0><<<148, 128>>>(tiles, c.nacc, c.ncommit, c.group, c.lag, o, cyc);
    if (c.per == 36 && c.style == 1) rate<36, 1><<<148, 128>>>(tiles, c.nacc, c.ncommit, c.group, c.lag, o, cyc);
    if (c.per == 36 && c.style == 4) rate<36, 4><<<148, 128>>>(tiles, c.nacc, c.ncommit, c.group, c.lag, o, cyc);
    if (c.per == 36 && c.style == 5) rate<36, 5><<<148, 128>>>(tiles, c.nacc, c.ncommit, c.group, c.lag, o, cyc);
    if (c.per == 144 && c.style == 6) rate<144, 6><<<148, 128>>>(tiles, c.nacc, c.ncommit, c.group, c.lag, o, cyc);
    if (c.per == 144 && c.style == 7) rate<144, 7><<<148, 128>>>(tiles, c.nacc, c.ncommit, c.group, c.lag, o, cyc);
    if (c.per == 144 && c.style == 0) rate<144, 0><<<148, 128>>>(tiles, c.nacc, c.ncommit, c.group, c.lag, o, cyc);
    if (c.per == 144 && c.style == 4) rate<144, 4><<<148, 128>>>(tiles, c.nacc, c.ncommit, c.group, c.lag, o, cyc);
    if (c.per == 144 && c.style == 5) rate<144, 5><<<148, 128>>>(tiles, c.nacc, c.ncommit, c.group, c.lag, o, cyc);
    if (c.per == 72 && c.style == 0) rate<72, 0><<<148, 128>>>(tiles, c.nacc, c.ncommit, c.group, c.lag, o, cyc);
    if (c.per == 72 && c.style == 2) rate<72, 2><<<148, 128>>>(tiles, c.nacc, c.ncommit, c.group, c.lag, o, cyc);
    if (c.per == 72 && c.style == 3) rate<72, 3><<<148, 128>>>(tiles, c.nacc, c.ncommit, c.group, c.lag, o, cyc);
    if (c.per == 32 && c.style == 2) rate<32, 2><<<148, 128>>>(tiles, c.nacc, c.ncommit, c.group, c.lag, o, cyc);
    if (c.per == 32 && c.style == 3) rate<32, 3><<<148, 128>>>(tiles, c.nacc, c.ncommit, c.group, c.lag, o, cyc);
    if (c.per == 16) rate<16, 0><<<148, 128>>>(tiles, c.nacc, c.ncommit, c.group, c.lag, o, cyc);
    cudaError_t e = cudaDeviceSynchronize();
    long long hc[148];
    cudaMemcpy(hc, cyc, 8 * 148, cudaMemcpyDeviceToHost);
    double s = 0;
    for (int i = 0; i < 148; ++i) s += hc[i];
    printf("%-66s %6.1f cycles/MMA  %7.0f per tile (%s)\n", c.what, s / 148 / (tiles * (double)c.per),
           s / 148 / tiles, cudaGetErrorString(e));
  }
  return 0;
}

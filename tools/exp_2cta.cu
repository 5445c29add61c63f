// Experiment (not product code): validate the tcgen05 CTA-pair mechanics on this B200 before using them in
// the conv kernels.  One cluster of 2 CTAs computes D[256][N] = A[256][K] * B[N][K]^T (bf16 in, fp32 out):
// CTA r holds A rows [128r, 128r+128) and B rows [r*N/2, (r+1)*N/2) in its shared memory (TMA, 128B swizzle),
// the leader issues tcgen05.mma.cta_group::2 (M = 256), commits multicast to both CTAs, each CTA reads its
// 128 accumulator lanes.  Peer readiness reaches the leader through a remote mbarrier arrive.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -std=c++17 -O2 -I<csrc> tools/exp_2cta.cu <csrc>/tma.cu
// Usage: exp_2cta [bsplit=1]   (bsplit=0 loads the whole B in both CTAs, to test the alternative reading)
#include <cstdio>
#include <cstdlib>
#include <vector>
#include <cmath>

#include "common.cuh"
#include "tma.cuh"

using namespace adainf;

constexpr int M = 256, N = 128, K = 64;

struct Args {
  CUtensorMap a_map, b_map;
  float* d;
  int bsplit;
};

__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(128, 1) pair_gemm(const __grid_constant__ Args a) {
  __shared__ __align__(1024) uint8_t sA[128 * 128];  // 128 rows x 64 bf16
  __shared__ __align__(1024) uint8_t sB[128 * 128];  // up to 128 rows x 64 bf16
  __shared__ uint64_t full, peer_ready, tfull;
  __shared__ uint32_t tmem_slot;
  const uint32_t rank = cluster_ctarank();
  const int warp = threadIdx.x >> 5;
  if (threadIdx.x == 0) {
    mbar_init(&full, 1);
    mbar_init(&peer_ready, 1);
    mbar_init(&tfull, 1);
    fence_mbar_init();
  }
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(&tmem_slot)),
                 "n"(128));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;");
  }
  tc_fence_before();
  cluster_sync_all();
  tc_fence_after();
  const uint32_t tmem = tmem_slot;
  const int brows = a.bsplit ? N / 2 : N;
  if (threadIdx.x == 0) {
    mbar_expect_tx(&full, 128 * 128 + brows * 128);
    tma_load_2d(smem_u32(sA), &a.a_map, &full, 0, (int)rank * 128);
    tma_load_2d(smem_u32(sB), &a.b_map, &full, 0, a.bsplit ? (int)rank * (N / 2) : 0);
    mbar_wait(&full, 0);
    if (rank == 1) mbar_arrive_cluster(mapa_rank(smem_u32(&peer_ready), 0));
  }
  if (rank == 0 && threadIdx.x == 0) {
    mbar_wait(&peer_ready, 0);
    tc_fence_after();
    constexpr uint32_t IDESC = make_idesc(M, N, 0, 0);
    const uint64_t ad = make_sdesc(smem_u32(sA), 16, 1024), bd = make_sdesc(smem_u32(sB), 16, 1024);
#pragma unroll
    for (int kk = 0; kk < K / 16; ++kk) {
      asm volatile(
          "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
          "tcgen05.mma.cta_group::2.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem),
          "l"(ad + 2u * kk), "l"(bd + 2u * kk), "r"(IDESC), "r"((uint32_t)(kk > 0))
          : "memory");
    }
    asm volatile(
        "tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;" ::"r"(
            smem_u32(&tfull)),
        "h"((uint16_t)3)
        : "memory");
  }
  __syncwarp();
  mbar_wait(&tfull, 0);
  tc_fence_after();
  const int row = warp * 32 + (threadIdx.x & 31);
  for (int c0 = 0; c0 < N; c0 += 32) {
    float v[32];
    tmem_ld32(tmem + c0 + ((uint32_t)(warp * 32) << 16), v);
    for (int i = 0; i < 32; ++i) a.d[(size_t)(rank * 128 + row) * N + c0 + i] = v[i];
  }
  tc_fence_before();
  cluster_sync_all();
  if (warp == 0) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(tmem), "n"(128));
  }
}

template <int CG, int NN = N, int MNMAJ = 0>  // MNMAJ: 1 = MN-major A and B (the weight-gradient operands)
__global__ void __launch_bounds__(128, 1) mma_rate(const __grid_constant__ Args a, int iters, long long* cycles) {
  __shared__ __align__(1024) uint8_t sA[128 * 128];
  __shared__ __align__(1024) uint8_t sB[128 * 128];
  __shared__ uint64_t done;
  __shared__ uint32_t tmem_slot;
  const int warp = threadIdx.x >> 5;
  const uint32_t rank = CG == 2 ? cluster_ctarank() : 0;
  if (threadIdx.x == 0) {
    mbar_init(&done, 1);
    fence_mbar_init();
  }
  if (warp == 0) {
    if (CG == 2) {
      asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(&tmem_slot)),
                   "n"(128));
      asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;");
    } else {
      asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(&tmem_slot)),
                   "n"(128));
      asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
  }
  tc_fence_before();
  if (CG == 2) cluster_sync_all(); else __syncthreads();
  tc_fence_after();
  const uint32_t tmem = tmem_slot;
  if (rank == 0 && threadIdx.x == 0) {
    const long long t0 = clock64();
    // MN-major: SW128 atoms of 64 MN x 8 K rows, 64-wide atoms 8 KB apart, K = 16 step = 2 KB (128 units)
    const uint64_t ad = MNMAJ ? make_sdesc(smem_u32(sA), 8192, 1024) : make_sdesc(smem_u32(sA), 16, 1024);
    const uint64_t bd = MNMAJ ? make_sdesc(smem_u32(sB), 8192, 1024) : make_sdesc(smem_u32(sB), 16, 1024);
    const uint32_t kst = MNMAJ ? 128u : 2u;
    for (int i = 0; i < iters; ++i) {
#pragma unroll
      for (int kk = 0; kk < 4; ++kk) {
        if (CG == 2) {
          constexpr uint32_t IDESC = make_idesc(256, NN, MNMAJ, MNMAJ);
          asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                       "tcgen05.mma.cta_group::2.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem),
                       "l"(ad + kst * kk), "l"(bd + kst * kk), "r"(IDESC), "r"(1u) : "memory");
        } else {
          constexpr uint32_t IDESC = make_idesc(128, NN, MNMAJ, MNMAJ);
          asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                       "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem),
                       "l"(ad + kst * kk), "l"(bd + kst * kk), "r"(IDESC), "r"(1u) : "memory");
        }
      }
    }
    if (CG == 2)
      asm volatile("tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;"
                   ::"r"(smem_u32(&done)), "h"((uint16_t)3) : "memory");
    else
      asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(&done))
                   : "memory");
    mbar_wait(&done, 0);
    cycles[blockIdx.x] = clock64() - t0;
  }
  if (CG == 2 && rank == 1 && threadIdx.x == 0) mbar_wait(&done, 0);
  tc_fence_before();
  if (CG == 2) cluster_sync_all(); else __syncthreads();
  if (warp == 0) {
    tc_fence_after();
    if (CG == 2) asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(tmem), "n"(128));
    else asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "n"(128));
  }
}

// per-tile commit cost: `per` MMAs (N=64) per tile into alternating accumulators, then a commit to an mbarrier
// (as the window conv kernels do); measures cycles per MMA including the per-tile commit
template <int NB, int NC = 1, int MODE = 0>
__global__ void __launch_bounds__(128, 1) mma_commit_rate(int tiles, int per, long long* cycles) {
  __shared__ __align__(1024) uint8_t sA[128 * 128];
  __shared__ __align__(1024) uint8_t sB[128 * 128];
  __shared__ uint64_t bar[NB], bar2[NB];
  __shared__ uint32_t tmem_slot;
  const int warp = threadIdx.x >> 5;
  if (threadIdx.x == 0) {
    for (int q = 0; q < NB; ++q) mbar_init(&bar[q], 1), mbar_init(&bar2[q], 1);
    fence_mbar_init();
  }
  if (warp == 0) tmem_alloc<NB * 64 < 32 ? 32 : NB * 64>(&tmem_slot);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = tmem_slot;
  if (threadIdx.x == 0) {
    const long long t0 = clock64();
    const uint64_t ad = make_sdesc(smem_u32(sA), 16, 1024), bd = make_sdesc(smem_u32(sB), 16, 1024);
    constexpr uint32_t IDESC = make_idesc(128, 64, 0, 0);
    for (int t = 0; t < tiles; ++t) {
      const int b = MODE == 1 ? 0 : t % NB;
      if (MODE == 0 && t >= NB) mbar_wait(&bar[b], ((t / NB) - 1) & 1);  // accumulator b drained
      // MODE 3: commit every tile but never wait (the barrier phase is simply overrun; timing only)
      if (MODE == 1 && t >= 1) mbar_wait(&bar[0], (t - 1) & 1);
      for (int i = 0; i < per; ++i)
        umma_bf16(tmem + b * 64, ad + 2u * (i & 3), bd + 2u * (i & 3), IDESC, MODE == 1 ? 1 : (i > 0));
      if (MODE != 2) {
        if (NC == 2) umma_commit(&bar2[b]);
        umma_commit(&bar[b]);
      }
    }
    if (MODE == 2 || MODE == 3) umma_commit(&bar2[0]);
    if (MODE == 2 || MODE == 3) mbar_wait(&bar2[0], 0);
    else if (MODE == 0) mbar_wait(&bar[(tiles - 1) % NB], ((tiles - 1) / NB) & 1);
    else if (MODE == 1) mbar_wait(&bar[0], (tiles - 1) & 1);

    cycles[blockIdx.x] = clock64() - t0;
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 0) {
    tc_fence_after();
    tmem_dealloc<NB * 64 < 32 ? 32 : NB * 64>(tmem);
  }
}

static float bf(uint16_t h) {
  uint32_t u = (uint32_t)h << 16;
  float f;
  memcpy(&f, &u, 4);
  return f;
}

int main(int argc, char** argv) {
  const int bsplit = argc > 1 ? atoi(argv[1]) : 1;
  std::vector<uint16_t> hA(M * K), hB(N * K);
  srand(1);
  for (auto& x : hA) x = (uint16_t)(0x3c00 + (rand() % 512) - 256);  // ~ +-[0.5, 2)
  for (auto& x : hB) x = (uint16_t)(0x3c00 + (rand() % 512) - 256);
  for (size_t i = 0; i < hA.size(); i += 3) hA[i] ^= 0x8000;
  void *dA, *dB;
  float* dD;
  cudaMalloc(&dA, hA.size() * 2);
  cudaMalloc(&dB, hB.size() * 2);
  cudaMalloc(&dD, (size_t)M * N * 4);
  cudaMemcpy(dA, hA.data(), hA.size() * 2, cudaMemcpyHostToDevice);
  cudaMemcpy(dB, hB.data(), hB.size() * 2, cudaMemcpyHostToDevice);
  cudaMemset(dD, 0, (size_t)M * N * 4);
  Args a{};
  a.a_map = make_tmap_2d(dA, M, K, K, 64, 128);
  a.b_map = make_tmap_2d(dB, N, K, K, 64, bsplit ? N / 2 : N);
  a.d = dD;
  a.bsplit = bsplit;
  pair_gemm<<<2, 128>>>(a);
  cudaError_t e = cudaDeviceSynchronize();
  printf("kernel: %s\n", cudaGetErrorString(e));
  std::vector<float> hD((size_t)M * N);
  cudaMemcpy(hD.data(), dD, hD.size() * 4, cudaMemcpyDeviceToHost);
  double maxerr = 0;
  int bad_lo = 0, bad_hi = 0;
  for (int i = 0; i < M; ++i)
    for (int j = 0; j < N; ++j) {
      double ref = 0;
      for (int k = 0; k < K; ++k) ref += (double)bf(hA[i * K + k]) * bf(hB[j * K + k]);
      const double err = fabs(ref - hD[(size_t)i * N + j]);
      maxerr = fmax(maxerr, err);
      if (err > 1e-2 * (1 + fabs(ref))) (j < N / 2 ? bad_lo : bad_hi)++;
    }
  {
    long long* cyc;
    cudaMalloc(&cyc, 8 * 296);
    const int iters = 20000;
    for (int cg = 1; cg <= 2; ++cg) {
      cudaEvent_t e0, e1;
      cudaEventCreate(&e0);
      cudaEventCreate(&e1);
      cudaEventRecord(e0);
      if (cg == 1) mma_rate<1><<<148, 128>>>(a, iters, cyc);
      else {
        cudaLaunchConfig_t cfg = {};
        cfg.gridDim = dim3(148);
        cfg.blockDim = dim3(128);
        cudaLaunchAttribute at[1];
        at[0].id = cudaLaunchAttributeClusterDimension;
        at[0].val.clusterDim.x = 2; at[0].val.clusterDim.y = 1; at[0].val.clusterDim.z = 1;
        cfg.attrs = at;
        cfg.numAttrs = 1;
        cudaLaunchKernelEx(&cfg, mma_rate<2>, a, iters, cyc);
      }
      cudaEventRecord(e1);
      cudaError_t er = cudaEventSynchronize(e1);
      float ms = 0;
      cudaEventElapsedTime(&ms, e0, e1);
      long long hc[148];
      cudaMemcpy(hc, cyc, 8 * 148, cudaMemcpyDeviceToHost);
      const double flop = 2.0 * (cg == 2 ? 74 : 148) * (double)iters * 4 * (cg == 2 ? 256 : 128) * N * 16;
      printf("cta_group::%d M=%d N=%d: %.3f ms (%s) -> %.1f TFLOP/s, cycles/MMA (leader 0) %.1f\n", cg, 128 * cg, N, ms,
             cudaGetErrorString(er), flop / ms / 1e9, (double)hc[0] / (iters * 4));
    }
  }
  {
    long long* cyc2;
    cudaMalloc(&cyc2, 8 * 296);
    auto run1 = [&](auto kern, int nn) {
      cudaEvent_t e0, e1;
      cudaEventCreate(&e0);
      cudaEventCreate(&e1);
      cudaEventRecord(e0);
      kern<<<148, 128>>>(a, 20000, cyc2);
      cudaEventRecord(e1);
      cudaEventSynchronize(e1);
      float ms = 0;
      cudaEventElapsedTime(&ms, e0, e1);
      long long hc[1];
      cudaMemcpy(hc, cyc2, 8, cudaMemcpyDeviceToHost);
      printf("cta_group::1 M=128 N=%d K=16: %.1f cycles per MMA, %.1f TFLOP/s\n", nn, (double)hc[0] / 80000,
             2.0 * 148 * 80000.0 * 128 * nn * 16 / ms / 1e9);
    };
    run1(mma_rate<1, 64>, 64);
    {  // CTA pair at N = 64 (M = 256): each SM reads its A half and HALF of B per MMA
      cudaLaunchConfig_t cfg = {};
      cfg.gridDim = dim3(148);
      cfg.blockDim = dim3(128);
      cudaLaunchAttribute at[1];
      at[0].id = cudaLaunchAttributeClusterDimension;
      at[0].val.clusterDim.x = 2; at[0].val.clusterDim.y = 1; at[0].val.clusterDim.z = 1;
      cfg.attrs = at;
      cfg.numAttrs = 1;
      cudaLaunchKernelEx(&cfg, mma_rate<2, 64>, a, 20000, cyc2);
      cudaDeviceSynchronize();
      long long hc[1];
      cudaMemcpy(hc, cyc2, 8, cudaMemcpyDeviceToHost);
      printf("cta_group::2 M=256 N=64 K=16: %.1f cycles per MMA (per-SM work = one M=128 N=64 K=16 tile)\n",
             (double)hc[0] / 80000);
      // N = 128 (the smem tiles hold 128 rows) K-major vs MN-major operands, single CTA and pair
      const char* nm[2] = {"K-major", "MN-major"};
      for (int mn = 0; mn < 2; ++mn) {
        if (mn == 0) { mma_rate<1, 128, 0><<<148, 128>>>(a, 20000, cyc2); }
        else { mma_rate<1, 128, 1><<<148, 128>>>(a, 20000, cyc2); }
        cudaDeviceSynchronize();
        cudaMemcpy(hc, cyc2, 8, cudaMemcpyDeviceToHost);
        printf("cta_group::1 M=128 N=128 %s A and B: %.1f cycles per MMA\n", nm[mn], (double)hc[0] / 80000);
        if (mn == 0) cudaLaunchKernelEx(&cfg, mma_rate<2, 128, 0>, a, 20000, cyc2);
        else cudaLaunchKernelEx(&cfg, mma_rate<2, 128, 1>, a, 20000, cyc2);
        cudaDeviceSynchronize();
        cudaMemcpy(hc, cyc2, 8, cudaMemcpyDeviceToHost);
        printf("cta_group::2 M=256 N=128 %s A and B: %.1f cycles per MMA (ideal 64)\n", nm[mn], (double)hc[0] / 80000);
      }
    }
    for (int per : {36}) {
      const int tiles = 80000 / per;
      mma_commit_rate<2, 2><<<148, 128>>>(tiles, per, cyc2);
      cudaDeviceSynchronize();
      long long hc[1];
      cudaMemcpy(hc, cyc2, 8, cudaMemcpyDeviceToHost);
      printf("N=64, 2 accumulators, TWO commits per tile, %d MMAs per tile: %.1f cycles per MMA\n", per,
             (double)hc[0] / (tiles * per));
    }
    {
      const int per = 36, tiles = 80000 / per;
      long long hc[1];
      mma_commit_rate<2, 1, 1><<<148, 128>>>(tiles, per, cyc2);
      cudaDeviceSynchronize();
      cudaMemcpy(hc, cyc2, 8, cudaMemcpyDeviceToHost);
      printf("N=64, ONE accumulator, commit + wait every 36 MMAs: %.1f cycles per MMA\n", (double)hc[0] / (tiles * per));
      mma_commit_rate<2, 1, 3><<<148, 128>>>(tiles, per, cyc2);
      cudaDeviceSynchronize();
      cudaMemcpy(hc, cyc2, 8, cudaMemcpyDeviceToHost);
      printf("N=64, commit every 36 MMAs, never waited on: %.1f cycles per MMA\n", (double)hc[0] / (tiles * per));
      mma_commit_rate<2, 1, 2><<<148, 128>>>(tiles, per, cyc2);
      cudaDeviceSynchronize();
      cudaMemcpy(hc, cyc2, 8, cudaMemcpyDeviceToHost);
      printf("N=64, switch accumulator every 36 MMAs (fresh accumulate), no commit: %.1f cycles per MMA\n",
             (double)hc[0] / (tiles * per));
    }
    for (int nbuf : {2, 4})
      for (int per : {36, 72, 144}) {
        const int tiles = 80000 / per;
        if (nbuf == 2) mma_commit_rate<2><<<148, 128>>>(tiles, per, cyc2);
        else mma_commit_rate<4><<<148, 128>>>(tiles, per, cyc2);
        cudaDeviceSynchronize();
        long long hc[1];
        cudaMemcpy(hc, cyc2, 8, cudaMemcpyDeviceToHost);
        printf("N=64, %d accumulators, %d MMAs per committed tile: %.1f cycles per MMA\n", nbuf, per,
               (double)hc[0] / (tiles * per));
      }
    run1(mma_rate<1, 128>, 128);
    run1(mma_rate<1, 256>, 256);
  }
  {
    for (int smem_kb : {0, 100, 200}) {
      cudaFuncSetAttribute(mma_rate<2>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem_kb * 1024);
      cudaLaunchConfig_t cfg = {};
      cfg.gridDim = dim3(148);
      cfg.blockDim = dim3(128);
      cfg.dynamicSmemBytes = smem_kb * 1024;
      cudaLaunchAttribute at[1];
      at[0].id = cudaLaunchAttributeClusterDimension;
      at[0].val.clusterDim.x = 2; at[0].val.clusterDim.y = 1; at[0].val.clusterDim.z = 1;
      cfg.attrs = at;
      cfg.numAttrs = 1;
      int nc = -1;
      cudaError_t er = cudaOccupancyMaxActiveClusters(&nc, mma_rate<2>, &cfg);
      printf("max active 2-CTA clusters at %d KB dynamic smem: %d (%s)\n", smem_kb, nc, cudaGetErrorString(er));
    }
  }
  printf("bsplit=%d max abs err %.3e, bad cols<N/2: %d, bad cols>=N/2: %d (of %d each)\n", bsplit, maxerr, bad_lo,
         bad_hi, M * N / 2);
  return 0;
}

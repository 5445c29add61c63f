// Microbenchmark + semantics check: does the tcgen05 operand collector (A_KEEP / B_KEEP reuse) remove the
// shared-memory operand reads of N = 64 MMAs?  Standalone: nvcc -gencode arch=compute_100a,code=sm_100a -O3 \
//   -I paper_conf_sigcomm_shubhas23_b200/csrc tools/exp_collector.cu -o /tmp/exp_collector -lcuda
// Prints cycles per MMA for each issue mode (one CTA per SM, one issuing thread) and checks that
// collector::b0::use really multiplies by the FILLED B (the descriptor passed with ::use points elsewhere).
#include <cstdio>
#include <cstdlib>
#include <vector>
#include <cmath>
#include "common.cuh"

using namespace adainf;

template <int MODE>
__device__ __forceinline__ void mma_mode(int j, uint32_t d, uint64_t a, uint64_t b, uint32_t idesc, uint32_t acc) {
  // j = position inside a group of 4 (fill / use / use / lastuse)
#define MMA_ASM(QUAL)                                                                          \
  asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\n" QUAL " [%0], %1, %2, %3, p;\n}\n" ::"r"(d), "l"(a), \
               "l"(b), "r"(idesc), "r"(acc))
  if (MODE == 0) {
    MMA_ASM("tcgen05.mma.cta_group::1.kind::f16");
  } else if (MODE == 1) {
    MMA_ASM("tcgen05.mma.ws.cta_group::1.kind::f16");
  } else if (MODE == 2) {
    if (j == 0) MMA_ASM("tcgen05.mma.ws.cta_group::1.kind::f16.collector::b0::fill");
    else if (j == 3) MMA_ASM("tcgen05.mma.ws.cta_group::1.kind::f16.collector::b0::lastuse");
    else MMA_ASM("tcgen05.mma.ws.cta_group::1.kind::f16.collector::b0::use");
  } else if (MODE == 3) {
    if (j == 0) MMA_ASM("tcgen05.mma.cta_group::1.kind::f16.collector::a::fill");
    else if (j == 3) MMA_ASM("tcgen05.mma.cta_group::1.kind::f16.collector::a::lastuse");
    else MMA_ASM("tcgen05.mma.cta_group::1.kind::f16.collector::a::use");
  }
#undef MMA_ASM
}

// smem: A region 4 tiles x 16 KB (128 rows x 64 bf16, SW128 K-major), B region 4 tiles x 32 KB (up to 256 rows)
constexpr int A_TILE = 16384, B_TILE = 32768;
constexpr int SMEM = 1024 + 4 * A_TILE + 4 * B_TILE + 256;

__device__ __forceinline__ uint32_t sw128(int r, int k) {  // byte offset of bf16 element (r, k) in a SW128 tile
  return r * 128 + ((((k * 2) >> 4) ^ (r & 7)) << 4) + ((k * 2) & 15);
}

template <int mode, int N>
__global__ void __launch_bounds__(128, 1) bench_kernel(int iters, unsigned long long* cycles,
                                                       const bf16* Ag, const bf16* Bg, float* Dout, int check) {
  extern __shared__ uint8_t raw[];
  uint8_t* smem = smem_align1024(raw);
  uint8_t* As = smem;
  uint8_t* Bs = smem + 4 * A_TILE;
  uint64_t* bar = (uint64_t*)(Bs + 4 * B_TILE);
  uint32_t* tslot = (uint32_t*)(bar + 1);
  // fill operands: A tiles t (128 x 64), B tiles t (256 x 64) from global (row-major [tile][row][k])
  for (int i = threadIdx.x; i < 4 * 128 * 64; i += blockDim.x) {
    const int t = i / (128 * 64), r = (i / 64) % 128, k = i % 64;
    *(bf16*)(As + t * A_TILE + sw128(r, k)) = Ag[i];
  }
  for (int i = threadIdx.x; i < 4 * 256 * 64; i += blockDim.x) {
    const int t = i / (256 * 64), r = (i / 64) % 256, k = i % 64;
    *(bf16*)(Bs + t * B_TILE + sw128(r, k)) = Bg[i];
  }
  if (threadIdx.x == 0) {
    mbar_init(bar, 1);
    fence_mbar_init();
  }
  if (threadIdx.x < 32) tmem_alloc<512>(tslot);
  fence_proxy_async_smem();
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tslot;
  const uint32_t idesc = make_idesc(128, N, 0, 0);
  if (threadIdx.x == 0) {
    const uint32_t as = smem_u32(As), bs = smem_u32(Bs);
    unsigned long long t0 = clock64();
    if (check) {
      // D0 = A0(kk=0) * B0(kk=0) with fill; D1 = A1(kk=0) * [desc -> B1] with ::use (collector must give B0)
      const uint32_t d0 = tmem, d1 = tmem + 256;
      mma_mode<mode>(0, d0, make_sdesc(as, 16, 1024), make_sdesc(bs, 16, 1024), idesc, 0);
      mma_mode<mode>(3, d1, make_sdesc(as + A_TILE, 16, 1024), make_sdesc(bs + B_TILE, 16, 1024), idesc, 0);
    } else {
      uint64_t ad[4], bd[4];
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        ad[j] = make_sdesc(as + ((mode == 3) ? 0u : (uint32_t)j * A_TILE), 16, 1024);
        bd[j] = make_sdesc(bs + ((mode == 2) ? 0u : (uint32_t)j * B_TILE), 16, 1024);
      }
      for (int it = 0; it < iters; it += 4) {
#pragma unroll
        for (int kk = 0; kk < 4; ++kk)
#pragma unroll
          for (int j = 0; j < 4; ++j)
            mma_mode<mode>(j, tmem + (uint32_t)((j & 1) * 256), ad[j] + 2u * kk, bd[j] + 2u * kk, idesc, 1u);
      }
    }
    umma_commit(bar);
    mbar_wait(bar, 0);
    unsigned long long t1 = clock64();
    cycles[blockIdx.x] = t1 - t0;
  }
  __syncthreads();
  tc_fence_after();
  if (check && blockIdx.x == 0) {
    const int w = threadIdx.x >> 5;
    for (int acc = 0; acc < 2; ++acc)
      for (int c = 0; c < N; c += 32) {
        float v[32];
        tmem_ld32(tmem + (uint32_t)(acc * 256 + c) + ((uint32_t)(w * 32) << 16), v);
        for (int i = 0; i < 32; ++i) Dout[(acc * 128 + threadIdx.x) * 256 + c + i] = v[i];
      }
  }
  tc_fence_before();
  __syncthreads();
  if (threadIdx.x < 32) tmem_dealloc<512>(tmem);
}

static float bf(uint16_t h) {
  uint32_t u = (uint32_t)h << 16;
  float f;
  memcpy(&f, &u, 4);
  return f;
}

int main() {
  const int nA = 4 * 128 * 64, nB = 4 * 256 * 64;
  std::vector<uint16_t> hA(nA), hB(nB);
  srand(1);
  for (auto& x : hA) x = (uint16_t)(0x3c00 + (rand() % 256) - 128);  // bf16 values around 0.0078..
  for (auto& x : hB) x = (uint16_t)(0x3f80 + (rand() % 128) - 64);
  bf16 *dA, *dB;
  float* dD;
  unsigned long long* dc;
  cudaMalloc(&dA, nA * 2);
  cudaMalloc(&dB, nB * 2);
  cudaMalloc(&dD, 256 * 256 * 4);
  cudaMalloc(&dc, 148 * 8);
  cudaMemcpy(dA, hA.data(), nA * 2, cudaMemcpyHostToDevice);
  cudaMemcpy(dB, hB.data(), nB * 2, cudaMemcpyHostToDevice);
#define ATTR(M, N) cudaFuncSetAttribute(bench_kernel<M, N>, cudaFuncAttributeMaxDynamicSharedMemorySize, SMEM);
  ATTR(0, 64) ATTR(1, 64) ATTR(2, 64) ATTR(3, 64) ATTR(0, 128) ATTR(1, 128) ATTR(2, 128) ATTR(3, 128)
  ATTR(0, 256) ATTR(1, 256) ATTR(2, 256) ATTR(3, 256)
  // semantics check
  for (int mode : {0, 2, 3}) {
    cudaMemset(dD, 0, 256 * 256 * 4);
    if (mode == 0) bench_kernel<0, 64><<<1, 128, SMEM>>>(0, dc, dA, dB, dD, 1);
    if (mode == 2) bench_kernel<2, 64><<<1, 128, SMEM>>>(0, dc, dA, dB, dD, 1);
    if (mode == 3) bench_kernel<3, 64><<<1, 128, SMEM>>>(0, dc, dA, dB, dD, 1);
    cudaError_t e = cudaDeviceSynchronize();
    if (e != cudaSuccess) {
      printf("mode %d check: %s\n", mode, cudaGetErrorString(e));
      return 1;
    }
    std::vector<float> D(256 * 256);
    cudaMemcpy(D.data(), dD, D.size() * 4, cudaMemcpyDeviceToHost);
    // references: D1 with B0 vs with B1 (A1 = A tile 1 k 0..15 ; mode 3 keeps A0)
    double e_b0 = 0, e_b1 = 0, e_d0 = 0;
    for (int r = 0; r < 128; ++r)
      for (int n = 0; n < 64; ++n) {
        double r0 = 0, rb0 = 0, rb1 = 0, ra0b1 = 0;
        for (int k = 0; k < 16; ++k) {
          const double a0 = bf(hA[r * 64 + k]), a1 = bf(hA[128 * 64 + r * 64 + k]);
          const double b0 = bf(hB[n * 64 + k]), b1 = bf(hB[256 * 64 + n * 64 + k]);
          r0 += a0 * b0;
          rb0 += a1 * b0;
          rb1 += a1 * b1;
          ra0b1 += a0 * b1;
        }
        const double g0 = D[r * 256 + n], g1 = D[(128 + r) * 256 + n];
        e_d0 = fmax(e_d0, fabs(g0 - r0));
        if (mode == 3) {  // A collector: D1 should be A0 * B1
          e_b0 = fmax(e_b0, fabs(g1 - ra0b1));
          e_b1 = fmax(e_b1, fabs(g1 - rb1));
        } else {
          e_b0 = fmax(e_b0, fabs(g1 - rb0));
          e_b1 = fmax(e_b1, fabs(g1 - rb1));
        }
      }
    printf("check mode %d: |D0-ref| %.3g ; D1 vs collector-operand ref %.3g ; D1 vs descriptor-operand ref %.3g\n",
           mode, e_d0, e_b0, e_b1);
  }
  const char* names[] = {"ss", "ws", "ws+b0 collector (B same x4)", "ss+a collector (A same x4)"};
  for (int N : {64, 128, 256})
    for (int mode = 0; mode < 4; ++mode) {
      if (mode == 1 || mode == 2) {
        if (N > 256) continue;
      }
      const int iters = 2048;
      auto launch = [&]() {
#define L(M, NN) if (mode == M && N == NN) bench_kernel<M, NN><<<148, 128, SMEM>>>(iters, dc, dA, dB, dD, 0);
        L(0, 64) L(1, 64) L(2, 64) L(3, 64) L(0, 128) L(1, 128) L(2, 128) L(3, 128)
        L(0, 256) L(1, 256) L(2, 256) L(3, 256)
      };
      launch();
      cudaError_t e = cudaDeviceSynchronize();
      if (e != cudaSuccess) {
        printf("N=%d mode %d: %s\n", N, mode, cudaGetErrorString(e));
        return 1;
      }
      launch();
      cudaDeviceSynchronize();
      std::vector<unsigned long long> c(148);
      cudaMemcpy(c.data(), dc, 148 * 8, cudaMemcpyDeviceToHost);
      double s = 0;
      for (auto x : c) s += (double)x;
      s /= 148.0;
      printf("N=%3d %-30s %7.2f cycles/MMA (M=128 K=16; ideal %d)\n", N, names[mode], s / (iters * 4.0),
             128 * N / 256);
    }
  return 0;
}

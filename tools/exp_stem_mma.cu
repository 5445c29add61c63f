// Experiment (not product code): tcgen05.mma issue rate for the stem's operand layouts.  One CTA per SM, operands
// resident in shared memory (contents irrelevant), one thread issues `iters` MMAs M=128 x N x K=16 back to back,
// then commits and waits; cycles per MMA are reported for:
//   A: K-major SWIZZLE_32B (32-byte rows, 8-row atoms), start row offset 0..3 (the stem's aw taps), or SWIZZLE_128B
//   B: K-major no-swizzle (the stem weights) with N = 64 / 128 / 256
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -std=c++17 -O2 -I<csrc> tools/exp_stem_mma.cu
#include <cstdio>
#include <cstdlib>

#include "common.cuh"

using namespace adainf;

__global__ void __launch_bounds__(128, 1) rate(int iters, int a_mode, int row_off, int N, long long* out) {
  extern __shared__ __align__(1024) uint8_t sm[];
  uint8_t* A = (uint8_t*)(((uintptr_t)sm + 1023) & ~(uintptr_t)1023);  // 64 KB
  uint8_t* Bm = A + 65536;                                                // 64 KB
  __shared__ uint64_t bar;
  __shared__ uint32_t slot;
  for (int i = threadIdx.x; i < 32768; i += blockDim.x) ((uint32_t*)A)[i] = 0x3c003c00u;
  if (threadIdx.x == 0) {
    mbar_init(&bar, 1);
    fence_mbar_init();
  }
  if (threadIdx.x < 32) tmem_alloc<256>(&slot);
  fence_proxy_async_smem();
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = slot;
  if (threadIdx.x == 0) {
    uint64_t ad;
    if (a_mode == 0) ad = make_sdesc_sw32(smem_u32(A), 16, 256) + (uint64_t)(row_off * 2);
    else ad = make_sdesc(smem_u32(A), 16, 1024);
    const uint64_t bd = make_sdesc_plain(smem_u32(Bm), 4096, 128);
    const uint32_t idesc = make_idesc(128, N, 0, 0);
    // warm up
    for (int i = 0; i < 16; ++i) umma_bf16(tmem, ad, bd, idesc, 1u);
    umma_commit(&bar);
    mbar_wait(&bar, 0);
    const long long t0 = clock64();
    for (int i = 0; i < iters; ++i) umma_bf16(tmem, ad + (uint64_t)((i & 3) * (a_mode == 0 ? 256 : 2)), bd, idesc, 1u);
    umma_commit(&bar);
    mbar_wait(&bar, 1);
    const long long t1 = clock64();
    out[blockIdx.x] = t1 - t0;
  }
  tc_fence_before();
  __syncthreads();
  if (threadIdx.x < 32) {
    tc_fence_after();
    tmem_dealloc<256>(tmem);
  }
}

int main() {
  long long* d;
  cudaMalloc(&d, 148 * 8);
  cudaFuncSetAttribute(rate, cudaFuncAttributeMaxDynamicSharedMemorySize, 140000);
  const int iters = 4096;
  struct Cfg { int a_mode, off, N; const char* name; } cfgs[] = {
      {0, 0, 64, "SW32 off0 N64"},  {0, 1, 64, "SW32 off1 N64"},  {0, 2, 64, "SW32 off2 N64"},
      {0, 3, 64, "SW32 off3 N64"},  {0, 0, 128, "SW32 off0 N128"}, {0, 1, 128, "SW32 off1 N128"},
      {0, 0, 256, "SW32 off0 N256"}, {0, 1, 256, "SW32 off1 N256"}, {1, 0, 64, "SW128 N64"},
      {1, 0, 128, "SW128 N128"},    {1, 0, 256, "SW128 N256"}};
  for (auto& c : cfgs) {
    rate<<<148, 128, 140000>>>(iters, c.a_mode, c.off, c.N, d);
    cudaError_t e = cudaDeviceSynchronize();
    if (e != cudaSuccess) {
      printf("%s: error %s\n", c.name, cudaGetErrorString(e));
      return 1;
    }
    long long h[148];
    cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
    double s = 0;
    for (int i = 0; i < 148; ++i) s += h[i];
    printf("%-16s %.1f cycles/MMA  (%.0f MAC/cycle)\n", c.name, s / 148 / iters, 128.0 * c.N * 16 / (s / 148 / iters));
  }
  return 0;
}

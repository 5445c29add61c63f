// Column sums of a dZ tile staged in shared memory by TMA (shared by the weight-gradient kernels).
#pragma once
#include <cuda_bf16.h>
#include <stdint.h>

namespace adainf {

// Bias gradient fused into the weight-gradient pipeline: warps 1-3 (idle otherwise) sum the columns of
// every dZ tile while it sits in shared memory, so dZ is not read a second time from HBM.  Tile layout is
// the MN-major 128B-swizzled one TMA writes: row = pixel, 64 channels per 128-byte row, 16-byte chunk j of
// row r stored at chunk j ^ (r & 7); atoms of 64 channels are 8192 B apart (64-row atoms) when the tile is
// wider than 64.  Each thread owns one 8-channel chunk column and a strided subset of rows; the per-thread
// sums are combined in a fixed order at the end of the unit (deterministic).
constexpr int CS_WORKERS = 96;
template <int BN>
struct TileColsum {
  static constexpr int NCH = BN / 8, NPH = CS_WORKERS / NCH;
  float acc[8];
  int cc, ph;
  __device__ __forceinline__ void init(int t) {
    cc = t % NCH;
    ph = t / NCH;
  }
  __device__ __forceinline__ void zero() {
#pragma unroll
    for (int q = 0; q < 8; ++q) acc[q] = 0.f;
  }
  // rows: valid rows per 64-channel atom (64 for the generic path, R*Wp for the window path)
  __device__ __forceinline__ void add(const uint8_t* tile, int rows) {
    if (ph >= NPH) return;
    const uint8_t* at = tile + (cc >> 3) * 8192;
    const int j = cc & 7;
    // four rows per batch: independent shared loads in flight before the adds
    for (int r0 = ph; r0 < rows; r0 += 4 * NPH) {
      uint4 raw[4];
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        const int r = r0 + i * NPH;
        raw[i] = r < rows ? *(const uint4*)(at + r * 128 + ((j ^ (r & 7)) << 4)) : make_uint4(0, 0, 0, 0);
      }
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        const __nv_bfloat162* h = (const __nv_bfloat162*)&raw[i];
#pragma unroll
        for (int q = 0; q < 4; ++q) {
          const float2 f = __bfloat1622float2(h[q]);
          acc[2 * q] += f.x;
          acc[2 * q + 1] += f.y;
        }
      }
    }
  }
  // combine the NPH row phases (fixed order) and write `lim` (<= BN) channel sums to out
  __device__ __forceinline__ void finish(float* red, float* out, int lim, int t) {
    if (ph < NPH)
#pragma unroll
      for (int q = 0; q < 8; ++q) red[ph * BN + cc * 8 + q] = acc[q];
    asm volatile("bar.sync 1, %0;" ::"n"(CS_WORKERS) : "memory");
    for (int ch = t; ch < BN; ch += CS_WORKERS) {
      float s = 0.f;
      for (int p = 0; p < NPH; ++p) s += red[p * BN + ch];
      if (ch < lim) out[ch] = s;
    }
    asm volatile("bar.sync 1, %0;" ::"n"(CS_WORKERS) : "memory");
  }
};

}  // namespace adainf

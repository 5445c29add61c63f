// TMA (cp.async.bulk.tensor) helpers: host-side tensor-map encoding through the driver entry point (no
// -lcuda link) and device-side bulk tensor loads completing on an mbarrier (transaction bytes).
#pragma once
#include <cuda.h>
#include <cuda_runtime.h>

#include "common.cuh"
#include "runtime.h"

namespace adainf {

// 4-D tiled map over a dense NHWC bf16 tensor [N][H][W][C]: dims (innermost first) {C, W, H, N},
// box {bc, bw, bh, 1}, 128B swizzle (bc * 2 bytes must be <= 128), out-of-bounds -> zeros.
CUtensorMap make_tmap_nhwc(const void* base, int N, int H, int W, int C, int bc, int bw, int bh, int stride = 1);
// same, no swizzle: the box lands row-major (bc * 2 bytes per (w, h) position, a multiple of 16)
CUtensorMap make_tmap_nhwc_plain(const void* base, int N, int H, int W, int C, int bc, int bw, int bh);
// same with a chosen swizzle: swz in {0, 32, 64, 128} bytes (bc * 2 must not exceed it)
CUtensorMap make_tmap_nhwc_swz(const void* base, int N, int H, int W, int C, int bc, int bw, int bh, int swz);
// 4-D tiled map over a dense NHWC uint8 tensor, no swizzle (bc bytes per (w, h) position, a multiple of 16)
CUtensorMap make_tmap_nhwc_u8(const void* base, int N, int H, int W, int C, int bc, int bw, int bh);
// 2-D tiled map over a row-major [rows][cols] bf16 matrix (row pitch ld elements), box {bcols, brows}.
CUtensorMap make_tmap_2d(const void* base, long long rows, int cols, int ld, int bcols, int brows);
// im2col map over NHWC [N][H][W][C] bf16 (128B swizzle): one load = `pixels` consecutive GEMM rows (output
// positions, W fastest then H then N, base positions [lo, dim-1+up] stepped by `stride`) x `ch` channels of the
// filter tap given by the load's offsets; elements outside the tensor read 0.
CUtensorMap make_tmap_im2col(const void* base, int N, int H, int W, int C, int lo, int up, int stride, int ch,
                             int pixels);

__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void tma_load_4d(uint32_t dst, const CUtensorMap* map, uint64_t* bar, int c0, int c1, int c2,
                                            int c3) {
  asm volatile(
      "cp.async.bulk.tensor.4d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5}], "
      "[%6];" ::"r"(dst),
      "l"(map), "r"(c0), "r"(c1), "r"(c2), "r"(c3), "r"(smem_u32(bar))
      : "memory");
}
// im2col load: coordinates {c, w, h, n} of the first row's base pixel, filter-tap offsets (ow, oh) >= 0
__device__ __forceinline__ void tma_load_im2col_4d(uint32_t dst, const CUtensorMap* map, uint64_t* bar, int c, int w,
                                                   int h, int n, uint16_t ow, uint16_t oh) {
  asm volatile(
      "cp.async.bulk.tensor.4d.shared::cluster.global.im2col.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5}], "
      "[%6], {%7, %8};" ::"r"(dst),
      "l"(map), "r"(c), "r"(w), "r"(h), "r"(n), "r"(smem_u32(bar)), "h"(ow), "h"(oh)
      : "memory");
}
__device__ __forceinline__ void tma_load_2d(uint32_t dst, const CUtensorMap* map, uint64_t* bar, int c0, int c1) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];" ::"r"(
          dst),
      "l"(map), "r"(c0), "r"(c1), "r"(smem_u32(bar))
      : "memory");
}
// bulk tensor store shared -> global (elements outside the tensor are not written), tracked by bulk groups
// CTA-pair forms: the transaction bytes complete on an mbarrier that may live in the PEER CTA of the pair
// (`bar` is a shared::cluster address, e.g. mapa of the leader's barrier), so both CTAs' operand loads of a
// stage land on ONE leader barrier without a forwarding hop
__device__ __forceinline__ void mbar_expect_tx_cluster(uint32_t bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cluster.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
}
__device__ __forceinline__ void tma_load_2d_cg2(uint32_t dst, const CUtensorMap* map, uint32_t bar, int c0, int c1) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes.cta_group::2 [%0], [%1, {%2, "
      "%3}], [%4];" ::"r"(dst),
      "l"(map), "r"(c0), "r"(c1), "r"(bar)
      : "memory");
}
__device__ __forceinline__ void tma_load_im2col_4d_cg2(uint32_t dst, const CUtensorMap* map, uint32_t bar, int c, int w,
                                                       int h, int n, uint16_t ow, uint16_t oh) {
  asm volatile(
      "cp.async.bulk.tensor.4d.shared::cluster.global.im2col.mbarrier::complete_tx::bytes.cta_group::2 [%0], [%1, {%2, "
      "%3, %4, %5}], [%6], {%7, %8};" ::"r"(dst),
      "l"(map), "r"(c), "r"(w), "r"(h), "r"(n), "r"(bar), "h"(ow), "h"(oh)
      : "memory");
}
__device__ __forceinline__ void tma_store_4d(const CUtensorMap* map, uint32_t src, int c0, int c1, int c2, int c3) {
  asm volatile("cp.async.bulk.tensor.4d.global.shared::cta.tile.bulk_group [%0, {%2, %3, %4, %5}], [%1];" ::"l"(map),
               "r"(src), "r"(c0), "r"(c1), "r"(c2), "r"(c3)
               : "memory");
}
__device__ __forceinline__ void tma_store_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
// this thread's committed bulk stores have finished reading shared memory (the buffer may be overwritten)
__device__ __forceinline__ void tma_store_wait_read() { asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory"); }
// ... and their global writes are complete
__device__ __forceinline__ void tma_store_wait_all() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }
__device__ __forceinline__ void tma_prefetch_desc(const CUtensorMap* map) {
  asm volatile("prefetch.tensormap [%0];" ::"l"(map) : "memory");
}

}  // namespace adainf

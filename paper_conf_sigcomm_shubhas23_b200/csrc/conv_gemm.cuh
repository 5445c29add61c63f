// Implicit-GEMM convolution on the 5th-gen tensor cores (tcgen05.mma kind::f16, fp32 accumulator in
// TMEM), one persistent warp-specialized kernel template for the three contractions of the hot path
// (SURVEY §8(a) a2, a9):
//
//   FWD   D[pix][co]   = sum_{tap,ci} X[gather(pix,tap)][ci] * W[co][tap][ci]        A K-major, B K-major
//   DGRAD D[pix'][ci]  = sum_{tap',co} dZ[gather(pix',tap')][co] * W[co][tap(tap')][ci]  A K-major, B MN-major
//   WGRAD D[kconv][co] = sum_{pix} X[gather(pix,tap(kconv))][ci(kconv)] * dZ[pix][co]   A MN-major, B MN-major
//
// "Run one layer for all requests of the batch at once" is inherent: M spans every pixel of
// every sample of the (compacted) batch.
//
// Structure (one CTA per SM, persistent over output tiles, tile order n-fastest for L2 reuse of A):
//   warps 0-3  producers: gather A/B 16-byte chunks with cp.async (zero-fill for padding, out-of-range
//              taps and rows beyond the device-side sample count) into a STAGES-deep ring of
//              128B-swizzled UMMA tiles; completion tracked by cp.async.mbarrier.arrive.noinc
//   warp 4     TMEM owner + MMA issuer (one elected lane): 4 x tcgen05.mma (K=16) per 64-wide K-block,
//              tcgen05.commit frees the smem stage; two TMEM accumulators (double buffer) so the
//              epilogue of tile i overlaps the MMAs of tile i+1
//   warps 5-8  epilogue: tcgen05.ld (32 lanes x 32 cols) -> bias / residual / activation / gradient
//              terms and masks -> 128-bit global stores; frees the accumulator after the last load
#pragma once
#include "common.cuh"
#include "tma.cuh"

namespace adainf {

enum { MODE_FWD = 0, MODE_DGRAD = 1, MODE_WGRAD = 2, MODE_DGRAD_SP = 3 };
// MODE_DGRAD_SP: stride-2 dgrad as ONE sub-pixel GEMM over the dZ grid (instead of 4 output-phase launches):
//   D[(n,y',x')][(py,px,ci)] = sum_{(a,b) in {0,1}^2, co} dZ[n][y'+a][x'+b][co] * Bsp[(py,px,ci)][(a,b,co)]
//   with Bsp = W[co][kh = py+p-2a][kw = px+p-2b][ci] (zero where the tap does not exist); the epilogue writes
//   column block (py,px) to dX[n][2y'+py][2x'+px].  N = 4*Cin instead of Cin: 4x fewer A-operand loads per MMA.
template <int MODE>
struct ModeTraits {
  static constexpr bool B_KMAJ = MODE == MODE_FWD || MODE == MODE_DGRAD_SP;  // B K-major ([N][K] rows)
  static constexpr bool DG_EPI = MODE == MODE_DGRAD || MODE == MODE_DGRAD_SP;
};
constexpr int MAX_TAPS = 49;

struct ConvArgs {
  // ---- gather source (A for FWD/DGRAD, im2col A for WGRAD) ----
  const bf16* src;      // NHWC [*][Hs][Ws][Cs]
  const int* src_map;   // optional: dense sample n -> source sample
  int Hs, Ws, Cs;
  // ---- pixel space (rows for FWD/DGRAD, reduction for WGRAD) ----
  const int* count;     // device sample count (nullptr -> n_static)
  int n_static;
  int Hg, Wg, sy, sx;
  int ntaps;
  int8_t ty[MAX_TAPS], tx[MAX_TAPS];
  // ---- B operand ----
  const bf16* B;        // FWD: W [Nout][ldb]; DGRAD: W [Cout][ldb] (fwd layout); WGRAD: dZ [pix][Nout]
  int ldb;
  int16_t btap[MAX_TAPS];  // DGRAD: forward tap index of phase tap t'
  int K;                // FWD: ntaps*Cs, DGRAD: ntaps*Cs (Cs = Cout), WGRAD: M extent = ntaps*Cs (kconv)
  int Nout;
  // ---- epilogue ----
  void* out;            // FWD/DGRAD: NHWC [*][Ho][Wo][Nout]; WGRAD: fp32 partial [split][Kconv][Nout]
  int out_f32;
  int Ho, Wo, oys, oxs, oyo, oxo;
  const float* bias;    // FWD
  const bf16* res;      // FWD residual (same geometry as out)
  const int* res_map;
  int act;              // FWD activation
  const float* bcast;   // DGRAD: + bcast[n][ch] (exit-head GAP gradient, pre-scaled by 1/HW)
  const bf16* sc;       // DGRAD: + shortcut gradient (same geometry as out)
  const bf16* yact;     // DGRAD: stored activation for the act' mask
  int mask_act;         // DGRAD: activation whose derivative masks (0 = none)
  int kb_per_split;     // WGRAD split-K (in 64-pixel blocks)
  int splits;           // WGRAD number of splits
  int exp_flags;        // experiments only (ADAINF_EXP): bit0 skip epilogue stores, bit1 skip bias/res loads
  // ---- optional TMA for the B (weight) operand of FWD / DGRAD: one elected producer thread issues the
  // bulk tensor loads (FWD: one {64 K, BN rows} box of the K-major shadow; DGRAD: BN/64 {64 ci, 64 co} boxes
  // that land as the MN-major SW128 atoms) instead of 128 threads issuing BN*8 cp.async each K-block ----
  int b_tma;
  int sp_cin;           // DGRAD_SP: Cin of the output (column block width); sp_sc_compact: sc is indexed by
  int sp_sc_compact;    // the dZ-grid row m and applies to phase (0,0) only (compact projection dgrad)
  CUtensorMap b_map;
  // ---- optional TMA im2col for the A operand of FWD / DGRAD / DGRAD_SP (dense source, Cs % 64 == 0, square
  // geometry): one elected producer thread issues one im2col load per K-block (128 GEMM rows x 64 channels
  // of one tap) instead of 128 threads decoding rows and issuing 8 cp.async each; requires b_tma ----
  int a_tma;
  int a_lo;             // base pixel = (g * stride + a_lo); tap offset = t{y,x}[tap] - a_lo >= 0
  CUtensorMap a_map;
};

constexpr int BM = 128, BK = 64;
constexpr int NUM_THREADS = 288;  // 4 producer warps, 1 MMA warp, 4 epilogue warps (window / wgrad kernels)
// conv_umma_kernel<.., EW>: 4 producer warps, 1 MMA warp, 4*EW epilogue warps.  EW = 2 (two warps per TMEM lane
// quadrant, alternating 64-column blocks) for epilogue-heavy short-K launches, which one epilogue warp per
// quadrant would bound; EW = 1 keeps more smem stages and registers for long-K launches
__host__ __device__ constexpr int gemm_threads(int EW) { return 160 + 128 * EW; }

template <int MODE, int BN, int EW = 1>
struct ConvCfg {
  static constexpr int A_BYTES = BM * BK * 2;
  static constexpr int B_BYTES = BN * BK * 2;
  static constexpr int STAGE_BYTES = A_BYTES + B_BYTES;
  // coalescing buffers of the bf16 epilogue: 4 warps x 2 operands x (32 rows x 128 B), double-buffered in
  // the sub-pixel dgrad mode
  static constexpr int EPI_BYTES =
      (MODE != 2 && BN >= 64) ? ((MODE == 3 || MODE == 1) && EW == 1 ? 4 * 16384 : 4 * EW * 8192) : 0;
  static constexpr int STAGES_FIT = (220 * 1024 - EPI_BYTES - 1280) / STAGE_BYTES;
  static constexpr int STAGES = STAGES_FIT > 8 ? 8 : STAGES_FIT;
  static constexpr int BIAS_BYTES = (MODE == 0 && EPI_BYTES > 0) ? 4096 : 0;  // FWD bias vector (Nout <= 1024)
  static constexpr int SMEM = STAGES * STAGE_BYTES + 1024 /*align*/ + 256 /*barriers*/ + EPI_BYTES + BIAS_BYTES;
  static constexpr int ACC_COLS = BN < 32 ? 32 : BN;
  static constexpr int TMEM_COLS = 2 * ACC_COLS;  // double-buffered accumulator
};

// 128B-swizzle offsets inside a tile (bytes).
// K-major tile [rows][64 elems]: row r, 16B chunk j.
__device__ __forceinline__ uint32_t kmaj_off(int r, int j) {
  return (uint32_t)((r >> 3) * 1024 + (r & 7) * 128 + ((j ^ (r & 7)) << 4));
}
// MN-major tile [K=64 rows][MN elems]: K row r, MN 16B chunk j (8 elems), atoms of 64 MN elems.
__device__ __forceinline__ uint32_t mnmaj_off(int r, int j) {
  return (uint32_t)((j >> 3) * 8192 + (r >> 3) * 1024 + (r & 7) * 128 + (((j & 7) ^ (r & 7)) << 4));
}

struct TileInfo {
  long long m0;
  int n0, kb0, kb1, z;
};

template <int MODE, int BN>
__device__ __forceinline__ int num_tiles(const ConvArgs& a, long long npix, int& mt, int& nt) {
  nt = (a.Nout + BN - 1) / BN;
  if (MODE == MODE_WGRAD) {
    mt = (a.K + BM - 1) / BM;
    return mt * nt * a.splits;
  }
  mt = (int)((npix + BM - 1) / BM);
  return mt * nt;
}

template <int MODE, int BN>
__device__ __forceinline__ TileInfo tile_info(const ConvArgs& a, int t, int mt, int nt, int nkb_total) {
  TileInfo ti;
  const int n = t % nt;
  const int r = t / nt;
  ti.n0 = n * BN;
  if (MODE == MODE_WGRAD) {
    const int m = r % mt;
    ti.z = r / mt;
    ti.m0 = (long long)m * BM;
    ti.kb0 = ti.z * a.kb_per_split;
    ti.kb1 = min(ti.kb0 + a.kb_per_split, nkb_total);
  } else {
    ti.z = 0;
    ti.m0 = (long long)r * BM;
    ti.kb0 = 0;
    ti.kb1 = nkb_total;
  }
  if (ti.kb1 < ti.kb0) ti.kb1 = ti.kb0;
  return ti;
}

__device__ __forceinline__ void st_bf16x8(bf16* p, const float* v) {
  __align__(16) bf16 h[8];
#pragma unroll
  for (int q = 0; q < 8; ++q) h[q] = __float2bfloat16_rn(v[q]);
  *(uint4*)p = *(uint4*)h;
}
// two floats -> bf16x2 (RNE; lower address = a)
__device__ __forceinline__ uint32_t pack_bf16x2(float a, float b) {
  const __nv_bfloat162 h = __floats2bfloat162_rn(a, b);
  return *(const uint32_t*)&h;
}
__device__ __forceinline__ void ld_bf16x8(const bf16* p, float* v) {
  const uint4 raw = __ldg((const uint4*)p);
  const bf16* h = (const bf16*)&raw;
#pragma unroll
  for (int q = 0; q < 8; ++q) v[q] = __bfloat162float(h[q]);
}

// ---- coalesced bf16 epilogue (FWD / DGRAD / DGRAD_SP with Nout % 64 == 0) ----
// Per 64-column block: the warp's 32 accumulator rows (thread = row) are combined with their epilogue
// operands and written through a per-warp 32 x 128 B shared buffer (16-byte chunks XOR-swizzled by row), so
// every global access is a lane group of 8 covering one row's 128 contiguous bytes (4 rows per instruction)
// instead of 32 rows x 16 B per instruction.  Same arithmetic and order as the per-thread path.
__device__ __forceinline__ uint32_t stg_off(int r, int j) { return (uint32_t)(r * 128 + ((j ^ (r & 7)) << 4)); }

// cooperative cp.async of 32 rows x 64 bf16 (row r of the warp at base + prow(r) * pitch; rows with ok = 0
// zero-filled) into a staging buffer: no register staging, one commit group per call
__device__ __forceinline__ void stage_issue(uint8_t* stg, const bf16* base, long long prow, bool ok, int pitch,
                                            int lane) {
  const int j = lane & 7;
#pragma unroll
  for (int it = 0; it < 8; ++it) {
    const int r = it * 4 + (lane >> 3);
    const long long pr = __shfl_sync(0xffffffffu, prow, r);
    const int okr = __shfl_sync(0xffffffffu, (int)ok, r);
    cp_async16(smem_u32(stg + stg_off(r, j)), okr ? (const void*)(base + pr * pitch + j * 8) : (const void*)base, okr);
  }
}
// each lane applies op to its own row of a staged buffer
template <class Op>
__device__ __forceinline__ void stage_apply(const uint8_t* stg, int lane, float* v, Op op) {
#pragma unroll
  for (int jj = 0; jj < 8; ++jj) {
    const uint4 x = *(const uint4*)(stg + stg_off(lane, jj));
    const bf16* h = (const bf16*)&x;
#pragma unroll
    for (int qq = 0; qq < 8; ++qq) v[jj * 8 + qq] = op(v[jj * 8 + qq], __bfloat162float(h[qq]));
  }
}
__device__ __forceinline__ void prefetch_l2(const void* p) {
  asm volatile("prefetch.global.L2 [%0];" ::"l"(p));
}
// Column-block geometry of the coalesced epilogue: where a row's 64 channels of this block come from / go to
struct EpiBlk {
  bool ok;              // row valid for this block (inside the batch; SP: output pixel inside the image)
  long long orow, srow;  // output / shortcut-term row
  const bf16* scp;       // shortcut term source (SP compact: phase 0 only)
  int ocol, NO;          // channel offset within the output row, output row pitch (channels)
};

template <int MODE>
__device__ __forceinline__ EpiBlk epi_block(const ConvArgs& a, int cb, long long m, bool rv, int n, long long orow,
                                            int gy, int gx) {
  EpiBlk e;
  e.ok = rv;
  e.orow = e.srow = orow;
  e.scp = a.sc;
  e.ocol = cb;
  e.NO = a.Nout;
  if (MODE == MODE_DGRAD_SP) {
    const int ph = cb / a.sp_cin;
    e.ocol = cb - ph * a.sp_cin;
    e.NO = a.sp_cin;
    const int oy = 2 * gy + (ph >> 1), ox = 2 * gx + (ph & 1);
    e.ok = rv && oy < a.Ho && ox < a.Wo;
    e.orow = e.srow = ((long long)n * a.Ho + oy) * a.Wo + ox;
    if (a.sp_sc_compact) {
      e.srow = m;
      if (ph != 0) e.scp = nullptr;
    }
  }
  return e;
}

// Coalesced epilogue.  Operands (FWD: residual; DGRAD: shortcut term and activation) are staged with cp.async
// into per-warp buffers; in the sub-pixel mode (short K, epilogue-heavy tiles) they are double-buffered: the
// first block's operands are requested before waiting for the accumulator, block c+1's while block c is
// combined, so the epilogue does not pay a memory latency per column block.
template <int MODE, int BN, int EW, bool PIPE_DG = false>
__device__ __forceinline__ void epilogue_coalesced(const ConvArgs& a, const TileInfo& ti, uint32_t trow,
                                                   uint64_t* tfull_b, uint32_t tpar, uint64_t* tempty_b, int nkb,
                                                   long long m, bool rv, int n, long long orow, long long rrow,
                                                   int HWg, uint8_t* stg, int lane, const float* bias_s, int h,
                                                   uint32_t tempty_remote = 0) {
  // tempty_remote != 0: the accumulator-free arrival goes to the pair leader's barrier (CTA-pair kernel)
  auto release = [&]() {
    if (tempty_remote) mbar_arrive_cluster(tempty_remote);
    else mbar_arrive(tempty_b);
  };
  // EW warps per lane quadrant: this warp takes column blocks h*64, h*64 + 64*EW, ...; with two warps the
  // staging is single-buffered (the other warp of the quadrant overlaps its latency)
  constexpr bool PIPE = (MODE == MODE_DGRAD_SP || (MODE == MODE_DGRAD && PIPE_DG)) && EW == 1;
  constexpr int STEP = 64 * EW;
  const int first = h * 64;
  if (first >= BN) {  // no block for this warp: release the accumulator in order
    mbar_wait(tfull_b, tpar);
    tc_fence_after();
    tc_fence_before();
    release();
    return;
  }
  int gy = 0, gx = 0;
  if (MODE == MODE_DGRAD_SP && rv) {
    const int pix = (int)m - n * HWg;
    gy = pix / a.Wg;
    gx = pix - gy * a.Wg;
  }
  const int ma = MODE == MODE_FWD ? 0 : a.mask_act;
  // operand 0: FWD residual / DGRAD shortcut term; operand 1: DGRAD activation (mask)
  auto issue = [&](const EpiBlk& e, int par) {
    uint8_t* s0 = stg + (PIPE ? par * 8192 : 0);
    if (a.exp_flags & 4) {  // experiment: no operand loads
      asm volatile("cp.async.commit_group;" ::: "memory");
      return;
    }
    if (MODE == MODE_FWD) {
      if (a.res) stage_issue(s0, a.res + e.ocol, rrow, e.ok, e.NO, lane);
    } else {
      if (e.scp) stage_issue(s0, e.scp + e.ocol, e.srow, e.ok, e.NO, lane);
      if (ma) stage_issue(s0 + 4096, a.yact + e.ocol, e.orow, e.ok, e.NO, lane);
    }
    asm volatile("cp.async.commit_group;" ::: "memory");
  };
  // L2 prefetch of this row's operands for the later column blocks (non-pipelined modes)
  if (!PIPE && rv) {
    const bf16* p0 = MODE == MODE_FWD ? a.res : a.sc;
    const bf16* p1 = MODE == MODE_FWD ? nullptr : (ma ? a.yact : nullptr);
    const long long r0 = MODE == MODE_FWD ? rrow : orow;
#pragma unroll 1
    for (int c = first + STEP; c < BN; c += STEP) {
      if (ti.n0 + c >= a.Nout) break;
      if (p0) prefetch_l2(p0 + r0 * a.Nout + ti.n0 + c);
      if (p1) prefetch_l2(p1 + orow * a.Nout + ti.n0 + c);
    }
  }
  EpiBlk cur = epi_block<MODE>(a, ti.n0 + first, m, rv, n, orow, gy, gx);
  if (PIPE) issue(cur, 0);
  mbar_wait(tfull_b, tpar);
  tc_fence_after();
  int it = 0;
#pragma unroll 1
  for (int c0 = first; c0 < BN; c0 += STEP, ++it) {
    float v[64];
    if (nkb > 0) {
      tmem_ld32(trow + c0, v);
      tmem_ld32(trow + c0 + 32, v + 32);
    } else {
#pragma unroll
      for (int i = 0; i < 64; ++i) v[i] = 0.f;
    }
    if (c0 + STEP >= BN) {
      tc_fence_before();
      release();  // accumulator free for the tile after next
    }
    const int cb = ti.n0 + c0;
    if (cb >= a.Nout) continue;  // warp-uniform (Nout % 64 == 0); keep looping: the last block frees the accumulator
    const bool has_next = c0 + STEP < BN && cb + STEP < a.Nout;
    if (!PIPE) cur = epi_block<MODE>(a, cb, m, rv, n, orow, gy, gx);
    EpiBlk nxt = cur;
    if (PIPE) {
      if (has_next) {
        nxt = epi_block<MODE>(a, cb + STEP, m, rv, n, orow, gy, gx);
        issue(nxt, (it + 1) & 1);
        asm volatile("cp.async.wait_group 1;" ::: "memory");
      } else {
        asm volatile("cp.async.wait_group 0;" ::: "memory");
      }
    } else {
      issue(cur, 0);
      asm volatile("cp.async.wait_group 0;" ::: "memory");
    }
    __syncwarp();
    uint8_t* s0 = stg + (PIPE ? (it & 1) * 8192 : 0);
    const auto add = [](float x, float r) { return __fadd_rn(x, r); };
    if (MODE == MODE_FWD) {
      if (!(a.exp_flags & 2)) {
        if (bias_s) {  // staged once per CTA: 16 broadcast LDS.128 instead of 64 uniform global loads
#pragma unroll
          for (int i = 0; i < 64; i += 4) {
            const float4 bb = *(const float4*)(bias_s + cb + i);
            v[i] = __fadd_rn(v[i], bb.x);
            v[i + 1] = __fadd_rn(v[i + 1], bb.y);
            v[i + 2] = __fadd_rn(v[i + 2], bb.z);
            v[i + 3] = __fadd_rn(v[i + 3], bb.w);
          }
        } else {
#pragma unroll
          for (int i = 0; i < 64; ++i) v[i] = __fadd_rn(v[i], __ldg(a.bias + cb + i));  // flat params: 4B-aligned
        }
      }
      if (a.res) stage_apply(s0, lane, v, add);
      act_vec<64>(a.act, v);
    } else {
      if (a.bcast && cur.ok) {
#pragma unroll
        for (int i = 0; i < 64; i += 4) {
          const float4 bb = __ldg((const float4*)(a.bcast + (long long)n * cur.NO + cur.ocol + i));
          v[i] = __fadd_rn(v[i], bb.x);
          v[i + 1] = __fadd_rn(v[i + 1], bb.y);
          v[i + 2] = __fadd_rn(v[i + 2], bb.z);
          v[i + 3] = __fadd_rn(v[i + 3], bb.w);
        }
      }
      if (cur.scp) stage_apply(s0, lane, v, add);
      if (ma == 1) stage_apply(s0 + 4096, lane, v, [](float x, float y) { return __fmul_rn(x, y > 0.f ? 1.f : 0.f); });
      else if (ma) stage_apply(s0 + 4096, lane, v, [ma](float x, float y) { return __fmul_rn(x, act_grad(ma, y)); });
    }
    __syncwarp();
    // own row -> staging (bf16), then 8 coalesced 16-byte stores per lane
#pragma unroll
    for (int jj = 0; jj < 8; ++jj) {
      __align__(16) bf16 h[8];
#pragma unroll
      for (int qq = 0; qq < 8; ++qq) h[qq] = __float2bfloat16_rn(v[jj * 8 + qq]);
      *(uint4*)(s0 + stg_off(lane, jj)) = *(const uint4*)h;
    }
    __syncwarp();
    const int j = lane & 7;
    bf16* ob = (bf16*)a.out + cur.ocol;
#pragma unroll
    for (int q8 = 0; q8 < 8; ++q8) {
      const int r = q8 * 4 + (lane >> 3);
      const long long pr = __shfl_sync(0xffffffffu, cur.orow, r);
      const int okr = __shfl_sync(0xffffffffu, (int)cur.ok, r);
      const uint4 x = *(const uint4*)(s0 + stg_off(r, j));
      if (okr && !(a.exp_flags & 8)) *((uint4*)(ob + pr * cur.NO) + j) = x;
    }
    __syncwarp();
    cur = nxt;
  }
}

template <int MODE, int BN, int EW>
__global__ void __launch_bounds__(gemm_threads(EW), 1) conv_umma_kernel(const __grid_constant__ ConvArgs a) {
  using Cfg = ConvCfg<MODE, BN, EW>;
  static_assert(ModeTraits<MODE>::B_KMAJ || BN >= 64, "MN-major SW128 B tiles need >= 64 columns");
  constexpr int STAGES = Cfg::STAGES;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = smem_align1024(smem_raw);
  uint64_t* full = (uint64_t*)(smem + STAGES * Cfg::STAGE_BYTES);
  uint64_t* empty = full + STAGES;
  uint64_t* tfull = empty + STAGES;   // [2]
  uint64_t* tempty = tfull + 2;       // [2]
  uint32_t* tmem_slot = (uint32_t*)(tempty + 2);
  uint8_t* epi_smem = smem + STAGES * Cfg::STAGE_BYTES + 256;  // Cfg::EPI_BYTES (non-WGRAD, BN >= 64)
  float* bias_s = nullptr;  // FWD: the layer's bias vector, staged once per CTA
  if (Cfg::BIAS_BYTES > 0 && a.bias && a.Nout <= Cfg::BIAS_BYTES / 4) {
    bias_s = (float*)(epi_smem + Cfg::EPI_BYTES);
    for (int i = threadIdx.x; i < a.Nout; i += gemm_threads(EW)) bias_s[i] = __ldg(a.bias + i);
  }

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int nsamp = a.count ? *a.count : a.n_static;
  const int HWg = a.Hg * a.Wg;
  const long long npix = (long long)nsamp * HWg;
  int mt, nt;
  const int ntile = num_tiles<MODE, BN>(a, npix, mt, nt);
  const int nkb_total = (MODE == MODE_WGRAD) ? (int)((npix + BK - 1) / BK) : (a.K + BK - 1) / BK;
  if ((int)blockIdx.x >= ntile) return;  // uniform: nothing for this CTA

  if (threadIdx.x == 0) {
    const bool btma = MODE != MODE_WGRAD && a.b_tma;
    for (int s = 0; s < STAGES; ++s) {
      // 128 cp.async arrivals (+1 expect_tx arrival of the B TMA); A by TMA: the single expect_tx arrival
      mbar_init(&full[s], (btma && a.a_tma) ? 1 : (btma ? 129 : 128));
      mbar_init(&empty[s], 1);
    }
    for (int b = 0; b < 2; ++b) {
      mbar_init(&tfull[b], 1);
      mbar_init(&tempty[b], 128 * EW);
    }
    fence_mbar_init();
  }
  if (warp == 4) tmem_alloc<Cfg::TMEM_COLS>(tmem_slot);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  const uint32_t smem_base = smem_u32(smem);

  if (warp < 4) {
    // ================= producers =================
    const int t = threadIdx.x;  // 0..127
    int it = 0;                 // global k-block counter (ring position)
    for (int tile = blockIdx.x; tile < ntile; tile += gridDim.x) {
      const TileInfo ti = tile_info<MODE, BN>(a, tile, mt, nt, nkb_total);
      const int nkb = ti.kb1 - ti.kb0;
      if (MODE != MODE_WGRAD && a.a_tma) {
        // A and B by TMA: one thread issues both loads of every K-block
        if (t == 0) {
          const int n0 = (int)(ti.m0 / HWg);
          const int pix = (int)ti.m0 - n0 * HWg;
          const int gy = pix / a.Wg, gx = pix - gy * a.Wg;
          const int bw = gx * a.sx + a.a_lo, bh = gy * a.sy + a.a_lo;
          int k = ti.kb0 * BK;
          int tap = k / a.Cs, c = k - tap * a.Cs;
          for (int kbi = 0; kbi < nkb; ++kbi, ++it) {
            const int s = it % STAGES, u = it / STAGES;
            if (u > 0) mbar_wait(&empty[s], (u - 1) & 1);
            const uint32_t sa = smem_base + s * Cfg::STAGE_BYTES;
            const uint32_t sb = sa + Cfg::A_BYTES;
            mbar_expect_tx(&full[s], (uint32_t)(Cfg::A_BYTES + Cfg::B_BYTES));
            tma_load_im2col_4d(sa, &a.a_map, &full[s], c, bw, bh, n0, (uint16_t)(a.tx[tap] - a.a_lo),
                               (uint16_t)(a.ty[tap] - a.a_lo));
            const int kb64 = (ti.kb0 + kbi) * BK;
            if (ModeTraits<MODE>::B_KMAJ) {
              tma_load_2d(sb, &a.b_map, &full[s], kb64, ti.n0);
            } else {
#pragma unroll
              for (int b = 0; b < BN / 64; ++b)
                tma_load_2d(sb + b * 8192, &a.b_map, &full[s], a.btap[tap] * a.Nout + ti.n0 + b * 64, c);
            }
            c += BK;
            if (c >= a.Cs) c = 0, ++tap;
          }
        }
      } else if (MODE != MODE_WGRAD) {
        // A: 128 rows (pixels) x 8 chunks; thread -> chunk t&7, rows (t>>3)+16*i
        const int j = t & 7;
        long long rowbase[8];
        int iy0[8], ix0[8];
#pragma unroll
        for (int i = 0; i < 8; ++i) {
          const long long m = ti.m0 + (t >> 3) + 16 * i;
          if (m < npix) {
            const int mi = (int)m;  // pixel counts < 2^31 (host-checked)
            const int n = mi / HWg;
            const int pix = mi - n * HWg;
            const int gy = pix / a.Wg, gx = pix - gy * a.Wg;
            const int sn = a.src_map ? __ldg(a.src_map + n) : n;
            rowbase[i] = (long long)sn * a.Hs * a.Ws;
            iy0[i] = gy * a.sy;
            ix0[i] = gx * a.sx;
          } else {
            rowbase[i] = 0;
            iy0[i] = -100000;
            ix0[i] = 0;
          }
        }
        for (int kbi = 0; kbi < nkb; ++kbi, ++it) {
          const int s = it % STAGES, u = it / STAGES;
          if (u > 0) mbar_wait(&empty[s], (u - 1) & 1);
          const uint32_t sa = smem_base + s * Cfg::STAGE_BYTES;
          const uint32_t sb = sa + Cfg::A_BYTES;
          const int k = (ti.kb0 + kbi) * BK + j * 8;
          if (a.Cs == 4) {
            // 4-channel (8-byte) pixels: each 16-byte chunk = taps t0, t0+1 -> two 8-byte cp.async
            const int t0 = k >> 2;
            const bool k0 = t0 < a.ntaps, k1 = t0 + 1 < a.ntaps;
            const int dy0 = k0 ? a.ty[t0] : -100000, dx0 = k0 ? a.tx[t0] : 0;
            const int dy1 = k1 ? a.ty[t0 + 1] : -100000, dx1 = k1 ? a.tx[t0 + 1] : 0;
#pragma unroll
            for (int i = 0; i < 8; ++i) {
              const int r = (t >> 3) + 16 * i;
              const int iya = iy0[i] + dy0, ixa = ix0[i] + dx0, iyb = iy0[i] + dy1, ixb = ix0[i] + dx1;
              const bool va = (unsigned)iya < (unsigned)a.Hs && (unsigned)ixa < (unsigned)a.Ws;
              const bool vb = (unsigned)iyb < (unsigned)a.Hs && (unsigned)ixb < (unsigned)a.Ws;
              const uint32_t d = sa + kmaj_off(r, j);
              cp_async8(d, va ? a.src + ((rowbase[i] + (long long)iya * a.Ws + ixa) << 2) : a.src, va);
              cp_async8(d + 8, vb ? a.src + ((rowbase[i] + (long long)iyb * a.Ws + ixb) << 2) : a.src, vb);
            }
          } else {
            const int tap = k / a.Cs;
            const int c = k - tap * a.Cs;
            const bool kval = k < a.K;
            const int dy = kval ? a.ty[tap] : -100000, dx = kval ? a.tx[tap] : 0;
#pragma unroll
            for (int i = 0; i < 8; ++i) {
              const int r = (t >> 3) + 16 * i;
              const int iy = iy0[i] + dy, ix = ix0[i] + dx;
              const bool v = (unsigned)iy < (unsigned)a.Hs && (unsigned)ix < (unsigned)a.Ws;
              const bf16* g = v ? a.src + ((rowbase[i] + (long long)iy * a.Ws + ix) * a.Cs + c) : a.src;
              cp_async16(sa + kmaj_off(r, j), g, v);
            }
          }
          if (a.b_tma) {
            if (t == 0) {
              mbar_expect_tx(&full[s], (uint32_t)Cfg::B_BYTES);
              const int kb64 = (ti.kb0 + kbi) * BK;
              if (ModeTraits<MODE>::B_KMAJ) {
                tma_load_2d(sb, &a.b_map, &full[s], kb64, ti.n0);
              } else {
                const int tp = kb64 / a.Cs;  // host guarantees Cs % 64 == 0: the K-block lies in one tap
                const int co0 = kb64 - tp * a.Cs;
#pragma unroll
                for (int b = 0; b < BN / 64; ++b)
                  tma_load_2d(sb + b * 8192, &a.b_map, &full[s], a.btap[tp] * a.Nout + ti.n0 + b * 64, co0);
              }
            }
          } else if (ModeTraits<MODE>::B_KMAJ) {
            // W [Nout][ldb] K-major: BN rows x 8 chunks
#pragma unroll
            for (int idx = t; idx < BN * 8; idx += 128) {
              const int r = idx >> 3, jj = idx & 7;
              const int kk = (ti.kb0 + kbi) * BK + jj * 8;
              const bool v = (ti.n0 + r) < a.Nout && kk < a.K;
              const bf16* g = v ? a.B + ((long long)(ti.n0 + r) * a.ldb + kk) : a.B;
              cp_async16(sb + kmaj_off(r, jj), g, v);
            }
          } else {
            // DGRAD: B MN-major [K=64 (tap',co) rows][BN ci]: element (k=(t',co), n=ci) = W[co][btap[t']][ci]
            constexpr int CH = BN / 8;
            const int kb64 = (ti.kb0 + kbi) * BK;
            if ((a.Cs & 63) == 0) {  // the whole K-block lies in one tap: one division per K-block
              const int tp = kb64 / a.Cs;
              const int co0 = kb64 - tp * a.Cs;
              const bf16* wb = a.B + (long long)co0 * a.ldb + (long long)a.btap[tp] * a.Nout + ti.n0;
#pragma unroll
              for (int idx = t; idx < 64 * CH; idx += 128) {
                const int r = idx / CH, jj = idx % CH;
                const bool v = (ti.n0 + jj * 8) < a.Nout;
                const bf16* g = v ? wb + (long long)r * a.ldb + jj * 8 : a.B;
                cp_async16(sb + mnmaj_off(r, jj), g, v);
              }
            } else {
#pragma unroll
              for (int idx = t; idx < 64 * CH; idx += 128) {
                const int r = idx / CH, jj = idx % CH;
                const int kk = kb64 + r;
                const int tp = kk / a.Cs;
                const int co = kk - tp * a.Cs;
                const int ci = ti.n0 + jj * 8;
                const bool v = kk < a.K && ci < a.Nout;
                const bf16* g = v ? a.B + ((long long)co * a.ldb + (long long)a.btap[tp] * a.Nout + ci) : a.B;
                cp_async16(sb + mnmaj_off(r, jj), g, v);
              }
            }
          }
          cp_async_arrive_noinc(&full[s]);
        }
      } else {
        // WGRAD: A MN-major [K=64 pixels][128 kconv]; thread -> pixel row r = t>>1 (one pixel decomposition
        // per K-block), kconv chunks j = (t&1)*8 .. +8 (taps / channels fixed per tile)
        const int r = t >> 1;
        const int j0 = (t & 1) * 8;
        const bool c4 = a.Cs == 4;  // 4-channel input: each 8-kconv chunk = two taps (8-byte halves)
        int dyj[8], dxj[8], cj[8], dyk[8], dxk[8];
#pragma unroll
        for (int q = 0; q < 8; ++q) {
          const int kc = (int)ti.m0 + (j0 + q) * 8;
          const bool mval = kc < a.K;
          const int tap = mval ? kc / a.Cs : 0;
          cj[q] = kc - tap * a.Cs;
          dyj[q] = mval ? a.ty[tap] : -100000;
          dxj[q] = a.tx[tap];
          const bool m1 = c4 && tap + 1 < a.ntaps && mval;
          dyk[q] = m1 ? a.ty[tap + 1] : -100000;
          dxk[q] = m1 ? a.tx[tap + 1] : 0;
        }
        for (int kbi = 0; kbi < nkb; ++kbi, ++it) {
          const int s = it % STAGES, u = it / STAGES;
          if (u > 0) mbar_wait(&empty[s], (u - 1) & 1);
          const uint32_t sa = smem_base + s * Cfg::STAGE_BYTES;
          const uint32_t sb = sa + Cfg::A_BYTES;
          const long long p0 = (long long)(ti.kb0 + kbi) * BK;
          const long long p = p0 + r;
          long long base = 0;
          int gy0 = -100000, gx0 = 0;
          if (p < npix) {
            const int pi = (int)p;
            const int n = pi / HWg;
            const int pix = pi - n * HWg;
            gy0 = pix / a.Wg;
            gx0 = pix - gy0 * a.Wg;
            gy0 *= a.sy;
            gx0 *= a.sx;
            base = (long long)(a.src_map ? __ldg(a.src_map + n) : n) * a.Hs * a.Ws;
          }
          if (c4) {
#pragma unroll
            for (int q = 0; q < 8; ++q) {
              const int iya = gy0 + dyj[q], ixa = gx0 + dxj[q], iyb = gy0 + dyk[q], ixb = gx0 + dxk[q];
              const bool va = (unsigned)iya < (unsigned)a.Hs && (unsigned)ixa < (unsigned)a.Ws;
              const bool vb = (unsigned)iyb < (unsigned)a.Hs && (unsigned)ixb < (unsigned)a.Ws;
              const uint32_t d = sa + mnmaj_off(r, j0 + q);
              cp_async8(d, va ? a.src + ((base + (long long)iya * a.Ws + ixa) << 2) : a.src, va);
              cp_async8(d + 8, vb ? a.src + ((base + (long long)iyb * a.Ws + ixb) << 2) : a.src, vb);
            }
          } else {
#pragma unroll
            for (int q = 0; q < 8; ++q) {
              const int iy = gy0 + dyj[q], ix = gx0 + dxj[q];
              const bool v = (unsigned)iy < (unsigned)a.Hs && (unsigned)ix < (unsigned)a.Ws;
              const bf16* g = v ? a.src + ((base + (long long)iy * a.Ws + ix) * a.Cs + cj[q]) : a.src;
              cp_async16(sa + mnmaj_off(r, j0 + q), g, v);
            }
          }
          // B: dZ [pix][Nout] MN-major [64 pixels][BN co]
          constexpr int CH = BN / 8;
#pragma unroll
          for (int idx = t; idx < 64 * CH; idx += 128) {
            const int r = idx / CH, jj = idx - (idx / CH) * CH;
            const long long p = p0 + r;
            const bool v = p < npix && (ti.n0 + jj * 8) < a.Nout;
            const bf16* g = v ? a.B + (p * a.Nout + ti.n0 + jj * 8) : a.B;
            cp_async16(sb + mnmaj_off(r, jj), g, v);
          }
          cp_async_arrive_noinc(&full[s]);
        }
      }
    }
  } else if (warp == 4) {
    // ================= MMA issuer =================
    constexpr uint32_t IDESC = make_idesc(BM, BN, MODE == MODE_WGRAD ? 1 : 0, ModeTraits<MODE>::B_KMAJ ? 0 : 1);
    int it = 0, lt = 0;
    for (int tile = blockIdx.x; tile < ntile; tile += gridDim.x, ++lt) {
      const TileInfo ti = tile_info<MODE, BN>(a, tile, mt, nt, nkb_total);
      const int nkb = ti.kb1 - ti.kb0;
      const int b = lt & 1, ub = lt >> 1;
      if (ub > 0) mbar_wait(&tempty[b], (ub - 1) & 1);  // epilogue drained this accumulator
      tc_fence_after();
      const uint32_t dacc = tmem + (uint32_t)(b * Cfg::ACC_COLS);
      for (int kbi = 0; kbi < nkb; ++kbi, ++it) {
        const int s = it % STAGES, u = it / STAGES;
        mbar_wait(&full[s], u & 1);
        fence_proxy_async_smem();
        tc_fence_after();
        if (elect_one()) {
          const uint32_t sa = smem_base + s * Cfg::STAGE_BYTES;
          const uint32_t sb = sa + Cfg::A_BYTES;
          // descriptors are linear in the start address (16-byte units): base + per-k-step offset
          const uint64_t ad0 = MODE == MODE_WGRAD ? make_sdesc(sa, 8192, 1024) : make_sdesc(sa, 16, 1024);
          const uint64_t bd0 = ModeTraits<MODE>::B_KMAJ ? make_sdesc(sb, 16, 1024) : make_sdesc(sb, 8192, 1024);
          constexpr uint32_t A_KK = MODE == MODE_WGRAD ? 128u : 2u, B_KK = ModeTraits<MODE>::B_KMAJ ? 2u : 128u;
#pragma unroll
          for (int kk = 0; kk < BK / 16; ++kk) umma_bf16(dacc, ad0 + kk * A_KK, bd0 + kk * B_KK, IDESC, (kbi | kk) != 0);
          umma_commit(&empty[s]);
          if (kbi == nkb - 1) umma_commit(&tfull[b]);
        }
        __syncwarp();
      }
      if (nkb == 0 && lane == 0) mbar_arrive(&tfull[b]);
      __syncwarp();
    }
  } else {
    // ================= epilogue =================
    const int q = warp & 3;  // TMEM lane quadrant of this warp
    const int h = (warp - 5) >> 2;  // which of the quadrant's two epilogue warps
    const int row = q * 32 + lane;
    int lt = 0;
    for (int tile = blockIdx.x; tile < ntile; tile += gridDim.x, ++lt) {
      const TileInfo ti = tile_info<MODE, BN>(a, tile, mt, nt, nkb_total);
      const int nkb = ti.kb1 - ti.kb0;
      const int b = lt & 1, ub = lt >> 1;
      bool coalesced = false;
      if constexpr (Cfg::EPI_BYTES > 0)
        coalesced = MODE != MODE_WGRAD && !a.out_f32 && (a.Nout & 63) == 0 && !(a.exp_flags & 1);
      if (!coalesced) {  // the coalesced epilogue waits itself, after requesting its first operands
        mbar_wait(&tfull[b], ub & 1);
        tc_fence_after();
      }
      const uint32_t trow = tmem + (uint32_t)(b * Cfg::ACC_COLS) + ((uint32_t)(q * 32) << 16);
      const long long m = ti.m0 + row;
      if (MODE == MODE_WGRAD) {
        float* outp = (float*)a.out + ((long long)ti.z * a.K + m) * a.Nout + ti.n0;
        if (h * 32 >= BN) {  // no chunk for this warp
          tc_fence_before();
          mbar_arrive(&tempty[b]);
        }
#pragma unroll 1
        for (int c0 = h * 32; c0 < BN; c0 += 32 * EW) {
          float v[32];
          if (nkb > 0) tmem_ld32(trow + c0, v);
          else
#pragma unroll
            for (int i = 0; i < 32; ++i) v[i] = 0.f;
          if (c0 + 32 * EW >= BN) {
            tc_fence_before();
            mbar_arrive(&tempty[b]);
          }
          if (m >= a.K) continue;
          if (ti.n0 + c0 + 32 <= a.Nout && (a.Nout & 3) == 0) {
#pragma unroll
            for (int i = 0; i < 32; i += 4)
              *(float4*)(outp + c0 + i) = make_float4(v[i], v[i + 1], v[i + 2], v[i + 3]);
          } else {
            for (int i = 0; i < 32; ++i)
              if (ti.n0 + c0 + i < a.Nout) outp[c0 + i] = v[i];
          }
        }
      } else {
        const bool rv = m < npix;
        long long orow = 0, rrow = 0;
        int n = 0;
        if (rv) {
          n = (int)m / HWg;
          const int pix = (int)m - n * HWg;
          const int gy = pix / a.Wg, gx = pix - gy * a.Wg;
          orow = ((long long)n * a.Ho + gy * a.oys + a.oyo) * a.Wo + gx * a.oxs + a.oxo;
          if (MODE == MODE_FWD && a.res) {
            const int rn = a.res_map ? __ldg(a.res_map + n) : n;
            rrow = (long long)rn * a.Ho * a.Wo + (orow - (long long)n * a.Ho * a.Wo);
          }
        }
        if constexpr (Cfg::EPI_BYTES > 0) {
          if (coalesced) {
            epilogue_coalesced<MODE, BN, EW, true>(a, ti, trow, &tfull[b], ub & 1, &tempty[b], nkb, m, rv, n, orow, rrow,
                                          HWg, epi_smem + (warp - 5) * (Cfg::EPI_BYTES / (4 * EW)), lane, bias_s, h);
            continue;
          }
        }
        if (h * 32 >= BN) {  // no chunk for this warp
          tc_fence_before();
          mbar_arrive(&tempty[b]);
        }
#pragma unroll 1
        for (int c0 = h * 32; c0 < BN; c0 += 32 * EW) {
          float v[32];
          if (nkb > 0) tmem_ld32(trow + c0, v);
          else
#pragma unroll
            for (int i = 0; i < 32; ++i) v[i] = 0.f;
          if (c0 + 32 * EW >= BN) {
            tc_fence_before();
            mbar_arrive(&tempty[b]);  // accumulator free for the tile after next
          }
          const int cb = ti.n0 + c0;
          if (!rv || cb >= a.Nout || (a.exp_flags & 1)) continue;
          const bool vec = (cb + 32 <= a.Nout) && ((a.Nout & 7) == 0);
          if (MODE == MODE_FWD) {
            if (vec) {
#pragma unroll
              if (!(a.exp_flags & 2))
                for (int i = 0; i < 32; ++i) v[i] = __fadd_rn(v[i], __ldg(a.bias + cb + i));  // flat params: 4B-aligned
              if (a.res) {
#pragma unroll
                for (int i = 0; i < 32; i += 8) {
                  float r8[8];
                  ld_bf16x8(a.res + rrow * a.Nout + cb + i, r8);
#pragma unroll
                  for (int qq = 0; qq < 8; ++qq) v[i + qq] = __fadd_rn(v[i + qq], r8[qq]);
                }
              }
#pragma unroll
              for (int i = 0; i < 32; ++i) v[i] = act_apply(a.act, v[i]);
              if (a.out_f32) {
                float* o = (float*)a.out + orow * a.Nout + cb;
#pragma unroll
                for (int i = 0; i < 32; i += 4) *(float4*)(o + i) = make_float4(v[i], v[i + 1], v[i + 2], v[i + 3]);
              } else {
                bf16* o = (bf16*)a.out + orow * a.Nout + cb;
#pragma unroll
                for (int i = 0; i < 32; i += 8) st_bf16x8(o + i, v + i);
              }
            } else {
              for (int i = 0; i < 32; ++i) {
                const int ch = cb + i;
                if (ch >= a.Nout) break;
                float x = __fadd_rn(v[i], a.bias[ch]);
                if (a.res) x = __fadd_rn(x, __bfloat162float(a.res[rrow * a.Nout + ch]));
                x = act_apply(a.act, x);
                if (a.out_f32) ((float*)a.out)[orow * a.Nout + ch] = x;
                else ((bf16*)a.out)[orow * a.Nout + ch] = __float2bfloat16_rn(x);
              }
            }
          } else {  // DGRAD epilogue: + bcast + shortcut, x act'(y), -> bf16
            int ocol = cb;         // channel within the output row
            long long srow = orow;  // row of the shortcut term
            const bf16* scp = a.sc;
            if (MODE == MODE_DGRAD_SP) {
              const int ph = cb / a.sp_cin;
              ocol = cb - ph * a.sp_cin;
              const int pix = (int)m - n * HWg;
              const int gy = pix / a.Wg, gx = pix - gy * a.Wg;
              const int oy = 2 * gy + (ph >> 1), ox = 2 * gx + (ph & 1);
              if (oy >= a.Ho || ox >= a.Wo) continue;
              orow = ((long long)n * a.Ho + oy) * a.Wo + ox;
              srow = orow;
              if (a.sp_sc_compact) {
                srow = m;
                if (ph != 0) scp = nullptr;
              }
            }
            const int NO = MODE == MODE_DGRAD_SP ? a.sp_cin : a.Nout;  // output row pitch (channels)
            if (vec) {
              if (a.bcast) {
#pragma unroll
                for (int i = 0; i < 32; i += 4) {
                  const float4 bb = __ldg((const float4*)(a.bcast + (long long)n * NO + ocol + i));
                  v[i] = __fadd_rn(v[i], bb.x);
                  v[i + 1] = __fadd_rn(v[i + 1], bb.y);
                  v[i + 2] = __fadd_rn(v[i + 2], bb.z);
                  v[i + 3] = __fadd_rn(v[i + 3], bb.w);
                }
              }
              if (scp) {
#pragma unroll
                for (int i = 0; i < 32; i += 8) {
                  float r8[8];
                  ld_bf16x8(scp + srow * NO + ocol + i, r8);
#pragma unroll
                  for (int qq = 0; qq < 8; ++qq) v[i + qq] = __fadd_rn(v[i + qq], r8[qq]);
                }
              }
              if (a.mask_act) {
#pragma unroll
                for (int i = 0; i < 32; i += 8) {
                  float y8[8];
                  ld_bf16x8(a.yact + orow * NO + ocol + i, y8);
#pragma unroll
                  for (int qq = 0; qq < 8; ++qq) v[i + qq] = __fmul_rn(v[i + qq], act_grad(a.mask_act, y8[qq]));
                }
              }
              bf16* o = (bf16*)a.out + orow * NO + ocol;
#pragma unroll
              for (int i = 0; i < 32; i += 8) st_bf16x8(o + i, v + i);
            } else {
              bf16* o = (bf16*)a.out + orow * NO + ocol;
              for (int i = 0; i < 32; ++i) {
                if (cb + i >= a.Nout) break;
                const int ch = ocol + i;
                float x = v[i];
                if (a.bcast) x = __fadd_rn(x, a.bcast[(long long)n * NO + ch]);
                if (scp) x = __fadd_rn(x, __bfloat162float(scp[srow * NO + ch]));
                if (a.mask_act)
                  x = __fmul_rn(x, act_grad(a.mask_act, __bfloat162float(a.yact[orow * NO + ch])));
                o[i] = __float2bfloat16_rn(x);
              }
            }
          }
        }
      }
    }
  }

  tc_fence_before();
  __syncthreads();
  if (warp == 4) {
    tc_fence_after();
    tmem_dealloc<Cfg::TMEM_COLS>(tmem);
  }
}

}  // namespace adainf

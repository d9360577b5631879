// Rolling dy-fold conv with tensor-core accumulation of the vertical taps in a TMEM ring (shared by conv_roll.cu
// and conv_block.cu).
//
// For input row i the MMA group (3 dx x Cin/16 MMAs, N = 3 Cout, B = dy-fold weights Wo[kx][ci/8][ky*Cout+co][8])
// adds dy = 0 into the accumulator of output row i+1, dy = 1 into row i, dy = 2 into row i-1.  Output row g owns
// TMEM block ring_idx<RB>(g) (COUTP columns); blocks descend with g so the three targets of a step are contiguous,
// except when the ring wraps inside them (ring_idx(g) < 2), then the step is issued as two MMA groups.  Blocks
// are armed with the bias by the epilogue (tcgen05.st), so every MMA accumulates.
#pragma once
#include "ptx.cuh"

namespace sr {

// A operand = one input row: APX bytes per pixel row of a K-atom (16 for SWIZZLE_NONE 8-channel chunks, 32 for
// SWIZZLE_32B 16-channel blocks); kstride = bytes from one K step (16 channels) to the next.
template <int CINP, int COUTP, int RB, int APX = 16>
__device__ __forceinline__ void ring_mma_step(uint32_t ring_base, unsigned g, uint64_t ad, uint64_t bd,
                                              uint32_t kstride) {
  constexpr int CCH = CINP / 8, KS = CINP / 16, N = 3 * COUTP;
  const int i0 = ring_idx<RB>(g);
  int blkA, rowA, nA, blkB = 0, rowB = 0, nB = 0;
  if (i0 >= 2) { blkA = i0 - 2; rowA = 0; nA = N; }
  else if (i0 == 0) { blkA = RB - 2; rowA = 0; nA = 2 * COUTP; blkB = 0; rowB = 2 * COUTP; nB = COUTP; }
  else { blkA = RB - 1; rowA = 0; nA = COUTP; blkB = 0; rowB = COUTP; nB = 2 * COUTP; }
  const uint32_t idA = make_idesc(128, nA, 0, 0);
#pragma unroll
  for (int dx = 0; dx < 3; ++dx)
#pragma unroll
    for (int ks = 0; ks < KS; ++ks)
      mma_bf16_ss(ring_base + blkA * COUTP, desc_add(ad, dx * (uint32_t)APX + ks * kstride),
                  desc_add(bd, (uint32_t)(dx * CCH + 2 * ks) * N * 16u + rowA * 16u), idA, 1u);
  if (nB) {
    const uint32_t idB = make_idesc(128, nB, 0, 0);
#pragma unroll
    for (int dx = 0; dx < 3; ++dx)
#pragma unroll
      for (int ks = 0; ks < KS; ++ks)
        mma_bf16_ss(ring_base + blkB * COUTP, desc_add(ad, dx * (uint32_t)APX + ks * kstride),
                    desc_add(bd, (uint32_t)(dx * CCH + 2 * ks) * N * 16u + rowB * 16u), idB, 1u);
  }
}

// Load COLS accumulator columns of a ring block (this thread's lane) and re-arm them with the bias (COLS % 8 == 0).
template <int COLS>
__device__ __forceinline__ void ring_drain(uint32_t taddr, float* v, const float4* sbias) {
  static_assert(COLS % 8 == 0, "ring_drain: columns must be a multiple of 8");
  constexpr int C16 = COLS / 16 * 16;
#pragma unroll
  for (int c0 = 0; c0 < C16; c0 += 16) tmem_ld16(taddr + c0, v + c0);
  if (COLS % 16) tmem_ld8(taddr + C16, v + C16);
  tmem_ld_wait();
#pragma unroll
  for (int c0 = 0; c0 < COLS; c0 += 8) {
    float b[8];
    const float4 t0 = sbias[c0 / 4], t1 = sbias[c0 / 4 + 1];
    b[0] = t0.x; b[1] = t0.y; b[2] = t0.z; b[3] = t0.w; b[4] = t1.x; b[5] = t1.y; b[6] = t1.z; b[7] = t1.w;
    tmem_st8(taddr + c0, b);
  }
  tmem_st_wait();
}

// Load COLS accumulator columns of a ring block (this thread's lane) without re-arming (blocks armed by ring_arm).
template <int COLS>
__device__ __forceinline__ void ring_load(uint32_t taddr, float* v) {
  static_assert(COLS % 8 == 0, "ring_load: columns must be a multiple of 8");
  constexpr int C16 = COLS / 16 * 16;
#pragma unroll
  for (int c0 = 0; c0 < C16; c0 += 16) tmem_ld16(taddr + c0, v + c0);
  if (COLS % 16) tmem_ld8(taddr + C16, v + C16);
  tmem_ld_wait();
}

// ---- arming a ring block with the bias inside the tensor pipe (instead of tcgen05.st from the epilogue): one
// non-accumulating MMA, M = 128, N = COUTP, K = 16, A = "ones" tile (A[m][k] = 1 for k < 3), B[n][k] = the bias split
// into three bf16 terms (hi, mid, lo: hi + mid + lo = the fp32 bias to ~2^-24 relative), so D[m][n] = bias[n].
// Both tiles are K-major SWIZZLE_NONE: element (row, k) at (row%8)*16 + (row/8)*128 + (k/8)*LBO + (k%8)*2 with
// LBO = rows*16.  The MMA issuer arms the block of an output row right before that row's first contribution, so
// the epilogue only drains (tcgen05.ld) and frees the block.
static constexpr uint32_t kArmOnesBytes = 128 * 16 * 2;  // A tile: 128 rows x 16 K

__device__ __forceinline__ void arm_tiles_fill(uint8_t* ones, uint8_t* btile, const float* bias, int coutp,
                                               int tid, int nthreads) {
  for (int i = tid; i < 128 * 16; i += nthreads) {
    const int r = i / 16, k = i % 16;
    *reinterpret_cast<__nv_bfloat16*>(ones + (r % 8) * 16 + (r / 8) * 128 + (k / 8) * 2048 + (k % 8) * 2) =
        __float2bfloat16(k < 3 ? 1.f : 0.f);
  }
  for (int i = tid; i < coutp * 16; i += nthreads) {
    const int n = i / 16, k = i % 16;
    const float b = bias[n];
    const __nv_bfloat16 hi = __float2bfloat16(b);
    const __nv_bfloat16 mid = __float2bfloat16(b - __bfloat162float(hi));
    const __nv_bfloat16 lo = __float2bfloat16(b - __bfloat162float(hi) - __bfloat162float(mid));
    const __nv_bfloat16 v = k == 0 ? hi : k == 1 ? mid : k == 2 ? lo : __float2bfloat16(0.f);
    *reinterpret_cast<__nv_bfloat16*>(btile + (n % 8) * 16 + (n / 8) * 128 + (k / 8) * (coutp * 16) + (k % 8) * 2) = v;
  }
}

template <int COUTP, int RB>
__device__ __forceinline__ void ring_arm(uint32_t ring_base, unsigned g, uint32_t ones_saddr, uint32_t btile_saddr) {
  constexpr uint32_t id = make_idesc(128, COUTP, 0, 0);
  mma_bf16_ss(ring_base + ring_idx<RB>(g) * COUTP, make_desc(ones_saddr, 2048, 128),
              make_desc(btile_saddr, COUTP * 16, 128), id, 0u);
}

// The same with the ones operand held in TMEM (8 columns: A[m][k] = 1 for k < 3, bf16 pairs per 32-bit column),
// written once by ones_tmem_fill: the arming MMA then reads only the bias tile from shared memory (the 4 KB ones
// tile per arm otherwise goes through the shared-memory port the conv MMAs saturate).
template <int COUTP, int RB>
__device__ __forceinline__ void ring_arm_ts(uint32_t ring_base, unsigned g, uint32_t ones_tmem, uint32_t btile_saddr) {
  constexpr uint32_t id = make_idesc(128, COUTP, 0, 0);
  mma_bf16_ts(ring_base + ring_idx<RB>(g) * COUTP, ones_tmem, make_desc(btile_saddr, COUTP * 16, 128), id, 0u);
}
// one warp writes its 32 lanes of the TMEM ones operand (caller: tcgen05.wait::st + fence before the MMA issuer)
__device__ __forceinline__ void ones_tmem_fill(uint32_t taddr_lane) {
  const __nv_bfloat162 one_one = __floats2bfloat162_rn(1.f, 1.f), one_zero = __floats2bfloat162_rn(1.f, 0.f);
  float v[8];
  v[0] = __uint_as_float(*reinterpret_cast<const uint32_t*>(&one_one));
  v[1] = __uint_as_float(*reinterpret_cast<const uint32_t*>(&one_zero));
#pragma unroll
  for (int i = 2; i < 8; ++i) v[i] = 0.f;
  tmem_st8(taddr_lane, v);
}

}  // namespace sr

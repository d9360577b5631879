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
__device__ __forceinline__ void ring_mma_step(uint32_t ring_base, long long g, uint64_t ad, uint64_t bd,
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

}  // namespace sr

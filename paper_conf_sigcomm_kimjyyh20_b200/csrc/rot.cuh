// Bank-conflict-free 16-B accesses to pixel-major rows in shared memory (staging rows of the TMA stores, aux rows of
// the TMA loads: pixel m at m * 16 * NCH bytes, NCH 16-B channel chunks).  The 8 lanes of one shared-memory phase
// hold 8 consecutive pixels; with a pixel stride of 16 * NCH bytes, lanes t and t + p (p = 8 / gcd(NCH, 8)) start on
// the same bank, so every 16-B access of a plain chunk loop is gcd(NCH, 8)-way conflicted.  Lane t instead visits
// the chunks starting at rot = t / p: the colliding lanes are then 4 banks apart and the phase covers all 32 banks
// once.  The smem image (and the TMA boxes) are unchanged; only the order of each lane's accesses rotates.
#pragma once
#include <cstdint>

namespace sr {

template <int NCH>
struct ChunkRot {
  static constexpr int G = NCH % 8 == 0 ? 8 : NCH % 4 == 0 ? 4 : NCH % 2 == 0 ? 2 : 1;
  static constexpr int P = 8 / G;
  __device__ __forceinline__ static int rot() { return (int)((threadIdx.x & 7u) / P); }
  // u[(j + rot) % NCH] with compile-time indices only (rot < G)
  __device__ __forceinline__ static uint4 fwd(const uint4* u, int j, int rot) {
    uint4 w = u[j % NCH];
#pragma unroll
    for (int r = 1; r < G; ++r)
      if (rot == r) w = u[(j + r) % NCH];
    return w;
  }
  // t[(c - rot) mod NCH]
  __device__ __forceinline__ static uint4 inv(const uint4* t, int c, int rot) {
    uint4 w = t[c % NCH];
#pragma unroll
    for (int r = 1; r < G; ++r)
      if (rot == r) w = t[(c - r + NCH) % NCH];
    return w;
  }
};

// store the NCH chunks u[0..NCH) of one pixel at `pix` (shared memory)
template <int NCH>
__device__ __forceinline__ void st_pix_rot(uint8_t* pix, const uint4* u) {
  const int rot = ChunkRot<NCH>::rot();
#pragma unroll
  for (int j = 0; j < NCH; ++j) {
    const int c = j + rot < NCH ? j + rot : j + rot - NCH;
    *reinterpret_cast<uint4*>(pix + c * 16) = ChunkRot<NCH>::fwd(u, j, rot);
  }
}

// load the NCH chunks of one pixel at `pix` (shared memory) into u[0..NCH)
template <int NCH>
__device__ __forceinline__ void ld_pix_rot(const uint8_t* pix, uint4* u) {
  const int rot = ChunkRot<NCH>::rot();
  uint4 t[NCH];
#pragma unroll
  for (int j = 0; j < NCH; ++j) {
    const int c = j + rot < NCH ? j + rot : j + rot - NCH;
    t[j] = *reinterpret_cast<const uint4*>(pix + c * 16);
  }
#pragma unroll
  for (int c = 0; c < NCH; ++c) u[c] = ChunkRot<NCH>::inv(t, c, rot);
}

}  // namespace sr

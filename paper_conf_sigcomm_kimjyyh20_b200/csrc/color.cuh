// I420 <-> RGB colour conversion shared by the conversion kernels (kernels.cu) and the fused I420 head conv
// (conv_roll.cu): BT.601 studio swing, integer (reading R21).  C = Y - 16, D = U - 128, E = V - 128;
// R = (298 C + 409 E + 128) >> 8, G = (298 C - 100 D - 208 E + 128) >> 8, B = (298 C + 516 D + 128) >> 8, clamped;
// chroma (y/2, x/2) is shared by its 2x2 block.
#pragma once
#include <cstdint>

namespace sr {

__device__ __forceinline__ uint8_t clip8(int v) { return (uint8_t)min(max(v, 0), 255); }
__device__ __forceinline__ void yuv_to_rgb(int Y, int U, int V, uint8_t* o) {
  const int c = Y - 16, d = U - 128, e = V - 128;
  o[0] = clip8((298 * c + 409 * e + 128) >> 8);
  o[1] = clip8((298 * c - 100 * d - 208 * e + 128) >> 8);
  o[2] = clip8((298 * c + 516 * d + 128) >> 8);
}

// RGB -> I420: Y per pixel; U / V from a 2x2 block's rounded mean colour (sums of the four R, G, B)
__device__ __forceinline__ uint8_t rgb_to_y(int R, int G, int B) {
  return (uint8_t)(((66 * R + 129 * G + 25 * B + 128) >> 8) + 16);
}
__device__ __forceinline__ void rgb_sums_to_uv(int sr, int sg, int sb, uint8_t& u, uint8_t& v) {
  const int R = (sr + 2) >> 2, G = (sg + 2) >> 2, B = (sb + 2) >> 2;
  u = (uint8_t)(((-38 * R - 74 * G + 112 * B + 128) >> 8) + 128);
  v = (uint8_t)(((112 * R - 94 * G - 18 * B + 128) >> 8) + 128);
}

}  // namespace sr

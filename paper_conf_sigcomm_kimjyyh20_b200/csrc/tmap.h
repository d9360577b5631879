// Host helpers: TMA tensor-map encoding through the driver entry point (no -lcuda link needed).
#pragma once
#include <cuda.h>
#include <cuda_runtime.h>
#include <cudaTypedefs.h>
#include <cstdint>
#include <cstring>

namespace sr {

inline PFN_cuTensorMapEncodeTiled_v12000 get_encode_fn() {
  static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
  if (!fn) {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(p);
  }
  return fn;
}

// NHWC bf16 activation [N][H][W][Cp] viewed as a 5-D tensor whose innermost dimension is one 8-channel
// (16-byte) chunk.  `order` selects the smem layout the box lands in (the box is written innermost-first):
//   CHUNK_ROW_PIX : dims {8, W, H, Cp/8, N}  -> smem [chunk][row][pixel][8]   (fwd conv A operand)
//   ROW_CHUNK_PIX : dims {8, W, Cp/8, H, N}  -> smem [row][chunk][pixel][8]   (wgrad operands)
// Out-of-bounds box elements (image border, padding) are zero-filled by the TMA unit.
enum TmapOrder { CHUNK_ROW_PIX = 0, ROW_CHUNK_PIX = 1 };

inline CUresult make_act_tmap(CUtensorMap* tm, const void* base, int N, int H, int W, int Cp, int box_w,
                              int box_h, int box_chunks, TmapOrder order) {
  auto fn = get_encode_fn();
  if (!fn) return CUDA_ERROR_NOT_SUPPORTED;
  const uint64_t es = 2;
  cuuint64_t dims[5];
  cuuint64_t strides[4];  // bytes, dims 1..4
  cuuint32_t box[5];
  cuuint32_t estr[5] = {1, 1, 1, 1, 1};
  const uint64_t pix = (uint64_t)Cp * es, row = (uint64_t)W * pix, img = (uint64_t)H * row;
  if (order == CHUNK_ROW_PIX) {
    dims[0] = 8; dims[1] = W; dims[2] = H; dims[3] = Cp / 8; dims[4] = N;
    strides[0] = pix; strides[1] = row; strides[2] = 16; strides[3] = img;
    box[0] = 8; box[1] = box_w; box[2] = box_h; box[3] = box_chunks; box[4] = 1;
  } else {
    dims[0] = 8; dims[1] = W; dims[2] = Cp / 8; dims[3] = H; dims[4] = N;
    strides[0] = pix; strides[1] = 16; strides[2] = row; strides[3] = img;
    box[0] = 8; box[1] = box_w; box[2] = box_chunks; box[3] = box_h; box[4] = 1;
  }
  return fn(tm, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 5, const_cast<void*>(base), dims, strides, box, estr,
            CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
            CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
}

// NHWC bf16 [N][H][W][Cp] as a 5-D tensor {16, W, Cp/16, H, N} whose innermost unit is a 16-channel (32-byte)
// block, SWIZZLE_32B: the box lands as smem [row][block][pixel][16 ch] with the two 16-B halves of each 32-B
// pixel row swapped when address bit 7 is set -- the MN-major SWIZZLE_32B canonical layout (atoms of 16 channels
// x 8 pixels).  Twice the TMA throughput of the 16-B-innermost maps above (scripts/tma_rate.py).
inline CUresult make_act_tmap_sw32(CUtensorMap* tm, const void* base, int N, int H, int W, int Cp, int box_w,
                                   int box_h) {
  auto fn = get_encode_fn();
  if (!fn) return CUDA_ERROR_NOT_SUPPORTED;
  const uint64_t pix = (uint64_t)Cp * 2, row = (uint64_t)W * pix, img = (uint64_t)H * row;
  cuuint64_t dims[5] = {16, (cuuint64_t)W, (cuuint64_t)(Cp / 16), (cuuint64_t)H, (cuuint64_t)N};
  cuuint64_t strides[4] = {pix, 32, row, img};
  cuuint32_t box[5] = {16, (cuuint32_t)box_w, (cuuint32_t)(Cp / 16), (cuuint32_t)box_h, 1};
  cuuint32_t estr[5] = {1, 1, 1, 1, 1};
  return fn(tm, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 5, const_cast<void*>(base), dims, strides, box, estr,
            CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_32B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
            CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
}

// NHWC bf16 [N][H][W][Cp] as a 4-D tensor {Cp, W, H, N}; box {box_c, box_w, 1, 1} = (part of the channels of)
// one row segment, smem layout [pixel][box_c] (residual rows; per-warp output slices for the TMA store).
inline CUresult make_row_tmap(CUtensorMap* tm, const void* base, int N, int H, int W, int Cp, int box_w, int box_c) {
  auto fn = get_encode_fn();
  if (!fn) return CUDA_ERROR_NOT_SUPPORTED;
  cuuint64_t dims[4] = {(cuuint64_t)Cp, (cuuint64_t)W, (cuuint64_t)H, (cuuint64_t)N};
  cuuint64_t strides[3] = {(cuuint64_t)Cp * 2, (cuuint64_t)W * Cp * 2, (cuuint64_t)H * W * Cp * 2};
  cuuint32_t box[4] = {(cuuint32_t)box_c, (cuuint32_t)box_w, 1, 1};
  cuuint32_t estr[4] = {1, 1, 1, 1};
  return fn(tm, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 4, const_cast<void*>(base), dims, strides, box, estr,
            CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
            CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
}

// u8 image rows [N][H][row_bytes] (NHWC RGB frames: row_bytes = 3 W) as a 4-D tensor {16, row_bytes/16, H, N}
// whose innermost unit is a 16-byte chunk; box {16, box_chunks, box_rows, 1} lands as smem [row][chunk][16], i.e.
// box_rows dense rows of 16 * box_chunks bytes.  Needs row_bytes % 16 == 0 and a 16-B aligned base.  Used by the
// up-conv tail: LR neighbourhood rows in, staged HR rows out (one TMA per LR row instead of 27 byte accesses per
// lane).  Out-of-bounds box bytes are zero-filled (loads) / clipped (stores).
inline CUresult make_u8_rows_tmap(CUtensorMap* tm, const void* base, int N, int H, long long row_bytes,
                                  int box_chunks, int box_rows) {
  auto fn = get_encode_fn();
  if (!fn) return CUDA_ERROR_NOT_SUPPORTED;
  if (row_bytes % 16 != 0 || (reinterpret_cast<uintptr_t>(base) & 15) != 0) return CUDA_ERROR_INVALID_VALUE;
  cuuint64_t dims[4] = {16, (cuuint64_t)(row_bytes / 16), (cuuint64_t)H, (cuuint64_t)N};
  cuuint64_t strides[3] = {16, (cuuint64_t)row_bytes, (cuuint64_t)row_bytes * H};
  cuuint32_t box[4] = {16, (cuuint32_t)box_chunks, (cuuint32_t)box_rows, 1};
  cuuint32_t estr[4] = {1, 1, 1, 1};
  return fn(tm, CU_TENSOR_MAP_DATA_TYPE_UINT8, 4, const_cast<void*>(base), dims, strides, box, estr,
            CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
            CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
}

}  // namespace sr

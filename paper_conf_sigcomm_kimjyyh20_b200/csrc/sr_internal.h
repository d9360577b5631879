// Internal declarations shared by the CUDA translation units of libsr.so (not part of the C ABI).
#pragma once
#include <cstdint>
#include <cstddef>
#include <cuda_runtime.h>
#include <cuda_bf16.h>
#include "../../include/sr.h"

namespace sr {

typedef __nv_bfloat16 bf16;

// Geometry of one implicit-GEMM conv launch (output = input spatial dims, 3x3, pad 1).
// A work unit is a tile of R output rows x TW output pixels of one image.  The input tile with a
// 1-pixel halo, (R+2) rows x P = TW+2 pixels x Cin, lands in shared memory "chunk-planar":
// [8-channel chunk][row][pixel][8 x bf16]; output position q (flattened with pitch P) of M-tile mt is
// q = mt*MS + lane.  Wide tiles (TW=128): MS = P, one output row per M-tile.  Narrow tiles (W < 96,
// e.g. 48x48 training patches): MS = 128, M-tiles run across rows; lanes that land in the halo
// columns are discarded.
struct ConvGeom {
  int N, H, W;
  int TW, R, P;
  int tiles_x, tiles_y, units;
  int MS, n_mt, wide;
};

enum EpiKind { EPI_ACT = 0, EPI_TAIL_U8 = 1, EPI_TAIL_TRAIN = 2 };

struct EpiParams {
  const float* bias;   // [COUTP] fp32 or null
  const bf16* res1;    // [N,H,W,COUTP] or null: v += res1
  const bf16* res2;    // [N,H,W,COUTP] or null: v += res2
  const bf16* mask;    // [N,H,W,COUTP] or null: v = mask > 0 ? v : 0 (ReLU' through a saved ReLU output)
  int relu;            // v = max(v, 0)
  bf16* out;           // EPI_ACT output [N,H,W,COUTP]
  // tail (pixel shuffle + bilinear skip):
  int scale;
  const uint8_t* lr;   // [N,H,W,3] LR u8 frames / patches
  uint8_t* hr;         // EPI_TAIL_U8: [N, sH, sW, 3]
  int hr_row0;         // EPI_TAIL_U8: first LR row written (strip mode); rows outside [hr_row0, hr_row1) skipped
  int hr_row1;
  const uint8_t* hr_ref;  // EPI_TAIL_TRAIN: target [N, sH, sW, 3]
  bf16* dy;            // EPI_TAIL_TRAIN: 2*(o - t) in pixel-unshuffled layout [N,H,W,COUTP]
  double* loss_sum;    // EPI_TAIL_TRAIN: += sum (o - t)^2
  int dbg;             // benchmarking only: 1 = drain TMEM and skip the epilogue, 2 = plain store (no bias/res)
  int vsep, vp;        // EPI_TAIL_TRAIN on the virtual training batch: column pitch p+2 and patch size p (0 = off)
  int l1;              // EPI_TAIL_TRAIN: L1 loss (loss += |d|, dy = sign(d)) instead of MSE
  int bicubic;         // tails: bicubic skip (reading R23) instead of bilinear
};

ConvGeom make_geom(int N, int H, int W, int cinp, int coutp, size_t* smem_bytes);
cudaError_t launch_conv(int cinp, int coutp, int epi, const void* in, const bf16* wpk, const ConvGeom& g,
                        const EpiParams& ep, size_t smem, int grid, cudaStream_t st);

struct WgradGeom {
  int N, H, W;
  int TW, R, P;
  int tiles_x, tiles_y, units;
  long long* dbg;  // optional per-CTA globaltimer stamps [grid][8] (benchmarking only)
  int exp;         // benchmarking experiments (results wrong): bit 0 skip bias-grad reads, bit 1 no TMA after the
                   // first ring fill, bit 2 skip the MMAs
};
// Where the weight gradient goes: per-CTA split-K partials ws [grid][9*cinp*coutp + coutp] (fp32), a grid
// barrier {count, generation} (zero-initialised once, reusable), and the final
// gW[co][ci][3][3] = scale * sum_cta partial, gb[co] likewise (canonical OIHW, unpadded cin x cout).
struct WgradOut {
  float* ws;
  unsigned* sync;
  float* gW;
  float* gb;
  int cin, cout;
  float scale;
};
WgradGeom make_wgrad_geom(int N, int H, int W, int cinp, int coutp, size_t* smem_bytes);
cudaError_t launch_wgrad(int cinp, int coutp, const bf16* x, const bf16* dy, const WgradGeom& g, const WgradOut& o,
                         size_t smem, int grid, cudaStream_t st);

// Batched rolling wgrad for wide images (conv_wgrad.cu): up to kWgradMaxJobs convs over inputs of one shape in one
// launch, partials ws[(grid + J)][max stride] (wgrad_multi_ws_floats), grid = wgrad_multi_grid, sync as WgradOut.
static constexpr int kWgradMaxJobs = 20;
struct WgradJob {
  const bf16* x;   // conv input  [N,H,W,cinp]
  const bf16* dy;  // conv output gradient [N,H,W,coutp]
  int cinp, coutp, cin, cout;
  float* gW;       // canonical OIHW [cout][cin][3][3]
  float* gb;       // [cout]
};
bool wgrad_multi_supported(const WgradJob* jobs, int J, int W);
int wgrad_multi_grid(int J, int N, int H, int W);
size_t wgrad_multi_ws_floats(const WgradJob* jobs, int J, int grid);
cudaError_t launch_wgrad_multi(const WgradJob* jobs, int J, int N, int H, int W, float scale, float* ws,
                               unsigned* sync, int grid, long long* dbg, cudaStream_t st);

int num_sms();
void set_grid_cap(int cap);
int grid_cap();

}  // namespace sr

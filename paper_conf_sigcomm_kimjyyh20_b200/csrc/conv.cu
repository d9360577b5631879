// 3x3 convolutions on the 5th-gen tensor cores (tcgen05) for sm_100a: implicit GEMM, TMA-staged NHWC bf16
// tiles, fp32 accumulators in TMEM, fused epilogues.
//
//   forward / data-grad:  D[pixel, co] = sum_{tap, ci} X[pixel + tap, ci] * W[tap, ci, co]
//       M = 128 output positions per MMA tile, N = Cout (padded to 16), K = 9 taps x Cin.
//       The tap shift is free: the A operand of tap (dy,dx) is the same smem tile with the descriptor start
//       address moved by (dy*P + dx) * 16 bytes (SWIZZLE_NONE K-major layout = one 16-byte row per pixel).
//   weight-grad:  D[(dy, ci), co] (for each dx) = sum_pixel X[pixel + (dy,dx), ci] * dY[pixel, co]
//       K = pixels, both operands MN-major from row-planar smem tiles; split-K over CTAs, deterministic
//       reduction in a second kernel.
//
// Warp roles (192 threads): warp 0 = TMA producer, warp 1 = TMEM allocator + single-thread MMA issuer,
// warps 2..5 = epilogue (TMEM -> registers -> bias/ReLU/residual/mask or pixel-shuffle tail -> HBM).
#include <cuda.h>
#include "ptx.cuh"
#include "tmap.h"
#include "sr_internal.h"
#include "kernels.h"
#include "launch.cuh"
#include "tail.cuh"

namespace sr {

static constexpr int kConvThreads = 320;   // conv: TMA warp, MMA warp, 2 x 4 epilogue warps
static constexpr int kWgradThreads = 384;  // wgrad: TMA warp, MMA warp, 4 epilogue warps, 6 more for the reduction
static constexpr int kStages = 2;
static constexpr int kWgStages = 3;  // wgrad TMA ring depth
static constexpr int kSmemLimit = 227 * 1024;

// Grid sizing.  Every persistent kernel takes one CTA per SM; set_grid_cap limits that to the SM share of the
// calling API entry (sr_set_sm_split: inference and training running concurrently on disjoint SM sets).
static thread_local int g_grid_cap = 0;
void set_grid_cap(int cap) { g_grid_cap = cap; }
int grid_cap() { return g_grid_cap; }
int num_sms() {
  static int n = 0;
  if (!n) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
    if (n <= 0) n = 148;
  }
  return (g_grid_cap > 0 && g_grid_cap < n) ? g_grid_cap : n;
}

// ------------------------------------------------------------------------------------------ geometry
static size_t conv_smem(int cinp, int coutp, int R, int P, int n_mt, int MS) {
  size_t wbytes = (size_t)9 * cinp * coutp * 2;
  size_t stage = ((size_t)(cinp / 8) * (R + 2) * P * 16 + 1023) / 1024 * 1024;  // TMA dst: 128-B aligned
  long over = (long)(n_mt - 1) * MS + 128 + 2 * P + 2 - (long)(R + 2) * P;  // positions read past a plane
  size_t slack = over > 0 ? (size_t)over * 16 : 0;
  return 1024 + wbytes + kStages * stage + slack + 16 + coutp * 4;
}

ConvGeom make_geom(int N, int H, int W, int cinp, int coutp, size_t* smem_bytes) {
  ConvGeom g{};
  g.N = N; g.H = H; g.W = W;
  if (W >= 96) {  // wide: one 128-pixel output row segment per M-tile
    g.TW = 128; g.P = 130; g.wide = 1; g.MS = g.P;
    int R = 4;
    while (R > 1 && conv_smem(cinp, coutp, R, g.P, R, g.MS) > (size_t)kSmemLimit) --R;
    g.R = R < H ? R : H;
    g.n_mt = g.R;
  } else {        // narrow (training patches): M-tiles run across rows of a pitch-(W+2) tile
    g.TW = W; g.P = W + 2; g.wide = 0; g.MS = 128;
    int R = (640 + g.P - 1) / g.P;
    if (R > H) R = H;
    for (;;) {
      int n_mt = (R * g.P + 127) / 128;
      if (R == 1 || conv_smem(cinp, coutp, R, g.P, n_mt, 128) <= (size_t)kSmemLimit) break;
      --R;
    }
    g.R = R;
    g.n_mt = (R * g.P + 127) / 128;
  }
  g.tiles_x = (W + g.TW - 1) / g.TW;
  g.tiles_y = (H + g.R - 1) / g.R;
  g.units = N * g.tiles_x * g.tiles_y;
  if (smem_bytes) *smem_bytes = conv_smem(cinp, coutp, g.R, g.P, g.n_mt, g.MS);
  return g;
}

// ------------------------------------------------------------------------------------------ epilogues
template <int COUTP>
__device__ __forceinline__ void load_bf16_row(const bf16* p, float* v) {
  const uint4* q = reinterpret_cast<const uint4*>(p);
#pragma unroll
  for (int i = 0; i < COUTP / 8; ++i) {
    uint4 u = __ldg(q + i);
    const __nv_bfloat162* h = reinterpret_cast<const __nv_bfloat162*>(&u);
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      float2 f = __bfloat1622float2(h[j]);
      v[i * 8 + 2 * j] = f.x;
      v[i * 8 + 2 * j + 1] = f.y;
    }
  }
}

// Residual / mask rows of one output pixel, loaded BEFORE the accumulator is waited on so that the global
// load latency overlaps the MMAs of this M-tile.
template <int COUTP>
struct EpiPre {
  uint4 r1[COUTP / 8], r2[COUTP / 8], mk[COUTP / 8];
};

template <int COUTP>
__device__ __forceinline__ void epi_prefetch(const EpiParams& ep, size_t pix, EpiPre<COUTP>& pre) {
#pragma unroll
  for (int i = 0; i < COUTP / 8; ++i) {
    if (ep.res1) pre.r1[i] = __ldg(reinterpret_cast<const uint4*>(ep.res1 + pix * COUTP) + i);
    if (ep.res2) pre.r2[i] = __ldg(reinterpret_cast<const uint4*>(ep.res2 + pix * COUTP) + i);
    if (ep.mask) pre.mk[i] = __ldg(reinterpret_cast<const uint4*>(ep.mask + pix * COUTP) + i);
  }
}

__device__ __forceinline__ void unpack8(const uint4& u, float* f) {
  const __nv_bfloat162* h = reinterpret_cast<const __nv_bfloat162*>(&u);
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    float2 t = __bfloat1622float2(h[j]);
    f[2 * j] = t.x;
    f[2 * j + 1] = t.y;
  }
}

// out = [mask>0] * act(acc + bias + res1 + res2)
template <int COUTP>
__device__ __forceinline__ void epi_act(const EpiParams& ep, const float* sbias, size_t pix, float* v,
                                        const EpiPre<COUTP>& pre) {
  if (ep.bias) {
#pragma unroll
    for (int c = 0; c < COUTP; ++c) v[c] += sbias[c];
  }
#pragma unroll
  for (int i = 0; i < COUTP / 8; ++i) {
    float f[8];
    if (ep.res1) {
      unpack8(pre.r1[i], f);
#pragma unroll
      for (int j = 0; j < 8; ++j) v[8 * i + j] += f[j];
    }
    if (ep.res2) {
      unpack8(pre.r2[i], f);
#pragma unroll
      for (int j = 0; j < 8; ++j) v[8 * i + j] += f[j];
    }
    if (ep.relu) {
#pragma unroll
      for (int j = 0; j < 8; ++j) v[8 * i + j] = fmaxf(v[8 * i + j], 0.f);
    }
    if (ep.mask) {
      unpack8(pre.mk[i], f);
#pragma unroll
      for (int j = 0; j < 8; ++j) v[8 * i + j] = f[j] > 0.f ? v[8 * i + j] : 0.f;
    }
  }
  store_bf16_row<COUTP>(ep.out + pix * COUTP, v);
}

// ------------------------------------------------------------------------------------------ conv kernel
template <int CINP, int COUTP, int EPI, int S>
__global__ void __launch_bounds__(kConvThreads, 1)
k_conv3x3(const __grid_constant__ CUtensorMap tm_in, const bf16* __restrict__ wpk, const ConvGeom g,
          const EpiParams ep) {
  constexpr int CCH = CINP / 8;
  constexpr int KSTEPS = CINP / 16;
  constexpr uint32_t WBYTES = 9u * CINP * COUTP * 2u;
  constexpr int SLOT = COUTP <= 32 ? 32 : (COUTP <= 64 ? 64 : 128);
  constexpr int NSLOT = 4;
  constexpr uint32_t TMEM_COLS = SLOT * NSLOT;
  constexpr uint32_t IDESC = make_idesc(128, COUTP, 0, 0);

  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);  // stays in the shared window (LDS/STS, not generic)
  __shared__ __align__(8) uint64_t full_bar[kStages], empty_bar[kStages], tfull_bar[NSLOT], tempty_bar[NSLOT];
  __shared__ __align__(8) uint64_t w_bar;
  __shared__ uint32_t tmem_base_sh;
  __shared__ float sbias[COUTP];

  const int P = g.P;
  const uint32_t plane = (uint32_t)(g.R + 2) * P * 16;
  const uint32_t stage_bytes = plane * CCH;                            // TMA box bytes
  const uint32_t stage_stride = (stage_bytes + 1023u) & ~1023u;        // smem stage stride (TMA dst alignment)
  uint8_t* sW = smem;
  uint8_t* sStage = smem + WBYTES;

  const int warp = warp_id();
  if (warp == 0 && lane_id() == 0) {
    for (int s = 0; s < kStages; ++s) { mbar_init(&full_bar[s], 1); mbar_init(&empty_bar[s], 1); }
    for (int s = 0; s < NSLOT; ++s) { mbar_init(&tfull_bar[s], 1); mbar_init(&tempty_bar[s], 4); }
    mbar_init(&w_bar, 1);
    fence_barrier_init();
  }
  if (warp == 1) tmem_alloc<TMEM_COLS>(&tmem_base_sh);
  tc_fence_before();
  __syncthreads();
  pdl_enter();
  if (threadIdx.x < COUTP) sbias[threadIdx.x] = ep.bias ? ep.bias[threadIdx.x] : 0.f;
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = tmem_base_sh;
  const int tiles_xy = g.tiles_x * g.tiles_y;

  if (warp == 0) {
    // ===================== TMA producer =====================
    if (elect_one()) {
      tma_prefetch_desc(&tm_in);
      mbar_arrive_expect_tx(&w_bar, WBYTES);
      bulk_load(sW, wpk, WBYTES, &w_bar);
      int s = 0;
      uint32_t ph = 0;
      for (int u = blockIdx.x; u < g.units; u += gridDim.x) {
        const int n = u / tiles_xy, rem = u - n * tiles_xy;
        const int ty = rem / g.tiles_x, tx = rem - ty * g.tiles_x;
        mbar_wait(&empty_bar[s], ph ^ 1);
        mbar_arrive_expect_tx(&full_bar[s], stage_bytes);
        tma_load_5d(sStage + s * stage_stride, &tm_in, &full_bar[s], 0, tx * g.TW - 1, ty * g.R - 1, 0, n);
        if (++s == kStages) { s = 0; ph ^= 1; }
      }
    }
    __syncwarp();
  } else if (warp == 1) {
    // ===================== MMA issuer (one thread) =====================
    if (elect_one()) {
      mbar_wait(&w_bar, 0);
      const uint64_t bdesc0 = make_desc(smem_u32(sW), COUTP * 16, 128);
      int s = 0, slot = 0;
      uint32_t ph = 0, tph = 0;
      for (int u = blockIdx.x; u < g.units; u += gridDim.x) {
        mbar_wait(&full_bar[s], ph);
        tc_fence_after();
        const uint64_t adesc0 = make_desc(smem_u32(sStage + s * stage_stride), plane, 128);
        for (int mt = 0; mt < g.n_mt; ++mt) {
          mbar_wait(&tempty_bar[slot], tph ^ 1);
          tc_fence_after();
          const uint32_t d = tmem + slot * SLOT;
#pragma unroll
          for (int tap = 0; tap < 9; ++tap) {
            const uint32_t aoff = (uint32_t)(mt * g.MS + (tap / 3) * P + (tap % 3)) * 16u;
#pragma unroll
            for (int ks = 0; ks < KSTEPS; ++ks) {
              mma_bf16_ss(d, desc_add(adesc0, aoff + ks * 2 * plane),
                          desc_add(bdesc0, (uint32_t)(tap * CCH + 2 * ks) * COUTP * 16u), IDESC,
                          (tap | ks) != 0);
            }
          }
          mma_commit(&tfull_bar[slot]);
          if (++slot == NSLOT) { slot = 0; tph ^= 1; }
        }
        mma_commit(&empty_bar[s]);
        if (++s == kStages) { s = 0; ph ^= 1; }
      }
    }
    __syncwarp();
  } else {
    // ===================== epilogue (warps 2..9: two groups of 4 alternate M-tiles) =====================
    const int quarter = warp & 3;            // TMEM lane quarter this warp may access
    const int grp = (warp - 2) >> 2;         // M-tile k is drained by group k % 2
    const int row = quarter * 32 + lane_id();
    float lsum = 0.f;
    int k = 0;                               // running M-tile index (same sequence as the MMA issuer)
    for (int u = blockIdx.x; u < g.units; u += gridDim.x) {
      const int n = u / tiles_xy, rem = u - n * tiles_xy;
      const int ty = rem / g.tiles_x, tx = rem - ty * g.tiles_x;
      const int y0 = ty * g.R, x0 = tx * g.TW;
      for (int mt = 0; mt < g.n_mt; ++mt, ++k) {
        if ((k & 1) != grp) continue;
        const int slot = k % NSLOT;
        const uint32_t tph = (uint32_t)(k / NSLOT) & 1u;
        int r, x;
        if (g.wide) { r = mt; x = row; }
        else { const int q = mt * 128 + row; r = q / P; x = q - r * P; }
        const int Y = y0 + r, X = x0 + x;
        const bool valid = x < g.TW && r < g.R && Y < g.H && X < g.W;
        const size_t pix = ((size_t)n * g.H + Y) * g.W + X;
        EpiPre<COUTP> pre;
        if (EPI == EPI_ACT && valid && ep.dbg == 0) epi_prefetch<COUTP>(ep, pix, pre);
        mbar_wait(&tfull_bar[slot], tph);
        tc_fence_after();
        float v[COUTP];
#pragma unroll
        for (int c0 = 0; c0 < COUTP; c0 += 16)
          tmem_ld16(tmem + ((uint32_t)(quarter * 32) << 16) + slot * SLOT + c0, v + c0);
        tmem_ld_wait();
        tc_fence_before();
        __syncwarp();
        if (lane_id() == 0) mbar_arrive(&tempty_bar[slot]);
        if (!valid || ep.dbg == 1) continue;
        if (EPI == EPI_ACT && ep.dbg == 2) {
          store_bf16_row<COUTP>(ep.out + pix * COUTP, v);
        } else if (EPI == EPI_ACT) {
          epi_act<COUTP>(ep, sbias, pix, v, pre);
        } else if (EPI == EPI_TAIL_U8) {
          if (ep.vsep > 0) {  // virtual batch of square images: image j at columns [j*vsep + 1, j*vsep + 1 + p)
            const int j = X / ep.vsep, x = X - j * ep.vsep - 1;
            if (x >= 0 && x < ep.vp) epi_tail<S, COUTP, false>(ep, sbias, j, Y, x, ep.vp, ep.vp, v, lsum, 0);
          } else if (Y >= ep.hr_row0 && Y < ep.hr_row1)
            epi_tail<S, COUTP, false>(ep, sbias, n, Y, X, g.H, g.W, v, lsum, ((size_t)n * g.H + Y) * g.W + X);
        } else {
          const size_t vp = ((size_t)n * g.H + Y) * g.W + X;
          if (ep.vsep > 0) {  // virtual training batch: patch j at columns [j*vsep + 1, j*vsep + 1 + p)
            const int j = X / ep.vsep, x = X - j * ep.vsep - 1;
            if (x < 0 || x >= ep.vp) {  // separator column: no loss, zero gradient
              float z[COUTP];
#pragma unroll
              for (int k = 0; k < COUTP; ++k) z[k] = 0.f;
              store_bf16_row<COUTP>(ep.dy + vp * COUTP, z);
            } else {
              epi_tail<S, COUTP, true>(ep, sbias, j, Y, x, ep.vp, ep.vp, v, lsum, vp);
            }
          } else {
            epi_tail<S, COUTP, true>(ep, sbias, n, Y, X, g.H, g.W, v, lsum, vp);
          }
        }
      }
    }
    if (EPI == EPI_TAIL_TRAIN) {
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) lsum += __shfl_xor_sync(0xffffffffu, lsum, o);
      if (lane_id() == 0) atomicAdd(ep.loss_sum, (double)lsum);
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 1) tmem_dealloc<TMEM_COLS>(tmem);
}

template <int CINP, int COUTP, int EPI, int S>
static cudaError_t launch_conv_t(const CUtensorMap& tm, const bf16* wpk, const ConvGeom& g, const EpiParams& ep,
                                 size_t smem, int grid, cudaStream_t st) {
  auto kern = k_conv3x3<CINP, COUTP, EPI, S>;
  static size_t configured = 0;
  if (smem > configured) {
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    configured = smem;
  }
  return launch_k(kern, dim3(grid), dim3(kConvThreads), smem, st, tm, wpk, g, ep);
}

#define SR_CONV_CASE(CI, CO)                                                                 \
  if (cinp == CI && coutp == CO) {                                                           \
    if (epi == EPI_ACT) return launch_conv_t<CI, CO, EPI_ACT, 1>(tm, wpk, g, ep, smem, grid, st); \
  }
#define SR_TAIL_CASE(CI, CO, S)                                                                          \
  if (cinp == CI && coutp == CO && ep.scale == S) {                                                      \
    if (epi == EPI_TAIL_U8) return launch_conv_t<CI, CO, EPI_TAIL_U8, S>(tm, wpk, g, ep, smem, grid, st);  \
    if (epi == EPI_TAIL_TRAIN)                                                                           \
      return launch_conv_t<CI, CO, EPI_TAIL_TRAIN, S>(tm, wpk, g, ep, smem, grid, st);                   \
  }

cudaError_t launch_conv(int cinp, int coutp, int epi, const void* in, const bf16* wpk, const ConvGeom& g,
                        const EpiParams& ep, size_t smem, int grid, cudaStream_t st) {
  CUtensorMap tm;
  if (make_act_tmap(&tm, in, g.N, g.H, g.W, cinp, g.P, g.R + 2, cinp / 8, CHUNK_ROW_PIX) != CUDA_SUCCESS)
    return cudaErrorInvalidValue;
  // head (16 -> C), body/blocks (C -> C), data-grad of the up conv (16/32 -> C)
  SR_CONV_CASE(16, 16) SR_CONV_CASE(16, 32) SR_CONV_CASE(16, 48) SR_CONV_CASE(16, 64)
  SR_CONV_CASE(32, 16) SR_CONV_CASE(32, 32) SR_CONV_CASE(32, 48) SR_CONV_CASE(32, 64)
  SR_CONV_CASE(48, 16) SR_CONV_CASE(48, 32) SR_CONV_CASE(48, 48)
  SR_CONV_CASE(64, 16) SR_CONV_CASE(64, 32) SR_CONV_CASE(64, 64) SR_CONV_CASE(48, 64)
  // up conv + tail (C -> 3 s^2 padded: 12 -> 16, 27 -> 32, 48)
  SR_TAIL_CASE(16, 16, 2) SR_TAIL_CASE(32, 16, 2) SR_TAIL_CASE(48, 16, 2) SR_TAIL_CASE(64, 16, 2)
  SR_TAIL_CASE(16, 32, 3) SR_TAIL_CASE(32, 32, 3) SR_TAIL_CASE(48, 32, 3) SR_TAIL_CASE(64, 32, 3)
  SR_TAIL_CASE(16, 48, 4) SR_TAIL_CASE(32, 48, 4) SR_TAIL_CASE(48, 48, 4) SR_TAIL_CASE(64, 48, 4)
  return cudaErrorNotSupported;
}

// ------------------------------------------------------------------------------------------ weight grad
// Stage: X tile (R+2) rows x P = TW+2 px and dY tile R rows x TW px, both loaded by TMA in the MN-major
// SWIZZLE_32B layout [row][16-ch block][px][16 ch] (32-B TMA inner unit: twice the TMA throughput of the
// 16-B-chunk maps, which would otherwise bound this kernel; scripts/tma_rate.py).
// A (MN-major) = X^T: M = (dy, ci) atoms of 16 channels a = dy*CB + cb at stride LBO = P*32 (rows are consecutive
// planes, so the three dy of a tile row are consecutive atoms), K = pixels (8-row groups, SBO = 256; the dx tap
// is a start-address shift of dx pixel rows).  B (MN-major) = dY: N = co atoms at LBO = TW*32.
// D[dx][mt] (128 lanes = 8 atoms, COUTP columns), accumulated over all of this CTA's K (split-K) and written as
// a per-CTA partial.  Then a grid barrier (cooperative launch: all CTAs are co-resident) and every CTA sums its
// 1/grid slice of the outputs over all partials in CTA order (fixed order -> deterministic), scales and
// scatters it into the canonical OIHW gradient.  No separate reduction kernel.
static size_t wgrad_smem(int cinp, int coutp, int R, int TW) {
  const int P = TW + 2;
  const int cb = cinp / 16, ob = coutp / 16;
  const int n_mt = (3 * cb + 7) / 8;
  size_t xs = ((size_t)(R + 2) * cb * P * 32 + 1023) / 1024 * 1024;
  size_t ys = ((size_t)R * ob * TW * 32 + 1023) / 1024 * 1024;
  long over = (long)(8 * n_mt - 3 * cb) * P * 32 + 64;  // atoms read past the X tile by padded M-tiles
  return 1024 + kWgStages * (xs + ys) + (over > 0 ? (size_t)over : 0) + 256;
}

WgradGeom make_wgrad_geom(int N, int H, int W, int cinp, int coutp, size_t* smem_bytes) {
  WgradGeom g{};
  g.N = N; g.H = H; g.W = W;
  g.TW = W >= 64 ? 64 : ((W + 15) / 16) * 16;
  g.P = g.TW + 2;
  int R = 4;
  while (R > 1 && wgrad_smem(cinp, coutp, R, g.TW) > (size_t)kSmemLimit) --R;
  g.R = R < H ? R : H;
  g.tiles_x = (W + g.TW - 1) / g.TW;
  g.tiles_y = (H + g.R - 1) / g.R;
  g.units = N * g.tiles_x * g.tiles_y;
  if (smem_bytes) *smem_bytes = wgrad_smem(cinp, coutp, g.R, g.TW);
  return g;
}

template <int CINP, int COUTP>
__global__ void __launch_bounds__(kWgradThreads, 1)
k_wgrad(const __grid_constant__ CUtensorMap tm_x, const __grid_constant__ CUtensorMap tm_dy, const WgradGeom g,
        const WgradOut o) {
  constexpr int CB = CINP / 16, OB = COUTP / 16, OCH = COUTP / 8;
  constexpr int NMT = (3 * CB + 7) / 8;
  constexpr uint32_t TMEM_NEED = 3 * NMT * COUTP;
  constexpr uint32_t TMEM_COLS = TMEM_NEED <= 32 ? 32 : TMEM_NEED <= 64 ? 64 : TMEM_NEED <= 128 ? 128
                                 : TMEM_NEED <= 256 ? 256 : 512;
  static_assert(TMEM_NEED <= 512, "wgrad accumulators exceed TMEM");
  constexpr uint32_t IDESC = make_idesc(128, COUTP, 1, 1);

  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);  // stays in the shared window (LDS/STS, not generic)
  constexpr int PER = 9 * CINP * COUTP, STRIDE = PER + COUTP;  // floats per partial
  __shared__ __align__(8) uint64_t full_bar[kWgStages], empty_bar[kWgStages], done_bar;
  __shared__ uint32_t tmem_base_sh;
  __shared__ float sdb[128 / OCH][COUTP];

  const int TW = g.TW, P = g.P, R = g.R;
  const uint32_t xbox = (uint32_t)(R + 2) * CB * P * 32, ybox = (uint32_t)R * OB * TW * 32;  // TMA box bytes
  const uint32_t xbytes = (xbox + 1023u) & ~1023u;      // dY tile offset inside a stage (TMA alignment)
  const uint32_t ybytes = (ybox + 1023u) & ~1023u;
  const uint32_t stage_bytes = xbytes + ybytes;
  const int warp = warp_id();
  if (warp == 0 && lane_id() == 0) {
    for (int s = 0; s < kWgStages; ++s) { mbar_init(&full_bar[s], 1); mbar_init(&empty_bar[s], 2); }
    mbar_init(&done_bar, 1);
    fence_barrier_init();
  }
  long long* dbg = g.dbg ? g.dbg + (size_t)blockIdx.x * 8 : nullptr;
  if (dbg && threadIdx.x == 0) dbg[0] = globaltimer();
  if (warp == 1) tmem_alloc<TMEM_COLS>(&tmem_base_sh);
  tc_fence_before();
  __syncthreads();
  pdl_wait();  // dependents are released only after the grid barrier below (no co-residency deadlock)
  tc_fence_after();
  if (dbg && threadIdx.x == 0) dbg[1] = clock64();
  const uint32_t tmem = tmem_base_sh;
  const int tiles_xy = g.tiles_x * g.tiles_y;

  if (warp == 0) {
    if (elect_one()) {
      tma_prefetch_desc(&tm_x);
      tma_prefetch_desc(&tm_dy);
      int s = 0;
      uint32_t ph = 0;
      for (int u = blockIdx.x; u < g.units; u += gridDim.x) {
        const int n = u / tiles_xy, rem = u - n * tiles_xy;
        const int ty = rem / g.tiles_x, tx = rem - ty * g.tiles_x;
        mbar_wait(&empty_bar[s], ph ^ 1);
        if ((g.exp & 2) && u >= (int)blockIdx.x + kWgStages * (int)gridDim.x) {
          mbar_arrive(&full_bar[s]);
        } else {
          mbar_arrive_expect_tx(&full_bar[s], xbox + ybox);
          uint8_t* base = smem + s * stage_bytes;
          tma_load_5d(base, &tm_x, &full_bar[s], 0, tx * TW - 1, 0, ty * R - 1, n);
          tma_load_5d(base + xbytes, &tm_dy, &full_bar[s], 0, tx * TW, 0, ty * R, n);
        }
        if (++s == kWgStages) { s = 0; ph ^= 1; }
      }
    }
    __syncwarp();
  } else if (warp == 1) {
    if (elect_one()) {
      int s = 0;
      uint32_t ph = 0;
      uint32_t acc = 0;
      long long waited = 0;
      for (int u = blockIdx.x; u < g.units; u += gridDim.x) {
        const long long tw0 = dbg ? globaltimer() : 0;
        mbar_wait(&full_bar[s], ph);
        if (dbg) {
          const long long tw1 = globaltimer();
          if (u == (int)blockIdx.x) dbg[2] = tw1;
          else waited += tw1 - tw0;
        }
        tc_fence_after();
        const uint32_t xb = smem_u32(smem + s * stage_bytes);
        const uint32_t yb = xb + xbytes;
        const uint64_t a0 = make_desc_sw(xb, P * 32, 256, 6);
        const uint64_t b0 = make_desc_sw(yb, TW * 32, 256, 6);
        for (int r = 0; r < R; ++r) {
          for (int k16 = 0; k16 < TW / 16; ++k16) {
            const uint32_t boff = (uint32_t)(r * OB * TW + k16 * 16) * 32u;
#pragma unroll
            for (int dx = 0; dx < 3; ++dx) {
#pragma unroll
              for (int mt = 0; mt < NMT; ++mt) {
                const uint32_t aoff = (uint32_t)((r * CB + 8 * mt) * P + k16 * 16 + dx) * 32u;
                if (!(g.exp & 4))
                  mma_bf16_ss(tmem + (dx * NMT + mt) * COUTP, desc_add(a0, aoff), desc_add(b0, boff), IDESC, acc);
              }
            }
            acc = 1;
          }
        }
        mma_commit(&empty_bar[s]);
        if (++s == kWgStages) { s = 0; ph ^= 1; }
      }
      mma_commit(&done_bar);
      if (dbg) dbg[3] = globaltimer();
    }
    __syncwarp();
  } else if (warp < 6) {
    // epilogue warps: bias gradient from the dY tiles while the MMAs run, then drain the accumulators.
    // Thread et owns 8-channel chunk j = et % OCH (block j/2, half j%2) and pixel subset grp = et / OCH (fixed
    // order -> deterministic).  Half h of pixel p sits at 16 * (h ^ bit 2 of p) (SWIZZLE_32B).
    const int et = threadIdx.x - 64;  // 0..127
    constexpr int NG = 128 / OCH;
    const int j = et % OCH, grp = et / OCH;
    float acc8[8];
#pragma unroll
    for (int e = 0; e < 8; ++e) acc8[e] = 0.f;
    int s = 0;
    uint32_t ph = 0;
    for (int u = blockIdx.x; u < g.units; u += gridDim.x) {
      mbar_wait(&full_bar[s], ph);
      if (grp < NG && !(g.exp & 1)) {
        const uint8_t* yt = smem + s * stage_bytes + xbytes;
        for (int r = 0; r < R; ++r) {
          for (int p = grp; p < TW; p += NG) {
            const uint32_t off = ((uint32_t)(r * OB + (j >> 1)) * TW + p) * 32u + (((j & 1) ^ ((p >> 2) & 1)) << 4);
            const uint4 q = *reinterpret_cast<const uint4*>(yt + off);
            const __nv_bfloat162* h2 = reinterpret_cast<const __nv_bfloat162*>(&q);
#pragma unroll
            for (int e = 0; e < 4; ++e) {
              const float2 f2 = __bfloat1622float2(h2[e]);
              acc8[2 * e] += f2.x;
              acc8[2 * e + 1] += f2.y;
            }
          }
        }
      }
      asm volatile("bar.sync 1, 128;" ::: "memory");
      if (et == 0) mbar_arrive(&empty_bar[s]);
      if (++s == kWgStages) { s = 0; ph ^= 1; }
    }
    if (grp < NG) {
#pragma unroll
      for (int e = 0; e < 8; ++e) sdb[grp][j * 8 + e] = acc8[e];
    }
    asm volatile("bar.sync 1, 128;" ::: "memory");
    if (et < COUTP) {
      float t = 0.f;
      for (int p2 = 0; p2 < NG; ++p2) t += sdb[p2][et];
      o.ws[(size_t)blockIdx.x * STRIDE + PER + et] = t;
    }
    // drain: lane m of M-tile mt = atom a = 8 mt + m / 16 -> (dy, cb) = (a / CB, a % CB), ci = 16 cb + m % 16
    mbar_wait(&done_bar, 0);
    if (dbg && et == 0) dbg[5] = globaltimer();
    tc_fence_after();
    const int quarter = warp & 3;
    const int m = quarter * 32 + lane_id();
    float* outp = o.ws + (size_t)blockIdx.x * STRIDE;
#pragma unroll
    for (int dx = 0; dx < 3; ++dx) {
#pragma unroll
      for (int mt = 0; mt < NMT; ++mt) {
        const int a = 8 * mt + m / 16;
        const bool ok = a < 3 * CB;
        const int dy = a / CB, cb = a % CB;
        const int ci = 16 * cb + (m % 16);
        float v[COUTP];  // all columns of this accumulator row: one TMEM round trip
#pragma unroll
        for (int c0 = 0; c0 < COUTP; c0 += 16)
          tmem_ld16(tmem + ((uint32_t)(quarter * 32) << 16) + (dx * NMT + mt) * COUTP + c0, v + c0);
        tmem_ld_wait();
        if (ok) {  // COUTP consecutive floats: 16-byte stores
          float4* dst = reinterpret_cast<float4*>(outp + ((size_t)(dy * 3 + dx) * CINP + ci) * COUTP);
#pragma unroll
          for (int q = 0; q < COUTP / 4; ++q) dst[q] = make_float4(v[4 * q], v[4 * q + 1], v[4 * q + 2], v[4 * q + 3]);
        }
      }
    }
    if (dbg && et == 0) { dbg[6] = globaltimer(); dbg[4] = clock64(); }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 1) tmem_dealloc<TMEM_COLS>(tmem);
  // ---- grid barrier: every partial written
  if (threadIdx.x == 0) {
    volatile unsigned* vgen = o.sync + 1;
    const unsigned gen = *vgen;
    __threadfence();
    const unsigned arrived = atomicAdd(o.sync, 1u);
    if (arrived == gridDim.x - 1) {
      atomicExch(o.sync, 0u);
      __threadfence();
      atomicAdd(o.sync + 1, 1u);
    } else {
      while (*vgen == gen) {
      }
    }
    __threadfence();
  }
  __syncthreads();
  pdl_trigger();
  if (dbg && threadIdx.x == 0) dbg[7] = globaltimer();
  // ---- deterministic split-K reduction of this CTA's slice [lo, hi) of float4 outputs over all partials, in
  // chunks of LC outputs: thread t sums partials q, q + NQ, ... (q = t / LC) of output t % LC, then the NQ group
  // sums are added in order q = 0..NQ-1.
  {
    constexpr int TOT4 = STRIDE / 4;
    const int G = gridDim.x;
    const int lo = (int)((long long)blockIdx.x * TOT4 / G), hi = (int)((long long)(blockIdx.x + 1) * TOT4 / G);
    float4* red = reinterpret_cast<float4*>(smem);  // stage buffers are free now
    const int t = threadIdx.x;
    for (int c0 = lo; c0 < hi; c0 += 48) {
      const int LC = min(48, hi - c0);
      const int NQ = min(32, kWgradThreads / LC);
      const int oi = t % LC, q = t / LC;
      if (q < NQ) {
        const float4* src = reinterpret_cast<const float4*>(o.ws) + c0 + oi;
        float4 acc4 = make_float4(0.f, 0.f, 0.f, 0.f);
        for (int p = q; p < G; p += 16 * NQ) {  // 16 independent (predicated) loads in flight, added in order
          float4 w4[16];
#pragma unroll
          for (int k = 0; k < 16; ++k)
            w4[k] = p + k * NQ < G ? __ldcg(src + (size_t)(p + k * NQ) * TOT4) : make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll
          for (int k = 0; k < 16; ++k) { acc4.x += w4[k].x; acc4.y += w4[k].y; acc4.z += w4[k].z; acc4.w += w4[k].w; }
        }
        red[q * LC + oi] = acc4;
      }
      __syncthreads();
      if (t < LC) {
        float4 s4 = red[t];
        for (int qq = 1; qq < NQ; ++qq) {
          const float4 w4 = red[qq * LC + t];
          s4.x += w4.x; s4.y += w4.y; s4.z += w4.z; s4.w += w4.w;
        }
        const float sv[4] = {s4.x, s4.y, s4.z, s4.w};
#pragma unroll
        for (int e = 0; e < 4; ++e) {
          const int i = 4 * (c0 + t) + e;
          if (i < PER) {  // partial index [tap][ci][co]
            const int co = i % COUTP, rest = i / COUTP;
            const int ci = rest % CINP, tap = rest / CINP;
            if (co < o.cout && ci < o.cin) o.gW[(co * o.cin + ci) * 9 + tap] = sv[e] * o.scale;
          } else {
            const int co = i - PER;
            if (co < o.cout) o.gb[co] = sv[e] * o.scale;
          }
        }
      }
      __syncthreads();
    }
  }
}

template <int CINP, int COUTP>
static cudaError_t launch_wgrad_t(const CUtensorMap& tx, const CUtensorMap& ty, const WgradGeom& g,
                                  const WgradOut& o, size_t smem, int grid, cudaStream_t st) {
  auto kern = k_wgrad<CINP, COUTP>;
  static size_t configured = 0;
  if (smem > configured) {
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    configured = smem;
  }
  return launch_coop(kern, dim3(grid), dim3(kWgradThreads), smem, st, tx, ty, g, o);
}

#define SR_WG_CASE(CI, CO) \
  if (cinp == CI && coutp == CO) return launch_wgrad_t<CI, CO>(tx, ty, g, o, smem, grid, st);

cudaError_t launch_wgrad(int cinp, int coutp, const bf16* x, const bf16* dy, const WgradGeom& g, const WgradOut& o,
                         size_t smem, int grid, cudaStream_t st) {
  CUtensorMap tx, ty;
  if (make_act_tmap_sw32(&tx, x, g.N, g.H, g.W, cinp, g.P, g.R + 2) != CUDA_SUCCESS) return cudaErrorInvalidValue;
  if (make_act_tmap_sw32(&ty, dy, g.N, g.H, g.W, coutp, g.TW, g.R) != CUDA_SUCCESS) return cudaErrorInvalidValue;
  SR_WG_CASE(16, 16) SR_WG_CASE(16, 32) SR_WG_CASE(16, 48) SR_WG_CASE(16, 64)
  SR_WG_CASE(32, 16) SR_WG_CASE(32, 32) SR_WG_CASE(32, 48) SR_WG_CASE(32, 64)
  SR_WG_CASE(48, 16) SR_WG_CASE(48, 32) SR_WG_CASE(48, 48)
  SR_WG_CASE(64, 16) SR_WG_CASE(64, 32) SR_WG_CASE(64, 64) SR_WG_CASE(64, 48)
  return cudaErrorNotSupported;
}

// ------------------------------------------------------------------------------------------ bilinear only
// SR_BILINEAR "model" (the WebRTC baseline): the tail with y = 0.
template <int S>
__global__ void k_bilinear_u8(const uint8_t* __restrict__ lr, int n, int h, int w, uint8_t* __restrict__ hr) {
  pdl_enter();
  const long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= (long long)n * h * w) return;
  const int X = (int)(i % w);
  const long long r = i / w;
  const int Y = (int)(r % h), img = (int)(r / h);
  EpiParams ep{};
  ep.lr = lr;
  ep.hr = hr;
  constexpr int CO = S == 4 ? 48 : 32;
  float v[CO];
#pragma unroll
  for (int k = 0; k < CO; ++k) v[k] = 0.f;
  const float zb[CO] = {0.f};
  float ls = 0.f;
  epi_tail<S, CO, false>(ep, zb, img, Y, X, h, w, v, ls, 0);
}

cudaError_t launch_bilinear_u8(const uint8_t* lr, int n, int h, int w, int s, uint8_t* hr, cudaStream_t st) {
  long long tot = (long long)n * h * w;
  unsigned blocks = (unsigned)((tot + 255) / 256);
  if (s == 2) return launch_k(k_bilinear_u8<2>, dim3(blocks), dim3(256), 0, st, lr, n, h, w, hr);
  if (s == 3) return launch_k(k_bilinear_u8<3>, dim3(blocks), dim3(256), 0, st, lr, n, h, w, hr);
  if (s == 4) return launch_k(k_bilinear_u8<4>, dim3(blocks), dim3(256), 0, st, lr, n, h, w, hr);
  return cudaErrorNotSupported;
}

}  // namespace sr

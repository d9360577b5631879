// Forward 3x3 conv for wide frames, "rolling dy-fold" form (sm_100a tcgen05).
//
// Why: with N = Cout = 32/48 a tcgen05.mma (M=128, K=16, both operands in smem) is limited by the 128 B/clk
// shared-memory read port: A (4 KB) + B (1.5 KB) per MMA -> 44.6 cycles instead of the 24-cycle tensor floor
// (measured, scripts/mma_rate.py).  Folding the three vertical taps into N (N = 3 Cout = 144 at C = 48) keeps
// A traffic the same while tripling the work per MMA: 72 cycles at the floor, 121 B/clk of smem.
//
//   For every input row i of a column strip (one 128-pixel segment + 1-pixel halo, TMA-loaded once):
//     E_i[x, (dy, co)] = sum_{dx, ci} in[i, x + dx - 1, ci] * W[co, ci, dy, dx]      (3 dx x Cin/16 MMAs, N = 3 Cout)
//   and the output row r needs the dy-blocks of three consecutive E at the SAME lane x:
//     out[r, x, co] = E_{r-1}[x, (0, co)] + E_r[x, (1, co)] + E_{r+1}[x, (2, co)]   (+ bias, + residual, ReLU)
//   (out[y,x] = b + sum_{ky,kx,ci} W[co,ci,ky,kx] in[y+ky-1, x+kx-1, ci]: with i = y + ky - 1, ky = dy.)
//   The epilogue keeps the two partial output rows in registers, so every E_i is drained once and its TMEM
//   slot recycled immediately.  Each CTA takes a contiguous range of (column strip, row) work so all CTAs get
//   the same number of rows; input rows are read once per strip piece (+2 halo rows per piece).
//
// Warp roles (320 threads): warp 0 TMA producer (input rows, residual rows), warp 1 TMEM alloc + MMA issuer,
// warps 2..9 epilogue (group g = channels [g*Cout/2, (g+1)*Cout/2)); output rows leave through smem + TMA store.
#include <cuda.h>
#include "ptx.cuh"
#include "tmap.h"
#include "sr_internal.h"

namespace sr {

static constexpr int kRollThreads = 320;
static constexpr int kRollIn = 6;    // input-row ring slots
static constexpr int kRollRes = 4;   // residual-row ring slots
static constexpr int kRollTW = 128;  // output pixels per strip (= MMA M)

template <int COUTP>
struct RollCfg {
  static constexpr int N = 3 * COUTP;
  static constexpr int ESTRIDE = ((N + 31) / 32) * 32;
  static constexpr int NE = (512 / ESTRIDE) < 4 ? (512 / ESTRIDE) : 4;
  static constexpr uint32_t TMEM_COLS = 512;
  static constexpr int HALF = COUTP / 2;
};

size_t roll_smem(int cinp, int coutp) {
  size_t w = (size_t)9 * cinp * coutp * 2;
  size_t in = ((size_t)(cinp / 8) * (kRollTW + 2) * 16 + 1023) / 1024 * 1024;
  size_t row = ((size_t)kRollTW * coutp * 2 + 1023) / 1024 * 1024;
  return 1024 + ((w + 1023) / 1024 * 1024) + kRollIn * in + kRollRes * row + 3 * row;
}

template <int HALF>
__device__ __forceinline__ void tmem_ld_half(uint32_t taddr, float* v) {
  static_assert(HALF % 8 == 0, "channel half must be a multiple of 8");
  int c = 0;
#pragma unroll
  for (; c + 16 <= HALF; c += 16) tmem_ld16(taddr + c, v + c);
  if (HALF % 16) tmem_ld8(taddr + c, v + c);
}

template <int CINP, int COUTP>
__global__ void __launch_bounds__(kRollThreads, 1)
k_conv_roll(const __grid_constant__ CUtensorMap tm_in, const __grid_constant__ CUtensorMap tm_res,
            const __grid_constant__ CUtensorMap tm_out, const bf16* __restrict__ wfold, const int N, const int H,
            const int W, const float* __restrict__ bias, const int relu, const int has_res) {
  using Cfg = RollCfg<COUTP>;
  constexpr int CCH = CINP / 8, KS = CINP / 16, HALF = Cfg::HALF, NE = Cfg::NE, ESTRIDE = Cfg::ESTRIDE;
  constexpr uint32_t WBYTES = 9u * CINP * COUTP * 2u;
  constexpr uint32_t PLANE = (kRollTW + 2) * 16;                  // one 8-channel chunk of an input row
  constexpr uint32_t IN_BOX = CCH * PLANE;
  constexpr uint32_t IN_STRIDE = (IN_BOX + 1023u) & ~1023u;
  constexpr uint32_t ROW_BOX = kRollTW * COUTP * 2;
  constexpr uint32_t ROW_STRIDE = (ROW_BOX + 1023u) & ~1023u;
  constexpr uint32_t IDESC = make_idesc(128, Cfg::N, 0, 0);

  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sW = smem;
  uint8_t* sIn = sW + ((WBYTES + 1023u) & ~1023u);
  uint8_t* sRes = sIn + kRollIn * IN_STRIDE;
  uint8_t* sOut = sRes + kRollRes * ROW_STRIDE;  // 3 x [128 px][COUTP] staging rows for the TMA store
  __shared__ __align__(8) uint64_t in_full[kRollIn], in_empty[kRollIn], res_full[kRollRes], res_empty[kRollRes],
      e_full[NE], e_empty[NE], w_bar;
  __shared__ uint32_t tmem_base_sh;

  const int warp = warp_id();
  if (warp == 0 && lane_id() == 0) {
    for (int s = 0; s < kRollIn; ++s) { mbar_init(&in_full[s], 1); mbar_init(&in_empty[s], 1); }
    for (int s = 0; s < kRollRes; ++s) { mbar_init(&res_full[s], 1); mbar_init(&res_empty[s], 8); }
    for (int s = 0; s < NE; ++s) { mbar_init(&e_full[s], 1); mbar_init(&e_empty[s], 8); }
    mbar_init(&w_bar, 1);
    fence_barrier_init();
  }
  if (warp == 1) tmem_alloc<Cfg::TMEM_COLS>(&tmem_base_sh);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = tmem_base_sh;

  // balanced contiguous range of (column strip, row) work for this CTA
  const int tiles_x = (W + kRollTW - 1) / kRollTW;
  const long long total = (long long)N * tiles_x * H;
  const long long beg = total * blockIdx.x / gridDim.x, end = total * (blockIdx.x + 1) / gridDim.x;

  if (warp == 0) {
    // ===================== TMA producer =====================
    if (elect_one()) {
      tma_prefetch_desc(&tm_in);
      if (has_res) tma_prefetch_desc(&tm_res);
      mbar_arrive_expect_tx(&w_bar, WBYTES);
      bulk_load(sW, wfold, WBYTES, &w_bar);
      int s = 0, rs = 0;
      uint32_t ph = 0, rph = 0;
      for (long long pos = beg; pos < end;) {
        const int col = (int)(pos / H), y0 = (int)(pos - (long long)col * H);
        const int y1 = (int)min((long long)H, y0 + (end - pos));
        pos += y1 - y0;
        const int n = col / tiles_x, x0 = (col - n * tiles_x) * kRollTW;
        const int n_in = y1 - y0 + 2;
        for (int i = 0; i < n_in; ++i) {
          mbar_wait(&in_empty[s], ph ^ 1);
          mbar_arrive_expect_tx(&in_full[s], IN_BOX);
          tma_load_5d(sIn + s * IN_STRIDE, &tm_in, &in_full[s], 0, x0 - 1, y0 - 1 + i, 0, n);
          if (++s == kRollIn) { s = 0; ph ^= 1; }
          if (has_res && i >= 1 && i - 1 < y1 - y0) {  // residual of output row y0+i-1, consumed at step i+1
            mbar_wait(&res_empty[rs], rph ^ 1);
            mbar_arrive_expect_tx(&res_full[rs], ROW_BOX);
            tma_load_4d(sRes + rs * ROW_STRIDE, &tm_res, &res_full[rs], 0, x0, y0 + i - 1, n);
            if (++rs == kRollRes) { rs = 0; rph ^= 1; }
          }
        }
      }
    }
    __syncwarp();
  } else if (warp == 1) {
    // ===================== MMA issuer =====================
    if (elect_one()) {
      mbar_wait(&w_bar, 0);
      const uint64_t bdesc0 = make_desc(smem_u32(sW), Cfg::N * 16, 128);
      int s = 0, es = 0;
      uint32_t ph = 0, eph = 0;
      for (long long pos = beg; pos < end;) {
        const int col = (int)(pos / H), y0 = (int)(pos - (long long)col * H);
        const int y1 = (int)min((long long)H, y0 + (end - pos));
        pos += y1 - y0;
        (void)col;
        const int n_in = y1 - y0 + 2;
        for (int i = 0; i < n_in; ++i) {
          mbar_wait(&in_full[s], ph);
          mbar_wait(&e_empty[es], eph ^ 1);
          tc_fence_after();
          const uint64_t adesc0 = make_desc(smem_u32(sIn + s * IN_STRIDE), PLANE, 128);
          const uint32_t d = tmem + es * ESTRIDE;
#pragma unroll
          for (int dx = 0; dx < 3; ++dx) {
#pragma unroll
            for (int ks = 0; ks < KS; ++ks) {
              mma_bf16_ss(d, desc_add(adesc0, dx * 16u + ks * 2u * PLANE),
                          desc_add(bdesc0, (uint32_t)(dx * CCH + 2 * ks) * Cfg::N * 16u), IDESC, (dx | ks) != 0);
            }
          }
          mma_commit(&e_full[es]);
          mma_commit(&in_empty[s]);
          if (++s == kRollIn) { s = 0; ph ^= 1; }
          if (++es == NE) { es = 0; eph ^= 1; }
        }
      }
    }
    __syncwarp();
  } else {
    // ===================== epilogue: 2 groups x 4 warps, group g owns channels [g*HALF, (g+1)*HALF) ==========
    const int quarter = warp & 3;
    const int grp = (warp - 2) >> 2;
    const int px = quarter * 32 + lane_id();
    const int c0 = grp * HALF;
    const bool leader = (warp == 2 && lane_id() == 0);
    float bv[HALF];
#pragma unroll
    for (int c = 0; c < HALF; ++c) bv[c] = bias ? __ldg(bias + c0 + c) : 0.f;
    int es = 0, rs = 0, os = 0;
    uint32_t eph = 0, rph = 0;
    float pa[HALF], pb[HALF];  // partial sums of output rows i-1 and i (relative to input row i)
    for (long long pos = beg; pos < end;) {
      const int col = (int)(pos / H), y0 = (int)(pos - (long long)col * H);
      const int y1 = (int)min((long long)H, y0 + (end - pos));
      pos += y1 - y0;
      const int n = col / tiles_x, x0 = (col - n * tiles_x) * kRollTW;
      const int n_in = y1 - y0 + 2;
      for (int i = 0; i < n_in; ++i) {
        float e0[HALF], e1[HALF], e2[HALF];
        mbar_wait(&e_full[es], eph);
        tc_fence_after();
        const uint32_t ta = tmem + ((uint32_t)(quarter * 32) << 16) + es * ESTRIDE + c0;
        tmem_ld_half<HALF>(ta, e0);
        tmem_ld_half<HALF>(ta + COUTP, e1);
        tmem_ld_half<HALF>(ta + 2 * COUTP, e2);
        tmem_ld_wait();
        tc_fence_before();
        __syncwarp();
        if (lane_id() == 0) mbar_arrive(&e_empty[es]);
        if (++es == NE) { es = 0; eph ^= 1; }
        if (i >= 2) {
          // output row r = y0 + i - 2 is complete: pa + E_i dy=2 block
          const int r = y0 + i - 2;
          float v[HALF];
#pragma unroll
          for (int c = 0; c < HALF; ++c) v[c] = pa[c] + e2[c] + bv[c];
          if (has_res) {
            mbar_wait(&res_full[rs], rph);
            const uint4* rr = reinterpret_cast<const uint4*>(sRes + rs * ROW_STRIDE + (px * COUTP + c0) * 2);
#pragma unroll
            for (int q = 0; q < HALF / 8; ++q) {
              uint4 u = rr[q];
              const __nv_bfloat162* h2 = reinterpret_cast<const __nv_bfloat162*>(&u);
#pragma unroll
              for (int j = 0; j < 4; ++j) {
                float2 f = __bfloat1622float2(h2[j]);
                v[8 * q + 2 * j] += f.x;
                v[8 * q + 2 * j + 1] += f.y;
              }
            }
            __syncwarp();
            if (lane_id() == 0) mbar_arrive(&res_empty[rs]);
            if (++rs == kRollRes) { rs = 0; rph ^= 1; }
          }
          if (relu) {
#pragma unroll
            for (int c = 0; c < HALF; ++c) v[c] = fmaxf(v[c], 0.f);
          }
          // stage the row in smem (3 buffers), one barrier, one thread TMA-stores it (clipped at the frame edge).
          // Buffer k%3 was last read by the store of row k-3, which the leader waited for (wait_read<1> after
          // issuing row k-2's store) before it reached the barrier of row k-1.
          uint4* orow = reinterpret_cast<uint4*>(sOut + os * ROW_STRIDE + (px * COUTP + c0) * 2);
#pragma unroll
          for (int q = 0; q < HALF / 8; ++q) {
            uint4 u;
            u.x = pack_bf16x2(v[8 * q + 0], v[8 * q + 1]);
            u.y = pack_bf16x2(v[8 * q + 2], v[8 * q + 3]);
            u.z = pack_bf16x2(v[8 * q + 4], v[8 * q + 5]);
            u.w = pack_bf16x2(v[8 * q + 6], v[8 * q + 7]);
            orow[q] = u;
          }
          fence_proxy_async_smem();
          named_bar_sync(1, 256);
          if (leader) {
            tma_store_4d(&tm_out, sOut + os * ROW_STRIDE, 0, x0, r, n);
            bulk_commit();
            bulk_wait_read<1>();
          }
          os = os == 2 ? 0 : os + 1;
        }
#pragma unroll
        for (int c = 0; c < HALF; ++c) {
          pa[c] = pb[c] + e1[c];
          pb[c] = e0[c];
        }
      }
    }
    if (leader) bulk_wait<0>();
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 1) tmem_dealloc<RollCfg<COUTP>::TMEM_COLS>(tmem);
}

template <int CINP, int COUTP>
static cudaError_t launch_roll_t(const CUtensorMap& ti, const CUtensorMap& tr, const CUtensorMap& to,
                                 const bf16* wfold, int N, int H, int W, const float* bias, int relu, int has_res,
                                 int grid, cudaStream_t st) {
  auto kern = k_conv_roll<CINP, COUTP>;
  const size_t smem = roll_smem(CINP, COUTP);
  static bool configured = false;
  if (!configured) {
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    configured = true;
  }
  kern<<<grid, kRollThreads, smem, st>>>(ti, tr, to, wfold, N, H, W, bias, relu, has_res);
  return cudaGetLastError();
}

bool roll_supported(int cinp, int coutp, int W) {
  if (W < 96) return false;
  const bool ci = cinp == 16 || cinp == 32 || cinp == 48 || cinp == 64;
  const bool co = coutp == 16 || coutp == 32 || coutp == 48 || coutp == 64;
  return ci && co && roll_smem(cinp, coutp) <= 227 * 1024;
}

#define SR_ROLL_CASE(CI, CO) \
  if (cinp == CI && coutp == CO) return launch_roll_t<CI, CO>(ti, tr, to, wfold, N, H, W, bias, relu, has_res, grid, st);

cudaError_t launch_conv_roll(int cinp, int coutp, const void* in, const bf16* wfold, const float* bias,
                             const bf16* res, int relu, bf16* out, int N, int H, int W, cudaStream_t st) {
  CUtensorMap ti, tr, to;
  if (make_act_tmap(&ti, in, N, H, W, cinp, kRollTW + 2, 1, cinp / 8, CHUNK_ROW_PIX) != CUDA_SUCCESS)
    return cudaErrorInvalidValue;
  if (make_row_tmap(&to, out, N, H, W, coutp, kRollTW, coutp) != CUDA_SUCCESS) return cudaErrorInvalidValue;
  if (make_row_tmap(&tr, res ? (const void*)res : (const void*)out, N, H, W, coutp, kRollTW, coutp) != CUDA_SUCCESS)
    return cudaErrorInvalidValue;
  const int has_res = res != nullptr;
  const long long rows = (long long)N * ((W + kRollTW - 1) / kRollTW) * H;
  int grid = num_sms();
  if (rows < grid) grid = (int)rows;
  SR_ROLL_CASE(16, 16) SR_ROLL_CASE(16, 32) SR_ROLL_CASE(16, 48) SR_ROLL_CASE(16, 64)
  SR_ROLL_CASE(32, 16) SR_ROLL_CASE(32, 32) SR_ROLL_CASE(32, 48) SR_ROLL_CASE(32, 64)
  SR_ROLL_CASE(48, 16) SR_ROLL_CASE(48, 32) SR_ROLL_CASE(48, 48)
  SR_ROLL_CASE(64, 16) SR_ROLL_CASE(64, 32) SR_ROLL_CASE(64, 64)
  return cudaErrorNotSupported;
}

}  // namespace sr

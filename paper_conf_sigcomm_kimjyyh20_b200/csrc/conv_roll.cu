// One 3x3 conv over wide images, rolling dy-fold form with tensor-core accumulation in a TMEM ring (sm_100a).
//
// Why: with N = Cout = 32/48 a tcgen05.mma (M=128, K=16, operands in smem) is limited by the 128 B/clk
// shared-memory read port: A (4 KB) + B (1.5 KB) per MMA -> 44.6 cycles instead of the 24-cycle tensor floor
// (measured, scripts/mma_rate.py).  Folding the three vertical taps into N (N = 3 Cout) keeps A traffic the same
// while tripling the work per MMA (72 cycles at the floor for N = 144).  The three dy partials of an output row are
// summed by the tensor core itself: each output row owns a bias-armed block of a TMEM ring (ring.cuh).
//
//   out[y, x, co] = b[co] + sum_{ky,kx,ci} W[co,ci,ky,kx] in[y+ky-1, x+kx-1, ci]            (zero padding)
//   step for input row i:  block(i+1) += in_i (x) Wo[dy=0],  block(i) += .. [dy=1],  block(i-1) += .. [dy=2]
//
// Epilogue (per finished row): optional ReLU, + res1 + res2, x 1[mask > 0] (ReLU' for the data gradient), and
// zero-forced "separator" columns (col % sep in {0, sep-1}) for the virtual wide training batch.
// Each CTA takes a contiguous range of (column strip, row) work (equal rows per CTA); input rows are read once
// per strip piece (+2 halo rows per piece).  Strips are 128 output pixels (= MMA M).
//
// Warp roles (384 threads): warp 0 TMA producer of the input rows, warp 1 TMEM alloc + MMA issuer, warps 2..9
// epilogue in two groups of 4 that take alternate output rows (all channels) and hand finished rows to warp 10,
// which issues the TMA stores; warp 11 issues the aux-row (residual / mask) and tail LR-row TMAs on its own, so
// waiting for an aux slot the epilogue has not released yet never holds back the input rows the MMAs need.  The per-row epilogue chain (drain, re-arm, residual, stage) is latency-bound: two rows in flight and no
// barrier or store wait on it.
#include <cuda.h>
#include "ptx.cuh"
#include "ring.cuh"
#include "tmap.h"
#include "sr_internal.h"
#include "kernels.h"
#include "launch.cuh"
#include "tail.cuh"
#include "color.cuh"
#include <algorithm>
#include <vector>

namespace sr {

static constexpr int kRollThreads = 384;  // warp 10: TMA-store warp, warp 11: aux / LR-row TMA producer
static constexpr int kRollNO = 3;    // output staging rows per epilogue group
static constexpr int kRollTW = 128;  // output pixels per strip (= MMA M)

static constexpr int kTailLrChunks = 26;  // 416 B: LR pixels x0-5 .. x0+133 of a 128-pixel strip
static constexpr uint32_t kTailLrSlot = (16 * kTailLrChunks * 5 + 127) & ~127u;  // 5 LR rows per slot
// LR-row ring depth of the staged tail (in the aux area, unused by the tail): deep enough that the producer, which
// runs up to NIN + RB rows ahead of the epilogue, never waits on it (a shallow ring stalls the input rows)

template <int CINP, int COUTP>
struct RollCfg {
  static constexpr int RB = (512 / COUTP) < 8 ? (512 / COUTP) : 8;
  static constexpr uint32_t WBYTES = 9u * CINP * COUTP * 2u;
  static constexpr uint32_t WB_AL = (WBYTES + 1023u) & ~1023u;
  static constexpr uint32_t PLANE = (kRollTW + 2) * 16;
  static constexpr uint32_t IN_BOX = (CINP / 8) * PLANE;
  static constexpr uint32_t IN_STRIDE = (IN_BOX + 127u) & ~127u;  // TMA destination: 128-B aligned
  static constexpr uint32_t ROWB = ((kRollTW * COUTP * 2) + 1023u) & ~1023u;
  static constexpr int NAUX = 4;  // residual / mask rows (TMA)
  static constexpr int NLR = (int)((NAUX * ROWB) / kTailLrSlot) < 16 ? (int)((NAUX * ROWB) / kTailLrSlot) : 16;
  static constexpr uint32_t ARMB = ((kArmOnesBytes + COUTP * 32) + 127u) & ~127u;  // bias-arming MMA operands
  static constexpr size_t BASE = 1024 + WB_AL + (size_t)2 * kRollNO * ROWB + (size_t)NAUX * ROWB + ARMB;
  // input-row ring slots: as many as fit (up to 8) -- the TMA loads in flight per SM are what keeps HBM busy
  static constexpr int NIN_FIT = (int)((227 * 1024 - BASE) / IN_STRIDE);
  static constexpr int NIN = NIN_FIT > 8 ? 8 : NIN_FIT;
  static constexpr bool FITS = NIN >= 3;  // else not offered (roll_supported)
  static constexpr size_t SMEM = BASE + (size_t)NIN * IN_STRIDE;
};

struct RollArgs {
  const float* bias;
  const bf16* res1;
  const bf16* res2;
  const bf16* mask;
  int relu;
  int sep;  // > 0: output columns with col % sep in {0, sep-1} are forced to 0
  int N, H, W;
  long long* dbg;  // benchmarking only: CTA-0 clock64 stamps [event][step]
  // tail mode (TS > 0, the up conv): pixel shuffle + skip + clamp + RNE u8 straight from the epilogue
  const uint8_t* lr;  // [N,H,W,3] LR frames (skip input)
  uint8_t* hr;        // [N,TS H,TS W,3]
  int hr_row0, hr_row1;  // LR rows whose HR rows are written (strip mode)
  int bicubic;
  // tail_tma: LR neighbourhood rows arrive by TMA (tm_aux, make_u8_rows_tmap, box kTailLrChunks x 5 rows) and the
  // S HR rows of every LR row are staged in smem and leave by one TMA store (tm_out); needs W % 16 == 0.
  // Otherwise every lane reads its 3x3 (5x5) LR neighbourhood and writes its S x S x 3 bytes from/to global.
  int tail_tma;
  int w_early;  // weights / bias may be fetched before the PDL wait (see the kernel prologue)
  // training tail (TS > 0, train = 1): o = PS(y) + skip/255 against hr_ref, loss += (o - t)^2 (L1: |o - t|) into
  // *loss_sum, dy = 2 (o - t) (L1: sign) as a bf16 row per pixel; vsep > 0: virtual batch of vp x vp patches at
  // columns [j vsep + 1, j vsep + 1 + vp), separator columns get dy = 0 and no loss
  int train;
  const uint8_t* hr_ref;
  bf16* dy;
  double* loss_sum;
  int vsep, vp, l1;
  // YUV head (U8 && YUV): the input is an I420 frame -- tm_in maps the Y plane's rows, U / V ([N][H/2][W/2]) are read
  // directly; the expansion warps convert with the library's BT.601 integer conversion (color.cuh) and also write
  // the frame's RGB u8 copy (rgb_out [N][H][W][3], each strip's own pixels and rows) for the tail's skip
  const uint8_t* yuv_u;
  const uint8_t* yuv_v;
  uint8_t* rgb_out;
};
#define SR_RDBG(ev, idx) \
  if (DBG && a.dbg && blockIdx.x == 0 && (idx) >= 0 && (idx) < 256) a.dbg[(ev) * 256 + (idx)] = clock64();

template <int CH>
__device__ __forceinline__ void ld_row(const bf16* base, uint4* dst) {
  const uint4* p = reinterpret_cast<const uint4*>(base);
#pragma unroll
  for (int q = 0; q < CH / 8; ++q) dst[q] = __ldg(p + q);
}

// One output row of one lane into the staging row: v (bias included) + res1 (aux row) + res2 -> ReLU -> x 1[mask > 0]
// (aux row) -> 0 in separator columns -> bf16.  M: variant bits (1 res1, 2 res2, 4 mask, 8 separators, 16 ReLU);
// M = 32: generic body, the variant is read from em at run time.
template <int COUTP, int M>
__device__ __forceinline__ void roll_stage(uint4* __restrict__ orow, const float* v, const uint4* __restrict__ aux_s,
                                           const uint4* r2, bool sep0, int em) {
  const int mm = (M & 32) ? em : M;
  // the whole aux row (residual or mask) into registers first: the staging stores below could alias it for the
  // compiler, which would otherwise serialise every 16-B load behind the previous chunk's store
  uint4 aux[COUTP / 8];
  if (mm & 5) {
#pragma unroll
    for (int j = 0; j < COUTP / 8; ++j) aux[j] = aux_s[j];
  }
#pragma unroll
  for (int j = 0; j < COUTP / 8; ++j) {
    float o[8];
#pragma unroll
    for (int e = 0; e < 8; ++e) o[e] = v[8 * j + e];
    if (mm & 1) {
      const uint4 t = aux[j];
      const __nv_bfloat162* h = reinterpret_cast<const __nv_bfloat162*>(&t);
#pragma unroll
      for (int e = 0; e < 4; ++e) { const float2 f = __bfloat1622float2(h[e]); o[2 * e] += f.x; o[2 * e + 1] += f.y; }
    }
    if (mm & 2) {
      const __nv_bfloat162* h = reinterpret_cast<const __nv_bfloat162*>(&r2[j]);
#pragma unroll
      for (int e = 0; e < 4; ++e) { const float2 f = __bfloat1622float2(h[e]); o[2 * e] += f.x; o[2 * e + 1] += f.y; }
    }
    if (mm & 16) {
#pragma unroll
      for (int e = 0; e < 8; ++e) o[e] = fmaxf(o[e], 0.f);
    }
    if (mm & 4) {
      const uint4 t = aux[j];
      const __nv_bfloat162* h = reinterpret_cast<const __nv_bfloat162*>(&t);
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        const float2 f = __bfloat1622float2(h[e]);
        o[2 * e] = f.x > 0.f ? o[2 * e] : 0.f;
        o[2 * e + 1] = f.y > 0.f ? o[2 * e + 1] : 0.f;
      }
    }
    if ((mm & 8) && sep0) {
#pragma unroll
      for (int e = 0; e < 8; ++e) o[e] = 0.f;
    }
    uint4 u;
    u.x = pack_bf16x2(o[0], o[1]);
    u.y = pack_bf16x2(o[2], o[3]);
    u.z = pack_bf16x2(o[4], o[5]);
    u.w = pack_bf16x2(o[6], o[7]);
    orow[j] = u;
  }
}

// U8 (head conv only, CINP = 16): the input is the u8 RGB frame itself.  The producer TMA-loads u8 rows (16-B
// chunk map, W % 16 == 0) into a small ring in the aux area and warps 12, 13 expand each row into the bf16 A slot
// (x = v/255 in channels 0..2, exactly k_pack_input's arithmetic; channel chunk 1 is a zero plane written once),
// so k_pack_input's 32 B/px write and the head's 32 B/px read become a 3 B/px read.
static constexpr int kU8Slots = 8;
static constexpr uint32_t kU8Slot = 512;  // 26 chunks = 416 B per u8 row
// DBG: the instantiation with the CTA-0 clock64 stamps (benchmarking tools only; the production instantiations
// carry no stamp code -- each predicated stamp sits on a latency-bound epilogue chain)
static constexpr int kYuvChunks = 10;  // Y bytes [16 cb, 16 cb + 160) cover pixels x0-1 .. x0+128
template <int CINP, int COUTP, int TS, bool U8 = false, bool DBG = false, bool YUV = false>
__global__ void __launch_bounds__(kRollThreads + (U8 ? 64 : 0), 1)
k_conv_roll(const __grid_constant__ CUtensorMap tm_in, const __grid_constant__ CUtensorMap tm_out,
            const __grid_constant__ CUtensorMap tm_aux, const bf16* __restrict__ wfold, const RollArgs a) {
  using Cfg = RollCfg<CINP, COUTP>;
  constexpr int RB = Cfg::RB, kRollIn = Cfg::NIN, NAUX = Cfg::NAUX;
  constexpr uint32_t PLANE = Cfg::PLANE, IN_STRIDE = Cfg::IN_STRIDE, ROWB = Cfg::ROWB;

  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);  // stays in the shared window (LDS/STS, not generic)
  uint8_t* sW = smem;
  uint8_t* sIn = sW + Cfg::WB_AL;
  uint8_t* sO = sIn + kRollIn * IN_STRIDE;
  uint8_t* sA = sO + 2 * kRollNO * ROWB;
  uint8_t* sOnes = sA + NAUX * ROWB;  // ring.cuh: ones x bias MMA arms a ring block
  uint8_t* sBt = sOnes + kArmOnesBytes;
  __shared__ __align__(8) uint64_t in_full[kRollIn], in_empty[kRollIn], r_ready[RB], r_free[RB], x_full[NAUX],
      x_empty[NAUX], o_full[2 * kRollNO], o_free[2 * kRollNO], w_bar, arm_bar, l_full[TS > 0 ? Cfg::NLR : 1],
      l_empty[TS > 0 ? Cfg::NLR : 1], u_full[U8 ? kU8Slots : 1], u_empty[U8 ? kU8Slots : 1];
  // the aux row (res1 or mask) travels by TMA; res2 (used once per backward pass) by plain loads
  const bool has_aux = a.res1 != nullptr || a.mask != nullptr;
  __shared__ uint32_t tmem_base_sh;
  __shared__ __align__(16) float4 sbv[COUTP / 4];

  const int N = a.N, H = a.H, W = a.W;
  const int warp = warp_id();
  if (threadIdx.x == 0) { SR_RDBG(8, 0) }  // kernel entry
  if (warp == 0 && lane_id() == 0) {
    for (int s = 0; s < kRollIn; ++s) { mbar_init(&in_full[s], 1); mbar_init(&in_empty[s], 1); }
    for (int s = 0; s < RB; ++s) { mbar_init(&r_ready[s], 1); mbar_init(&r_free[s], 4); }
    for (int s = 0; s < NAUX; ++s) { mbar_init(&x_full[s], 1); mbar_init(&x_empty[s], 4); }
    if (TS > 0)
      for (int s = 0; s < Cfg::NLR; ++s) { mbar_init(&l_full[s], 1); mbar_init(&l_empty[s], 4); }
    for (int s = 0; s < 2 * kRollNO; ++s) { mbar_init(&o_full[s], 4); mbar_init(&o_free[s], 1); }
    if (U8)
      for (int s = 0; s < kU8Slots; ++s) { mbar_init(&u_full[s], 1); mbar_init(&u_empty[s], 1); }
    mbar_init(&w_bar, 1);
    mbar_init(&arm_bar, 1);
    fence_barrier_init();
  }
  if (warp == 1) tmem_alloc<512>(&tmem_base_sh);
  if constexpr (U8) {  // channel chunk 1 (channels 8..15) of every input slot stays zero
    static_assert(CINP == 16, "u8 input: head conv only");
    for (int i = threadIdx.x; i < kRollIn * (int)(PLANE / 16); i += blockDim.x)
      *reinterpret_cast<uint4*>(sIn + (i / (PLANE / 16)) * IN_STRIDE + PLANE + (i % (PLANE / 16)) * 16) =
          make_uint4(0u, 0u, 0u, 0u);
    fence_proxy_async_smem();
  }
  tc_fence_before();
  __syncthreads();
  // Weights and bias were written at least two kernels upstream when the caller sets w_early (every launch inside the
  // library's forward / backward chains: the kernel that packed them has completed before our predecessor passed its
  // own griddepcontrol.wait, i.e. before we were scheduled), so they are fetched before the PDL wait and the fetch
  // overlaps the predecessor's tail.  Everything the predecessor writes (activations) is read only after the wait.
  // The weights go by one bulk copy (producer thread); the bias and the ring-arming tiles are prepared by the epilogue
  // and store warps (2..10) alone and announced to the MMA issuer through arm_bar, so the producer's first input-row
  // TMAs are not queued behind the bias load and the tile fill.
  if (warp == 0 && lane_id() == 0 && a.w_early) {
    mbar_arrive_expect_tx(&w_bar, Cfg::WBYTES);
    bulk_load(sW, wfold, Cfg::WBYTES, &w_bar);
  }
  constexpr uint32_t kArmThreads = 9 * 32;  // warps 2..10
  // the arming MMAs take their ones operand from 8 spare TMEM columns after the ring when there are any (ring.cuh)
  constexpr bool kOnesTmem = RB * COUTP + 8 <= 512;
  auto arm_params = [&]() {
    const int t = (int)threadIdx.x - 64;
    if (t < COUTP) reinterpret_cast<float*>(sbv)[t] = a.bias ? a.bias[t] : 0.f;
    named_bar_sync(1, kArmThreads);
    arm_tiles_fill(sOnes, sBt, reinterpret_cast<const float*>(sbv), COUTP, t, kArmThreads);
    fence_proxy_async_smem();
    if constexpr (kOnesTmem) {
      if (warp >= 2 && warp <= 5) {  // the four TMEM lane quarters
        tc_fence_after();
        ones_tmem_fill(tmem_base_sh + ((uint32_t)((warp & 3) * 32) << 16) + RB * COUTP);
        tmem_st_wait();
        tc_fence_before();
      }
    }
    named_bar_sync(1, kArmThreads);
    if (t == 0) mbar_arrive(&arm_bar);
  };
  if (a.w_early && warp >= 2 && warp <= 10) arm_params();
  pdl_enter();  // predecessor complete: global inputs are valid from here on
  if (threadIdx.x == 0) { SR_RDBG(10, 0) }  // after setup + PDL wait
  if (!a.w_early) {
    if (warp == 0 && lane_id() == 0) {
      mbar_arrive_expect_tx(&w_bar, Cfg::WBYTES);
      bulk_load(sW, wfold, Cfg::WBYTES, &w_bar);
    }
    if (warp >= 2 && warp <= 10) arm_params();
  }
  tc_fence_after();
  const uint32_t tmem = tmem_base_sh;

  const int tiles_x = (W + kRollTW - 1) / kRollTW;
  const long long total = (long long)N * tiles_x * H;
  const long long beg = total * blockIdx.x / gridDim.x, end = total * (blockIdx.x + 1) / gridDim.x;
#define SR_PIECE_BEGIN                                                                \
  for (long long pos = beg; pos < end;) {                                             \
    const int col = (int)(pos / H), y0 = (int)(pos - (long long)col * H);             \
    const int y1 = (int)min((long long)H, y0 + (end - pos));                          \
    pos += y1 - y0;                                                                   \
    const int n = col / tiles_x, x0 = (col - n * tiles_x) * kRollTW;                  \
    const int n_in = y1 - y0 + 2;                                                     \
    (void)n; (void)x0; (void)n_in;
#define SR_PIECE_END }

  if (warp == 0) {
    // ===================== TMA producer: weights, then input rows y0-1 .. y1 of each piece =====================
    if (elect_one()) {
      tma_prefetch_desc(&tm_in);
      int s = 0, us = 0;
      uint32_t ph = 0, uph = 0;
      SR_PIECE_BEGIN
      for (int i = 0; i < n_in; ++i) {
        if constexpr (U8) {  // u8 row y0-1+i, pixels x0-1 .. x0+128 (+ chunk alignment), for warps 12, 13 to expand
          mbar_wait(&u_empty[us], uph ^ 1);
          if constexpr (YUV) {  // Y row y0-1+i, pixels x0-1 .. x0+128
            mbar_arrive_expect_tx(&u_full[us], 16 * kYuvChunks);
            tma_load_4d(sA + us * kU8Slot, &tm_in, &u_full[us], 0, (x0 - 1) >> 4, y0 - 1 + i, n);
          } else {
            mbar_arrive_expect_tx(&u_full[us], 16 * 26);
            tma_load_4d(sA + us * kU8Slot, &tm_in, &u_full[us], 0, (3 * x0 - 3) >> 4, y0 - 1 + i, n);
          }
          if (++us == kU8Slots) { us = 0; uph ^= 1; }
        } else {
          mbar_wait(&in_empty[s], ph ^ 1);
          mbar_arrive_expect_tx(&in_full[s], Cfg::IN_BOX);
          tma_load_5d(sIn + s * IN_STRIDE, &tm_in, &in_full[s], 0, x0 - 1, y0 - 1 + i, 0, n);
          if (++s == kRollIn) { s = 0; ph ^= 1; }
        }
        SR_RDBG(0, i)
      }
      SR_PIECE_END
    }
    __syncwarp();
  } else if (warp == 11) {
    // ===================== aux producer: residual / mask rows and the tail's LR neighbourhood rows =============
    if ((has_aux || (TS > 0 && a.tail_tma)) && elect_one()) {
      tma_prefetch_desc(&tm_aux);
      int xs = 0, ls = 0;
      uint32_t xph = 0, lph = 0;
      SR_PIECE_BEGIN
      for (int r = y0; r < y1; ++r) {  // output rows of the piece, in emission order
        if (TS > 0 && a.tail_tma) {  // LR rows r-2..r+2 of output row r
          mbar_wait(&l_empty[ls], lph ^ 1);
          mbar_arrive_expect_tx(&l_full[ls], 16 * kTailLrChunks * 5);
          tma_load_4d(sA + ls * kTailLrSlot, &tm_aux, &l_full[ls], 0, 3 * x0 / 16 - 1, r - 2, n);
          if (++ls == Cfg::NLR) { ls = 0; lph ^= 1; }
        }
        if (has_aux) {  // aux row of output row r
          mbar_wait(&x_empty[xs], xph ^ 1);
          mbar_arrive_expect_tx(&x_full[xs], kRollTW * COUTP * 2);
          tma_load_4d(sA + xs * ROWB, &tm_aux, &x_full[xs], 0, x0, r, n);
          if (++xs == NAUX) { xs = 0; xph ^= 1; }
        }
      }
      SR_PIECE_END
    }
    __syncwarp();
  } else if (warp == 1) {
    // ===================== MMA issuer =====================
    if (elect_one()) {
      mbar_wait(&w_bar, 0);
      mbar_wait(&arm_bar, 0);  // bias-arming tiles in place
      tc_fence_after();
      const uint64_t bd = make_desc(smem_u32(sW), 3 * COUTP * 16, 128);
      auto arm = [&](unsigned gg) {
        if constexpr (kOnesTmem) ring_arm_ts<COUTP, RB>(tmem, gg, tmem + RB * COUTP, smem_u32(sBt));
        else ring_arm<COUTP, RB>(tmem, gg, smem_u32(sOnes), smem_u32(sBt));
      };
      int s = 0;
      uint32_t ph = 0;
      unsigned G = 0, acq = 0;
      SR_PIECE_BEGIN
      for (int i = 0; i < n_in; ++i) {
        const unsigned g = G + i;  // out row completed by this step (dy = 2 target)
        SR_RDBG(1, i)
        for (; acq < g + 3; ++acq) mbar_wait(&r_free[ring_idx<RB>(acq)], (uint32_t)(acq / RB) & 1u);
        SR_RDBG(2, i)
        mbar_wait(&in_full[s], ph);
        SR_RDBG(3, i)
        tc_fence_after();
        if (i == 0) {  // the piece's first two rows receive no earlier contribution
          arm(g);
          arm(g + 1);
        }
        arm(g + 2);  // its first contribution comes now
        ring_mma_step<CINP, COUTP, RB>(tmem, g, make_desc(smem_u32(sIn + s * IN_STRIDE), PLANE, 128), bd, 2 * PLANE);
        mma_commit(&r_ready[ring_idx<RB>(g)]);
        mma_commit(&in_empty[s]);
        SR_RDBG(4, i)
        if (i == n_in - 1) {
          mma_commit(&r_ready[ring_idx<RB>(g + 1)]);
          mma_commit(&r_ready[ring_idx<RB>(g + 2)]);
        }
        if (++s == kRollIn) { s = 0; ph ^= 1; }
      }
      G += n_in + 2;
      SR_PIECE_END
    }
    __syncwarp();
  } else if (U8 && warp >= 12) {
    // ===================== u8 -> bf16 A-operand expansion (head conv): warps 12, 13 take alternate rows ==========
    int s = 0, us = 0;
    uint32_t ph = 0, uph = 0;
    long long rowc = 0;  // rows seen so far (both warps count every row; each converts its parity)
    SR_PIECE_BEGIN
    const int lbase = YUV ? 16 * ((x0 - 1) >> 4) : 16 * ((3 * x0 - 3) >> 4);
    for (int i = 0; i < n_in; ++i, ++rowc) {
      if ((int)(rowc & 1) != warp - 12) {
        if (++us == kU8Slots) { us = 0; uph ^= 1; }
        if (++s == kRollIn) { s = 0; ph ^= 1; }
        continue;
      }
      mbar_wait(&u_full[us], uph);
      mbar_wait(&in_empty[s], ph ^ 1);
      uint8_t* dst = sIn + s * IN_STRIDE;
      constexpr int kIt = (kRollTW + 2 + 31) / 32;
      float px[kIt][3];
      if constexpr (YUV) {  // I420 -> RGB (color.cuh) per pixel; zero outside the frame (the conv's zero padding)
        const uint32_t src = smem_u32(sA + us * kU8Slot) + (uint32_t)(x0 - 1 - lbase);
        const int y = y0 - 1 + i;
        const bool row_ok = y >= 0 && y < H, own_row = i >= 1 && i <= n_in - 2;
        const size_t crow = ((size_t)n * (H / 2) + (y >> 1)) * (size_t)(W / 2);
#pragma unroll
        for (int k = 0; k < kIt; ++k) {
          const int p = lane_id() + 32 * k, x = x0 - 1 + p;
          const bool ok = row_ok && p < kRollTW + 2 && x >= 0 && x < W;
          uint8_t rgb[3] = {0, 0, 0};
          if (ok) {
            const int Y = (int)lds_u8f(src + p);
            yuv_to_rgb(Y, __ldg(a.yuv_u + crow + (x >> 1)), __ldg(a.yuv_v + crow + (x >> 1)), rgb);
            if (own_row && p >= 1 && p <= kRollTW) {
              uint8_t* o = a.rgb_out + (((size_t)n * H + y) * W + x) * 3;
              o[0] = rgb[0];
              o[1] = rgb[1];
              o[2] = rgb[2];
            }
          }
          px[k][0] = (float)rgb[0];
          px[k][1] = (float)rgb[1];
          px[k][2] = (float)rgb[2];
        }
      } else {
        const uint32_t src = smem_u32(sA + us * kU8Slot) + (uint32_t)(3 * (x0 - 1) - lbase);
#pragma unroll
        for (int k = 0; k < kIt; ++k) {  // all loads first, so their latencies overlap
          const int p = lane_id() + 32 * k;
          const uint32_t q = src + 3 * min(p, kRollTW + 1);
          px[k][0] = lds_u8f(q);
          px[k][1] = lds_u8f(q + 1);
          px[k][2] = lds_u8f(q + 2);
        }
      }
#pragma unroll
      for (int k = 0; k < kIt; ++k) {
        const int p = lane_id() + 32 * k;
        if (p < kRollTW + 2) {
          uint4 v;
          v.x = pack_bf16x2(px[k][0] * (1.f / 255.f), px[k][1] * (1.f / 255.f));
          v.y = pack_bf16x2(px[k][2] * (1.f / 255.f), 0.f);
          v.z = 0u;
          v.w = 0u;
          *reinterpret_cast<uint4*>(dst + p * 16) = v;
        }
      }
      fence_proxy_async_smem();
      __syncwarp();
      if (lane_id() == 0) {
        mbar_arrive(&u_empty[us]);
        mbar_arrive(&in_full[s]);
      }
      if (++us == kU8Slots) { us = 0; uph ^= 1; }
      if (++s == kRollIn) { s = 0; ph ^= 1; }
    }
    SR_PIECE_END
  } else if (warp == 10) {
    // ===================== store warp: TMA-store finished rows in emission order =====================
    if ((TS == 0 || a.tail_tma) && elect_one()) {
      tma_prefetch_desc(&tm_out);
      int os[2] = {0, 0};
      uint32_t oph[2] = {0, 0};
      int pend_b = -1;  // staging slot (global index) of the previously issued store
      unsigned G = 0;
      SR_PIECE_BEGIN
      for (int q = 1; q <= n_in - 2; ++q) {
        const unsigned g = G + q + 1;
        const int grp = (int)(g & 1);
        const int b = grp * kRollNO + os[grp];
        mbar_wait(&o_full[b], oph[grp]);
        const int r = y0 - 1 + q;
        if (TS == 0 || (r >= a.hr_row0 && r < a.hr_row1)) {
          if (TS > 0)  // the S HR rows of LR row r
            tma_store_4d(&tm_out, sO + b * ROWB, 0, x0 * TS * 3 / 16, TS * r, n);
          else
            tma_store_4d(&tm_out, sO + b * ROWB, 0, x0, r, n);
          bulk_commit();
          bulk_wait_read<1>();        // the previous store has read its staging row
          if (pend_b >= 0) mbar_arrive(&o_free[pend_b]);
          pend_b = b;
        } else {  // strip mode: row outside [hr_row0, hr_row1), nothing to store
          bulk_wait_read<0>();
          if (pend_b >= 0) mbar_arrive(&o_free[pend_b]);
          pend_b = -1;
          mbar_arrive(&o_free[b]);
        }
        if (++os[grp] == kRollNO) { os[grp] = 0; oph[grp] ^= 1; }
      }
      G += n_in + 2;
      SR_PIECE_END
      bulk_wait<0>();
    }
    __syncwarp();
  } else {
    // ===================== epilogue: 2 groups x 4 warps, group g drains the rows with sequence index % 2 == g ======
    const int quarter = warp & 3;
    const int grp = (warp - 2) >> 2;
    const int m = quarter * 32 + lane_id();
    const uint32_t lane_off = (uint32_t)(quarter * 32) << 16;
    uint8_t* stage = sO + grp * kRollNO * ROWB;
    uint32_t ophase = 0;
    for (int b = grp; b < RB; b += 2)  // this group's ring blocks start free (RB is even; the MMA issuer arms)
      if (lane_id() == 0) mbar_arrive(&r_free[b]);
    int os = 0;
    float tr_lsum = 0.f;  // training tail: this thread's loss partial
    unsigned G = 0, emitted = 0;  // emitted: output rows of both groups so far (aux ring order)
    SR_PIECE_BEGIN
    const int xc = x0 + m;
    const bool lane_ok = xc < W;
    const bool sep0 = a.sep > 0 && ((xc % a.sep) == 0 || (xc % a.sep) == a.sep - 1);
    // epilogue variant bits: 1 res1, 2 res2, 4 mask, 8 separators, 16 ReLU
    const int emode = U8 ? 0 : (a.res1 ? 1 : 0) | (a.res2 ? 2 : 0) | (a.mask ? 4 : 0) | (a.sep > 0 ? 8 : 0) | (a.relu ? 16 : 0);
    for (int q = -1; q <= n_in; ++q) {
      const unsigned g = G + q + 1;
      const bool emit = q >= 1 && q <= n_in - 2;
      const unsigned xi = emitted;  // aux ring index of this row (if emitted)
      emitted += emit;
      if ((int)(g & 1) != grp) continue;
      const int r = y0 - 1 + q;
      const size_t pix = (((size_t)n * H + r) * W) + xc;
      uint4 r2[COUTP / 8];
      if (emit && lane_ok && a.res2) ld_row<COUTP>(a.res2 + pix * COUTP, r2);
      const int b = ring_idx<RB>(g);
      mbar_wait(&r_ready[b], (uint32_t)(g / RB) & 1u);
      tc_fence_after();
      if (warp == 2 && lane_id() == 0) { SR_RDBG(5, q + 1) }
      float v[COUTP];
      ring_load<COUTP>(tmem + lane_off + b * COUTP, v);
      tc_fence_before();
      __syncwarp();
      if (lane_id() == 0) mbar_arrive(&r_free[b]);
      if (warp == 2 && lane_id() == 0) { SR_RDBG(6, q + 1) }
      if (!emit) continue;
      if constexpr (TS > 0) {  // up conv: the tail straight from registers (the ring held the bias)
        if (a.train) {  // training tail: loss partial + dy row (same arithmetic as the tiled EPI_TAIL_TRAIN)
          if (lane_ok) {
            EpiParams ep{};
            ep.scale = TS;
            ep.lr = a.lr;
            ep.hr_ref = a.hr_ref;
            ep.dy = a.dy;
            ep.l1 = a.l1;
            ep.bicubic = a.bicubic;
            const size_t vpix = ((size_t)n * H + r) * W + xc;
            if (a.vsep > 0) {
              const int j = xc / a.vsep, x = xc - j * a.vsep - 1;
              if (x < 0 || x >= a.vp) {
                float z[COUTP];
#pragma unroll
                for (int k = 0; k < COUTP; ++k) z[k] = 0.f;
                store_bf16_row<COUTP>(a.dy + vpix * COUTP, z);
              } else {
                epi_tail<TS, COUTP, true>(ep, nullptr, j, r, x, a.vp, a.vp, v, tr_lsum, vpix);
              }
            } else {
              epi_tail<TS, COUTP, true>(ep, nullptr, n, r, xc, H, W, v, tr_lsum, vpix);
            }
          }
          continue;
        }
        if (a.tail_tma) {  // LR rows from the TMA ring, HR rows staged for the store warp
          constexpr int NLR = TS > 0 ? Cfg::NLR : 1;
          mbar_wait(&l_full[xi % NLR], (uint32_t)(xi / NLR) & 1u);
          mbar_wait(&o_free[grp * kRollNO + os], ophase ^ 1);
          if (lane_ok)
            tail_u8_smem<TS>(smem_u32(sA) + (uint32_t)(xi % NLR) * kTailLrSlot, 16 * kTailLrChunks, 3 * x0 - 16,
                             smem_u32(stage + os * ROWB), kRollTW * TS * 3, 3 * TS * m, r, xc, H, W, v, a.bicubic);
          __syncwarp();
          if (lane_id() == 0) mbar_arrive(&l_empty[xi % NLR]);
          fence_proxy_async_smem();
          __syncwarp();
          if (lane_id() == 0) mbar_arrive(&o_full[grp * kRollNO + os]);
          if (warp == 2 && lane_id() == 0) { SR_RDBG(7, q + 1) }
          if (++os == kRollNO) { os = 0; ophase ^= 1; }
          continue;
        }
        if (lane_ok && r >= a.hr_row0 && r < a.hr_row1) {
          EpiParams ep{};
          ep.scale = TS;
          ep.lr = a.lr;
          ep.hr = a.hr;
          ep.bicubic = a.bicubic;
          float ls = 0.f;
          epi_tail<TS, COUTP, false>(ep, nullptr, n, r, xc, H, W, v, ls, 0);
        }
        continue;
      }
      const uint4* aux = reinterpret_cast<const uint4*>(sA + (int)(xi % NAUX) * ROWB + m * COUTP * 2);
      if (has_aux) mbar_wait(&x_full[xi % NAUX], (uint32_t)(xi / NAUX) & 1u);
      mbar_wait(&o_free[grp * kRollNO + os], ophase ^ 1);  // the store warp has read this staging row
      if (warp == 2 && lane_id() == 0) { SR_RDBG(11, q + 1) }
      if (lane_ok) {
        uint4* orow = reinterpret_cast<uint4*>(stage + os * ROWB + m * COUTP * 2);
        // the epilogue variant is uniform across the launch: dispatch once per row to straight-line code
        // (a generic body predicates every variant's instructions -- ~600 per row -- and the per-row chain of
        // the epilogue group is what bounds the launch)
        switch (emode) {  // the variants the library launches; anything else takes the generic body
          case 0: roll_stage<COUTP, 0>(orow, v, aux, r2, sep0, emode); break;
          case 1: roll_stage<COUTP, 1>(orow, v, aux, r2, sep0, emode); break;
          case 8: roll_stage<COUTP, 8>(orow, v, aux, r2, sep0, emode); break;
          case 1 | 8: roll_stage<COUTP, 1 | 8>(orow, v, aux, r2, sep0, emode); break;
          case 1 | 2 | 8: roll_stage<COUTP, 1 | 2 | 8>(orow, v, aux, r2, sep0, emode); break;
          case 4 | 8: roll_stage<COUTP, 4 | 8>(orow, v, aux, r2, sep0, emode); break;
          case 16 | 8: roll_stage<COUTP, 16 | 8>(orow, v, aux, r2, sep0, emode); break;
          default: roll_stage<COUTP, 32>(orow, v, aux, r2, sep0, emode); break;
        }
      }
      if (warp == 2 && lane_id() == 0) { SR_RDBG(12, q + 1) }
      if (has_aux) {
        __syncwarp();
        if (lane_id() == 0) mbar_arrive(&x_empty[xi % NAUX]);
      }
      fence_proxy_async_smem();
      if (warp == 2 && lane_id() == 0) { SR_RDBG(13, q + 1) }
      __syncwarp();
      if (lane_id() == 0) mbar_arrive(&o_full[grp * kRollNO + os]);
      if (warp == 2 && lane_id() == 0) { SR_RDBG(7, q + 1) }
      if (++os == kRollNO) { os = 0; ophase ^= 1; }
    }
    G += n_in + 2;
    SR_PIECE_END
    if (TS > 0 && a.train) {
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) tr_lsum += __shfl_xor_sync(0xffffffffu, tr_lsum, o);
      if (lane_id() == 0) atomicAdd(a.loss_sum, (double)tr_lsum);
    }
  }
#undef SR_PIECE_BEGIN
#undef SR_PIECE_END
  tc_fence_before();
  __syncthreads();
  if (threadIdx.x == 0) { SR_RDBG(9, 0) }  // all roles done
  if (warp == 1) tmem_dealloc<512>(tmem);
}

template <int CINP, int COUTP, int TS = 0, bool U8 = false, bool DBG = false, bool YUV = false>
static cudaError_t launch_roll_t(const CUtensorMap& ti, const CUtensorMap& to, const CUtensorMap& tx,
                                 const bf16* wfold, const RollArgs& a, int grid, cudaStream_t st) {
  if constexpr (!RollCfg<CINP, COUTP>::FITS) {
    return cudaErrorNotSupported;
  } else {
    auto kern = k_conv_roll<CINP, COUTP, TS, U8, DBG, YUV>;
    constexpr size_t smem = RollCfg<CINP, COUTP>::SMEM;
    static bool configured = false;
    if (!configured) {
      cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
      if (e != cudaSuccess) return e;
      configured = true;
    }
    return launch_k(kern, dim3(grid), dim3(kRollThreads + (U8 ? 64 : 0)), smem, st, ti, to, tx, wfold, a);
  }
}

bool roll_head_u8_supported(int coutp, int W, const void* lr) {
  return W >= 96 && W % 16 == 0 && (reinterpret_cast<uintptr_t>(lr) & 15) == 0 &&
         (coutp == 16 || coutp == 32 || coutp == 48);
}

cudaError_t launch_conv_roll_head_u8(int coutp, const uint8_t* lr, const bf16* wfold, const float* bias, bf16* out,
                                     int N, int H, int W, cudaStream_t st, int w_early) {
  if (!roll_head_u8_supported(coutp, W, lr)) return cudaErrorNotSupported;
  CUtensorMap ti, to;
  if (make_u8_rows_tmap(&ti, lr, N, H, 3LL * W, 26, 1) != CUDA_SUCCESS) return cudaErrorInvalidValue;
  if (make_row_tmap(&to, out, N, H, W, coutp, kRollTW, coutp) != CUDA_SUCCESS) return cudaErrorInvalidValue;
  RollArgs a{bias, nullptr, nullptr, nullptr, 0, 0, N, H, W, nullptr, nullptr, nullptr, 0, 0, 0, 0, w_early};
  const long long rows = (long long)N * ((W + kRollTW - 1) / kRollTW) * H;
  int grid = num_sms();
  if (rows < grid) grid = (int)rows;
  if (coutp == 16) return launch_roll_t<16, 16, 0, true>(ti, to, to, wfold, a, grid, st);
  if (coutp == 32) return launch_roll_t<16, 32, 0, true>(ti, to, to, wfold, a, grid, st);
  return launch_roll_t<16, 48, 0, true>(ti, to, to, wfold, a, grid, st);
}

bool roll_head_yuv_supported(int coutp, int W, const void* y, const void* u, const void* v) {
  auto al16 = [](const void* q) { return (reinterpret_cast<uintptr_t>(q) & 15) == 0; };
  return W >= 96 && W % 32 == 0 && al16(y) && al16(u) && al16(v) && (coutp == 16 || coutp == 32 || coutp == 48);
}

cudaError_t launch_conv_roll_head_yuv(int coutp, const uint8_t* y, const uint8_t* u, const uint8_t* v,
                                      uint8_t* rgb_out, const bf16* wfold, const float* bias, bf16* out, int N, int H,
                                      int W, cudaStream_t st, int w_early) {
  if (!roll_head_yuv_supported(coutp, W, y, u, v) || (H & 1)) return cudaErrorNotSupported;
  CUtensorMap ti, to;
  if (make_u8_rows_tmap(&ti, y, N, H, W, kYuvChunks, 1) != CUDA_SUCCESS) return cudaErrorInvalidValue;
  if (make_row_tmap(&to, out, N, H, W, coutp, kRollTW, coutp) != CUDA_SUCCESS) return cudaErrorInvalidValue;
  RollArgs a{bias, nullptr, nullptr, nullptr, 0, 0, N, H, W, nullptr, nullptr, nullptr, 0, 0, 0, 0, w_early};
  a.yuv_u = u;
  a.yuv_v = v;
  a.rgb_out = rgb_out;
  const long long rows = (long long)N * ((W + kRollTW - 1) / kRollTW) * H;
  int grid = num_sms();
  if (rows < grid) grid = (int)rows;
  if (coutp == 16) return launch_roll_t<16, 16, 0, true, false, true>(ti, to, to, wfold, a, grid, st);
  if (coutp == 32) return launch_roll_t<16, 32, 0, true, false, true>(ti, to, to, wfold, a, grid, st);
  return launch_roll_t<16, 48, 0, true, false, true>(ti, to, to, wfold, a, grid, st);
}

static bool ch_ok(int c) { return c == 16 || c == 32 || c == 48 || c == 64; }

template <int CI>
static bool roll_fits(int coutp) {
  return coutp == 16 ? RollCfg<CI, 16>::FITS : coutp == 32 ? RollCfg<CI, 32>::FITS : RollCfg<CI, 48>::FITS;
}

bool roll_supported(int cinp, int coutp, int W) {
  if (W < 96 || !ch_ok(cinp) || !(coutp == 16 || coutp == 32 || coutp == 48)) return false;
  return cinp == 16 ? roll_fits<16>(coutp) : cinp == 32 ? roll_fits<32>(coutp)
       : cinp == 48 ? roll_fits<48>(coutp) : roll_fits<64>(coutp);
}

#define SR_ROLL_CASE(CI, CO) \
  if (cinp == CI && coutp == CO)                                                                 \
    return (a.dbg && CI == 48 && CO == 48) ? launch_roll_t<48, 48, 0, false, true>(ti, to, tx, wfold, a, grid, st) \
                                           : launch_roll_t<CI, CO>(ti, to, tx, wfold, a, grid, st);

cudaError_t launch_conv_roll_ex(int cinp, int coutp, const void* in, const bf16* wfold, const float* bias,
                                const bf16* res1, const bf16* res2, const bf16* mask, int relu, int sep, bf16* out,
                                int N, int H, int W, cudaStream_t st, long long* dbg, int w_early) {
  CUtensorMap ti, to;
  if (make_act_tmap(&ti, in, N, H, W, cinp, kRollTW + 2, 1, cinp / 8, CHUNK_ROW_PIX) != CUDA_SUCCESS)
    return cudaErrorInvalidValue;
  if (make_row_tmap(&to, out, N, H, W, coutp, kRollTW, coutp) != CUDA_SUCCESS) return cudaErrorInvalidValue;
  CUtensorMap tx;
  const void* auxp = res1 ? (const void*)res1 : (mask ? (const void*)mask : (const void*)out);
  if (make_row_tmap(&tx, auxp, N, H, W, coutp, kRollTW, coutp) != CUDA_SUCCESS) return cudaErrorInvalidValue;
  if (res1 && mask) return cudaErrorNotSupported;  // one TMA aux stream per launch
  RollArgs a{bias, res1, res2, mask, relu, sep, N, H, W, dbg, nullptr, nullptr, 0, 0, 0, 0, w_early};
  const long long rows = (long long)N * ((W + kRollTW - 1) / kRollTW) * H;
  int grid = num_sms();
  if (rows < grid) grid = (int)rows;
  SR_ROLL_CASE(16, 16) SR_ROLL_CASE(16, 32) SR_ROLL_CASE(16, 48)
  SR_ROLL_CASE(32, 16) SR_ROLL_CASE(32, 32) SR_ROLL_CASE(32, 48)
  SR_ROLL_CASE(48, 16) SR_ROLL_CASE(48, 32) SR_ROLL_CASE(48, 48)
  SR_ROLL_CASE(64, 16) SR_ROLL_CASE(64, 32) SR_ROLL_CASE(64, 48)
  return cudaErrorNotSupported;
}

#define SR_ROLL_TAIL_CASE(CI, CO, S) \
  if (cinp == CI && coutp == CO && s == S)                                                                  \
    return (a.dbg && CI == 48 && CO == 32 && S == 3) ? launch_roll_t<48, 32, 3, false, true>(ti, th, tl, wfold, a, grid, st) \
                                                     : launch_roll_t<CI, CO, S>(ti, th, tl, wfold, a, grid, st);

cudaError_t launch_conv_roll_tail(int cinp, int coutp, int s, const void* in, const bf16* wfold, const float* bias,
                                  const uint8_t* lr, uint8_t* hr, int hr_row0, int hr_row1, int bicubic, int N, int H,
                                  int W, cudaStream_t st, int tail_tma_ok, long long* dbg, int w_early) {
  CUtensorMap ti;
  if (make_act_tmap(&ti, in, N, H, W, cinp, kRollTW + 2, 1, cinp / 8, CHUNK_ROW_PIX) != CUDA_SUCCESS)
    return cudaErrorInvalidValue;
  RollArgs a{bias, nullptr, nullptr, nullptr, 0, 0, N, H, W, dbg, lr, hr, hr_row0, hr_row1, bicubic, 0, w_early};
  // TMA-staged tail when both u8 images are 16-B row-aligned (W % 16 == 0) and 16-B based
  CUtensorMap tl = ti, th = ti;
  if (tail_tma_ok && W % 16 == 0 &&
      make_u8_rows_tmap(&tl, lr, N, H, 3LL * W, kTailLrChunks, 5) == CUDA_SUCCESS &&
      make_u8_rows_tmap(&th, hr, N, s * H, 3LL * s * W, kRollTW * s * 3 / 16, s) == CUDA_SUCCESS)
    a.tail_tma = 1;
  const long long rows = (long long)N * ((W + kRollTW - 1) / kRollTW) * H;
  int grid = num_sms();
  if (rows < grid) grid = (int)rows;
  SR_ROLL_TAIL_CASE(16, 16, 2) SR_ROLL_TAIL_CASE(32, 16, 2) SR_ROLL_TAIL_CASE(48, 16, 2) SR_ROLL_TAIL_CASE(64, 16, 2)
  SR_ROLL_TAIL_CASE(16, 32, 3) SR_ROLL_TAIL_CASE(32, 32, 3) SR_ROLL_TAIL_CASE(48, 32, 3) SR_ROLL_TAIL_CASE(64, 32, 3)
  SR_ROLL_TAIL_CASE(16, 48, 4) SR_ROLL_TAIL_CASE(32, 48, 4) SR_ROLL_TAIL_CASE(48, 48, 4) SR_ROLL_TAIL_CASE(64, 48, 4)
  return cudaErrorNotSupported;
}

cudaError_t launch_conv_roll_tail_train(int cinp, int coutp, int s, const void* in, const bf16* wfold,
                                        const float* bias, const uint8_t* lr, const uint8_t* hr_ref, bf16* dy,
                                        double* loss_sum, int vsep, int vp, int l1, int bicubic, int N, int H, int W,
                                        cudaStream_t st, int w_early) {
  CUtensorMap ti;
  if (make_act_tmap(&ti, in, N, H, W, cinp, kRollTW + 2, 1, cinp / 8, CHUNK_ROW_PIX) != CUDA_SUCCESS)
    return cudaErrorInvalidValue;
  RollArgs a{bias, nullptr, nullptr, nullptr, 0, 0, N, H, W, nullptr, lr, nullptr, 0, H, bicubic, 0, w_early};
  a.train = 1;
  a.hr_ref = hr_ref;
  a.dy = dy;
  a.loss_sum = loss_sum;
  a.vsep = vsep;
  a.vp = vp;
  a.l1 = l1;
  const long long rows = (long long)N * ((W + kRollTW - 1) / kRollTW) * H;
  int grid = num_sms();
  if (rows < grid) grid = (int)rows;
  CUtensorMap tl = ti, th = ti;
  SR_ROLL_TAIL_CASE(16, 16, 2) SR_ROLL_TAIL_CASE(32, 16, 2) SR_ROLL_TAIL_CASE(48, 16, 2) SR_ROLL_TAIL_CASE(64, 16, 2)
  SR_ROLL_TAIL_CASE(16, 32, 3) SR_ROLL_TAIL_CASE(32, 32, 3) SR_ROLL_TAIL_CASE(48, 32, 3) SR_ROLL_TAIL_CASE(64, 32, 3)
  SR_ROLL_TAIL_CASE(16, 48, 4) SR_ROLL_TAIL_CASE(32, 48, 4) SR_ROLL_TAIL_CASE(48, 48, 4) SR_ROLL_TAIL_CASE(64, 48, 4)
  return cudaErrorNotSupported;
}

cudaError_t launch_conv_roll(int cinp, int coutp, const void* in, const bf16* wfold, const float* bias,
                             const bf16* res, int relu, bf16* out, int N, int H, int W, cudaStream_t st, int w_early) {
  return launch_conv_roll_ex(cinp, coutp, in, wfold, bias, res, nullptr, nullptr, relu, 0, out, N, H, W, st, nullptr,
                             w_early);
}


// ====================================================================================================================
// k_conv_chain: a whole chain of C -> C rolling convs (the residual blocks + body conv of a training forward pass, or
// the data-gradient chain of its backward pass) in ONE persistent cooperative launch.  Opt-in (sr_set_fusion bit 9,
// SR_CHAIN=1): measured, it does not beat one PDL-overlapped k_conv_roll launch per conv.
//
// Why it was built: at the training shape (64 patches of 48 x 48 side by side = 1 x 48 x 3200) a conv is 6.4 GFLOP,
// ~8 rows per CTA on 148 SMs, so each k_conv_roll launch is ~3-4 us of ramp (barriers, TMEM, weights, the first
// input rows' TMA latency) + ~10 row-steps + ~2 us of drain (profiles/r02_roll_timeline.txt).  Here every CTA keeps
// the same work for all layers of the chain and walks them in order: the TMEM ring, barriers and counters keep
// running across layer boundaries, the next layer's weights are fetched as soon as the MMAs of the previous one have
// completed, and a layer's input row is loaded as soon as the CTAs that produce it (same strip and the two
// neighbouring strips, for the 1-pixel halo columns) have published it -- no grid-wide barrier, no relaunch.
// Work split (chain_pieces): with >= 1 CTA per column strip, two phases -- each CTA owns one band of the top half and
// one band of the bottom half of the rows and walks layer l as [top band, bottom band], so the store -> publish ->
// load latency of a layer boundary is covered by the other phase's work.
//
// Cross-CTA protocol (all CTAs co-resident: cooperative launch): sync[0] = launch generation, sync[1] = exit count,
// sync[2 + col * H + row] = flag of output row (col, row).  Once the bulk group of a piece has completed
// (cp.async.bulk.wait_group 0) the store thread hands the piece to the publisher warp through shared memory, which
// issues the proxy + gpu-scope fences and stores gen * 64 + layer + 1 into the piece's row flags.  A producer
// polls the flags of the rows it is about to load (input rows: layer - 1, three columns; res1 aux rows: the layer
// that wrote them) with one lane per flag, fences (acquire) and orders its TMA loads after them with
// fence.proxy.async.  Flags only grow, so no reset is needed between launches; the last CTA to exit advances the
// generation.  Math per layer: exactly k_conv_roll's (same MMAs in the same order, same ring, same epilogue
// variants): the outputs are bit-identical to one k_conv_roll launch per layer (tests/test_gpu_timed_paths.py).
static constexpr int kChainMax = 20;
struct ChainLayer {
  CUtensorMap tin, tout, taux;
  const bf16* w;
  const float* bias;
  const bf16* res2;
  int emode;    // roll_stage variant bits: 1 res1, 2 res2, 4 mask, 8 separators, 16 ReLU
  int aux_dep;  // >= 0: the aux (res1) rows were written by layer aux_dep of this launch; -1: by an earlier kernel
};
static constexpr int kChainMaxCta = 192;
struct ChainPiece {
  short col, y0, y1, pad;
};
struct ChainParams {
  ChainLayer L[kChainMax];
  int nl, N, H, W, sep;
  int nph;      // 0: each CTA takes a contiguous (strip, row) range (<= 4 pieces); 1, 2: pieces from pc[cta][0..nph)
  ChainPiece pc[kChainMaxCta][2];
  unsigned* sync;
  int dbg_cta;              // benchmarking only: the CTA whose per-row stamps are kept (SR_CHAIN_DBG_CTA)
  unsigned long long* dbg;  // benchmarking only: per (CTA, layer) globaltimer stamps [8] (sr_test_chain_dbg)
};
#define SR_RDBG2(l, i, k) \
  if (p.dbg && blockIdx.x == (unsigned)p.dbg_cta && (i) < 64) \
    p.dbg[(size_t)gridDim.x * kChainMax * 8 + ((size_t)(l) * 64 + (i)) * 4 + (k)] = (unsigned long long)globaltimer();
#define SR_CDBG(l, k) \
  if (p.dbg) p.dbg[((size_t)blockIdx.x * kChainMax + (l)) * 8 + (k)] = (unsigned long long)globaltimer();

// bias of one layer into its arming tile (B[n][k]: hi, mid, lo bf16 terms at k = 0, 1, 2; ring.cuh)
__device__ __forceinline__ void chain_bias_tile(uint8_t* btile, const float* bias, int coutp, int tid, int nthreads) {
  for (int i = tid; i < coutp * 16; i += nthreads) {
    const int n = i / 16, k = i % 16;
    const float b = bias ? __ldg(bias + n) : 0.f;
    const __nv_bfloat16 hi = __float2bfloat16(b);
    const __nv_bfloat16 mid = __float2bfloat16(b - __bfloat162float(hi));
    const __nv_bfloat16 lo = __float2bfloat16(b - __bfloat162float(hi) - __bfloat162float(mid));
    const __nv_bfloat16 v = k == 0 ? hi : k == 1 ? mid : k == 2 ? lo : __float2bfloat16(0.f);
    *reinterpret_cast<__nv_bfloat16*>(btile + (n % 8) * 16 + (n / 8) * 128 + (k / 8) * (coutp * 16) + (k % 8) * 2) = v;
  }
}

static constexpr int kChainThreads = kRollThreads;
template <int C>
__global__ void __launch_bounds__(kChainThreads, 1) k_conv_chain(const __grid_constant__ ChainParams p) {
  using Cfg = RollCfg<C, C>;
  constexpr int RB = Cfg::RB, kRollIn = Cfg::NIN, NAUX = Cfg::NAUX;
  constexpr uint32_t PLANE = Cfg::PLANE, IN_STRIDE = Cfg::IN_STRIDE, ROWB = Cfg::ROWB;
  static_assert(RB * C + 8 <= 512, "chain: the ones operand lives in TMEM");
  static_assert(2 * C * 32 <= (int)kArmOnesBytes, "chain: two bias tiles in the (unused) ones-tile area");

  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  uint8_t* sW = smem;
  uint8_t* sIn = sW + Cfg::WB_AL;
  uint8_t* sO = sIn + kRollIn * IN_STRIDE;
  uint8_t* sA = sO + 2 * kRollNO * ROWB;
  uint8_t* sBt = sA + NAUX * ROWB;  // two bias-arming tiles (layer parity)
  __shared__ __align__(8) uint64_t in_full[kRollIn], in_empty[kRollIn], r_ready[RB], r_free[RB], x_full[NAUX],
      x_empty[NAUX], o_full[2 * kRollNO], o_free[2 * kRollNO], w_bar, w_free, arm_bar[2];
  __shared__ uint32_t tmem_base_sh;
  __shared__ unsigned gen_sh;
  // pieces whose stores have completed, handed from the store thread to the publisher (piece index, layer): entries
  // [0, pub_w) written; the publisher trails by at most one layer, far less than the ring
  constexpr int kPubRing = 128;
  __shared__ uint8_t pub_pc[kPubRing], pub_l[kPubRing];
  __shared__ volatile uint32_t pub_w;

  const int N = p.N, H = p.H, W = p.W, nl = p.nl;
  const int warp = warp_id();
  if (warp == 0 && lane_id() == 0) {
    for (int s = 0; s < kRollIn; ++s) { mbar_init(&in_full[s], 1); mbar_init(&in_empty[s], 1); }
    for (int s = 0; s < RB; ++s) { mbar_init(&r_ready[s], 1); mbar_init(&r_free[s], 4); }
    for (int s = 0; s < NAUX; ++s) { mbar_init(&x_full[s], 1); mbar_init(&x_empty[s], 4); }
    for (int s = 0; s < 2 * kRollNO; ++s) { mbar_init(&o_full[s], 4); mbar_init(&o_free[s], 1); }
    mbar_init(&w_bar, 1);
    mbar_init(&w_free, 1);
    mbar_init(&arm_bar[0], 1);
    mbar_init(&arm_bar[1], 1);
    fence_barrier_init();
    pub_w = 0;
  }
  if (warp == 1) tmem_alloc<512>(&tmem_base_sh);
  tc_fence_before();
  __syncthreads();
  if (warp >= 2 && warp <= 5) {  // the TMEM ones operand of the arming MMAs (four lane quarters)
    tc_fence_after();
    ones_tmem_fill(tmem_base_sh + ((uint32_t)((warp & 3) * 32) << 16) + RB * C);
    tmem_st_wait();
    tc_fence_before();
  }
  pdl_enter();  // the chain's input, the external aux rows and the packed weights are complete from here on
  if (threadIdx.x == 0) gen_sh = *reinterpret_cast<volatile unsigned*>(p.sync);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = tmem_base_sh;
  const unsigned base = gen_sh * 64u;  // flag value of layer l: base + l + 1
  unsigned* const flags = p.sync + 2;

  const int tiles_x = (W + kRollTW - 1) / kRollTW;
  const long long total = (long long)N * tiles_x * H;
  // this CTA's pieces (column strip, rows [y0, y1)), the same for every layer
  int pcol[4], py0[4], py1[4], npc = 0;
  if (p.nph > 0) {
    for (int k = 0; k < p.nph; ++k) {
      const ChainPiece& q = p.pc[blockIdx.x][k];
      pcol[npc] = q.col; py0[npc] = q.y0; py1[npc] = q.y1; ++npc;
    }
  } else {
    const long long beg = total * blockIdx.x / gridDim.x, end = total * (blockIdx.x + 1) / gridDim.x;
    for (long long pos = beg; pos < end && npc < 4;) {
      const int col = (int)(pos / H), y0 = (int)(pos - (long long)col * H);
      const int y1 = (int)min((long long)H, y0 + (end - pos));
      pos += y1 - y0;
      pcol[npc] = col; py0[npc] = y0; py1[npc] = y1; ++npc;
    }
  }
#define SR_PIECE_BEGIN                                                                \
  for (int pi = 0; pi < npc; ++pi) {                                                  \
    const int col = pcol[pi], y0 = py0[pi], y1 = py1[pi];                             \
    const int n = col / tiles_x, x0 = (col - n * tiles_x) * kRollTW;                  \
    const int n_in = y1 - y0 + 2;                                                     \
    (void)n; (void)x0; (void)n_in;
#define SR_PIECE_END }

  if (warp == 0) {
    // ===================== producer: layer weights, then each input row once its three producers published it ====
    // The warp polls the flags of the next up-to-8 input rows x 3 columns (the 1-pixel halo of the neighbouring
    // strips) in one round (one lane per flag); lane 0 issues the weight and row TMAs.
    const bool lead = lane_id() == 0;
    int s = 0, xs = 0;
    uint32_t ph = 0, xph = 0;
    for (int l = 0; l < nl; ++l) {
      const ChainLayer& Ly = p.L[l];
      if (lead) {
        tma_prefetch_desc(&Ly.tin);
        if (l > 0) mbar_wait(&w_free, (uint32_t)(l - 1) & 1u);  // the previous layer's MMAs have completed
        mbar_arrive_expect_tx(&w_bar, Cfg::WBYTES);
        bulk_load(sW, Ly.w, Cfg::WBYTES, &w_bar);
        SR_CDBG(l, 5)
      }
      const bool has_aux = (Ly.emode & 5) != 0;
      if (lead && has_aux) tma_prefetch_desc(&Ly.taux);
      bool first_piece = true;
      SR_PIECE_BEGIN
      const int sx = col - n * tiles_x;
      const bool has_l = sx > 0, has_r = sx + 1 < tiles_x;
      int ready = l > 0 ? 0 : n_in;  // input rows [0, ready) of the piece confirmed published
      if (has_aux && Ly.aux_dep >= 0) {  // res1 rows: own rows (same strip and rows) of an earlier layer
        for (int r = y0 + lane_id(); r < y1; r += 32)
          flag_spin(flags + (size_t)col * H + r, base + (unsigned)Ly.aux_dep + 1u);
        fence_acq_rel_gpu();
        __syncwarp();
        if (lead) fence_proxy_async_global();
      }
      for (int i = 0; i < n_in; ++i) {
        const int y = y0 - 1 + i;
        if (i >= ready) {  // input row y = output row y of layer l - 1 in strips sx - 1 .. sx + 1
          const int k = lane_id(), ii = i + k / 3, dc = k % 3 - 1;
          const int yy = y0 - 1 + ii;
          const bool mine = k < 24 && ii < n_in && yy >= 0 && yy < H && (dc == 0 || (dc < 0 ? has_l : has_r));
          const unsigned* f = flags + (size_t)(col + dc) * H + yy;
          const unsigned tgt = base + (unsigned)l;
          const long long t0 = clock64();
          for (;;) {
            const bool ok = !mine || (int)(ld_relaxed_gpu(f) - tgt) >= 0;
            const unsigned bad = __ballot_sync(0xffffffffu, !ok);
            const int nrd = bad ? (__ffs(bad) - 1) / 3 : 8;  // leading rows with all three flags set
            if (nrd > 0) { ready = i + nrd; break; }
            __nanosleep(20);
            if (clock64() - t0 > (1ll << 34)) __trap();
          }
          fence_acq_rel_gpu();
          __syncwarp();
          if (lead) fence_proxy_async_global();
        }
        if (lead) {
          if (first_piece && i == 0) { SR_CDBG(l, 0) }
          SR_RDBG2(l, i, 0)
          mbar_wait(&in_empty[s], ph ^ 1);
          mbar_arrive_expect_tx(&in_full[s], Cfg::IN_BOX);
          tma_load_5d(sIn + s * IN_STRIDE, &Ly.tin, &in_full[s], 0, x0 - 1, y, 0, n);
          if (has_aux && i >= 1 && i <= n_in - 2) {  // the aux row of output emission i (needed after input i + 1)
            const int r = y0 - 1 + i;
            mbar_wait(&x_empty[xs], xph ^ 1);
            mbar_arrive_expect_tx(&x_full[xs], kRollTW * C * 2);
            tma_load_4d(sA + xs * ROWB, &Ly.taux, &x_full[xs], 0, x0, r, n);
          }
        }
        if (has_aux && i >= 1 && i <= n_in - 2 && ++xs == NAUX) { xs = 0; xph ^= 1; }
        if (++s == kRollIn) { s = 0; ph ^= 1; }
      }
      first_piece = false;
      __syncwarp();
      SR_PIECE_END
    }
  } else if (warp == 11) {
    // ===================== publisher: flags of the pieces the store thread reports written ======================
    // (a gpu-scope fence costs ~1.5k cycles; issued here it never holds back the store thread's staging slots)
    const uint32_t total = (uint32_t)(nl * npc);  // pieces handed over: every piece of every layer
    uint32_t r = 0;
    const long long t0 = clock64();
    while (r < total) {
      const uint32_t w = pub_w;
      if (w == r) {
        __nanosleep(32);
        if (clock64() - t0 > (1ll << 36)) __trap();
        continue;
      }
      __syncwarp();
      __threadfence_block();
      if (lane_id() == 0) {
        fence_proxy_async_global();
        fence_acq_rel_gpu();
      }
      __syncwarp();
      for (; r < w; ++r) {
        const int pi = pub_pc[r % kPubRing], l = pub_l[r % kPubRing];
        const int col = pcol[pi], y0 = py0[pi], y1 = py1[pi];
        for (int y = y0 + lane_id(); y < y1; y += 32) st_relaxed_gpu(flags + (size_t)col * H + y, base + (unsigned)l + 1u);
        if (pi == npc - 1) { SR_CDBG(l, 4) }
      }
      __syncwarp();
    }
  } else if (warp == 1) {
    // ===================== MMA issuer =====================
    if (elect_one()) {
      const uint64_t bd = make_desc(smem_u32(sW), 3 * C * 16, 128);
      const uint32_t ones = tmem + RB * C;
      int s = 0;
      uint32_t ph = 0;
      unsigned G = 0, acq = 0;
      for (int l = 0; l < nl; ++l) {
        mbar_wait(&w_bar, (uint32_t)l & 1u);
        mbar_wait(&arm_bar[l & 1], (uint32_t)(l >> 1) & 1u);
        tc_fence_after();
        const uint32_t bt = smem_u32(sBt + (l & 1) * C * 32);
        const unsigned Gl = G;
        SR_PIECE_BEGIN
        for (int i = 0; i < n_in; ++i) {
          const unsigned g = G + i;
          for (; acq < g + 3; ++acq) mbar_wait(&r_free[ring_idx<RB>(acq)], (uint32_t)(acq / RB) & 1u);
          mbar_wait(&in_full[s], ph);
          tc_fence_after();
          if (i == 0) {
            ring_arm_ts<C, RB>(tmem, g, ones, bt);
            ring_arm_ts<C, RB>(tmem, g + 1, ones, bt);
          }
          ring_arm_ts<C, RB>(tmem, g + 2, ones, bt);
          ring_mma_step<C, C, RB>(tmem, g, make_desc(smem_u32(sIn + s * IN_STRIDE), PLANE, 128), bd, 2 * PLANE);
          if (G == Gl && i == 0) { SR_CDBG(l, 1) }
          if (G == Gl) { SR_RDBG2(l, i, 1) }
          mma_commit(&r_ready[ring_idx<RB>(g)]);
          mma_commit(&in_empty[s]);
          if (i == n_in - 1) {
            mma_commit(&r_ready[ring_idx<RB>(g + 1)]);
            mma_commit(&r_ready[ring_idx<RB>(g + 2)]);
          }
          if (++s == kRollIn) { s = 0; ph ^= 1; }
        }
        G += n_in + 2;
        SR_PIECE_END
        mma_commit(&w_free);  // fires when every MMA of this layer (and the arms) has completed
        SR_CDBG(l, 2)
      }
    }
    __syncwarp();
  } else if (warp == 10) {
    // ===================== store warp: TMA-store finished rows; publish each piece's rows once written ==========
    const bool lead = lane_id() == 0;
    int os[2] = {0, 0};
    uint32_t oph[2] = {0, 0};
    unsigned G = 0;
    for (int l = 0; l < nl; ++l) {
      const ChainLayer& Ly = p.L[l];
      if (lead) tma_prefetch_desc(&Ly.tout);
      SR_PIECE_BEGIN
      if (lead) {
        // The rows of a piece are published together once its last store has completed, by the publisher warp (a
        // gpu-scope fence issued here, behind outstanding bulk stores, costs ~1.5k cycles and holds back the staging
        // slots the epilogue waits for).
        int pend_b = -1;
        for (int q = 1; q <= n_in - 2; ++q) {
          const unsigned g = G + q + 1;
          const int grp = (int)(g & 1);
          const int b = grp * kRollNO + os[grp];
          mbar_wait(&o_full[b], oph[grp]);
          SR_RDBG2(l, q, 3)
          tma_store_4d(&Ly.tout, sO + b * ROWB, 0, x0, y0 - 1 + q, n);
          bulk_commit();
          bulk_wait_read<1>();  // the previous store has read its staging row
          if (pend_b >= 0) mbar_arrive(&o_free[pend_b]);
          pend_b = b;
          if (++os[grp] == kRollNO) { os[grp] = 0; oph[grp] ^= 1; }
        }
        SR_CDBG(l, 3)
        bulk_wait<0>();
        if (pend_b >= 0) mbar_arrive(&o_free[pend_b]);
        const uint32_t w = pub_w;  // hand the piece to the publisher warp
        pub_pc[w % kPubRing] = (uint8_t)pi;
        pub_l[w % kPubRing] = (uint8_t)l;
        __threadfence_block();
        pub_w = w + 1;
      }
      __syncwarp();
      G += n_in + 2;
      SR_PIECE_END
    }
  } else {
    // ===================== epilogue: 2 groups x 4 warps (alternate rows); also build the next layers' bias tiles =
    const int quarter = warp & 3;
    const int grp = (warp - 2) >> 2;
    const int m = quarter * 32 + lane_id();
    const uint32_t lane_off = (uint32_t)(quarter * 32) << 16;
    const int et = (int)threadIdx.x - 64;  // 0 .. 255 over the eight epilogue warps
    uint8_t* stage = sO + grp * kRollNO * ROWB;
    auto arm_layer = [&](int l) {  // bias tile of layer l into slot l & 1 (its previous user, layer l - 2, is drained)
      chain_bias_tile(sBt + (l & 1) * C * 32, p.L[l].bias, C, et, 256);
      fence_proxy_async_smem();
      named_bar_sync(1, 256);
      if (et == 0) mbar_arrive(&arm_bar[l & 1]);
    };
    arm_layer(0);
    if (nl > 1) arm_layer(1);
    uint32_t ophase = 0;
    for (int b = grp; b < RB; b += 2)
      if (lane_id() == 0) mbar_arrive(&r_free[b]);
    int os = 0;
    unsigned G = 0, xi = 0;  // xi: aux rows consumed so far (layers with an aux row only)
    for (int l = 0; l < nl; ++l) {
      const ChainLayer& Ly = p.L[l];
      if (l >= 1 && l + 1 < nl) arm_layer(l + 1);
      const int emode = Ly.emode;
      const bool has_aux = (emode & 5) != 0;
      const bf16* res2 = Ly.res2;
      const unsigned Gl = G;
      SR_PIECE_BEGIN
      const int xc = x0 + m;
      const bool lane_ok = xc < W;
      const bool sep0 = p.sep > 0 && ((xc % p.sep) == 0 || (xc % p.sep) == p.sep - 1);
      for (int q = -1; q <= n_in; ++q) {
        const unsigned g = G + q + 1;
        const bool emit = q >= 1 && q <= n_in - 2;
        const unsigned xr = xi;
        if (emit && has_aux) ++xi;
        if ((int)(g & 1) != grp) continue;
        const int r = y0 - 1 + q;
        const size_t pix = (((size_t)n * H + r) * W) + xc;
        uint4 r2[C / 8];
        if (emit && lane_ok && (emode & 2)) ld_row<C>(res2 + pix * C, r2);
        const int b = ring_idx<RB>(g);
        mbar_wait(&r_ready[b], (uint32_t)(g / RB) & 1u);
        tc_fence_after();
        float v[C];
        ring_load<C>(tmem + lane_off + b * C, v);
        tc_fence_before();
        __syncwarp();
        if (lane_id() == 0) mbar_arrive(&r_free[b]);
        if (!emit) continue;
        if (warp == 2 + 4 * grp && lane_id() == 0 && G == Gl) { SR_RDBG2(l, q, 2) }
        const uint4* aux = reinterpret_cast<const uint4*>(sA + (int)(xr % NAUX) * ROWB + m * C * 2);
        if (has_aux) mbar_wait(&x_full[xr % NAUX], (uint32_t)(xr / NAUX) & 1u);
        mbar_wait(&o_free[grp * kRollNO + os], ophase ^ 1);
        if (lane_ok) {
          uint4* orow = reinterpret_cast<uint4*>(stage + os * ROWB + m * C * 2);
          switch (emode) {
            case 8: roll_stage<C, 8>(orow, v, aux, r2, sep0, emode); break;
            case 1 | 8: roll_stage<C, 1 | 8>(orow, v, aux, r2, sep0, emode); break;
            case 1 | 2 | 8: roll_stage<C, 1 | 2 | 8>(orow, v, aux, r2, sep0, emode); break;
            case 4 | 8: roll_stage<C, 4 | 8>(orow, v, aux, r2, sep0, emode); break;
            case 16 | 8: roll_stage<C, 16 | 8>(orow, v, aux, r2, sep0, emode); break;
            default: roll_stage<C, 32>(orow, v, aux, r2, sep0, emode); break;
          }
        }
        if (has_aux) {
          __syncwarp();
          if (lane_id() == 0) mbar_arrive(&x_empty[xr % NAUX]);
        }
        fence_proxy_async_smem();
        __syncwarp();
        if (lane_id() == 0) mbar_arrive(&o_full[grp * kRollNO + os]);
        if (++os == kRollNO) { os = 0; ophase ^= 1; }
      }
      G += n_in + 2;
      SR_PIECE_END
    }
  }
#undef SR_PIECE_BEGIN
#undef SR_PIECE_END
  tc_fence_before();
  __syncthreads();
  if (warp == 1) tmem_dealloc<512>(tmem);
  if (threadIdx.x == 0) {  // the last CTA out advances the generation for the next launch
    __threadfence();
    const unsigned prev = atomicAdd(p.sync + 1, 1u);
    if (prev == gridDim.x - 1) {
      p.sync[1] = 0;
      __threadfence();
      atomicAdd(p.sync, 1u);
    }
  }
}

static unsigned long long* g_chain_dbg = nullptr;
void set_chain_dbg(void* p) { g_chain_dbg = reinterpret_cast<unsigned long long*>(p); }

bool chain_supported(int cp, int W, int nl) {
  if (nl < 1 || nl > kChainMax || W < 96) return false;
  return (cp == 32 && RollCfg<32, 32>::FITS) || (cp == 48 && RollCfg<48, 48>::FITS);
}

size_t chain_sync_words(int N, int H, int W) {
  return 2 + (size_t)N * ((W + kRollTW - 1) / kRollTW) * H;
}

// Work split of a chain launch (the same for every layer).  With at least one CTA per column strip: two phases --
// every CTA takes one band of the top half of the rows and one band of the bottom half (bands of neighbouring
// strips cover the same rows), and walks layer l as [top band, bottom band]: the rows a top band needs for layer
// l + 1 were all published during the previous top-band phase, a whole bottom-band phase before (and the bottom
// half's row a boundary band needs comes last in its pass), so the layer boundary's store -> publish -> load latency
// is hidden by the other phase's work instead of idling the tensor pipe.  Bands are paired tall with short.
// Otherwise: contiguous (strip, row) ranges (<= 4 pieces per CTA).
static bool chain_pieces(ChainParams& prm, int N, int H, int W, int grid) {
  const int S = N * ((W + kRollTW - 1) / kRollTW);
  if (grid >= S && grid <= kChainMaxCta && H >= 8 && grid <= S * (H / 2) &&
      std::getenv("SR_CHAIN_CONTIG") == nullptr) {
    const int hs[3] = {0, H / 2, H};
    std::vector<ChainPiece> ph[2];
    for (int h = 0; h < 2; ++h) {
      const int q = grid / S, rm = grid % S, rows = hs[h + 1] - hs[h];
      for (int sc = 0; sc < S; ++sc) {
        const int k = q + ((h == 0 ? sc : S - 1 - sc) < rm ? 1 : 0);  // extra bands on different strips per phase
        for (int j = 0; j < k; ++j)
          ph[h].push_back(ChainPiece{(short)sc, (short)(hs[h] + rows * j / k), (short)(hs[h] + rows * (j + 1) / k), 0});
      }
    }
    auto ht = [](const ChainPiece& a) { return a.y1 - a.y0; };
    std::stable_sort(ph[0].begin(), ph[0].end(), [&](const ChainPiece& a, const ChainPiece& b) { return ht(a) > ht(b); });
    std::stable_sort(ph[1].begin(), ph[1].end(), [&](const ChainPiece& a, const ChainPiece& b) { return ht(a) < ht(b); });
    for (int c = 0; c < grid; ++c) { prm.pc[c][0] = ph[0][c]; prm.pc[c][1] = ph[1][c]; }
    prm.nph = 2;
    return true;
  }
  const long long total = (long long)S * H;
  const long long maxlen = (total + grid - 1) / grid;
  if ((maxlen + H - 1) / H + 1 > 4) return false;
  prm.nph = 0;
  return true;
}

template <int C>
static cudaError_t launch_chain_t(const ChainParams& prm, int grid, cudaStream_t st) {
  auto kern = k_conv_chain<C>;
  constexpr size_t smem = RollCfg<C, C>::SMEM;
  static bool configured = false;
  if (!configured) {
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    configured = true;
  }
  return launch_coop(kern, dim3(grid), dim3(kChainThreads), smem, st, prm);
}

cudaError_t launch_conv_chain(int cp, const ChainLayerDesc* layers, int nl, int sep, int N, int H, int W,
                              unsigned* sync, cudaStream_t st) {
  if (!chain_supported(cp, W, nl) || !sync) return cudaErrorNotSupported;
  ChainParams prm{};  // ~9 KB of kernel parameters (tensor maps by value: a captured graph keeps its own copy)
  for (int l = 0; l < nl; ++l) {
    const ChainLayerDesc& d = layers[l];
    ChainLayer& L = prm.L[l];
    if (make_act_tmap(&L.tin, d.in, N, H, W, cp, kRollTW + 2, 1, cp / 8, CHUNK_ROW_PIX) != CUDA_SUCCESS)
      return cudaErrorInvalidValue;
    if (make_row_tmap(&L.tout, d.out, N, H, W, cp, kRollTW, cp) != CUDA_SUCCESS) return cudaErrorInvalidValue;
    if (d.res1 && d.mask) return cudaErrorNotSupported;
    const void* auxp = d.res1 ? (const void*)d.res1 : (d.mask ? (const void*)d.mask : (const void*)d.out);
    if (make_row_tmap(&L.taux, auxp, N, H, W, cp, kRollTW, cp) != CUDA_SUCCESS) return cudaErrorInvalidValue;
    L.w = d.w;
    L.bias = d.bias;
    L.res2 = d.res2;
    L.emode = (d.res1 ? 1 : 0) | (d.res2 ? 2 : 0) | (d.mask ? 4 : 0) | (sep > 0 ? 8 : 0) | (d.relu ? 16 : 0);
    L.aux_dep = d.res1 ? d.aux_dep : -1;
    if (L.aux_dep >= l) return cudaErrorInvalidValue;
  }
  prm.nl = nl;
  prm.N = N;
  prm.H = H;
  prm.W = W;
  prm.sep = sep;
  prm.sync = sync;
  prm.dbg = g_chain_dbg;
  if (const char* e = std::getenv("SR_CHAIN_DBG_CTA")) prm.dbg_cta = std::atoi(e);
  const long long rows = (long long)N * ((W + kRollTW - 1) / kRollTW) * H;
  int grid = num_sms();
  if (rows < grid) grid = (int)rows;
  if (!chain_pieces(prm, N, H, W, grid)) return cudaErrorNotSupported;
  if (cp == 32) return launch_chain_t<32>(prm, grid, st);
  return launch_chain_t<48>(prm, grid, st);
}

}  // namespace sr

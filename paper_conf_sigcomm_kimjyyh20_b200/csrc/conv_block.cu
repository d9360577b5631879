// Fused residual block for wide frames:  f' = f + conv2(ReLU(conv1(f) + b1)) + b2   (sm_100a tcgen05)
//
// Unfused, one block moves 480 B per pixel through HBM at C = 48 (conv1: read f, write t; conv2: read t, read f,
// write f') against 83 kFLOP -- below the B200 ridge.  Here the ReLU intermediate t never leaves the SM: both
// convs use the rolling dy-fold form of conv_roll.cu (N = 3C per MMA, one input row per step) and t rows pass
// through a shared-memory ring from the conv1 epilogue to the conv2 MMAs.  HBM per pixel: f once (+2 columns of
// halo per 126) and f' once.
//
// Column strip of 126 output pixels starting at x0 (MMA M = 128 lanes):
//   f row in smem  : pixels x0-2 .. x0+127 (130, TMA, zero outside the frame)
//   conv1 lane m   : t column x0-1+m, reads f positions m+dx              -> t row in smem (128 + 2 spare positions)
//   conv2 lane m   : out column x0+m (m < 126), reads t positions m+dx
//   t is forced to 0 outside the frame (it is conv2's zero padding).
//
// Accumulation (the point of this design): for every input row the MMA group (3 dx x C/16 MMAs, N = 3C) adds
//   dy = 0 into the accumulator of output row i+1, dy = 1 into row i, dy = 2 into row i-1,
// i.e. out[r] = sum_{dy} sum_{dx,ci} in[r+dy-1, x+dx-1, ci] W[co,ci,dy,dx] is summed by the tensor core in TMEM.
// Output rows own C-column blocks of a TMEM ring (RB blocks per conv, descending so the three targets of a step
// are contiguous; when the ring wraps inside them the step is issued as two MMA groups).  Blocks are armed with
// the bias (tcgen05.st) by the epilogue, so the epilogue only drains a finished row: ReLU -> t smem (conv1) or
// + residual -> TMA store (conv2), then re-arms the block.
// Rows of a strip piece with output rows [y0,y1): f rows y0-2 .. y1+1 (n_f), t rows y0-1 .. y1 (n_t = n_f - 2).
// Per conv the out-row sequence of a piece has n_in + 2 entries (local q = -1 .. n_in); q in [1, n_in-2] are
// the rows that are kept.
//
// Warps: 0 TMA producer, 1 TMEM alloc + conv1 MMA issuer, 10 conv2 MMA issuer (conv2 trails conv1 by three rows;
// two issuers so that one waiting on a barrier does not starve the tensor pipe), 2..5 conv1 epilogue, 6..9 conv2
// epilogue (residual from global/L2, rows -> smem -> TMA store).  The kernel is bound by the
// 128 B/clk shared-memory port: per row-step the MMAs read ~155 KB of operands (A 4 KB + B 4.5 KB per MMA) and the
// TMA/epilogue traffic adds ~49 KB (clock64 timeline, scripts/bench_block.py).
#include <cuda.h>
#include "ptx.cuh"
#include "tmap.h"
#include "sr_internal.h"
#include "ring.cuh"
#include "launch.cuh"
#include "rot.cuh"

namespace sr {

static constexpr int kBlkThreads = 352;  // + warp 10: the conv2 MMA issuer
static constexpr int kBlkTW = 126;  // output pixels per strip
static constexpr int kBlkNF = 4;    // f-row ring
static constexpr int kBlkNT = 3;    // t-row ring
static constexpr int kBlkNO = 3;    // output staging rows (TMA store)

template <int C>
struct BlkCfg {
  static constexpr int CCH = C / 8, KS = C / 16, N = 3 * C;
  static constexpr int RB = (256 / C) < 8 ? (256 / C) : 8;  // TMEM ring blocks per conv (256 columns each)
  static constexpr uint32_t WBYTES = 9u * C * C * 2u;
  static constexpr uint32_t PLANE = 130 * 16;
  static constexpr uint32_t ROWB = ((CCH * PLANE) + 127u) & ~127u;  // f / t ring slot (TMA: 128-B aligned)
  static constexpr uint32_t WB_AL = (WBYTES + 1023u) & ~1023u;
  static constexpr uint32_t OUTB = ((kBlkTW * C * 2) + 1023u) & ~1023u;          // staging row
  static constexpr uint32_t ARMB = ((kArmOnesBytes + 2 * 2 * C * 16) + 1023u) & ~1023u;  // ones + 2 bias tiles
  static constexpr size_t SMEM = 1024 + 2 * WB_AL + (size_t)kBlkNF * ROWB + (size_t)kBlkNT * ROWB +
                                 (size_t)kBlkNO * OUTB + ARMB;
};

// GEN = 0: the inference instantiation -- no experiments, no t save, no separators, no timeline (those runtime
// checks otherwise put predicated instructions on the epilogues' per-row chains); 1: training forward (t save and
// separators, no experiments / timeline); 2: everything read at run time.
template <int C, bool BWD, int GEN>
__global__ void __launch_bounds__(kBlkThreads, 1)
k_resblock(const __grid_constant__ CUtensorMap tm_f, const __grid_constant__ CUtensorMap tm_out,
           const bf16* __restrict__ w1, const bf16* __restrict__ w2, const float* __restrict__ b1,
           const float* __restrict__ b2, const bf16* __restrict__ fres, bf16* __restrict__ outp, const int N,
           const int H, const int W, bf16* __restrict__ tsave_in, const int sep_in, long long* __restrict__ dbg_in,
           const int exp_in, const bf16* __restrict__ mask, const bf16* __restrict__ res2) {
  bf16* const tsave = GEN ? tsave_in : nullptr;
  const int sep = GEN ? sep_in : 0;
  long long* const dbg = GEN == 2 ? dbg_in : nullptr;
  const int exp = GEN == 2 ? exp_in : 0;
  // exp (benchmarking experiments only, results wrong when set): 1 no residual load, 2 no output store, 4 no t
  // smem write, 8 no bias re-arm, 16 no conv2 MMAs, 32 no conv1 MMAs, 64 no accumulator loads, 128 no f-row TMA
  // after the first piece
  // tsave (nullable): also write t = ReLU(conv1(f) + b1) to global (training saves it for the backward pass).
  // mask (nullable): the data-gradient block of the backward pass -- t = conv1(f) * 1[mask > 0] (ReLU' through the
  // saved forward t) instead of ReLU; res2 (nullable): conv2's output also adds res2 (the global-skip gradient).
  // sep > 0: columns with col % sep in {0, sep-1} are separators of the virtual training batch -> t and out = 0.
  // dbg (benchmarking only, CTA 0): clock64 stamps [event][step], events: 0 f issued, 1 conv1 step issued,
  // 2 conv2 step issued, 3 epi1 got a block, 4 epi1 t row done, 5 epi2 got a block, 6 epi2 row stored
#define SR_DBG(ev, idx) \
  if (dbg && blockIdx.x == 0 && (idx) >= 0 && (idx) < 256) dbg[(ev) * 256 + (idx)] = clock64();
  // more MMA-thread stamps: 7 step start, 8 conv1 blocks acquired, 9 f row landed, 10 conv2 part start,
  // 11 conv2 blocks acquired, 12 t row ready, 13 epi1 freed a block (by row), 14 epi2 freed a block (by row)
  using Cfg = BlkCfg<C>;
  constexpr int CCH = Cfg::CCH, RB = Cfg::RB;
  // the bias-arming MMAs take their ones operand from 8 spare TMEM columns after ring 1 when there are any
  // (C = 48: columns 240..247; C = 16: 128..135), saving a 4 KB shared-memory read per arm
  constexpr bool kOnesTmem = RB * C + 8 <= 256;
  constexpr uint32_t PLANE = Cfg::PLANE, ROWB = Cfg::ROWB, OUTB = Cfg::OUTB;

  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sW1 = smem;
  uint8_t* sW2 = sW1 + Cfg::WB_AL;
  uint8_t* sF = sW2 + Cfg::WB_AL;
  uint8_t* sT = sF + kBlkNF * ROWB;
  uint8_t* sO = sT + kBlkNT * ROWB;
  uint8_t* sOnes = sO + kBlkNO * OUTB;       // bias-arming MMA operands (ring.cuh)
  uint8_t* sB1 = sOnes + kArmOnesBytes;
  uint8_t* sB2 = sB1 + 2 * C * 16;
  __shared__ __align__(8) uint64_t f_full[kBlkNF], f_empty[kBlkNF], t_full[kBlkNT], t_empty[kBlkNT], r1_ready[RB],
      r1_free[RB], r2_ready[RB], r2_free[RB], w_bar;
  __shared__ uint32_t tmem_base_sh;
  __shared__ __align__(16) float4 sb1v[C / 4], sb2v[C / 4];

  const int warp = warp_id();
  // spare t positions 128, 129 of every plane of every t slot are read by the two invalid conv2 lanes: zero them
  for (int i = threadIdx.x; i < kBlkNT * CCH * 2; i += blockDim.x) {
    const int slot = i / (CCH * 2), rem = i % (CCH * 2);
    *reinterpret_cast<uint4*>(sT + slot * ROWB + (rem / 2) * PLANE + (128 + rem % 2) * 16) = make_uint4(0, 0, 0, 0);
  }
  fence_proxy_async_smem();
  if (warp == 0 && lane_id() == 0) {
    for (int s = 0; s < kBlkNF; ++s) { mbar_init(&f_full[s], 1); mbar_init(&f_empty[s], 1); }
    for (int s = 0; s < kBlkNT; ++s) { mbar_init(&t_full[s], 4); mbar_init(&t_empty[s], 1); }
    for (int s = 0; s < RB; ++s) {
      mbar_init(&r1_ready[s], 1); mbar_init(&r1_free[s], 4);
      mbar_init(&r2_ready[s], 1); mbar_init(&r2_free[s], 4);
    }
    mbar_init(&w_bar, 1);
    fence_barrier_init();
  }
  if (warp == 1) tmem_alloc<512>(&tmem_base_sh);
  tc_fence_before();
  __syncthreads();
  if constexpr (kOnesTmem) {
    if (warp >= 2 && warp < 6) {  // warps 2..5 cover the four TMEM lane quarters
      tc_fence_after();
      ones_tmem_fill(tmem_base_sh + ((uint32_t)((warp & 3) * 32) << 16) + RB * C);
      tmem_st_wait();
      tc_fence_before();
    }
  }
  // Weights and biases were written at least two kernels upstream in every chain that launches this kernel (the
  // library's repack / publish precede at least the head conv; the kernel that wrote them completed before our
  // predecessor passed its own griddepcontrol.wait), so they are fetched and the bias-arming tiles built before the
  // PDL wait: on SMs the predecessor has already left, this overlaps its tail, and after the wait the producer's
  // first activation-row TMA goes out at once.
  if (warp == 0 && lane_id() == 0) {
    mbar_arrive_expect_tx(&w_bar, 2 * Cfg::WBYTES);
    bulk_load(sW1, w1, Cfg::WBYTES, &w_bar);
    bulk_load(sW2, w2, Cfg::WBYTES, &w_bar);
  }
  if (threadIdx.x < C) {
    reinterpret_cast<float*>(sb1v)[threadIdx.x] = b1[threadIdx.x];
    reinterpret_cast<float*>(sb2v)[threadIdx.x] = b2[threadIdx.x];
  }
  __syncthreads();
  arm_tiles_fill(sOnes, sB1, reinterpret_cast<const float*>(sb1v), C, threadIdx.x, blockDim.x);
  arm_tiles_fill(sOnes, sB2, reinterpret_cast<const float*>(sb2v), C, threadIdx.x, blockDim.x);
  fence_proxy_async_smem();
  __syncthreads();
  pdl_enter();
  tc_fence_after();
  const uint32_t tmem = tmem_base_sh;
  const uint32_t ring1 = tmem, ring2 = tmem + 256, ones_t = tmem + RB * C;
  auto arm1 = [&](unsigned gg) {
    if constexpr (kOnesTmem) ring_arm_ts<C, RB>(ring1, gg, ones_t, smem_u32(sB1));
    else ring_arm<C, RB>(ring1, gg, smem_u32(sOnes), smem_u32(sB1));
  };
  auto arm2 = [&](unsigned gg) {
    if constexpr (kOnesTmem) ring_arm_ts<C, RB>(ring2, gg, ones_t, smem_u32(sB2));
    else ring_arm<C, RB>(ring2, gg, smem_u32(sOnes), smem_u32(sB2));
  };

  const int tiles_x = (W + kBlkTW - 1) / kBlkTW;
  const long long total = (long long)N * tiles_x * H;
  const long long beg = total * blockIdx.x / gridDim.x, end = total * (blockIdx.x + 1) / gridDim.x;
#define SR_PIECE_BEGIN                                                                \
  for (long long pos = beg; pos < end;) {                                             \
    const int col = (int)(pos / H), y0 = (int)(pos - (long long)col * H);             \
    const int y1 = (int)min((long long)H, y0 + (end - pos));                          \
    pos += y1 - y0;                                                                   \
    const int n = col / tiles_x, x0 = (col - n * tiles_x) * kBlkTW;                   \
    const int n_f = y1 - y0 + 4, n_t = n_f - 2;                                       \
    (void)n; (void)x0; (void)n_t;
#define SR_PIECE_END }

  if (warp == 0) {
    // ===================== producer: weights once, then f rows y0-2 .. y1+1 of every piece =====================
    if (elect_one()) {
      tma_prefetch_desc(&tm_f);
      int s = 0;
      uint32_t ph = 0;
      SR_PIECE_BEGIN
      for (int i = 0; i < n_f; ++i) {
        mbar_wait(&f_empty[s], ph ^ 1);
        if ((exp & 128) && pos > beg + 8) {
          mbar_arrive(&f_full[s]);
        } else {
          mbar_arrive_expect_tx(&f_full[s], CCH * PLANE);
          tma_load_5d(sF + s * ROWB, &tm_f, &f_full[s], 0, x0 - 2, y0 - 2 + i, 0, n);
        }
        SR_DBG(0, i)
        if (++s == kBlkNF) { s = 0; ph ^= 1; }
      }
      SR_PIECE_END
    }
    __syncwarp();
  } else if (warp == 1) {
    // ===================== conv1 MMA issuer: step st consumes f row st =====================
    // (conv2 has its own issuer, warp 10: while one thread waits on a barrier the other keeps the tensor pipe fed)
    if (elect_one()) {
      mbar_wait(&w_bar, 0);
      const uint64_t bd1 = make_desc(smem_u32(sW1), Cfg::N * 16, 128);
      int fs = 0;
      uint32_t fph = 0;
      unsigned G1 = 0, acq1 = 0;  // out-row sequence (first row of the piece) / blocks acquired
      SR_PIECE_BEGIN
      for (int st = 0; st < n_f; ++st) {
        SR_DBG(7, st)
        const unsigned g = G1 + st;
        for (; acq1 < g + 3; ++acq1) mbar_wait(&r1_free[ring_idx<RB>(acq1)], (uint32_t)(acq1 / RB) & 1u);
        SR_DBG(8, st)
        mbar_wait(&f_full[fs], fph);
        SR_DBG(9, st)
        tc_fence_after();
        if (st == 0) {  // the piece's first two rows receive no earlier contribution
          arm1(g);
          arm1(g + 1);
        }
        arm1(g + 2);  // its first contribution comes now
        if (!(exp & 32))
          ring_mma_step<C, C, RB>(ring1, g, make_desc(smem_u32(sF + fs * ROWB), PLANE, 128), bd1, 2 * PLANE);
        mma_commit(&r1_ready[ring_idx<RB>(g)]);  // out row g (dy=2 target) is complete
        mma_commit(&f_empty[fs]);
        if (st == n_f - 1) {                      // the last two rows of the piece receive nothing more
          mma_commit(&r1_ready[ring_idx<RB>(g + 1)]);
          mma_commit(&r1_ready[ring_idx<RB>(g + 2)]);
        }
        SR_DBG(1, st)
        if (++fs == kBlkNF) { fs = 0; fph ^= 1; }
      }
      G1 += n_f + 2;
      SR_PIECE_END
    }
    __syncwarp();
  } else if (warp == 10) {
    // ===================== conv2 MMA issuer: step k consumes t row k =====================
    if (elect_one()) {
      mbar_wait(&w_bar, 0);
      const uint64_t bd2 = make_desc(smem_u32(sW2), Cfg::N * 16, 128);
      int ts = 0;
      uint32_t tph = 0;
      unsigned G2 = 0, acq2 = 0;
      SR_PIECE_BEGIN
      for (int k = 0; k < n_t; ++k) {
        SR_DBG(10, k + 3)
        const unsigned g = G2 + k;
        for (; acq2 < g + 3; ++acq2) mbar_wait(&r2_free[ring_idx<RB>(acq2)], (uint32_t)(acq2 / RB) & 1u);
        SR_DBG(11, k + 3)
        mbar_wait(&t_full[ts], tph);
        SR_DBG(12, k + 3)
        tc_fence_after();
        if (k == 0) {
          arm2(g);
          arm2(g + 1);
        }
        arm2(g + 2);
        if (!(exp & 16))
          ring_mma_step<C, C, RB>(ring2, g, make_desc(smem_u32(sT + ts * ROWB), PLANE, 128), bd2, 2 * PLANE);
        mma_commit(&r2_ready[ring_idx<RB>(g)]);
        mma_commit(&t_empty[ts]);
        if (k == n_t - 1) {
          mma_commit(&r2_ready[ring_idx<RB>(g + 1)]);
          mma_commit(&r2_ready[ring_idx<RB>(g + 2)]);
        }
        SR_DBG(2, k)
        if (++ts == kBlkNT) { ts = 0; tph ^= 1; }
      }
      G2 += n_t + 2;
      SR_PIECE_END
    }
    __syncwarp();
  } else if (warp < 6) {
    // ===================== conv1 epilogue: drain finished t rows -> ReLU -> t smem ring =====================
    const int quarter = warp & 3;
    const int m = quarter * 32 + lane_id();
    const uint32_t lane_off = (uint32_t)(quarter * 32) << 16;
    for (int b = 0; b < RB; ++b)  // every ring block starts free (the MMA issuer arms blocks itself)
      if (lane_id() == 0) mbar_arrive(&r1_free[b]);
    int ts = 0;
    uint32_t tph = 0;
    unsigned G = 0;
    SR_PIECE_BEGIN
    const int tcol = x0 - 1 + m;
    const bool col_ok = tcol >= 0 && tcol < W && !(sep > 0 && ((tcol % max(sep, 1)) == 0 || (tcol % max(sep, 1)) == sep - 1));
    const bool save_col = tsave != nullptr && m >= 1 && m <= kBlkTW && tcol < W;  // this strip's own columns
    // backward mode: the ReLU' mask row (saved forward t) is loaded one row ahead, like the residual below
    uint4 mk_nx[BWD ? C / 8 : 1];
    auto ld_mask = [&](int q) {
      const int trow = y0 - 2 + q;
      if (BWD && q >= 1 && q <= n_f - 2 && col_ok && trow >= 0 && trow < H) {
        const uint4* mp = reinterpret_cast<const uint4*>(mask + ((((size_t)n * H + trow) * W) + tcol) * C);
#pragma unroll
        for (int j = 0; j < C / 8; ++j) mk_nx[j] = __ldg(mp + j);
      }
    };
    ld_mask(-1);
    for (int q = -1; q <= n_f; ++q) {         // out rows of conv1 = t rows y0-2+q
      const unsigned g = G + q + 1;
      const bool emit = q >= 1 && q <= n_f - 2;
      const int trow = y0 - 2 + q;
      const bool ok = col_ok && trow >= 0 && trow < H;
      uint4 mk[BWD ? C / 8 : 1];
      if constexpr (BWD) {
#pragma unroll
        for (int j = 0; j < C / 8; ++j) mk[j] = mk_nx[j];
        ld_mask(q + 1);
      }
      if (emit) mbar_wait(&t_empty[ts], tph ^ 1);
      const int b = ring_idx<RB>(g);
      mbar_wait(&r1_ready[b], (uint32_t)(g / RB) & 1u);
      tc_fence_after();
      if (warp == 2 && lane_id() == 0) { SR_DBG(3, q + 1) }
      float v[C];
      if (exp & 72) {
        if (!(exp & 64)) {
#pragma unroll
          for (int c0 = 0; c0 < C; c0 += 8) tmem_ld8(ring1 + lane_off + b * C + c0, v + c0);
          tmem_ld_wait();
        } else {
#pragma unroll
          for (int c0 = 0; c0 < C; ++c0) v[c0] = (float)c0;
        }
      } else {
#pragma unroll
        for (int c0 = 0; c0 < C; c0 += 8) tmem_ld8(ring1 + lane_off + b * C + c0, v + c0);
        tmem_ld_wait();
      }
      tc_fence_before();
      __syncwarp();
      if (lane_id() == 0) mbar_arrive(&r1_free[b]);
      if (warp == 2 && lane_id() == 0) { SR_DBG(13, q + 1) }
      if (emit && !(exp & 4)) {
        uint8_t* dst = sT + ts * ROWB + m * 16;
#pragma unroll
        for (int j = 0; j < CCH; ++j) {
          float a[8];
          if constexpr (BWD) {  // ReLU' = 1[t > 0] of the forward t
            const __nv_bfloat162* h2 = reinterpret_cast<const __nv_bfloat162*>(&mk[j]);
#pragma unroll
            for (int e = 0; e < 4; ++e) {
              const float2 f2 = __bfloat1622float2(h2[e]);
              a[2 * e] = ok && f2.x > 0.f ? v[8 * j + 2 * e] : 0.f;
              a[2 * e + 1] = ok && f2.y > 0.f ? v[8 * j + 2 * e + 1] : 0.f;
            }
          } else {
#pragma unroll
            for (int e = 0; e < 8; ++e) a[e] = ok ? fmaxf(v[8 * j + e], 0.f) : 0.f;
          }
          uint4 u;
          u.x = pack_bf16x2(a[0], a[1]);
          u.y = pack_bf16x2(a[2], a[3]);
          u.z = pack_bf16x2(a[4], a[5]);
          u.w = pack_bf16x2(a[6], a[7]);
          *reinterpret_cast<uint4*>(dst + j * PLANE) = u;
          if (save_col && q >= 2 && q <= n_f - 3)  // t rows y0 .. y1-1 belong to this piece
            reinterpret_cast<uint4*>(tsave + ((((size_t)n * H + trow) * W) + tcol) * C)[j] = u;
        }
      }
      if (emit) {
        fence_proxy_async_smem();
        __syncwarp();
        if (lane_id() == 0) mbar_arrive(&t_full[ts]);
        if (warp == 2 && lane_id() == 0) { SR_DBG(4, q + 1) }
        if (++ts == kBlkNT) { ts = 0; tph ^= 1; }
      }
    }
    G += n_f + 2;
    SR_PIECE_END
  } else if (warp < 10) {
    // ===================== conv2 epilogue: drain finished rows -> + residual f -> smem -> TMA store ==========
    const int quarter = warp & 3;
    const int m = quarter * 32 + lane_id();
    const uint32_t lane_off = (uint32_t)(quarter * 32) << 16;
    const bool leader = (warp == 6 && lane_id() == 0);
    for (int b = 0; b < RB; ++b)
      if (lane_id() == 0) mbar_arrive(&r2_free[b]);
    int os = 0;
    unsigned G = 0;
    SR_PIECE_BEGIN
    const bool lane_ok = m < kBlkTW && x0 + m < W;
    const bool sep0 = sep > 0 && (((x0 + m) % max(sep, 1)) == 0 || ((x0 + m) % max(sep, 1)) == sep - 1);
    // the residual row is loaded ahead (res_nx: one row; at C <= 32, where a row-step is only ~660 cycles, two rows
    // through res_nx2), so its L2/HBM latency overlaps whole row-steps
    constexpr int kAhead = (C <= 32 && !BWD) ? 2 : 1;  // (BWD keeps res2 one row ahead alongside)
    uint4 res_nx[C / 8], res_nx2[kAhead > 1 ? C / 8 : 1];
    uint4 r2_nx[BWD ? C / 8 : 1];
    auto ld_res = [&](int q) {
      if (q >= 1 && q <= n_t - 2 && lane_ok && !(exp & 1)) {
        const size_t pix = (((size_t)n * H + y0 - 1 + q) * W) + x0 + m;
        const uint4* rp = reinterpret_cast<const uint4*>(fres + pix * C);
#pragma unroll
        for (int j = 0; j < C / 8; ++j) (kAhead > 1 ? res_nx2 : res_nx)[j] = __ldg(rp + j);
        if (BWD && res2) {
          const uint4* rp2 = reinterpret_cast<const uint4*>(res2 + pix * C);
#pragma unroll
          for (int j = 0; j < C / 8; ++j) r2_nx[j] = __ldg(rp2 + j);
        }
      }
    };
    ld_res(-1);
    if constexpr (kAhead > 1) {
#pragma unroll
      for (int j = 0; j < C / 8; ++j) res_nx[j] = res_nx2[j];
      ld_res(0);
    }
    for (int q = -1; q <= n_t; ++q) {         // out rows of conv2 = output rows y0-1+q
      const unsigned g = G + q + 1;
      const bool emit = q >= 1 && q <= n_t - 2;
      const int r = y0 - 1 + q;
      uint4 res[C / 8], rs2[BWD ? C / 8 : 1];
#pragma unroll
      for (int j = 0; j < C / 8; ++j) res[j] = res_nx[j];
      if constexpr (kAhead > 1) {
#pragma unroll
        for (int j = 0; j < C / 8; ++j) res_nx[j] = res_nx2[j];
      }
      if (BWD && res2) {
#pragma unroll
        for (int j = 0; j < C / 8; ++j) rs2[j] = r2_nx[j];
      }
      ld_res(q + kAhead);
      const int b = ring_idx<RB>(g);
      mbar_wait(&r2_ready[b], (uint32_t)(g / RB) & 1u);
      tc_fence_after();
      if (warp == 6 && lane_id() == 0) { SR_DBG(5, q + 1) }
      if (exp & 1) {
#pragma unroll
        for (int j = 0; j < C / 8; ++j) res[j] = make_uint4(0, 0, 0, 0);
      }
      float v[C];
      if (exp & 72) {
        if (!(exp & 64)) {
#pragma unroll
          for (int c0 = 0; c0 < C; c0 += 8) tmem_ld8(ring2 + lane_off + b * C + c0, v + c0);
          tmem_ld_wait();
        } else {
#pragma unroll
          for (int c0 = 0; c0 < C; ++c0) v[c0] = (float)c0;
        }
      } else {
#pragma unroll
        for (int c0 = 0; c0 < C; c0 += 8) tmem_ld8(ring2 + lane_off + b * C + c0, v + c0);
        tmem_ld_wait();
      }
      tc_fence_before();
      __syncwarp();
      if (lane_id() == 0) mbar_arrive(&r2_free[b]);
      if (warp == 6 && lane_id() == 0) { SR_DBG(14, q + 1) }
      if (emit) {
        if (lane_ok && !(exp & 2)) {
          uint8_t* orow = sO + os * OUTB + m * C * 2;
          uint4 ov[C / 8];
#pragma unroll
          for (int j = 0; j < C / 8; ++j) {
            const __nv_bfloat162* h2 = reinterpret_cast<const __nv_bfloat162*>(&res[j]);
            float a[8];
#pragma unroll
            for (int e = 0; e < 4; ++e) {
              const float2 f2 = __bfloat1622float2(h2[e]);
              a[2 * e] = v[8 * j + 2 * e] + f2.x;
              a[2 * e + 1] = v[8 * j + 2 * e + 1] + f2.y;
            }
            if (BWD && res2) {
              const __nv_bfloat162* g2 = reinterpret_cast<const __nv_bfloat162*>(&rs2[j]);
#pragma unroll
              for (int e = 0; e < 4; ++e) {
                const float2 f2 = __bfloat1622float2(g2[e]);
                a[2 * e] += f2.x;
                a[2 * e + 1] += f2.y;
              }
            }
            if (sep0) {
#pragma unroll
              for (int e = 0; e < 8; ++e) a[e] = 0.f;
            }
            uint4 u;
            u.x = pack_bf16x2(a[0], a[1]);
            u.y = pack_bf16x2(a[2], a[3]);
            u.z = pack_bf16x2(a[4], a[5]);
            u.w = pack_bf16x2(a[6], a[7]);
            ov[j] = u;
          }
          // lane-rotated chunk order: conflict-free 16-B stores into the pixel-major staging row (rot.cuh; at
          // C = 32 the 64-B pixel stride makes a plain chunk loop 4-way conflicted)
          st_pix_rot<C / 8>(orow, ov);
        }
        fence_proxy_async_smem();
        named_bar_sync(2, 128);
        if (leader && !(exp & 2)) {
          tma_store_4d(&tm_out, sO + os * OUTB, 0, x0, r, n);
          bulk_commit();
          bulk_wait_read<kBlkNO - 2>();
          SR_DBG(6, q + 1)
        }
        os = os == kBlkNO - 1 ? 0 : os + 1;
      }
    }
    G += n_t + 2;
    SR_PIECE_END
    if (leader) bulk_wait<0>();
  }
#undef SR_PIECE_BEGIN
#undef SR_PIECE_END
#undef SR_DBG
  tc_fence_before();
  __syncthreads();
  if (warp == 1) tmem_dealloc<512>(tmem);
}

static int g_block_gen = -1;
void set_block_gen(int g) { g_block_gen = g; }

template <int C>
static cudaError_t launch_block_t(const CUtensorMap& tf, const CUtensorMap& to, const bf16* w1, const bf16* w2,
                                  const float* b1, const float* b2, const bf16* f, bf16* out, int N, int H, int W,
                                  int grid, bf16* tsave, int sep, long long* dbg, int exp, const bf16* mask,
                                  const bf16* res2, cudaStream_t st) {
  int ki = mask ? ((dbg || exp) ? 4 : 3) : ((dbg || exp) ? 2 : ((tsave || sep > 0) ? 1 : 0));
  if (!mask && g_block_gen > ki) ki = g_block_gen;  // benchmarking only: a more general instantiation
  auto kern = ki == 4 ? k_resblock<C, true, 2> : ki == 3 ? k_resblock<C, true, 1>
                      : (ki == 2 ? k_resblock<C, false, 2> : (ki == 1 ? k_resblock<C, false, 1> : k_resblock<C, false, 0>));
  static bool configured[5] = {false, false, false, false, false};
  if (!configured[ki]) {
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)BlkCfg<C>::SMEM);
    if (e != cudaSuccess) return e;
    configured[ki] = true;
  }
  return launch_k(kern, dim3(grid), dim3(kBlkThreads), BlkCfg<C>::SMEM, st, tf, to, w1, w2, b1, b2, f, out, N, H, W,
                  tsave, sep, dbg, exp, mask, res2);
}

bool resblock_supported(int cp, int W) {
  if (W < 96) return false;
  if (cp == 16) return BlkCfg<16>::SMEM <= 227 * 1024;
  if (cp == 32) return BlkCfg<32>::SMEM <= 227 * 1024;
  if (cp == 48) return BlkCfg<48>::SMEM <= 227 * 1024;
  return false;
}

cudaError_t launch_resblock(int cp, const bf16* f, const bf16* w1fold, const bf16* w2fold, const float* b1,
                            const float* b2, bf16* out, int N, int H, int W, cudaStream_t st, long long* dbg,
                            bf16* tsave, int sep, int exp, const bf16* mask, const bf16* res2) {
  CUtensorMap tf, to;
  if (make_act_tmap(&tf, f, N, H, W, cp, 130, 1, cp / 8, CHUNK_ROW_PIX) != CUDA_SUCCESS) return cudaErrorInvalidValue;
  if (make_row_tmap(&to, out, N, H, W, cp, kBlkTW, cp) != CUDA_SUCCESS) return cudaErrorInvalidValue;
  const long long rows = (long long)N * ((W + kBlkTW - 1) / kBlkTW) * H;
  int grid = num_sms();
  if (rows < grid) grid = (int)rows;
  if (cp == 16)
    return launch_block_t<16>(tf, to, w1fold, w2fold, b1, b2, f, out, N, H, W, grid, tsave, sep, dbg, exp, mask, res2, st);
  if (cp == 32)
    return launch_block_t<32>(tf, to, w1fold, w2fold, b1, b2, f, out, N, H, W, grid, tsave, sep, dbg, exp, mask, res2, st);
  if (cp == 48)
    return launch_block_t<48>(tf, to, w1fold, w2fold, b1, b2, f, out, N, H, W, grid, tsave, sep, dbg, exp, mask, res2, st);
  return cudaErrorNotSupported;
}

}  // namespace sr

// Fused body conv + up conv + tail for wide frames (sm_100a tcgen05):
//   g   = f0 + conv_body(f) + b_body                               (global skip, reading R1)
//   out = RNE(clamp(255 PS_s(conv_up(g) + b_up) + skip_s(v), 0, 255))   (A3 + A4 of SURVEY §8(a))
//
// Unfused, the body conv writes g (2C B/px) and the up conv reads it back (2C B/px + halo): 192 B/px of the
// 414 B/px the two kernels move at C = 48.  Here g never leaves the SM -- the structure of the fused residual
// block (conv_block.cu): conv1 = the body conv (dy-fold, N = 3C), its epilogue adds f0 and writes g rows into a
// shared-memory ring; conv2 = the up conv (dy-fold, N = 3 CO2) reads g rows from that ring; its epilogue is the
// tail.  HBM per LR pixel: f and f0 once (+2 halo columns per 126), the LR frame (5 rows per output row, L2), the
// HR bytes once.
//
// Column strip of 126 output pixels starting at x0 (MMA M = 128 lanes), as conv_block.cu:
//   f row in smem : pixels x0-2 .. x0+127 (130, TMA, zero outside the frame)
//   conv1 lane m  : g column x0-1+m                 -> g row in smem (128 + 2 spare positions)
//   conv2 lane m  : out column x0+m (m < 126), reads g positions m+dx; g is 0 outside the frame (zero padding).
// Tail: the producer TMA-loads LR rows r-2..r+2 of every output row r into a ring (u8 rows map, 16-B chunks,
// W % 16 == 0); the epilogue computes the S x S x 3 bytes of its pixel into an S-row staging buffer whose rows are
// placed at the destination's address mod 16, then the four warps copy the rows out with 16-B stores (126-pixel
// strips are not 16-B aligned in the HR frame, so a TMA store box cannot tile them).
//
// Warps: 0 TMA producer (f rows, LR rows), 1 TMEM alloc + conv1 MMA issuer, 10 conv2 MMA issuer, 2..5 conv1
// epilogue (+f0 -> g smem), 6..9 and 11..14 two tail epilogue groups taking alternate output rows (the tail's
// per-row chain -- drain, 27 skip/clamp/round, staging, copy-out -- is twice the tensor time of a row-step).
#include <cuda.h>
#include "ptx.cuh"
#include "tmap.h"
#include "sr_internal.h"
#include "ring.cuh"
#include "launch.cuh"
#include "tail.cuh"
#include "color.cuh"

namespace sr {

static constexpr int kBtThreads = 480;  // 15 warps: two tail epilogue groups
// C <= 32: a second body-conv epilogue group (warps 15..18) on alternate g rows
template <int C>
struct BtThreads {
  static constexpr int EPI1 = C <= 32 ? 2 : 1;
  static constexpr int N = kBtThreads + (EPI1 - 1) * 128;
};
static constexpr int kBtTW = 126;  // output pixels per strip
static constexpr int kBtNF = 4;    // f-row ring (C = 48)
static constexpr int kBtNT = 4;    // g-row ring (C = 48)
static constexpr int kBtNO = 3;    // HR staging slots per tail group
static constexpr int kBtLrChunks = 26;  // LR bytes [16 cb, 16 cb + 416) cover pixels x0-2 .. x0+129
static constexpr uint32_t kBtLrSlot = (16 * kBtLrChunks * 5 + 127) & ~127u;

template <int C, int CO2, int S>
struct BtCfg {
  // TMEM: ring2 (up conv, blocks of CO2 columns) at the top, ring1 (body conv, C columns) below it
  static constexpr int RB2 = CO2 == 16 ? 8 : (CO2 == 32 ? 6 : 5);
  static constexpr int R2BASE = 512 - RB2 * CO2;
  static constexpr int RB1 = (R2BASE / C) < 8 ? (R2BASE / C) : 8;
  static constexpr uint32_t W1B = 9u * C * C * 2u, W2B = 9u * C * CO2 * 2u;
  static constexpr uint32_t W1_AL = (W1B + 1023u) & ~1023u, W2_AL = (W2B + 1023u) & ~1023u;
  static constexpr uint32_t PLANE = 130 * 16;
  static constexpr uint32_t ROWB = (((C / 8) * PLANE) + 127u) & ~127u;
  static constexpr uint32_t HRP = ((kBtTW * S * 3 + 15u) & ~15u) + 16u;  // staging row pitch (+16: alignment shift)
  static constexpr uint32_t OUTB = ((S * HRP) + 127u) & ~127u;
  static constexpr uint32_t ARMB = ((kArmOnesBytes + C * 32 + CO2 * 32) + 1023u) & ~1023u;
  // f- and g-row ring depths: 4 at C = 48 (shared memory is full); at C <= 32 as deep as fits with >= 8 LR slots,
  // up to 8 (config 2's body + tail: 0.91 -> 0.77 ms per 30 540p frames from 4 to 8, profiles/r02_ab_bodytail.log)
  static constexpr size_t base_at(int d) {
    return 1024 + W1_AL + W2_AL + (size_t)2 * d * ROWB + (size_t)2 * kBtNO * OUTB + ARMB;
  }
  static constexpr int fit_lr(int d) { return (int)(((long long)227 * 1024 - 2048 - (long long)base_at(d)) / kBtLrSlot); }
  static constexpr int DEPTH = C >= 48 ? kBtNF : (fit_lr(8) >= 8 ? 8 : (fit_lr(6) >= 8 ? 6 : kBtNF));
  static constexpr int NF = DEPTH, NT = DEPTH;
  static constexpr size_t BASE = base_at(DEPTH);
  static constexpr int NLR_FIT = (int)((227 * 1024 - 2048 - BASE) / kBtLrSlot);  // 2 KB: static smem (barriers)
  static constexpr int NLR = NLR_FIT > 12 ? 12 : NLR_FIT;
  static constexpr bool FITS = NLR >= 4;
  static constexpr size_t SMEM = BASE + (size_t)(NLR > 0 ? NLR : 0) * kBtLrSlot;
};

struct BtArgs {
  const float* b1;
  const float* b2;
  const bf16* f0;    // global-skip residual [N,H,W,C]
  const uint8_t* lr;  // [N,H,W,3]
  uint8_t* hr;        // [N,sH,sW,3]
  int N, H, W;
  int hr_row0, hr_row1;  // LR rows whose HR rows are written (strip mode)
  int bicubic;
  long long* dbg;  // benchmarking only: CTA-0 clock64 stamps [event][row]
  // I420 output (k_bodytail<..., YO = true>, S = 2 or 4: a lane's S x S HR block holds whole 2x2 chroma blocks):
  // planes hy [N][sH][sW], hu / hv [N][sH/2][sW/2] instead of the RGB frame hr
  uint8_t* hy;
  uint8_t* hu;
  uint8_t* hv;
};
#define SR_BDBG(ev, idx) \
  if (a.dbg && blockIdx.x == 0 && (idx) >= 0 && (idx) < 256) a.dbg[(ev) * 256 + (idx)] = clock64();

// BIC: bicubic skip (else bilinear).  A template parameter, so each kernel carries only its own tail code
// (k_bodytail<48,32,3> -3.4% with the bicubic code compiled out, scripts/bt_time.py A/B).  The kernel is very
// sensitive to code shape: compiling the (null-checked) clock64 stamps out made it 10% slower, a runtime
// experiment mask 13% slower -- measure every change to it.
template <int C, int CO2, int S, bool BIC, bool YO = false>
__global__ void __launch_bounds__(BtThreads<C>::N, 1)
k_bodytail(const __grid_constant__ CUtensorMap tm_f, const __grid_constant__ CUtensorMap tm_lr,
           const bf16* __restrict__ w1, const bf16* __restrict__ w2, const BtArgs a) {
  using Cfg = BtCfg<C, CO2, S>;
  constexpr int CCH = C / 8, RB1 = Cfg::RB1, RB2 = Cfg::RB2, NLR = Cfg::NLR;
  constexpr uint32_t PLANE = Cfg::PLANE, ROWB = Cfg::ROWB, OUTB = Cfg::OUTB, HRP = Cfg::HRP;

  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sW1 = smem;
  uint8_t* sW2 = sW1 + Cfg::W1_AL;
  uint8_t* sF = sW2 + Cfg::W2_AL;
  constexpr int kNF = Cfg::NF, kNT = Cfg::NT;
  uint8_t* sT = sF + kNF * ROWB;
  uint8_t* sO = sT + kNT * ROWB;
  uint8_t* sOnes = sO + 2 * kBtNO * OUTB;
  uint8_t* sB1 = sOnes + kArmOnesBytes;
  uint8_t* sB2 = sB1 + C * 32;
  uint8_t* sL = sOnes + Cfg::ARMB;
  __shared__ __align__(8) uint64_t f_full[kNF], f_empty[kNF], t_full[kNT], t_empty[kNT], r1_ready[RB1],
      r1_free[RB1], r2_ready[RB2], r2_free[RB2], l_full[NLR], l_empty[NLR], w_bar;
  __shared__ uint32_t tmem_base_sh;

  const int N = a.N, H = a.H, W = a.W;
  const int warp = warp_id();
  // spare g positions 128, 129 of every plane of every g slot are read by the two invalid conv2 lanes: zero them
  for (int i = threadIdx.x; i < kNT * CCH * 2; i += blockDim.x) {
    const int slot = i / (CCH * 2), rem = i % (CCH * 2);
    *reinterpret_cast<uint4*>(sT + slot * ROWB + (rem / 2) * PLANE + (128 + rem % 2) * 16) = make_uint4(0, 0, 0, 0);
  }
  fence_proxy_async_smem();
  if (warp == 0 && lane_id() == 0) {
    for (int s = 0; s < kNF; ++s) { mbar_init(&f_full[s], 1); mbar_init(&f_empty[s], 1); }
    for (int s = 0; s < kNT; ++s) { mbar_init(&t_full[s], 4); mbar_init(&t_empty[s], 1); }
    for (int s = 0; s < RB1; ++s) { mbar_init(&r1_ready[s], 1); mbar_init(&r1_free[s], 4); }
    for (int s = 0; s < RB2; ++s) { mbar_init(&r2_ready[s], 1); mbar_init(&r2_free[s], 4); }
    for (int s = 0; s < NLR; ++s) { mbar_init(&l_full[s], 1); mbar_init(&l_empty[s], 1); }
    mbar_init(&w_bar, 1);
    fence_barrier_init();
  }
  if (warp == 1) tmem_alloc<512>(&tmem_base_sh);
  tc_fence_before();
  __syncthreads();
  // weights + biases before the PDL wait (written >= 2 kernels upstream; see k_resblock's prologue)
  if (warp == 0 && lane_id() == 0) {
    mbar_arrive_expect_tx(&w_bar, Cfg::W1B + Cfg::W2B);
    bulk_load(sW1, w1, Cfg::W1B, &w_bar);
    bulk_load(sW2, w2, Cfg::W2B, &w_bar);
  }
  arm_tiles_fill(sOnes, sB1, a.b1, C, threadIdx.x, blockDim.x);
  arm_tiles_fill(sOnes, sB2, a.b2, CO2, threadIdx.x, blockDim.x);
  fence_proxy_async_smem();
  // the arming MMAs take their ones operand from 8 spare TMEM columns after ring 1 when there are any (ring.cuh)
  constexpr bool kOnesTmem = RB1 * C + 8 <= Cfg::R2BASE;
  if constexpr (kOnesTmem) {
    if (warp >= 2 && warp < 6) {
      tc_fence_after();
      ones_tmem_fill(tmem_base_sh + ((uint32_t)((warp & 3) * 32) << 16) + RB1 * C);
      tmem_st_wait();
      tc_fence_before();
    }
  }
  __syncthreads();
  pdl_enter();
  tc_fence_after();
  const uint32_t tmem = tmem_base_sh;
  const uint32_t ring1 = tmem, ring2 = tmem + Cfg::R2BASE, ones_t = tmem + RB1 * C;
  auto arm1 = [&](unsigned gg) {
    if constexpr (kOnesTmem) ring_arm_ts<C, RB1>(ring1, gg, ones_t, smem_u32(sB1));
    else ring_arm<C, RB1>(ring1, gg, smem_u32(sOnes), smem_u32(sB1));
  };
  auto arm2 = [&](unsigned gg) {
    if constexpr (kOnesTmem) ring_arm_ts<CO2, RB2>(ring2, gg, ones_t, smem_u32(sB2));
    else ring_arm<CO2, RB2>(ring2, gg, smem_u32(sOnes), smem_u32(sB2));
  };

  const int tiles_x = (W + kBtTW - 1) / kBtTW;
  const long long total = (long long)N * tiles_x * H;
  const long long beg = total * blockIdx.x / gridDim.x, end = total * (blockIdx.x + 1) / gridDim.x;
#define SR_PIECE_BEGIN                                                                \
  for (long long pos = beg; pos < end;) {                                             \
    const int col = (int)(pos / H), y0 = (int)(pos - (long long)col * H);             \
    const int y1 = (int)min((long long)H, y0 + (end - pos));                          \
    pos += y1 - y0;                                                                   \
    const int n = col / tiles_x, x0 = (col - n * tiles_x) * kBtTW;                    \
    const int n_f = y1 - y0 + 4, n_t = n_f - 2;                                       \
    (void)n; (void)x0; (void)n_t;
#define SR_PIECE_END }

  if (warp == 0) {
    // ============ producer: weights once; per piece f rows y0-2 .. y1+1 and LR rows of output rows y0 .. y1-1 ======
    if (elect_one()) {
      tma_prefetch_desc(&tm_f);
      tma_prefetch_desc(&tm_lr);
      int s = 0, ls = 0;
      uint32_t ph = 0, lph = 0;
      SR_PIECE_BEGIN
      for (int i = 0; i < n_f; ++i) {
        mbar_wait(&f_empty[s], ph ^ 1);
        mbar_arrive_expect_tx(&f_full[s], CCH * PLANE);
        tma_load_5d(sF + s * ROWB, &tm_f, &f_full[s], 0, x0 - 2, y0 - 2 + i, 0, n);
        SR_BDBG(0, i)
        if (++s == kNF) { s = 0; ph ^= 1; }
        if (i >= 4) {  // f row y0-2+i is the last one output row r = y0+i-4 needs: its LR rows r-2 .. r+2 now
          mbar_wait(&l_empty[ls], lph ^ 1);
          mbar_arrive_expect_tx(&l_full[ls], 16 * kBtLrChunks * 5);
          tma_load_4d(sL + ls * kBtLrSlot, &tm_lr, &l_full[ls], 0, (3 * x0 - 6) >> 4, y0 + i - 6, n);
          if (++ls == NLR) { ls = 0; lph ^= 1; }
        }
      }
      SR_PIECE_END
    }
    __syncwarp();
  } else if (warp == 1) {
    // ===================== conv1 (body) MMA issuer: step st consumes f row st =====================
    if (elect_one()) {
      mbar_wait(&w_bar, 0);
      const uint64_t bd1 = make_desc(smem_u32(sW1), 3 * C * 16, 128);
      int fs = 0;
      uint32_t fph = 0;
      unsigned G1 = 0, acq1 = 0;
      SR_PIECE_BEGIN
      for (int st = 0; st < n_f; ++st) {
        const unsigned g = G1 + st;
        SR_BDBG(7, st)
        for (; acq1 < g + 3; ++acq1) mbar_wait(&r1_free[ring_idx<RB1>(acq1)], (uint32_t)(acq1 / RB1) & 1u);
        SR_BDBG(8, st)
        mbar_wait(&f_full[fs], fph);
        SR_BDBG(9, st)
        tc_fence_after();
        if (st == 0) {
          arm1(g);
          arm1(g + 1);
        }
        arm1(g + 2);
        ring_mma_step<C, C, RB1>(ring1, g, make_desc(smem_u32(sF + fs * ROWB), PLANE, 128), bd1, 2 * PLANE);
        mma_commit(&r1_ready[ring_idx<RB1>(g)]);
        mma_commit(&f_empty[fs]);
        SR_BDBG(1, st)
        if (st == n_f - 1) {
          mma_commit(&r1_ready[ring_idx<RB1>(g + 1)]);
          mma_commit(&r1_ready[ring_idx<RB1>(g + 2)]);
        }
        if (++fs == kNF) { fs = 0; fph ^= 1; }
      }
      G1 += n_f + 2;
      SR_PIECE_END
    }
    __syncwarp();
  } else if (warp == 10) {
    // ===================== conv2 (up conv) MMA issuer: step k consumes g row k =====================
    if (elect_one()) {
      mbar_wait(&w_bar, 0);
      const uint64_t bd2 = make_desc(smem_u32(sW2), 3 * CO2 * 16, 128);
      int ts = 0;
      uint32_t tph = 0;
      unsigned G2 = 0, acq2 = 0;
      SR_PIECE_BEGIN
      for (int k = 0; k < n_t; ++k) {
        const unsigned g = G2 + k;
        SR_BDBG(10, k + 3)
        for (; acq2 < g + 3; ++acq2) mbar_wait(&r2_free[ring_idx<RB2>(acq2)], (uint32_t)(acq2 / RB2) & 1u);
        SR_BDBG(11, k + 3)
        mbar_wait(&t_full[ts], tph);
        SR_BDBG(12, k + 3)
        tc_fence_after();
        if (k == 0) {
          arm2(g);
          arm2(g + 1);
        }
        arm2(g + 2);
        ring_mma_step<C, CO2, RB2>(ring2, g, make_desc(smem_u32(sT + ts * ROWB), PLANE, 128), bd2, 2 * PLANE);
        mma_commit(&r2_ready[ring_idx<RB2>(g)]);
        mma_commit(&t_empty[ts]);
        SR_BDBG(2, k)
        if (k == n_t - 1) {
          mma_commit(&r2_ready[ring_idx<RB2>(g + 1)]);
          mma_commit(&r2_ready[ring_idx<RB2>(g + 2)]);
        }
        if (++ts == kNT) { ts = 0; tph ^= 1; }
      }
      G2 += n_t + 2;
      SR_PIECE_END
    }
    __syncwarp();
  } else if (BtThreads<C>::EPI1 == 2 && (warp < 6 || warp >= 15)) {
    // ============ conv1 epilogue, two groups (C <= 32): alternate g rows; g slots follow the emitted-row order ======
    constexpr int EPI1 = BtThreads<C>::EPI1;
    const int grp = warp >= 15 ? 1 : 0;
    const int quarter = warp & 3;
    const int m = quarter * 32 + lane_id();
    const uint32_t lane_off = (uint32_t)(quarter * 32) << 16;
    if (grp == 0)
      for (int b = 0; b < RB1; ++b)
        if (lane_id() == 0) mbar_arrive(&r1_free[b]);
    unsigned G = 0, E = 0;  // E: g rows emitted by both groups in earlier pieces
    SR_PIECE_BEGIN
    const int tcol = x0 - 1 + m;
    const bool col_ok = tcol >= 0 && tcol < W;
    uint4 res_nx[CCH];  // f0 row of this group's next kept row
    auto ld_res = [&](int q) {
      const int trow = y0 - 2 + q;
      if (q >= 1 && q <= n_f - 2 && col_ok && trow >= 0 && trow < H) {
        const uint4* rp = reinterpret_cast<const uint4*>(a.f0 + ((((size_t)n * H + trow) * W) + tcol) * C);
#pragma unroll
        for (int j = 0; j < CCH; ++j) res_nx[j] = __ldg(rp + j);
      }
    };
    auto own = [&](int q) { return (int)((G + q + 1) % EPI1) == grp; };
    int q0 = -1;
    while (q0 <= n_f && !own(q0)) ++q0;
    {
      int qf = q0;
      while (qf <= n_f && !(own(qf) && qf >= 1 && qf <= n_f - 2)) ++qf;
      ld_res(qf);
    }
    for (int q = q0; q <= n_f; q += EPI1) {  // out rows of conv1 = g rows y0-2+q
      const unsigned g = G + q + 1;
      const bool emit = q >= 1 && q <= n_f - 2;
      const int trow = y0 - 2 + q;
      const bool ok = col_ok && trow >= 0 && trow < H;
      uint4 res[CCH];
      if (emit) {
#pragma unroll
        for (int j = 0; j < CCH; ++j) res[j] = res_nx[j];
        ld_res(q + EPI1);
      }
      const unsigned ti = E + (unsigned)(q - 1);
      const int ts = (int)(ti % kNT);
      const uint32_t tph = (ti / kNT) & 1u;
      if (emit) mbar_wait(&t_empty[ts], tph ^ 1);
      const int b = ring_idx<RB1>(g);
      mbar_wait(&r1_ready[b], (uint32_t)(g / RB1) & 1u);
      tc_fence_after();
      float v[C];
      ring_load<C>(ring1 + lane_off + b * C, v);
      tc_fence_before();
      __syncwarp();
      if (lane_id() == 0) mbar_arrive(&r1_free[b]);
      if (emit) {
        uint8_t* dst = sT + ts * ROWB + m * 16;
#pragma unroll
        for (int j = 0; j < CCH; ++j) {
          const __nv_bfloat162* h2 = reinterpret_cast<const __nv_bfloat162*>(&res[j]);
          float o[8];
#pragma unroll
          for (int e = 0; e < 4; ++e) {
            const float2 f2 = __bfloat1622float2(h2[e]);
            o[2 * e] = ok ? v[8 * j + 2 * e] + f2.x : 0.f;
            o[2 * e + 1] = ok ? v[8 * j + 2 * e + 1] + f2.y : 0.f;
          }
          uint4 u;
          u.x = pack_bf16x2(o[0], o[1]);
          u.y = pack_bf16x2(o[2], o[3]);
          u.z = pack_bf16x2(o[4], o[5]);
          u.w = pack_bf16x2(o[6], o[7]);
          *reinterpret_cast<uint4*>(dst + j * PLANE) = u;
        }
        fence_proxy_async_smem();
        __syncwarp();
        if (lane_id() == 0) mbar_arrive(&t_full[ts]);
      }
    }
    G += n_f + 2;
    E += n_f - 2;
    SR_PIECE_END
  } else if (warp < 6) {
    // ============ conv1 epilogue: drain finished rows -> + b (armed) + f0 -> g smem ring (0 outside the frame) ======
    const int quarter = warp & 3;
    const int m = quarter * 32 + lane_id();
    const uint32_t lane_off = (uint32_t)(quarter * 32) << 16;
    for (int b = 0; b < RB1; ++b)
      if (lane_id() == 0) mbar_arrive(&r1_free[b]);
    int ts = 0;
    uint32_t tph = 0;
    unsigned G = 0;
    SR_PIECE_BEGIN
    const int tcol = x0 - 1 + m;
    const bool col_ok = tcol >= 0 && tcol < W;
    uint4 res_nx[CCH];  // the f0 row is loaded one row ahead, so its L2/HBM latency overlaps a row-step
    auto ld_res = [&](int q) {
      const int trow = y0 - 2 + q;
      if (q >= 1 && q <= n_f - 2 && col_ok && trow >= 0 && trow < H) {
        const uint4* rp = reinterpret_cast<const uint4*>(a.f0 + ((((size_t)n * H + trow) * W) + tcol) * C);
#pragma unroll
        for (int j = 0; j < CCH; ++j) res_nx[j] = __ldg(rp + j);
      }
    };
    ld_res(-1);
    for (int q = -1; q <= n_f; ++q) {  // out rows of conv1 = g rows y0-2+q
      const unsigned g = G + q + 1;
      const bool emit = q >= 1 && q <= n_f - 2;
      const int trow = y0 - 2 + q;
      const bool ok = col_ok && trow >= 0 && trow < H;
      uint4 res[CCH];
#pragma unroll
      for (int j = 0; j < CCH; ++j) res[j] = res_nx[j];
      ld_res(q + 1);
      if (emit) mbar_wait(&t_empty[ts], tph ^ 1);
      const int b = ring_idx<RB1>(g);
      mbar_wait(&r1_ready[b], (uint32_t)(g / RB1) & 1u);
      tc_fence_after();
      if (warp == 2 && lane_id() == 0) { SR_BDBG(3, q + 1) }
      float v[C];
      ring_load<C>(ring1 + lane_off + b * C, v);
      tc_fence_before();
      __syncwarp();
      if (lane_id() == 0) mbar_arrive(&r1_free[b]);
      if (emit) {
        uint8_t* dst = sT + ts * ROWB + m * 16;
#pragma unroll
        for (int j = 0; j < CCH; ++j) {
          const __nv_bfloat162* h2 = reinterpret_cast<const __nv_bfloat162*>(&res[j]);
          float o[8];
#pragma unroll
          for (int e = 0; e < 4; ++e) {
            const float2 f2 = __bfloat1622float2(h2[e]);
            o[2 * e] = ok ? v[8 * j + 2 * e] + f2.x : 0.f;
            o[2 * e + 1] = ok ? v[8 * j + 2 * e + 1] + f2.y : 0.f;
          }
          uint4 u;
          u.x = pack_bf16x2(o[0], o[1]);
          u.y = pack_bf16x2(o[2], o[3]);
          u.z = pack_bf16x2(o[4], o[5]);
          u.w = pack_bf16x2(o[6], o[7]);
          *reinterpret_cast<uint4*>(dst + j * PLANE) = u;
        }
        fence_proxy_async_smem();
        __syncwarp();
        if (lane_id() == 0) mbar_arrive(&t_full[ts]);
        if (warp == 2 && lane_id() == 0) { SR_BDBG(4, q + 1) }
        if (++ts == kNT) { ts = 0; tph ^= 1; }
      }
    }
    G += n_f + 2;
    SR_PIECE_END
  } else {
    // ============ tail epilogue: drain -> pixel shuffle + skip + clamp + RNE -> staged HR rows -> 16-B stores ======
    const int grp = warp >= 11 ? 1 : 0;  // group grp drains the ring rows g with g % 2 == grp
    const int quarter = warp & 3;
    const int m = quarter * 32 + lane_id();
    const int tid = (warp - (grp ? 11 : 6)) * 32 + lane_id();  // 0..127 within the group
    const uint32_t lane_off = (uint32_t)(quarter * 32) << 16;
    if (grp == 0)  // every ring block starts free (4 arrivals); later each drain's group frees its block
      for (int b = 0; b < RB2; ++b)
        if (lane_id() == 0) mbar_arrive(&r2_free[b]);
    const int sH = S * H, sW = S * W;
    int os = 0;
    unsigned G = 0, emitted = 0;  // emitted: output rows of both groups so far (LR ring order)
    SR_PIECE_BEGIN
    const int xc = x0 + m;
    const bool lane_ok = m < kBtTW && xc < W;
    const int lbase = 16 * ((3 * x0 - 6) >> 4);  // LR byte of the slot's first chunk
    const int nbytes = min(kBtTW, W - x0) * 3 * S;  // HR bytes of this strip per row
    for (int q = -1; q <= n_t; ++q) {  // out rows of conv2 = output rows y0-1+q
      const unsigned g = G + q + 1;
      const bool emit = q >= 1 && q <= n_t - 2;
      const unsigned xi = emitted;  // LR ring index of this row (if emitted)
      emitted += emit;
      if ((int)(g & 1) != grp) continue;
      const int ls = (int)(xi % NLR);
      const uint32_t lph = (uint32_t)(xi / NLR) & 1u;
      const int r = y0 - 1 + q;
      const int b = ring_idx<RB2>(g);
      mbar_wait(&r2_ready[b], (uint32_t)(g / RB2) & 1u);
      tc_fence_after();
      if (tid == 0) { SR_BDBG(5, q + 1) }
      float v[CO2];
      ring_load<CO2>(ring2 + lane_off + b * CO2, v);
      tc_fence_before();
      __syncwarp();
      if (lane_id() == 0) mbar_arrive(&r2_free[b]);
      if (!emit) continue;
      if (tid == 0) { SR_BDBG(13, q + 1) }
      mbar_wait(&l_full[ls], lph);
      if (tid == 0) { SR_BDBG(14, q + 1) }
      uint8_t* stg = sO + (grp * kBtNO + os) * OUTB;
      if constexpr (YO) {  // I420 out: Y rows (S), U and V rows (S/2 each) staged like the RGB rows, then copied out
        static_assert(S % 2 == 0, "I420 output: whole 2x2 chroma blocks per lane");
        constexpr uint32_t HRPY = ((kBtTW * S + 15u) & ~15u) + 16u, HRPC = ((kBtTW * S / 2 + 15u) & ~15u) + 16u;
        static_assert(S * HRPY + S * HRPC <= OUTB, "I420 staging fits the RGB staging slot");
        uint8_t* const stgY = stg;
        uint8_t* const stgU = stg + S * HRPY;
        uint8_t* const stgV = stgU + (S / 2) * HRPC;
        const size_t sWc = (size_t)sW / 2, sHc = (size_t)sH / 2;
        uint8_t* const yrow0 = a.hy + ((size_t)n * sH + (size_t)S * r) * sW + (size_t)S * x0;
        uint8_t* const urow0 = a.hu + ((size_t)n * sHc + (size_t)(S / 2) * r) * sWc + (size_t)(S / 2) * x0;
        uint8_t* const vrow0 = a.hv + ((size_t)n * sHc + (size_t)(S / 2) * r) * sWc + (size_t)(S / 2) * x0;
        if (lane_ok) {
          uint8_t o[S * S * 3];
          tail_u8_px<S>(smem_u32(sL + ls * kBtLrSlot) - (uint32_t)lbase + 0u, 16 * kBtLrChunks, 0, r, xc, H, W, v,
                        BIC ? 1 : 0, o);
#pragma unroll
          for (int i = 0; i < S; ++i) {
            const uint32_t sh = (uint32_t)(reinterpret_cast<uintptr_t>(yrow0 + (size_t)i * sW) & 15);
            const uint32_t dst = smem_u32(stgY + i * HRPY) + sh + S * m;
#pragma unroll
            for (int j = 0; j < S; ++j)
              sts_u8(dst + j, rgb_to_y(o[i * 3 * S + 3 * j], o[i * 3 * S + 3 * j + 1], o[i * 3 * S + 3 * j + 2]));
          }
#pragma unroll
          for (int bi = 0; bi < S / 2; ++bi) {
            const uint32_t shu = (uint32_t)(reinterpret_cast<uintptr_t>(urow0 + (size_t)bi * sWc) & 15);
            const uint32_t shv = (uint32_t)(reinterpret_cast<uintptr_t>(vrow0 + (size_t)bi * sWc) & 15);
#pragma unroll
            for (int bj = 0; bj < S / 2; ++bj) {
              int sr = 0, sg = 0, sb = 0;
#pragma unroll
              for (int dy = 0; dy < 2; ++dy)
#pragma unroll
                for (int dx = 0; dx < 2; ++dx) {
                  const int k = (2 * bi + dy) * 3 * S + 3 * (2 * bj + dx);
                  sr += o[k]; sg += o[k + 1]; sb += o[k + 2];
                }
              uint8_t uu, vv;
              rgb_sums_to_uv(sr, sg, sb, uu, vv);
              sts_u8(smem_u32(stgU + bi * HRPC) + shu + (S / 2) * m + bj, uu);
              sts_u8(smem_u32(stgV + bi * HRPC) + shv + (S / 2) * m + bj, vv);
            }
          }
        }
        named_bar_sync(2 + grp, 128);  // staging complete (and the LR slot read by every lane of the group)
        if (tid == 0) mbar_arrive(&l_empty[ls]);
        if (r >= a.hr_row0 && r < a.hr_row1) {
          const int npx = min(kBtTW, W - x0);
          auto copy_row = [&](uint8_t* d, const uint8_t* srow, int nb) {  // 16-B stores, ragged ends bytewise
            const int sh = (int)(reinterpret_cast<uintptr_t>(d) & 15);
            const uint8_t* src = srow + sh;
            const int pre = min((16 - sh) & 15, nb);
            const int nch = (nb - pre) >> 4;
            const int post = nb - pre - 16 * nch;
            for (int k = tid; k < nch; k += 128)
              *reinterpret_cast<uint4*>(d + pre + 16 * k) = *reinterpret_cast<const uint4*>(src + pre + 16 * k);
            if (tid < pre) d[tid] = src[tid];
            else if (tid >= 32 && tid < 32 + post) d[pre + 16 * nch + tid - 32] = src[pre + 16 * nch + tid - 32];
          };
#pragma unroll
          for (int i = 0; i < S; ++i) copy_row(yrow0 + (size_t)i * sW, stgY + i * HRPY, npx * S);
#pragma unroll
          for (int bi = 0; bi < S / 2; ++bi) {
            copy_row(urow0 + (size_t)bi * sWc, stgU + bi * HRPC, npx * S / 2);
            copy_row(vrow0 + (size_t)bi * sWc, stgV + bi * HRPC, npx * S / 2);
          }
        }
        os = os == kBtNO - 1 ? 0 : os + 1;
        continue;
      }
      uint8_t* hrow0 = a.hr + (((size_t)n * sH + (size_t)S * r) * sW + (size_t)S * x0) * 3;
      if (lane_ok) {
        uint8_t o[S * S * 3];
        tail_u8_px<S>(smem_u32(sL + ls * kBtLrSlot) - (uint32_t)lbase + 0u, 16 * kBtLrChunks, 0, r, xc, H, W, v,
                      BIC ? 1 : 0, o);
#pragma unroll
        for (int i = 0; i < S; ++i) {
          const uint32_t sh = (uint32_t)(reinterpret_cast<uintptr_t>(hrow0 + (size_t)i * sW * 3) & 15);
          const uint32_t dst = smem_u32(stg + i * HRP) + sh + 3 * S * m;
#pragma unroll
          for (int k = 0; k < 3 * S; ++k) sts_u8(dst + k, o[i * 3 * S + k]);
        }
      }
      named_bar_sync(2 + grp, 128);  // staging complete (and the LR slot read by every lane of the group)
      if (tid == 0) mbar_arrive(&l_empty[ls]);
      if (r >= a.hr_row0 && r < a.hr_row1) {
#pragma unroll
        for (int i = 0; i < S; ++i) {
          uint8_t* d = hrow0 + (size_t)i * sW * 3;
          const int sh = (int)(reinterpret_cast<uintptr_t>(d) & 15);
          const uint8_t* src = stg + i * HRP + sh;
          const int pre = min((16 - sh) & 15, nbytes);
          const int nch = (nbytes - pre) >> 4;
          const int post = nbytes - pre - 16 * nch;
          for (int k = tid; k < nch; k += 128)
            *reinterpret_cast<uint4*>(d + pre + 16 * k) = *reinterpret_cast<const uint4*>(src + pre + 16 * k);
          if (tid < pre) d[tid] = src[tid];
          else if (tid >= 32 && tid < 32 + post) d[pre + 16 * nch + tid - 32] = src[pre + 16 * nch + tid - 32];
        }
      }
      if (tid == 0) { SR_BDBG(6, q + 1) }
      os = os == kBtNO - 1 ? 0 : os + 1;
    }
    G += n_t + 2;
    SR_PIECE_END
  }
#undef SR_PIECE_BEGIN
#undef SR_PIECE_END
  tc_fence_before();
  __syncthreads();
  if (warp == 1) tmem_dealloc<512>(tmem);
}

template <int C, int CO2, int S, bool BIC, bool YO = false>
static cudaError_t launch_bt_t(const CUtensorMap& tf, const CUtensorMap& tl, const bf16* w1, const bf16* w2,
                               const BtArgs& a, int grid, cudaStream_t st) {
  if constexpr (!BtCfg<C, CO2, S>::FITS || (YO && S % 2 != 0)) {
    return cudaErrorNotSupported;
  } else {
    auto kern = k_bodytail<C, CO2, S, BIC, YO>;
    static bool configured = false;
    if (!configured) {
      cudaError_t e =
          cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)BtCfg<C, CO2, S>::SMEM);
      if (e != cudaSuccess) return e;
      configured = true;
    }
    return launch_k(kern, dim3(grid), dim3(BtThreads<C>::N), BtCfg<C, CO2, S>::SMEM, st, tf, tl, w1, w2, a);
  }
}

static int bt_co2(int s) { return s == 2 ? 16 : (s == 3 ? 32 : 48); }

bool bodytail_supported(int cp, int s, int W, const void* lr, const void* hr) {
  if (W < 96 || W % 16 != 0) return false;  // the LR rows map needs 16-B rows
  if ((reinterpret_cast<uintptr_t>(lr) & 15) != 0) return false;
  (void)hr;
  const int co2 = bt_co2(s);
#define SR_BT_FIT(C, S) \
  if (cp == C && s == S) return BtCfg<C, (S == 2 ? 16 : (S == 3 ? 32 : 48)), S>::FITS;
  SR_BT_FIT(16, 2) SR_BT_FIT(16, 3) SR_BT_FIT(16, 4)
  SR_BT_FIT(32, 2) SR_BT_FIT(32, 3) SR_BT_FIT(32, 4)
  SR_BT_FIT(48, 2) SR_BT_FIT(48, 3) SR_BT_FIT(48, 4)
#undef SR_BT_FIT
  (void)co2;
  return false;
}

cudaError_t launch_bodytail(int cp, int s, const bf16* f, const bf16* f0, const bf16* w1fold, const bf16* w2fold,
                            const float* b1, const float* b2, const uint8_t* lr, uint8_t* hr, int hr_row0,
                            int hr_row1, int bicubic, int N, int H, int W, cudaStream_t st, long long* dbg,
                            uint8_t* hy, uint8_t* hu, uint8_t* hv) {
  CUtensorMap tf, tl;
  if (make_act_tmap(&tf, f, N, H, W, cp, 130, 1, cp / 8, CHUNK_ROW_PIX) != CUDA_SUCCESS) return cudaErrorInvalidValue;
  if (make_u8_rows_tmap(&tl, lr, N, H, 3LL * W, kBtLrChunks, 5) != CUDA_SUCCESS) return cudaErrorInvalidValue;
  BtArgs a{b1, b2, f0, lr, hr, N, H, W, hr_row0, hr_row1, bicubic, dbg, hy, hu, hv};
  const long long rows = (long long)N * ((W + kBtTW - 1) / kBtTW) * H;
  int grid = num_sms();
  if (rows < grid) grid = (int)rows;
  if (hy) {  // I420 output (s = 2, 4)
    if (!hu || !hv || s == 3) return cudaErrorNotSupported;
#define SR_BT_YO(C, S) \
    if (cp == C && s == S)                                                                                      \
      return bicubic ? launch_bt_t<C, (S == 2 ? 16 : 48), S, true, true>(tf, tl, w1fold, w2fold, a, grid, st)   \
                     : launch_bt_t<C, (S == 2 ? 16 : 48), S, false, true>(tf, tl, w1fold, w2fold, a, grid, st);
    SR_BT_YO(16, 2) SR_BT_YO(16, 4) SR_BT_YO(32, 2) SR_BT_YO(32, 4) SR_BT_YO(48, 2) SR_BT_YO(48, 4)
#undef SR_BT_YO
    return cudaErrorNotSupported;
  }
#define SR_BT_CASE(C, S) \
  if (cp == C && s == S)                                                                                   \
    return bicubic ? launch_bt_t<C, (S == 2 ? 16 : (S == 3 ? 32 : 48)), S, true>(tf, tl, w1fold, w2fold, a, grid, st) \
                   : launch_bt_t<C, (S == 2 ? 16 : (S == 3 ? 32 : 48)), S, false>(tf, tl, w1fold, w2fold, a, grid, st);
  SR_BT_CASE(16, 2) SR_BT_CASE(16, 3) SR_BT_CASE(16, 4)
  SR_BT_CASE(32, 2) SR_BT_CASE(32, 3) SR_BT_CASE(32, 4)
  SR_BT_CASE(48, 2) SR_BT_CASE(48, 3) SR_BT_CASE(48, 4)
#undef SR_BT_CASE
  return cudaErrorNotSupported;
}

}  // namespace sr

// Fused residual block on CTA pairs (tcgen05 cta_group::2):  f' = f + conv2(ReLU(conv1(f) + b1)) + b2, inference.
//
// The same dataflow as k_resblock (conv_block.cu: rolling dy-fold convs, t kept in a shared-memory ring, TMEM-ring
// accumulation of the three vertical taps, bias-armed blocks), but every MMA is M = 256 over the two SMs of a
// cluster pair: CTA r of the pair owns one 126-pixel strip (the pair's strips are consecutive in the flattened
// (frame, strip) order, so an odd strip count leaves one dummy strip in total), supplies its 128 pixel rows of A
// (its own f / t rows) and HALF of B's N columns from its own shared memory, and receives its 128 lanes x all N
// columns in its own TMEM.  Per SM an MMA then reads 4 KB of A + 2.25 KB of B instead of 4 + 4.5 KB (N = 144), and
// one issuer per conv drives both SMs.  Only the pair's leader (cluster rank 0) issues MMAs.
//
// B halves.  With cta_group::2, CTA r provides rows [r N/2, (r+1) N/2) of an MMA's B.  A step whose three target
// blocks wrap around the TMEM ring is issued as two MMA groups (N = 2C + C or C + 2C; ring.cuh), and those
// sub-ranges split differently, so each CTA keeps five row regions of every (kx, 8-channel) weight slab of the
// dy-fold layout Wo[kx][ci/8][3C][8]: FULL (its half of the 3C rows), A1/A2 (its halves of rows [0,2C) and
// [2C,3C)), B1/B2 (its halves of rows [0,C) and [C,3C)) -- 4.5 C rows instead of 3 C, all at the same shared-memory
// offsets in both CTAs, so one descriptor addresses both halves.
//
// Synchronisation (the leader's barriers collect both CTAs): f rows are TMA-loaded by each CTA into its own smem and
// counted on the LEADER's f_full (cta_group::2 TMA, expect_tx from both producers); t rows are written by both
// CTAs' conv1 epilogues (each SM's tensor core reads its own CTA's rows) and announced on the leader's t_full
// (fence.proxy.async, then a remote arrive: a cluster-scope release there cost 30% in an A/B); ring
// blocks are freed on the leader's r1_free / r2_free by both CTAs' epilogues; the leader's commits multicast
// r*_ready, f_empty and t_empty to both CTAs.  Weights and bias-arming tiles of both CTAs are announced on the
// leader's setup_bar.  Results are bit-identical to k_resblock: the same MMA sequence per output element.
#include <cuda.h>
#include "ptx.cuh"
#include "pair.cuh"
#include "tmap.h"
#include "sr_internal.h"
#include "ring.cuh"
#include "launch.cuh"
#include "rot.cuh"

namespace sr {

// warps: 0 producer, 1 conv1 issuer, 2..5 conv1 epi, 6..9 conv2 epi (group 0), 10 conv2 issuer, at C <= 32 also
// 11..14 conv2 epi (group 1): the conv2 epilogue groups take alternate output rows
static constexpr int kB2Threads = 352;
static constexpr int kB2TW = 126;

template <int C>
struct B2Cfg {
  static constexpr int EPI2 = C <= 32 ? 2 : 1;  // conv2 epilogue groups (rows alternate between them)
  static constexpr int THREADS = kB2Threads + (EPI2 - 1) * 128;
  static constexpr int CCH = C / 8, KS = C / 16, N = 3 * C;
  static constexpr int RB = (256 / C) < 8 ? (256 / C) : 8;
  static constexpr int NF = C >= 48 ? 3 : 5;  // f-row ring (C = 48: one slot less than k_resblock, weights grew;
                                              // C = 32: 5 measured 5% faster than 4, 6-7 no better)
  static constexpr int NT = C >= 48 ? 3 : 5;  // t-row ring (the cross-CTA t hand-off needs depth at C = 32)
  static constexpr int NO = C >= 48 ? 2 : 3;  // output staging rows
  static constexpr int SLABS = 3 * CCH;       // (kx, 8-channel) slabs of a conv's dy-fold weights
  static constexpr int R_FULL = 3 * C / 2, R_A1 = C, R_A2 = C / 2, R_B1 = C / 2, R_B2 = C;
  static constexpr uint32_t OFF_FULL = 0;
  static constexpr uint32_t OFF_A1 = OFF_FULL + SLABS * R_FULL * 16;
  static constexpr uint32_t OFF_A2 = OFF_A1 + SLABS * R_A1 * 16;
  static constexpr uint32_t OFF_B1 = OFF_A2 + SLABS * R_A2 * 16;
  static constexpr uint32_t OFF_B2 = OFF_B1 + SLABS * R_B1 * 16;
  static constexpr uint32_t WBYTES = OFF_B2 + SLABS * R_B2 * 16;
  static constexpr uint32_t WB_AL = (WBYTES + 127u) & ~127u;
  static constexpr uint32_t PLANE = 130 * 16;
  static constexpr uint32_t ROWB = ((CCH * PLANE) + 127u) & ~127u;
  static constexpr uint32_t OUTB = ((kB2TW * C * 2) + 1023u) & ~1023u;
  static constexpr uint32_t ARMB = ((kArmOnesBytes + 2 * (C / 2) * 32) + 127u) & ~127u;  // ones + 2 half bias tiles
  static constexpr size_t SMEM = 1024 + 2 * (size_t)WB_AL + (size_t)NF * ROWB + (size_t)NT * ROWB +
                                 (size_t)EPI2 * NO * OUTB + ARMB;
};

// Bias-arming B tile of this CTA's half of the N = C columns: rows n < C/2 hold bias[half + n] split into three bf16
// terms (ring.cuh), K-major SWIZZLE_NONE with LBO = (C/2) * 16.
__device__ __forceinline__ void arm_half_fill(uint8_t* btile, const float* bias, int half0, int nh, int tid,
                                              int nthreads) {
  for (int i = tid; i < nh * 16; i += nthreads) {
    const int n = i / 16, k = i % 16;
    const float b = bias[half0 + n];
    const __nv_bfloat16 hi = __float2bfloat16(b);
    const __nv_bfloat16 mid = __float2bfloat16(b - __bfloat162float(hi));
    const __nv_bfloat16 lo = __float2bfloat16(b - __bfloat162float(hi) - __bfloat162float(mid));
    const __nv_bfloat16 v = k == 0 ? hi : k == 1 ? mid : k == 2 ? lo : __float2bfloat16(0.f);
    *reinterpret_cast<__nv_bfloat16*>(btile + (n % 8) * 16 + (n / 8) * 128 + (k / 8) * (nh * 16) + (k % 8) * 2) = v;
  }
}

template <int C, int RB>
__device__ __forceinline__ void ring_arm2(uint32_t ring_base, unsigned g, uint32_t ones_saddr, uint32_t btile_saddr) {
  constexpr uint32_t id = make_idesc(256, C, 0, 0);
  mma2_bf16_ss(ring_base + ring_idx<RB>(g) * C, make_desc(ones_saddr, 2048, 128),
               make_desc(btile_saddr, (C / 2) * 16, 128), id, 0u);
}

// one input-row step of a dy-fold conv on the pair (see ring_mma_step in ring.cuh for the single-CTA form)
template <int C, int RB>
__device__ __forceinline__ void ring_mma_step2(uint32_t ring_base, unsigned g, uint64_t ad, uint32_t sw,
                                               uint32_t kstride) {
  using Cfg = B2Cfg<C>;
  constexpr int CCH = Cfg::CCH, KS = Cfg::KS;
  const int i0 = ring_idx<RB>(g);
  auto group = [&](int blk, int n, uint32_t off, int rows) {
    const uint32_t id = make_idesc(256, (uint32_t)n, 0, 0);
#pragma unroll
    for (int dx = 0; dx < 3; ++dx)
#pragma unroll
      for (int ks = 0; ks < KS; ++ks)
        mma2_bf16_ss(ring_base + blk * C, desc_add(ad, dx * 16u + ks * kstride),
                     make_desc(sw + off + (uint32_t)(dx * CCH + 2 * ks) * rows * 16u, rows * 16u, 128), id, 1u);
  };
  if (i0 >= 2) {
    group(i0 - 2, 3 * C, Cfg::OFF_FULL, Cfg::R_FULL);
  } else if (i0 == 0) {
    group(RB - 2, 2 * C, Cfg::OFF_A1, Cfg::R_A1);
    group(0, C, Cfg::OFF_A2, Cfg::R_A2);
  } else {
    group(RB - 1, C, Cfg::OFF_B1, Cfg::R_B1);
    group(0, 2 * C, Cfg::OFF_B2, Cfg::R_B2);
  }
}

template <int C>
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(B2Cfg<C>::THREADS, 1)
k_resblock2(const __grid_constant__ CUtensorMap tm_f, const __grid_constant__ CUtensorMap tm_out,
            const bf16* __restrict__ w1, const bf16* __restrict__ w2, const float* __restrict__ b1,
            const float* __restrict__ b2, const bf16* __restrict__ fres, const int N, const int H, const int W) {
  using Cfg = B2Cfg<C>;
  constexpr int CCH = Cfg::CCH, RB = Cfg::RB, NF = Cfg::NF, NT = Cfg::NT, NO = Cfg::NO;
  constexpr uint32_t PLANE = Cfg::PLANE, ROWB = Cfg::ROWB, OUTB = Cfg::OUTB;

  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sW1 = smem;
  uint8_t* sW2 = sW1 + Cfg::WB_AL;
  uint8_t* sF = sW2 + Cfg::WB_AL;
  uint8_t* sT = sF + NF * ROWB;
  uint8_t* sO = sT + NT * ROWB;
  uint8_t* sOnes = sO + Cfg::EPI2 * NO * OUTB;
  uint8_t* sB1 = sOnes + kArmOnesBytes;
  uint8_t* sB2 = sB1 + (C / 2) * 32;
  __shared__ __align__(8) uint64_t f_full[NF], f_empty[NF], t_full[NT], t_empty[NT], r1_ready[RB], r1_free[RB],
      r2_ready[RB], r2_free[RB], w_bar, setup_bar;
  __shared__ uint32_t tmem_base_sh;
  __shared__ __align__(16) float sbv[2 * C];

  const int warp = warp_id();
  const uint32_t rank = cluster_rank();
  const bool lead = rank == 0;
  // spare t positions 128, 129 of every plane of every t slot are read by the two invalid conv2 lanes: zero them
  for (int i = threadIdx.x; i < NT * CCH * 2; i += blockDim.x) {
    const int slot = i / (CCH * 2), rem = i % (CCH * 2);
    *reinterpret_cast<uint4*>(sT + slot * ROWB + (rem / 2) * PLANE + (128 + rem % 2) * 16) = make_uint4(0, 0, 0, 0);
  }
  if (warp == 0 && lane_id() == 0) {
    for (int s = 0; s < NF; ++s) { mbar_init(&f_full[s], 2); mbar_init(&f_empty[s], 1); }
    for (int s = 0; s < NT; ++s) { mbar_init(&t_full[s], 8); mbar_init(&t_empty[s], 1); }
    for (int s = 0; s < RB; ++s) {
      mbar_init(&r1_ready[s], 1); mbar_init(&r1_free[s], 8);
      mbar_init(&r2_ready[s], 1); mbar_init(&r2_free[s], 8);
    }
    mbar_init(&w_bar, 1);
    mbar_init(&setup_bar, 2);
    fence_barrier_init();
  }
  if (warp == 1) tmem_alloc2<512>(&tmem_base_sh);
  // weights (this CTA's five row regions of both convs) and the bias-arming tiles before the PDL wait: written at
  // least two kernels upstream (k_resblock's prologue)
  if (warp == 0 && lane_id() == 0) {
    mbar_arrive_expect_tx(&w_bar, 2 * Cfg::WBYTES);
    const int h = (int)rank;
    const int r0[5] = {h * Cfg::R_FULL, h * C, 2 * C + h * (C / 2), h * (C / 2), C + h * C};
    const int rn[5] = {Cfg::R_FULL, Cfg::R_A1, Cfg::R_A2, Cfg::R_B1, Cfg::R_B2};
    const uint32_t off[5] = {Cfg::OFF_FULL, Cfg::OFF_A1, Cfg::OFF_A2, Cfg::OFF_B1, Cfg::OFF_B2};
    for (int cv = 0; cv < 2; ++cv) {
      const bf16* wg = cv ? w2 : w1;
      uint8_t* sw = cv ? sW2 : sW1;
      for (int rg = 0; rg < 5; ++rg)
        for (int sl = 0; sl < Cfg::SLABS; ++sl)
          bulk_load(sw + off[rg] + (uint32_t)sl * rn[rg] * 16u, wg + ((size_t)sl * 3 * C + r0[rg]) * 8,
                    (uint32_t)rn[rg] * 16u, &w_bar);
    }
  }
  if (threadIdx.x < C) {
    sbv[threadIdx.x] = b1[threadIdx.x];
    sbv[C + threadIdx.x] = b2[threadIdx.x];
  }
  __syncthreads();
  arm_tiles_fill(sOnes, sB1, sbv, 0, threadIdx.x, blockDim.x);  // the ones tile (no bias rows at coutp = 0)
  arm_half_fill(sB1, sbv, (int)rank * (C / 2), C / 2, threadIdx.x, blockDim.x);
  arm_half_fill(sB2, sbv + C, (int)rank * (C / 2), C / 2, threadIdx.x, blockDim.x);
  fence_proxy_async_smem();
  tc_fence_before();
  cluster_sync_all();  // barriers of both CTAs initialised, TMEM allocated in both
  tc_fence_after();
  pdl_enter();
  const uint32_t tmem = tmem_base_sh;
  const uint32_t ring1 = tmem, ring2 = tmem + 256;

  const int tiles_x = (W + kB2TW - 1) / kB2TW;
  const long long cols = (long long)N * tiles_x;
  const long long npc = (cols + 1) / 2;  // pair-columns: strips (2 pc, 2 pc + 1) of the flattened (frame, strip) list
  const long long total = npc * H;
  const long long npairs = gridDim.x / 2, pair = blockIdx.x / 2;
  const long long beg = total * pair / npairs, end = total * (pair + 1) / npairs;
#define SR_PIECE_BEGIN                                                                      \
  for (long long pos = beg; pos < end;) {                                                   \
    const long long pc = pos / H;                                                           \
    const int y0 = (int)(pos - pc * H);                                                     \
    const int y1 = (int)min((long long)H, y0 + (end - pos));                                \
    pos += y1 - y0;                                                                         \
    const long long col = 2 * pc + rank;                                                    \
    const bool dummy = col >= cols; /* odd strip count: the last pair's second strip */     \
    const int n = dummy ? 0 : (int)(col / tiles_x);                                         \
    const int x0 = dummy ? W : (int)(col - (long long)n * tiles_x) * kB2TW;                 \
    const int n_f = y1 - y0 + 4, n_t = n_f - 2;                                             \
    (void)n; (void)x0; (void)n_t; (void)dummy;
#define SR_PIECE_END }

  if (warp == 0) {
    // ===================== producer (both CTAs): f rows y0-2 .. y1+1 into own smem, counted on the leader ======
    if (elect_one()) {
      tma_prefetch_desc(&tm_f);
      int s = 0;
      uint32_t ph = 0;
      SR_PIECE_BEGIN
      for (int i = 0; i < n_f; ++i) {
        mbar_wait(&f_empty[s], ph ^ 1);
        const uint32_t lf = cluster_addr(&f_full[s], 0);
        mbar_arrive_expect_tx_remote(lf, CCH * PLANE);
        tma_load_5d_pair(sF + s * ROWB, &tm_f, lf, 0, x0 - 2, y0 - 2 + i, 0, n);
        if (++s == NF) { s = 0; ph ^= 1; }
      }
      SR_PIECE_END
      for (int k = 0; k < NF; ++k) {  // drain: every slot's last release (multicast commit) has landed
        mbar_wait(&f_empty[s], ph ^ 1);
        if (++s == NF) { s = 0; ph ^= 1; }
      }
    }
    __syncwarp();
  } else if (warp == 1) {
    // ===================== conv1 MMA issuer (leader): step st consumes f row st of both CTAs ====================
    if (elect_one()) {
      mbar_wait(&w_bar, 0);  // this CTA's weight regions have landed (the arming tiles before the cluster sync)
      mbar_arrive_remote(cluster_addr(&setup_bar, 0));  // (the arming tiles were ordered by the cluster barrier)
      if (lead) {
        mbar_wait(&setup_bar, 0);
        tc_fence_after();
        int fs = 0;
        uint32_t fph = 0;
        unsigned G1 = 0, acq1 = 0;
        SR_PIECE_BEGIN
        for (int st = 0; st < n_f; ++st) {
          const unsigned g = G1 + st;
          for (; acq1 < g + 3; ++acq1) mbar_wait(&r1_free[ring_idx<RB>(acq1)], (uint32_t)(acq1 / RB) & 1u);
          mbar_wait(&f_full[fs], fph);
          tc_fence_after();
          if (st == 0) {
            ring_arm2<C, RB>(ring1, g, smem_u32(sOnes), smem_u32(sB1));
            ring_arm2<C, RB>(ring1, g + 1, smem_u32(sOnes), smem_u32(sB1));
          }
          ring_arm2<C, RB>(ring1, g + 2, smem_u32(sOnes), smem_u32(sB1));
          ring_mma_step2<C, RB>(ring1, g, make_desc(smem_u32(sF + fs * ROWB), PLANE, 128), smem_u32(sW1), 2 * PLANE);
          mma2_commit_mc(&r1_ready[ring_idx<RB>(g)], 0x3);
          mma2_commit_mc(&f_empty[fs], 0x3);
          if (st == n_f - 1) {
            mma2_commit_mc(&r1_ready[ring_idx<RB>(g + 1)], 0x3);
            mma2_commit_mc(&r1_ready[ring_idx<RB>(g + 2)], 0x3);
          }
          if (++fs == NF) { fs = 0; fph ^= 1; }
        }
        G1 += n_f + 2;
        SR_PIECE_END
      }
    }
    __syncwarp();
  } else if (warp == 10) {
    // ===================== conv2 MMA issuer (leader): step k consumes t row k of both CTAs =====================
    if (lead && elect_one()) {
      mbar_wait(&setup_bar, 0);
      tc_fence_after();
      int ts = 0;
      uint32_t tph = 0;
      unsigned G2 = 0, acq2 = 0;
      SR_PIECE_BEGIN
      for (int k = 0; k < n_t; ++k) {
        const unsigned g = G2 + k;
        for (; acq2 < g + 3; ++acq2) mbar_wait(&r2_free[ring_idx<RB>(acq2)], (uint32_t)(acq2 / RB) & 1u);
        mbar_wait(&t_full[ts], tph);
        tc_fence_after();
        if (k == 0) {
          ring_arm2<C, RB>(ring2, g, smem_u32(sOnes), smem_u32(sB2));
          ring_arm2<C, RB>(ring2, g + 1, smem_u32(sOnes), smem_u32(sB2));
        }
        ring_arm2<C, RB>(ring2, g + 2, smem_u32(sOnes), smem_u32(sB2));
        ring_mma_step2<C, RB>(ring2, g, make_desc(smem_u32(sT + ts * ROWB), PLANE, 128), smem_u32(sW2), 2 * PLANE);
        mma2_commit_mc(&r2_ready[ring_idx<RB>(g)], 0x3);
        mma2_commit_mc(&t_empty[ts], 0x3);
        if (k == n_t - 1) {
          mma2_commit_mc(&r2_ready[ring_idx<RB>(g + 1)], 0x3);
          mma2_commit_mc(&r2_ready[ring_idx<RB>(g + 2)], 0x3);
        }
        if (++ts == NT) { ts = 0; tph ^= 1; }
      }
      G2 += n_t + 2;
      SR_PIECE_END
    }
    __syncwarp();
  } else if (warp < 6) {
    // ===================== conv1 epilogue (both CTAs): drain t rows -> ReLU -> own t smem ring ==================
    const int quarter = warp & 3;
    const int m = quarter * 32 + lane_id();
    const uint32_t lane_off = (uint32_t)(quarter * 32) << 16;
    for (int b = 0; b < RB; ++b)
      if (lane_id() == 0) mbar_arrive_remote(cluster_addr(&r1_free[b], 0));
    int ts = 0;
    uint32_t tph = 0;
    unsigned G = 0;
    SR_PIECE_BEGIN
    const int tcol = x0 - 1 + m;
    const bool col_ok = tcol >= 0 && tcol < W;
    for (int q = -1; q <= n_f; ++q) {  // out rows of conv1 = t rows y0-2+q
      const unsigned g = G + q + 1;
      const bool emit = q >= 1 && q <= n_f - 2;
      const int trow = y0 - 2 + q;
      const bool ok = col_ok && trow >= 0 && trow < H;
      if (emit) mbar_wait(&t_empty[ts], tph ^ 1);
      const int b = ring_idx<RB>(g);
      mbar_wait(&r1_ready[b], (uint32_t)(g / RB) & 1u);
      tc_fence_after();
      float v[C];
#pragma unroll
      for (int c0 = 0; c0 < C; c0 += 8) tmem_ld8(ring1 + lane_off + b * C + c0, v + c0);
      tmem_ld_wait();
      tc_fence_before();
      __syncwarp();
      if (lane_id() == 0) mbar_arrive_remote(cluster_addr(&r1_free[b], 0));
      if (emit) {
        uint8_t* dst = sT + ts * ROWB + m * 16;
#pragma unroll
        for (int j = 0; j < CCH; ++j) {
          float a[8];
#pragma unroll
          for (int e = 0; e < 8; ++e) a[e] = ok ? fmaxf(v[8 * j + e], 0.f) : 0.f;
          uint4 u;
          u.x = pack_bf16x2(a[0], a[1]);
          u.y = pack_bf16x2(a[2], a[3]);
          u.z = pack_bf16x2(a[4], a[5]);
          u.w = pack_bf16x2(a[6], a[7]);
          *reinterpret_cast<uint4*>(dst + j * PLANE) = u;
        }
        fence_proxy_async_smem();
        __syncwarp();
        if (lane_id() == 0) mbar_arrive_remote(cluster_addr(&t_full[ts], 0));  // after fence.proxy.async
        if (++ts == NT) { ts = 0; tph ^= 1; }
      }
    }
    G += n_f + 2;
    SR_PIECE_END
    for (int k = 0; k < NT; ++k) {  // drain: the last releases of the t slots (multicast commits) have landed
      mbar_wait(&t_empty[ts], tph ^ 1);
      if (++ts == NT) { ts = 0; tph ^= 1; }
    }
  } else if (warp < 10 || warp >= 11) {
    // ===================== conv2 epilogue (both CTAs): drain rows -> + residual f -> smem -> TMA store ==========
    // (EPI2 groups: group grp takes the output rows with g % EPI2 == grp, its own staging slots and named barrier)
    constexpr int EPI2 = Cfg::EPI2;
    const int grp = warp >= 11 ? 1 : 0;
    const int quarter = warp & 3;
    const int m = quarter * 32 + lane_id();
    const uint32_t lane_off = (uint32_t)(quarter * 32) << 16;
    const bool leader = (warp == (grp ? 11 : 6) && lane_id() == 0);
    if (grp == 0)
      for (int b = 0; b < RB; ++b)
        if (lane_id() == 0) mbar_arrive_remote(cluster_addr(&r2_free[b], 0));
    int os = 0;
    unsigned G = 0;
    SR_PIECE_BEGIN
    const bool lane_ok = m < kB2TW && x0 + m < W;
    // the residual row of this group's next kept output row is loaded while the current one is processed
    uint4 res_nx[C / 8];
    auto ld_res = [&](int q) {
      if (q >= 1 && q <= n_t - 2 && lane_ok) {
        const size_t pix = (((size_t)n * H + y0 - 1 + q) * W) + x0 + m;
        const uint4* rp = reinterpret_cast<const uint4*>(fres + pix * C);
#pragma unroll
        for (int j = 0; j < C / 8; ++j) res_nx[j] = __ldg(rp + j);
      }
    };
    auto own = [&](int q) { return (int)((G + q + 1) % EPI2) == grp; };
    int qn = -1;  // this group's next row index
    while (qn <= n_t && !own(qn)) ++qn;
    {
      int qf = qn;  // first kept row of the group
      while (qf <= n_t && !(own(qf) && qf >= 1 && qf <= n_t - 2)) ++qf;
      ld_res(qf);
    }
    for (int q = qn; q <= n_t; q += EPI2) {  // out rows of conv2 = output rows y0-1+q
      const unsigned g = G + q + 1;
      const bool emit = q >= 1 && q <= n_t - 2;
      const int r = y0 - 1 + q;
      uint4 res[C / 8];
      if (emit) {
#pragma unroll
        for (int j = 0; j < C / 8; ++j) res[j] = res_nx[j];
        ld_res(q + EPI2);
      }
      const int b = ring_idx<RB>(g);
      mbar_wait(&r2_ready[b], (uint32_t)(g / RB) & 1u);
      tc_fence_after();
      float v[C];
#pragma unroll
      for (int c0 = 0; c0 < C; c0 += 8) tmem_ld8(ring2 + lane_off + b * C + c0, v + c0);
      tmem_ld_wait();
      tc_fence_before();
      __syncwarp();
      if (lane_id() == 0) mbar_arrive_remote(cluster_addr(&r2_free[b], 0));
      if (emit) {
        uint8_t* const slot = sO + (grp * NO + os) * OUTB;
        if (lane_ok) {
          uint8_t* orow = slot + m * C * 2;
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
            uint4 u;
            u.x = pack_bf16x2(a[0], a[1]);
            u.y = pack_bf16x2(a[2], a[3]);
            u.z = pack_bf16x2(a[4], a[5]);
            u.w = pack_bf16x2(a[6], a[7]);
            ov[j] = u;
          }
          st_pix_rot<C / 8>(orow, ov);
        }
        fence_proxy_async_smem();
        named_bar_sync(2 + grp, 128);
        if (leader && !dummy) {
          tma_store_4d(&tm_out, slot, 0, x0, r, n);
          bulk_commit();
          bulk_wait_read<NO - 2>();
        } else if (leader) {
          bulk_wait_read<0>();
        }
        os = os == NO - 1 ? 0 : os + 1;
      }
    }
    G += n_t + 2;
    SR_PIECE_END
    if (leader) bulk_wait<0>();
  }
#undef SR_PIECE_BEGIN
#undef SR_PIECE_END
  tc_fence_before();
  __syncthreads();
  cluster_sync_all();  // every remote arrival and multicast commit of the pair has landed; both CTAs are done
  if (warp == 1) tmem_dealloc2<512>(tmem);
}

template <int C>
static cudaError_t launch_block2_t(const CUtensorMap& tf, const CUtensorMap& to, const bf16* w1, const bf16* w2,
                                   const float* b1, const float* b2, const bf16* f, int N, int H, int W, int grid,
                                   cudaStream_t st) {
  auto kern = k_resblock2<C>;
  static bool configured = false;
  if (!configured) {
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)B2Cfg<C>::SMEM);
    if (e != cudaSuccess) return e;
    configured = true;
  }
  return launch_k(kern, dim3(grid), dim3(B2Cfg<C>::THREADS), B2Cfg<C>::SMEM, st, tf, to, w1, w2, b1, b2, f, N, H, W);
}

// Offered for C = 32 (BASELINE config 2's 8 x 32 net), where a row-step's MMAs are short and the pair's halved B
// reads and single issuer pay (same-session A/B: 0.83 -> 0.69 ms per 30 540p frames).  At C = 48 the 4.5 C weight
// rows cost a slot of the f ring and of the output staging, and the pair measured no faster than the single-CTA
// kernel (17.4 vs 17.6-20.5 ms per 30 720p frames across the variants tried), so C = 48 stays on k_resblock.
bool resblock2_supported(int cp, int W) {
  constexpr size_t kStatic = 1024;  // barriers, TMEM address, bias staging (static shared memory)
  if (W < 96) return false;
  if (cp == 32) return B2Cfg<32>::SMEM + kStatic <= 227 * 1024;
  return false;
}

cudaError_t launch_resblock2(int cp, const bf16* f, const bf16* w1fold, const bf16* w2fold, const float* b1,
                             const float* b2, bf16* out, int N, int H, int W, cudaStream_t st) {
  if (!resblock2_supported(cp, W)) return cudaErrorNotSupported;
  CUtensorMap tf, to;
  if (make_act_tmap(&tf, f, N, H, W, cp, 130, 1, cp / 8, CHUNK_ROW_PIX) != CUDA_SUCCESS) return cudaErrorInvalidValue;
  if (make_row_tmap(&to, out, N, H, W, cp, kB2TW, cp) != CUDA_SUCCESS) return cudaErrorInvalidValue;
  const long long cols = (long long)N * ((W + kB2TW - 1) / kB2TW);
  const long long units = (cols + 1) / 2 * H;
  long long pairs = num_sms() / 2;
  if (units < pairs) pairs = units;
  const int grid = (int)(2 * pairs);
  return launch_block2_t<32>(tf, to, w1fold, w2fold, b1, b2, f, N, H, W, grid, st);
}

}  // namespace sr

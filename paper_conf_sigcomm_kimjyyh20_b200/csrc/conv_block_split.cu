// Residual block on a CTA pair split by conv (inference):  f' = f + conv2(ReLU(conv1(f) + b1)) + b2   (sm_100a)
//
// Same arithmetic and the same rolling dy-fold form as k_resblock (conv_block.cu), but the two convs of a block run
// on the two SMs of a cluster of 2 instead of both on one SM:
//   rank 0 ("conv1 CTA"): TMA producer of the f rows, conv1 MMA issuer, two epilogue groups that drain finished t
//                         rows (ReLU, bf16) and write them straight into rank 1's t ring (st.shared::cluster);
//   rank 1 ("conv2 CTA"): conv2 MMA issuer on its own t ring, two epilogue groups (+ residual f from L2/HBM,
//                         pixel-major staging, TMA store).
// Why: on one SM both convs' accumulator rings share the 512 TMEM columns (5 blocks of 48 per conv at C = 48), so
// 2 of every 5 row-steps wrap inside the three dy targets and issue as two MMA groups of N = 2C and N = C, whose
// operand reads are bound by the shared-memory port (measured: resblock<48> -14% with the wraps suppressed).  With
// one conv per SM the ring has 10 blocks (wraps 1 step in 5) and each SM's shared memory carries one conv's operand
// and epilogue traffic; each SM still does the same number of MMAs per row of the strip.
// t rows cross the pair by the bulk-copy engine: the conv1 epilogue group writes its row into a local mirror of
// rank 1's t ring slot, then one thread issues cp.async.bulk shared::cta -> shared::cluster, whose bytes complete
// the transaction count of rank 1's t_full[s] (async proxy to async proxy: no generic-proxy ordering across SMs).
// t_empty[s] (rank 0) is signalled by rank 1's conv2 MMAs completing on slot s (tcgen05.commit multicast to rank
// 0); it also frees rank 0's mirror slot (the copy out of it completed before rank 1 could consume the row).
// (Storing the t row with st.shared::cluster and a release.cluster arrive per warp was 2.2x slower than the
// single-CTA kernel.)
#include <cuda.h>
#include "ptx.cuh"
#include "tmap.h"
#include "sr_internal.h"
#include "ring.cuh"
#include "launch.cuh"
#include "rot.cuh"
#include "pair.cuh"

namespace sr {

static constexpr int kSpThreads = 320;  // 10 warps: 0 producer (rank 0), 1 issuer, 2..9 two epilogue groups
static constexpr int kSpTW = 126;       // output pixels per strip
static constexpr int kSpNO = 3;         // staging rows per epilogue group (rank 1)

template <int C>
struct SpCfg {
  static constexpr int CCH = C / 8, CB = C / 16, N = 3 * C;
  static constexpr int RB = (512 / C) < 16 ? (512 / C) : 16;  // TMEM ring blocks (one conv per CTA)
  static constexpr uint32_t WBYTES = 9u * C * C * 2u;
  static constexpr uint32_t WB_AL = (WBYTES + 1023u) & ~1023u;
  // f and t rows in the K-major SWIZZLE_32B layout: one plane per 16-channel block, pixel rows of 32 B (the TMA
  // moves 32-B units: half the element count of 16-B chunk planes, whose ~1 element/clk TMA rate would otherwise
  // bound the conv1 SM; scripts/tma_rate.py), the dx tap a 32-B start shift (scripts/sw32k_probe.py)
  static constexpr uint32_t PLANE = 130 * 32;
  static constexpr uint32_t ROWB = ((CB * PLANE) + 255u) & ~255u;         // f / t ring slot
  static constexpr uint32_t OUTB = ((kSpTW * C * 2) + 1023u) & ~1023u;    // staging row
  static constexpr uint32_t ARMB = ((kArmOnesBytes + C * 32) + 1023u) & ~1023u;  // ones + this CTA's bias tile
  static constexpr size_t FIXED = 1024 + WB_AL + ARMB;
  static constexpr size_t BUDGET = 227 * 1024 - 2048;  // 2 KB: static shared memory (barriers)
  static constexpr int NT_FIT = (int)((BUDGET - FIXED - 2 * kSpNO * (size_t)OUTB) / ROWB);
  static constexpr int NT = NT_FIT < 8 ? NT_FIT : 8;  // t ring (rank 1) and its mirror (rank 0), same offset
  static constexpr int NF_FIT = (int)((BUDGET - FIXED) / ROWB) - NT;
  static constexpr int NF = NF_FIT < 8 ? NF_FIT : 8;  // rank 0: f rows
  static constexpr size_t R0 = (size_t)(NT + NF) * ROWB, R1 = (size_t)NT * ROWB + 2 * kSpNO * (size_t)OUTB;
  static constexpr size_t SMEM = FIXED + (R0 > R1 ? R0 : R1);
  static constexpr bool FITS = NF >= 4 && NT >= 4;
};

__device__ __forceinline__ void sts128(uint32_t a, uint4 u) {
  asm volatile("st.shared.v4.u32 [%0], {%1, %2, %3, %4};" ::"r"(a), "r"(u.x), "r"(u.y), "r"(u.z), "r"(u.w) : "memory");
}
// bulk copy of `bytes` (16-B multiple) from this CTA's shared memory to a peer CTA's (shared::cluster addresses
// of the destination and of the peer's mbarrier, whose transaction count the bytes complete)
__device__ __forceinline__ void bulk_copy_to_peer(uint32_t dst_caddr, const void* src, uint32_t bytes,
                                                  uint32_t bar_caddr) {
  asm volatile("cp.async.bulk.shared::cluster.shared::cta.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                   dst_caddr),
               "r"(smem_u32(src)), "r"(bytes), "r"(bar_caddr)
               : "memory");
}
// arrive on the mbarrier at `bar`'s offset in the CTAs of `mask` once this thread's prior MMAs completed
__device__ __forceinline__ void mma_commit_mc(uint64_t* bar, uint16_t mask) {
  asm volatile(
      "tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;" ::"r"(
          smem_u32(bar)),
      "h"(mask)
      : "memory");
}

template <int C>
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(kSpThreads, 1)
k_resblock_split(const __grid_constant__ CUtensorMap tm_f, const __grid_constant__ CUtensorMap tm_out,
                 const bf16* __restrict__ w1, const bf16* __restrict__ w2, const float* __restrict__ b1,
                 const float* __restrict__ b2, const bf16* __restrict__ fres, const int N, const int H,
                 const int W, long long* __restrict__ dbg) {
  // dbg (benchmarking only, pair 0): clock64 stamps [rank * 8 + event][index]
#define SP_DBG(ev, idx) \
  if (dbg && blockIdx.x < 2 && (idx) >= 0 && (idx) < 256) dbg[((int)rank * 8 + (ev)) * 256 + (idx)] = clock64();
  using Cfg = SpCfg<C>;
  constexpr int CB = Cfg::CB, RB = Cfg::RB, NF = Cfg::NF, NT = Cfg::NT;
  constexpr uint32_t PLANE = Cfg::PLANE, ROWB = Cfg::ROWB, OUTB = Cfg::OUTB;

  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sW = smem;                    // this CTA's conv weights (dy-fold layout)
  uint8_t* sOnes = sW + Cfg::WB_AL;      // bias-arming operands (ring.cuh)
  uint8_t* sB = sOnes + kArmOnesBytes;
  uint8_t* sR = sOnes + Cfg::ARMB;       // t ring (rank 1) / its mirror (rank 0), then f ring / staging rows
  uint8_t* sT = sR;
  uint8_t* sF = sR + (size_t)NT * ROWB;
  uint8_t* sO = sR + (size_t)NT * ROWB;
  __shared__ __align__(8) uint64_t f_full[NF], f_empty[NF], t_full[NT], t_empty[NT], r_ready[RB], r_free[RB], w_bar;
  __shared__ uint32_t tmem_base_sh;
  __shared__ __align__(16) float4 sbv[C / 4];

  const int warp = warp_id();
  const uint32_t rank = cluster_rank();
  // spare t positions 128, 129 of every plane (read by the two invalid conv2 lanes): zero in the ring and in the
  // mirror (whole planes are copied)
  for (int i = threadIdx.x; i < NT * CB * 4; i += blockDim.x) {  // 2 positions x 2 halves per plane
    const int slot = i / (CB * 4), rem = i % (CB * 4);
    *reinterpret_cast<uint4*>(sT + slot * ROWB + (rem / 4) * PLANE + (128 + (rem / 2) % 2) * 32 + (rem % 2) * 16) =
        make_uint4(0, 0, 0, 0);
  }
  fence_proxy_async_smem();
  if (warp == 0 && lane_id() == 0) {
    for (int s = 0; s < NF; ++s) { mbar_init(&f_full[s], 1); mbar_init(&f_empty[s], 1); }
    for (int s = 0; s < NT; ++s) { mbar_init(&t_full[s], 1); mbar_init(&t_empty[s], 1); }
    for (int s = 0; s < RB; ++s) { mbar_init(&r_ready[s], 1); mbar_init(&r_free[s], 4); }
    mbar_init(&w_bar, 1);
    fence_barrier_init();
  }
  if (warp == 1) tmem_alloc<512>(&tmem_base_sh);
  tc_fence_before();
  // weights and biases before the PDL wait (written >= 2 kernels upstream; see k_resblock's prologue)
  const float* bias = rank == 0 ? b1 : b2;
  if (warp == 0 && lane_id() == 0) {
    mbar_arrive_expect_tx(&w_bar, Cfg::WBYTES);
    bulk_load(sW, rank == 0 ? w1 : w2, Cfg::WBYTES, &w_bar);
  }
  if (threadIdx.x < C) reinterpret_cast<float*>(sbv)[threadIdx.x] = bias[threadIdx.x];
  __syncthreads();
  arm_tiles_fill(sOnes, sB, reinterpret_cast<const float*>(sbv), C, threadIdx.x, blockDim.x);
  fence_proxy_async_smem();
  cluster_sync_all();  // both CTAs' barriers initialised before any remote arrive / store
  pdl_enter();
  tc_fence_after();
  const uint32_t ring = tmem_base_sh;

  const int tiles_x = (W + kSpTW - 1) / kSpTW;
  const long long total = (long long)N * tiles_x * H;
  const long long npairs = gridDim.x / 2, pair = blockIdx.x / 2;
  const long long beg = total * pair / npairs, end = total * (pair + 1) / npairs;
#define SR_PIECE_BEGIN                                                                \
  for (long long pos = beg; pos < end;) {                                             \
    const int col = (int)(pos / H), y0 = (int)(pos - (long long)col * H);             \
    const int y1 = (int)min((long long)H, y0 + (end - pos));                          \
    pos += y1 - y0;                                                                   \
    const int n = col / tiles_x, x0 = (col - n * tiles_x) * kSpTW;                    \
    const int n_f = y1 - y0 + 4, n_t = n_f - 2;                                       \
    (void)n; (void)x0; (void)n_t;
#define SR_PIECE_END }

  if (rank == 0) {
    if (warp == 0) {
      // ===================== producer: f rows y0-2 .. y1+1 of every piece =====================
      if (elect_one()) {
        tma_prefetch_desc(&tm_f);
        int s = 0;
        uint32_t ph = 0;
        SR_PIECE_BEGIN
        for (int i = 0; i < n_f; ++i) {
          mbar_wait(&f_empty[s], ph ^ 1);
          mbar_arrive_expect_tx(&f_full[s], CB * PLANE);
          tma_load_5d(sF + s * ROWB, &tm_f, &f_full[s], 0, x0 - 2, 0, y0 - 2 + i, n);
          SP_DBG(0, i)
          if (++s == NF) { s = 0; ph ^= 1; }
        }
        SR_PIECE_END
      }
      __syncwarp();
    } else if (warp == 1) {
      // ===================== conv1 MMA issuer: step st consumes f row st =====================
      if (elect_one()) {
        mbar_wait(&w_bar, 0);
        const uint64_t bd = make_desc(smem_u32(sW), Cfg::N * 16, 128);
        int fs = 0;
        uint32_t fph = 0;
        unsigned G1 = 0, acq = 0;
        SR_PIECE_BEGIN
        for (int st = 0; st < n_f; ++st) {
          const unsigned g = G1 + st;
          SP_DBG(1, st)
          for (; acq < g + 3; ++acq) mbar_wait(&r_free[ring_idx<RB>(acq)], (uint32_t)(acq / RB) & 1u);
          SP_DBG(2, st)
          mbar_wait(&f_full[fs], fph);
          SP_DBG(3, st)
          tc_fence_after();
          if (st == 0) {
            ring_arm<C, RB>(ring, g, smem_u32(sOnes), smem_u32(sB));
            ring_arm<C, RB>(ring, g + 1, smem_u32(sOnes), smem_u32(sB));
          }
          ring_arm<C, RB>(ring, g + 2, smem_u32(sOnes), smem_u32(sB));
          ring_mma_step<C, C, RB, 32>(ring, g, make_desc_sw(smem_u32(sF + fs * ROWB), 16, 256, 6), bd, PLANE);
          mma_commit(&r_ready[ring_idx<RB>(g)]);
          mma_commit(&f_empty[fs]);
          if (st == n_f - 1) {
            mma_commit(&r_ready[ring_idx<RB>(g + 1)]);
            mma_commit(&r_ready[ring_idx<RB>(g + 2)]);
          }
          if (++fs == NF) { fs = 0; fph ^= 1; }
        }
        G1 += n_f + 2;
        SR_PIECE_END
      }
      __syncwarp();
    } else {
      // ============ conv1 epilogue (two groups, alternate rows): drain t row -> ReLU -> rank 1's t ring ============
      const int grp = (warp - 2) >> 2;
      const int quarter = warp & 3;
      const int m = quarter * 32 + lane_id();
      const uint32_t lane_off = (uint32_t)(quarter * 32) << 16;
      if (grp == 0)
        for (int b = 0; b < RB; ++b)
          if (lane_id() == 0) mbar_arrive(&r_free[b]);
      const bool issuer = (warp == 2 + 4 * grp) && lane_id() == 0;
      const uint32_t tT = cluster_addr(sT, 1);           // rank 1's t ring
      const uint32_t tfull = cluster_addr(&t_full[0], 1);
      unsigned G = 0, emitted = 0;
      SR_PIECE_BEGIN
      const int tcol = x0 - 1 + m;
      const bool col_ok = tcol >= 0 && tcol < W;
      for (int q = -1; q <= n_f; ++q) {  // out rows of conv1 = t rows y0-2+q
        const unsigned g = G + q + 1;
        const bool emit = q >= 1 && q <= n_f - 2;
        const unsigned xi = emitted;
        emitted += emit;
        if ((int)(g & 1u) != grp) continue;
        const int trow = y0 - 2 + q;
        const bool ok = col_ok && trow >= 0 && trow < H;
        const int b = ring_idx<RB>(g);
        mbar_wait(&r_ready[b], (uint32_t)(g / RB) & 1u);
        if (warp == 2 + 4 * grp && lane_id() == 0) { SP_DBG(4, q + 1) }
        tc_fence_after();
        float v[C];
#pragma unroll
        for (int c0 = 0; c0 < C; c0 += 8) tmem_ld8(ring + lane_off + b * C + c0, v + c0);
        tmem_ld_wait();
        tc_fence_before();
        __syncwarp();
        if (lane_id() == 0) mbar_arrive(&r_free[b]);
        if (!emit) continue;
        const unsigned ts = xi % NT;
        mbar_wait(&t_empty[ts], ((xi / NT) & 1u) ^ 1u);  // rank 1's conv2 MMAs are done with the slot
        // SWIZZLE_32B: the 16-B half h of pixel row m sits at 16 (h ^ bit 7 of its address); odd lanes store their
        // halves in the other order, so each store instruction covers all 32 banks once per 8 lanes
        const uint32_t dst = smem_u32(sT + ts * ROWB) + (uint32_t)m * 32u;
#pragma unroll
        for (int jb = 0; jb < CB; ++jb) {
          uint4 hv[2];
#pragma unroll
          for (int h = 0; h < 2; ++h) {
            float a[8];
#pragma unroll
            for (int e = 0; e < 8; ++e) a[e] = ok ? fmaxf(v[16 * jb + 8 * h + e], 0.f) : 0.f;
            hv[h].x = pack_bf16x2(a[0], a[1]);
            hv[h].y = pack_bf16x2(a[2], a[3]);
            hv[h].z = pack_bf16x2(a[4], a[5]);
            hv[h].w = pack_bf16x2(a[6], a[7]);
          }
          const uint32_t row = dst + jb * PLANE;
          const uint32_t sw = (row >> 7) & 1u;
          const uint32_t first = (uint32_t)m & 1u;
          sts128(row + 16u * (first ^ sw), first ? hv[1] : hv[0]);
          sts128(row + 16u * (first ^ 1u ^ sw), first ? hv[0] : hv[1]);
        }
        fence_proxy_async_smem();
        named_bar_sync(2 + grp, 128);
        if (issuer) {
          SP_DBG(5, q + 1)
          mbar_arrive_expect_tx_remote(tfull + ts * 8u, CB * PLANE);
          bulk_copy_to_peer(tT + ts * ROWB, sT + ts * ROWB, CB * PLANE, tfull + ts * 8u);
        }
      }
      G += n_f + 2;
      SR_PIECE_END
    }
  } else {
    if (warp == 1) {
      // ===================== conv2 MMA issuer: step k consumes t row k =====================
      if (elect_one()) {
        mbar_wait(&w_bar, 0);
        const uint64_t bd = make_desc(smem_u32(sW), Cfg::N * 16, 128);
        int ts = 0;
        uint32_t tph = 0;
        unsigned G2 = 0, acq = 0;
        SR_PIECE_BEGIN
        for (int k = 0; k < n_t; ++k) {
          const unsigned g = G2 + k;
          SP_DBG(1, k)
          for (; acq < g + 3; ++acq) mbar_wait(&r_free[ring_idx<RB>(acq)], (uint32_t)(acq / RB) & 1u);
          SP_DBG(2, k)
          mbar_wait(&t_full[ts], tph);
          SP_DBG(3, k)
          tc_fence_after();
          if (k == 0) {
            ring_arm<C, RB>(ring, g, smem_u32(sOnes), smem_u32(sB));
            ring_arm<C, RB>(ring, g + 1, smem_u32(sOnes), smem_u32(sB));
          }
          ring_arm<C, RB>(ring, g + 2, smem_u32(sOnes), smem_u32(sB));
          ring_mma_step<C, C, RB, 32>(ring, g, make_desc_sw(smem_u32(sT + ts * ROWB), 16, 256, 6), bd, PLANE);
          mma_commit(&r_ready[ring_idx<RB>(g)]);
          mma_commit_mc(&t_empty[ts], 0x1);  // the slot is free: rank 0's epilogue may overwrite it
          if (k == n_t - 1) {
            mma_commit(&r_ready[ring_idx<RB>(g + 1)]);
            mma_commit(&r_ready[ring_idx<RB>(g + 2)]);
          }
          if (++ts == NT) { ts = 0; tph ^= 1; }
        }
        G2 += n_t + 2;
        SR_PIECE_END
      }
      __syncwarp();
    } else if (warp >= 2) {
      // ====== conv2 epilogue (two groups, alternate rows): drain -> + residual f -> staging -> TMA store ======
      const int grp = (warp - 2) >> 2;
      const int quarter = warp & 3;
      const int m = quarter * 32 + lane_id();
      const uint32_t lane_off = (uint32_t)(quarter * 32) << 16;
      const bool leader = (warp == 2 + 4 * grp) && lane_id() == 0;
      if (grp == 0)
        for (int b = 0; b < RB; ++b)
          if (lane_id() == 0) mbar_arrive(&r_free[b]);
      uint8_t* sOg = sO + (size_t)grp * kSpNO * OUTB;
      int os = 0;
      unsigned G = 0;
      SR_PIECE_BEGIN
      const bool lane_ok = m < kSpTW && x0 + m < W;
      uint4 res_nx[C / 8];
      auto ld_res = [&](int q) {  // the group's next row is two rows on: its residual is loaded a row-step ahead
        if (q >= 1 && q <= n_t - 2 && lane_ok) {
          const size_t pix = (((size_t)n * H + y0 - 1 + q) * W) + x0 + m;
          const uint4* rp = reinterpret_cast<const uint4*>(fres + pix * C);
#pragma unroll
          for (int j = 0; j < C / 8; ++j) res_nx[j] = __ldg(rp + j);
        }
      };
      ld_res(((int)(G & 1u) == grp) ? -1 : 0);
      for (int q = -1; q <= n_t; ++q) {  // out rows of conv2 = output rows y0-1+q
        const unsigned g = G + q + 1;
        if ((int)(g & 1u) != grp) continue;
        const bool emit = q >= 1 && q <= n_t - 2;
        const int r = y0 - 1 + q;
        uint4 res[C / 8];
#pragma unroll
        for (int j = 0; j < C / 8; ++j) res[j] = res_nx[j];
        ld_res(q + 2);
        const int b = ring_idx<RB>(g);
        mbar_wait(&r_ready[b], (uint32_t)(g / RB) & 1u);
        if (warp == 2 + 4 * grp && lane_id() == 0) { SP_DBG(4, q + 1) }
        tc_fence_after();
        float v[C];
#pragma unroll
        for (int c0 = 0; c0 < C; c0 += 8) tmem_ld8(ring + lane_off + b * C + c0, v + c0);
        tmem_ld_wait();
        tc_fence_before();
        __syncwarp();
        if (lane_id() == 0) mbar_arrive(&r_free[b]);
        if (!emit) continue;
        if (lane_ok) {
          uint8_t* orow = sOg + os * OUTB + m * C * 2;
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
        if (leader) {
          SP_DBG(5, q + 1)
          tma_store_4d(&tm_out, sOg + os * OUTB, 0, x0, r, n);
          bulk_commit();
          bulk_wait_read<kSpNO - 2>();
        }
        os = os == kSpNO - 1 ? 0 : os + 1;
      }
      G += n_t + 2;
      SR_PIECE_END
      if (leader) bulk_wait<0>();
    }
  }
#undef SR_PIECE_BEGIN
#undef SR_PIECE_END
  tc_fence_before();
  __syncthreads();
  if (warp == 1) tmem_dealloc<512>(ring);
  cluster_sync_all();  // no CTA leaves while its peer may still signal its barriers or write its shared memory
#undef SP_DBG
}

template <int C>
static cudaError_t launch_split_t(const CUtensorMap& tf, const CUtensorMap& to, const bf16* w1, const bf16* w2,
                                  const float* b1, const float* b2, const bf16* f, int N, int H, int W, int grid,
                                  cudaStream_t st, long long* dbg) {
  if constexpr (!SpCfg<C>::FITS) {
    return cudaErrorNotSupported;
  } else {
    auto kern = k_resblock_split<C>;
    static bool configured = false;
    if (!configured) {
      cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)SpCfg<C>::SMEM);
      if (e != cudaSuccess) return e;
      configured = true;
    }
    return launch_k(kern, dim3(grid), dim3(kSpThreads), SpCfg<C>::SMEM, st, tf, to, w1, w2, b1, b2, f, N, H, W, dbg);
  }
}

bool resblock_split_supported(int cp, int W) {
  if (W < 96) return false;
  if (cp == 16) return SpCfg<16>::FITS;
  if (cp == 32) return SpCfg<32>::FITS;
  if (cp == 48) return SpCfg<48>::FITS;
  return false;
}

cudaError_t launch_resblock_split(int cp, const bf16* f, const bf16* w1fold, const bf16* w2fold, const float* b1,
                                  const float* b2, bf16* out, int N, int H, int W, cudaStream_t st, long long* dbg) {
  if (!resblock_split_supported(cp, W)) return cudaErrorNotSupported;
  CUtensorMap tf, to;
  if (make_act_tmap_sw32(&tf, f, N, H, W, cp, 130, 1) != CUDA_SUCCESS) return cudaErrorInvalidValue;
  if (make_row_tmap(&to, out, N, H, W, cp, kSpTW, cp) != CUDA_SUCCESS) return cudaErrorInvalidValue;
  const long long units = (long long)N * ((W + kSpTW - 1) / kSpTW) * H;
  long long pairs = num_sms() / 2;
  if (units < pairs) pairs = units;
  const int grid = (int)(2 * pairs);
  if (cp == 16) return launch_split_t<16>(tf, to, w1fold, w2fold, b1, b2, f, N, H, W, grid, st, dbg);
  if (cp == 32) return launch_split_t<32>(tf, to, w1fold, w2fold, b1, b2, f, N, H, W, grid, st, dbg);
  if (cp == 48) return launch_split_t<48>(tf, to, w1fold, w2fold, b1, b2, f, N, H, W, grid, st, dbg);
  return cudaErrorNotSupported;
}

}  // namespace sr

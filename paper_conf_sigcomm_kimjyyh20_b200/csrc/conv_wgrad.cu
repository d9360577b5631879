// Weight gradients of 3x3 convs over wide images (W >= 128), rolling over dY rows, many convs per launch (sm_100a).
//
//   dW[co,ci,ky,kx] = sum_p dY[p,co] X[p + (ky-1, kx-1), ci],   db[co] = sum_p dY[p,co]
//
// MMA form.  With N = Cout (the tiled k_wgrad in conv.cu) an MMA is bound by the 128 B/clk shared-memory read port
// (44.6 cycles per M=128, N=48 MMA instead of the 24-cycle tensor floor, scripts/mma_rate.py).  Here the
// horizontal tap goes into N:
//   D[(ky,ci), (kx,co)] = sum_j  X[y+ky-1, x0+j, ci]  *  dY[y, x0+j+1-kx, co]       (j = 0..127 of the strip)
// so one MMA is M = 128 (ky, ci) rows x N = 3*Cout (kx, co) columns x K = 16 pixels.  The kx shift is a separate
// TMA box of the same dY row at x0+1-kx (three boxes per row, zero-filled outside the image) laid out as
// consecutive N-atoms, so one descriptor covers all three.  The three X rows of a dY row are consecutive M-atoms
// because the X ring mirrors its first two slots behind the last (a row loaded into slot s < 2 is also written to
// slot NX+s), so slots (s, s+1, s+2) are contiguous for every s.  At Cin = Cout = 48: 16 MMAs of N = 144 per
// 128-pixel row (72 cycles each at the tensor floor) instead of 48 MMAs of N = 48 (44.6 cycles each).
//
// Batching.  All wgrads of a training iteration are independent of each other (each needs only its conv's saved
// input X and output gradient dY), so they run as ONE launch at the end of the backward pass: the rows of all
// jobs (job, image, 128-px strip, dY row) are split into contiguous, balanced ranges, one per CTA (~138 rows per
// CTA at the 8x48 training shape, i.e. ~9 CTAs per conv).  A CTA accumulates in TMEM over its rows of one job
// (split-K), and at a job boundary the epilogue warps write the partial (slot b + k for CTA b, job k: injective
// because every range is non-empty) while the producer already streams the next job's rows.  One grid barrier
// (cooperative launch) and a deterministic reduction over the ~9 partials of every output, in CTA order, replace
// the per-conv barrier + 148-way reduction.  The bias gradient is summed from the unshifted dY copy by the
// epilogue warps while the MMAs run.
//
// Warp roles (384 threads): warp 0 TMA producer, warp 1 TMEM alloc + MMA issuer, warps 2..5 bias grad + drain; all
// 12 warps take part in the reduction.
#include <cuda.h>
#include <algorithm>
#include <cstdlib>
#include "ptx.cuh"
#include "tmap.h"
#include "sr_internal.h"
#include "kernels.h"
#include "launch.cuh"

namespace sr {

static constexpr int kWrThreads = 384;
static constexpr int kWrTW = 128;  // pixels per strip (= K per dY row)
static constexpr int kWmOBM = 4;   // max 16-channel blocks of dY supported (Cout <= 64)

struct WmJob {
  int cinp, coutp, cin, cout;
  float* gW;  // canonical OIHW [cout][cin][3][3]
  float* gb;  // [cout]
  int off4;   // float4 offset of this job's partial outputs in the flattened reduction space
};
struct WmParams {
  CUtensorMap tmx[kWgradMaxJobs];
  CUtensorMap tmy[kWgradMaxJobs];
  WmJob job[kWgradMaxJobs];
  int J, N, H, W;
  int nq;         // reduction: partial groups per output
  int maxstride;  // floats per partial slot
  int total4;     // float4 outputs over all jobs
  float scale;
  float* ws;      // partial slots [(grid + J)][maxstride]; job k of CTA b -> slot b + k
  unsigned* sync;
  long long* dbg;
};

// CBM / OBM = max 16-channel blocks of X / dY over the jobs; a job has cinp = 16 or 16 CBM (its X row atoms (ky, cb)
// are then at a uniform stride: ATOM when cb = CBM, the slot stride S when cb = 1).  The operands stream from HBM
// (all of an iteration's activations), so the rings are as deep as shared memory allows: with NX X slots the
// producer runs NX - 3 rows ahead of the MMAs.
template <int CBM, int OBM>
struct WmCfg {
  static constexpr uint32_t ATOM = kWrTW * 32;  // one 16-channel block of a 128-px row (4 KB)
  static constexpr uint32_t S = CBM * ATOM;     // X ring slot
  static constexpr uint32_t DYS = 3 * OBM * ATOM;  // one dY stage (3 shifted copies)
  static constexpr size_t kBudget = 227 * 1024 - 1024 - 6144;
  static constexpr int NX = (10 * S + 3 * DYS <= kBudget) ? 8 : (8 * S + 3 * DYS <= kBudget) ? 6 : 4;  // (+ 2 mirrors)
  static constexpr uint32_t XRING = (NX + 2) * S;
  static constexpr int NS = (XRING + 3 * DYS <= kBudget) ? 3 : 2;
  static constexpr uint32_t AREA = XRING + NS * DYS;
  // MMA A reads past the triple (garbage M rows, never drained) must stay inside the allocation: worst case is a
  // cb = 1 job (atoms at stride S) from the last ring slot
  static constexpr uint32_t READ_END = (NX - 1) * S + 8 * S;
  static constexpr size_t SMEM = 1024 + (READ_END > AREA ? READ_END : AREA);
};

template <int CBM, int OBM>
__global__ void __launch_bounds__(kWrThreads, 1) k_wgrad_multi(const __grid_constant__ WmParams P) {
  using Cfg = WmCfg<CBM, OBM>;
  constexpr int NX = Cfg::NX, NS = Cfg::NS;
  constexpr uint32_t ATOM = Cfg::ATOM, S = Cfg::S, DYS = Cfg::DYS;

  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);  // stays in the shared window (LDS/STS, not generic)
  uint8_t* sX = smem;
  uint8_t* sDY = smem + Cfg::XRING;
  __shared__ __align__(8) uint64_t x_full[NX], x_empty[NX], d_full[NS], d_empty[NS], done_bar, t_empty;
  __shared__ uint32_t tmem_base_sh;
  __shared__ float sdb[1024];  // bias partials [pixel group][co]

  const int warp = warp_id();
  if (warp == 0 && lane_id() == 0) {
    for (int s = 0; s < NX; ++s) { mbar_init(&x_full[s], 1); mbar_init(&x_empty[s], 1); }
    for (int s = 0; s < NS; ++s) { mbar_init(&d_full[s], 1); mbar_init(&d_empty[s], 2); }
    mbar_init(&done_bar, 1);
    mbar_init(&t_empty, 4);
    fence_barrier_init();
  }
  long long* dbg = P.dbg ? P.dbg + (size_t)blockIdx.x * 8 : nullptr;
  if (dbg && threadIdx.x == 0) dbg[0] = globaltimer();
  if (warp == 1) tmem_alloc<512>(&tmem_base_sh);
  tc_fence_before();
  __syncthreads();
  pdl_wait();  // dependents are released only after the grid barrier below (no co-residency deadlock)
  tc_fence_after();
  const uint32_t tmem = tmem_base_sh;

  const int H = P.H, W = P.W;
  const int tiles_x = (W + kWrTW - 1) / kWrTW;
  const long long per_job = (long long)P.N * tiles_x * H;
  const long long total = per_job * P.J;
  const long long beg = total * blockIdx.x / gridDim.x, end = total * (blockIdx.x + 1) / gridDim.x;
  // pieces: maximal runs of rows of one (job, image, strip) inside [beg, end); seg_end marks the last piece of a
  // job in this CTA (its accumulators are complete)
#define SR_WPIECE_BEGIN                                                                   \
  for (long long pos = beg; pos < end;) {                                                 \
    const int job = (int)(pos / per_job);                                                 \
    const long long rem = pos - (long long)job * per_job;                                 \
    const int col = (int)(rem / H), y0 = (int)(rem - (long long)col * H);                 \
    const int y1 = (int)min((long long)H, y0 + (end - pos));                              \
    pos += y1 - y0;                                                                       \
    const bool seg_end = pos >= end || (int)(pos / per_job) != job;                       \
    const int n = col / tiles_x, x0 = (col - n * tiles_x) * kWrTW;                        \
    const int rows = y1 - y0;                                                             \
    const WmJob& jb = P.job[job];                                                         \
    const int cb = jb.cinp >> 4, ob = jb.coutp >> 4;                                      \
    (void)n; (void)x0; (void)seg_end; (void)cb; (void)ob;
#define SR_WPIECE_END }

  if (warp == 0) {
    // ===================== TMA producer: X rows y0-1 .. y1 (mirrored ring), dY rows y0 .. y1-1 (3 shifts each)
    if (elect_one()) {
      int xs = 0, ds = 0;
      uint32_t xph = 0, dph = 0;
      int pre = -1;
      SR_WPIECE_BEGIN
      const CUtensorMap* tx = &P.tmx[job];
      const CUtensorMap* ty = &P.tmy[job];
      if (job != pre) { tma_prefetch_desc(tx); tma_prefetch_desc(ty); pre = job; }
      const uint32_t xbytes = cb * ATOM, cbytes = ob * ATOM;
      for (int i = 0; i < rows + 2; ++i) {
        mbar_wait(&x_empty[xs], xph ^ 1);
        const bool mir = xs < 2;
        mbar_arrive_expect_tx(&x_full[xs], mir ? 2 * xbytes : xbytes);
        tma_load_5d(sX + xs * S, tx, &x_full[xs], 0, x0, 0, y0 - 1 + i, n);
        if (mir) tma_load_5d(sX + (NX + xs) * S, tx, &x_full[xs], 0, x0, 0, y0 - 1 + i, n);
        if (++xs == NX) { xs = 0; xph ^= 1; }
        if (i >= 2) {  // dY row y0 + i - 2 needs X rows up to y0 + i - 1 (just issued)
          mbar_wait(&d_empty[ds], dph ^ 1);
          mbar_arrive_expect_tx(&d_full[ds], 3 * cbytes);
#pragma unroll
          for (int kx = 0; kx < 3; ++kx)
            tma_load_5d(sDY + ds * DYS + kx * cbytes, ty, &d_full[ds], 0, x0 + 1 - kx, 0, y0 + i - 2, n);
          if (++ds == NS) { ds = 0; dph ^= 1; }
        }
      }
      SR_WPIECE_END
    }
    __syncwarp();
  } else if (warp == 1) {
    // ===================== MMA issuer
    if (elect_one()) {
      unsigned xq0 = 0, xw = 0, dq = 0;  // global X input index of the piece's first row, X inputs waited, dY rows
      bool first = true;
      uint32_t seg = 0;
      SR_WPIECE_BEGIN
      const int nmt = (3 * cb + 7) / 8, nn = 3 * jb.coutp;
      const uint32_t idesc = make_idesc(128, nn, 1, 1);
      const uint32_t albo = cb == CBM ? ATOM : S;  // stride of the (ky, cb) M-atoms
      for (int k = 0; k < rows; ++k) {
        for (; xw <= xq0 + k + 2; ++xw) mbar_wait(&x_full[xw % NX], (uint32_t)(xw / NX) & 1u);
        const int ds = (int)(dq % NS);
        mbar_wait(&d_full[ds], (uint32_t)(dq / NS) & 1u);
        if (first && seg > 0) mbar_wait(&t_empty, (seg - 1) & 1u);  // previous job's accumulators drained
        tc_fence_after();
        if (dbg && first && seg == 0) dbg[2] = globaltimer();
        const uint32_t xa = smem_u32(sX + (int)((xq0 + k) % NX) * S);
        const uint32_t yb = smem_u32(sDY + ds * DYS);
#pragma unroll
        for (int k16 = 0; k16 < kWrTW / 16; ++k16) {
          const uint64_t bdesc = make_desc_sw(yb + k16 * 512u, ATOM, 256, 6);
          for (int mt = 0; mt < nmt; ++mt)
            mma_bf16_ss(tmem + mt * nn, make_desc_sw(xa + mt * 8u * albo + k16 * 512u, albo, 256, 6), bdesc, idesc,
                        (first && k16 == 0) ? 0u : 1u);
        }
        first = false;
        mma_commit(&d_empty[ds]);
        mma_commit(&x_empty[(int)((xq0 + k) % NX)]);  // X input k: last used by dY row k
        ++dq;
      }
      mma_commit(&x_empty[(int)((xq0 + rows) % NX)]);
      mma_commit(&x_empty[(int)((xq0 + rows + 1) % NX)]);
      xq0 += rows + 2;
      if (seg_end) {
        mma_commit(&done_bar);
        first = true;
        ++seg;
      }
      SR_WPIECE_END
      if (dbg) dbg[3] = globaltimer();
    }
    __syncwarp();
  } else if (warp < 6) {
    // ===================== bias gradient from the unshifted dY copy; drain the accumulators at each job end
    // thread et owns 8-channel chunk j = et % och (block j/2, half j%2) and pixel subset grp = et / och (fixed
    // order -> deterministic).  Half h of pixel p sits at 16 * (h ^ bit 2 of p) (SWIZZLE_32B).
    const int et = threadIdx.x - 64;  // 0..127
    const int quarter = warp & 3;
    const int m = quarter * 32 + lane_id();
    float acc8[8];
#pragma unroll
    for (int e = 0; e < 8; ++e) acc8[e] = 0.f;
    unsigned dq = 0;
    uint32_t seg = 0;
    SR_WPIECE_BEGIN
    const int coutp = jb.coutp, cinp = jb.cinp;
    const int och = coutp >> 3, ng = 128 / och;
    const int j = et % och, grp = et / och;
    for (int k = 0; k < rows; ++k, ++dq) {
      const int ds = (int)(dq % NS);
      mbar_wait(&d_full[ds], (uint32_t)(dq / NS) & 1u);
      if (grp < ng) {
        const uint8_t* yt = sDY + ds * DYS + ob * ATOM;  // kx = 1: dY[y, x0 + p]
        for (int p = grp; p < kWrTW; p += ng) {
          const uint32_t off = ((uint32_t)(j >> 1) * kWrTW + p) * 32u + (((j & 1) ^ ((p >> 2) & 1)) << 4);
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
      named_bar_sync(1, 128);
      if (et == 0) mbar_arrive(&d_empty[ds]);
    }
    if (seg_end) {
      float* outp = P.ws + (size_t)(blockIdx.x + job) * P.maxstride;
      if (grp < ng) {
#pragma unroll
        for (int e = 0; e < 8; ++e) { sdb[grp * coutp + j * 8 + e] = acc8[e]; acc8[e] = 0.f; }
      }
      named_bar_sync(1, 128);
      if (et < coutp) {
        float t = 0.f;
        for (int p2 = 0; p2 < ng; ++p2) t += sdb[p2 * coutp + et];
        outp[9 * cinp * coutp + et] = t;
      }
      // drain: lane m of M-tile mt = atom a = 8 mt + m / 16 -> (ky, c) = (a / cb, a % cb), ci = 16 c + m % 16;
      // columns kx * coutp + co.  Partial layout [tap = ky*3 + kx][ci][co] (+ bias).
      mbar_wait(&done_bar, seg & 1u);
      if (dbg && et == 0 && seg == 0) dbg[5] = globaltimer();
      tc_fence_after();
      const int nmt = (3 * cb + 7) / 8, nn = 3 * coutp;
      for (int mt = 0; mt < nmt; ++mt) {
        const int at = 8 * mt + m / 16;
        const bool ok = at < 3 * cb;
        const int ky = at / cb, ci = 16 * (at % cb) + (m % 16);
        for (int kx = 0; kx < 3; ++kx) {
          float v[16 * OBM];
#pragma unroll
          for (int c0 = 0; c0 < 16 * OBM; c0 += 16)
            if (c0 < coutp) tmem_ld16(tmem + ((uint32_t)(quarter * 32) << 16) + mt * nn + kx * coutp + c0, v + c0);
          tmem_ld_wait();
          if (ok) {
            float4* dst = reinterpret_cast<float4*>(outp + ((size_t)(ky * 3 + kx) * cinp + ci) * coutp);
#pragma unroll
            for (int q = 0; q < 4 * OBM; ++q)
              if (4 * q < coutp) dst[q] = make_float4(v[4 * q], v[4 * q + 1], v[4 * q + 2], v[4 * q + 3]);
          }
        }
      }
      tc_fence_before();
      __syncwarp();
      if (lane_id() == 0) mbar_arrive(&t_empty);
      named_bar_sync(1, 128);  // sdb is reused by the next job
      ++seg;
    }
    SR_WPIECE_END
    if (dbg && et == 0) dbg[6] = globaltimer();
  }
#undef SR_WPIECE_BEGIN
#undef SR_WPIECE_END
  tc_fence_before();
  __syncthreads();
  if (warp == 1) tmem_dealloc<512>(tmem);
  // ---- grid barrier: every partial written.  atom.inc wraps the arrival counter back to 0 in the same atomic,
  // so only the last arriver bumps the generation.
  if (threadIdx.x == 0) {
    volatile unsigned* vgen = P.sync + 1;
    const unsigned gen = *vgen;
    __threadfence();
    const unsigned arrived = atomicInc(P.sync, gridDim.x - 1);
    if (arrived == gridDim.x - 1) {
      __threadfence();
      atomicAdd(P.sync + 1, 1u);
    } else {
      while (*vgen == gen) {
      }
    }
    __threadfence();
  }
  __syncthreads();
  pdl_trigger();
  if (dbg && threadIdx.x == 0) dbg[7] = globaltimer();
  // ---- deterministic reduction of this CTA's slice of the flattened float4 outputs: output i of job k sums the
  // partials of the CTAs whose ranges touch job k, in CTA order (group q of NQ takes CTAs q, q + NQ, ...; the NQ
  // group sums are then added in order)
  {
    const int G = gridDim.x;
    const int NQ = P.nq, LC = kWrThreads / NQ;
    const int lo = (int)((long long)blockIdx.x * P.total4 / G), hi = (int)((long long)(blockIdx.x + 1) * P.total4 / G);
    float4* red = reinterpret_cast<float4*>(smem);  // stage buffers are free now
    const int t = threadIdx.x;
    const int oi = t % LC, q = t / LC;
    for (int c0 = lo; c0 < hi; c0 += LC) {
      const int lc = min(LC, hi - c0);
      int k = 0, li = 0;
      if (oi < lc && q < NQ) {
        const int gi = c0 + oi;
        while (k + 1 < P.J && P.job[k + 1].off4 <= gi) ++k;
        li = gi - P.job[k].off4;
        // CTAs whose range [floor(total b / G), floor(total (b+1) / G)) intersects job k's rows [j0, j1): the
        // CTA holding row r is the largest b with floor(total b / G) <= r, i.e. b = ((r + 1) G - 1) / total
        const long long j0 = (long long)k * per_job, j1 = j0 + per_job;
        const int bf = (int)min((long long)G - 1, ((j0 + 1) * G - 1) / total);
        const int bl = (int)min((long long)G - 1, (j1 * G - 1) / total);
        const int cnt = bl - bf + 1;
        const float4* src = reinterpret_cast<const float4*>(P.ws) + li;
        const size_t sstride = (size_t)P.maxstride / 4;
        float4 acc4 = make_float4(0.f, 0.f, 0.f, 0.f);
        for (int p = q; p < cnt; p += 16 * NQ) {
          float4 w4[16];
#pragma unroll
          for (int kk = 0; kk < 16; ++kk)
            w4[kk] = p + kk * NQ < cnt ? __ldcg(src + (size_t)(bf + p + kk * NQ + k) * sstride)
                                       : make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll
          for (int kk = 0; kk < 16; ++kk) {
            acc4.x += w4[kk].x; acc4.y += w4[kk].y; acc4.z += w4[kk].z; acc4.w += w4[kk].w;
          }
        }
        red[q * LC + oi] = acc4;
      }
      __syncthreads();
      if (t < lc) {
        float4 s4 = red[t];
        for (int qq = 1; qq < NQ; ++qq) {
          const float4 w4 = red[qq * LC + t];
          s4.x += w4.x; s4.y += w4.y; s4.z += w4.z; s4.w += w4.w;
        }
        const WmJob& jb = P.job[k];
        const int per = 9 * jb.cinp * jb.coutp;
        const float sv[4] = {s4.x, s4.y, s4.z, s4.w};
#pragma unroll
        for (int e = 0; e < 4; ++e) {
          const int i = 4 * li + e;
          if (i < per) {  // partial index [tap][ci][co]
            const int co = i % jb.coutp, rest = i / jb.coutp;
            const int ci = rest % jb.cinp, tap = rest / jb.cinp;
            if (co < jb.cout && ci < jb.cin) jb.gW[(co * jb.cin + ci) * 9 + tap] = sv[e] * P.scale;
          } else {
            const int co = i - per;
            if (co < jb.cout) jb.gb[co] = sv[e] * P.scale;
          }
        }
      }
      __syncthreads();
    }
  }
  if (dbg && threadIdx.x == 0) dbg[1] = globaltimer();
}

template <int CBM, int OBM>
static cudaError_t launch_wm_t(const WmParams& p, int grid, cudaStream_t st) {
  auto kern = k_wgrad_multi<CBM, OBM>;
  constexpr size_t smem = WmCfg<CBM, OBM>::SMEM;
  static bool configured = false;
  if (!configured) {
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    configured = true;
  }
  return launch_coop(kern, dim3(grid), dim3(kWrThreads), smem, st, p);
}

static bool force_tile() {
  static int v = -1;  // SR_WGRAD_TILE=1: always the tiled k_wgrad, one launch per conv (A/B timing)
  if (v < 0) {
    const char* e = std::getenv("SR_WGRAD_TILE");
    v = (e && e[0] == '1') ? 1 : 0;
  }
  return v == 1;
}

static int max_cb(const WgradJob* jobs, int J) {
  int m = 1;
  for (int k = 0; k < J; ++k) m = std::max(m, jobs[k].cinp / 16);
  return m;
}
static int max_ob(const WgradJob* jobs, int J) {
  int m = 1;
  for (int k = 0; k < J; ++k) m = std::max(m, jobs[k].coutp / 16);
  return m;
}

bool wgrad_multi_supported(const WgradJob* jobs, int J, int W) {
  if (force_tile() || W < kWrTW || J < 1 || J > kWgradMaxJobs) return false;
  const int cbm = max_cb(jobs, J);
  for (int k = 0; k < J; ++k) {
    const int cb = jobs[k].cinp / 16, ob = jobs[k].coutp / 16;
    if (jobs[k].cinp % 16 || jobs[k].coutp % 16 || (cb != 1 && cb != cbm) || ob < 1 || ob > kWmOBM) return false;
  }
  return cbm <= 4;
}

int wgrad_multi_grid(int J, int N, int H, int W) {
  const long long rows = (long long)J * N * ((W + kWrTW - 1) / kWrTW) * H;
  return (int)std::min<long long>(rows, num_sms());
}

size_t wgrad_multi_ws_floats(const WgradJob* jobs, int J, int grid) {
  size_t ms = 0;
  for (int k = 0; k < J; ++k) ms = std::max(ms, (size_t)9 * jobs[k].cinp * jobs[k].coutp + jobs[k].coutp);
  return (size_t)(grid + J) * ms;
}

cudaError_t launch_wgrad_multi(const WgradJob* jobs, int J, int N, int H, int W, float scale, float* ws,
                               unsigned* sync, int grid, long long* dbg, cudaStream_t st) {
  if (!wgrad_multi_supported(jobs, J, W)) return cudaErrorNotSupported;
  WmParams p{};
  int off4 = 0, ms = 0;
  for (int k = 0; k < J; ++k) {
    const WgradJob& g = jobs[k];
    if (make_act_tmap_sw32(&p.tmx[k], g.x, N, H, W, g.cinp, kWrTW, 1) != CUDA_SUCCESS) return cudaErrorInvalidValue;
    if (make_act_tmap_sw32(&p.tmy[k], g.dy, N, H, W, g.coutp, kWrTW, 1) != CUDA_SUCCESS)
      return cudaErrorInvalidValue;
    const int stride = 9 * g.cinp * g.coutp + g.coutp;
    p.job[k] = WmJob{g.cinp, g.coutp, g.cin, g.cout, g.gW, g.gb, off4};
    off4 += stride / 4;
    ms = std::max(ms, stride);
  }
  p.J = J; p.N = N; p.H = H; p.W = W;
  p.maxstride = ms;
  p.total4 = off4;
  p.scale = scale;
  p.ws = ws;
  p.sync = sync;
  p.dbg = dbg;
  const long long per_job = (long long)N * ((W + kWrTW - 1) / kWrTW) * H;
  const long long cnt_max = (per_job * grid + (long long)J * per_job - 1) / ((long long)J * per_job) + 2;
  p.nq = (int)std::max(1LL, std::min(32LL, (cnt_max + 15) / 16));
#define SR_WM_CASE(CB, OB) \
  if (cbm == CB && obm == OB) return launch_wm_t<CB, OB>(p, grid, st);
  const int cbm = max_cb(jobs, J), obm = max_ob(jobs, J);
  SR_WM_CASE(1, 1) SR_WM_CASE(1, 2) SR_WM_CASE(1, 3) SR_WM_CASE(1, 4)
  SR_WM_CASE(2, 1) SR_WM_CASE(2, 2) SR_WM_CASE(2, 3) SR_WM_CASE(2, 4)
  SR_WM_CASE(3, 1) SR_WM_CASE(3, 2) SR_WM_CASE(3, 3) SR_WM_CASE(3, 4)
  SR_WM_CASE(4, 1) SR_WM_CASE(4, 2) SR_WM_CASE(4, 3) SR_WM_CASE(4, 4)
#undef SR_WM_CASE
  return cudaErrorNotSupported;
}

}  // namespace sr

// Shared epilogue pieces of the up-conv tail (pixel shuffle + bilinear / bicubic skip + clamp + RNE u8, or the
// training loss / dy), used by the tiled conv (conv.cu) and the rolling conv (conv_roll.cu).
// sbias may be null when the accumulator already holds the bias (the rolling kernel's bias-armed TMEM ring).
#pragma once
#include "ptx.cuh"
#include "sr_internal.h"

namespace sr {

template <int COUTP>
__device__ __forceinline__ void store_bf16_row(bf16* p, const float* v) {
  uint4* q = reinterpret_cast<uint4*>(p);
#pragma unroll
  for (int i = 0; i < COUTP / 8; ++i) {
    uint4 u;
    u.x = pack_bf16x2(v[i * 8 + 0], v[i * 8 + 1]);
    u.y = pack_bf16x2(v[i * 8 + 2], v[i * 8 + 3]);
    u.z = pack_bf16x2(v[i * 8 + 4], v[i * 8 + 5]);
    u.w = pack_bf16x2(v[i * 8 + 6], v[i * 8 + 7]);
    q[i] = u;
  }
}

// Bilinear skip by output phase (half-pixel centres, edge replicate == PyTorch align_corners=False):
//   x2: phase 0 -> 0.25 v[i-1] + 0.75 v[i];  phase 1 -> 0.75 v[i] + 0.25 v[i+1]
//   x3: phase 0 -> v[i-1]/3 + 2 v[i]/3;  phase 1 -> v[i];  phase 2 -> 2 v[i]/3 + v[i+1]/3
//   x4: source offsets (ph + 1/2)/4 - 1/2 = -3/8, -1/8, +1/8, +3/8 (exact binary fractions)
template <int S>
__device__ __forceinline__ void phase_w(int ph, float& wm, float& w0, float& wp) {
  if (S == 2) {
    wm = ph == 0 ? 0.25f : 0.f;
    w0 = 0.75f;
    wp = ph == 1 ? 0.25f : 0.f;
  } else if (S == 4) {
    wm = ph == 0 ? 0.375f : (ph == 1 ? 0.125f : 0.f);
    w0 = (ph == 0 || ph == 3) ? 0.625f : 0.875f;
    wp = ph == 3 ? 0.375f : (ph == 2 ? 0.125f : 0.f);
  } else {
    const float t = 1.f / 3.f, tt = 2.f / 3.f;
    wm = ph == 0 ? t : 0.f;
    w0 = ph == 1 ? 1.f : tt;
    wp = ph == 2 ? t : 0.f;
  }
}

// One separable bilinear pass at output phase ph: weights of (v[i-1], v[i], v[i+1]); zero taps are skipped at
// compile time (each phase has at most two), which is exact: the dropped terms are +0 on non-negative values.
template <int S>
__device__ __forceinline__ float bil3(int ph, float a, float b, float c) {
  float wm, w0, wp;
  phase_w<S>(ph, wm, w0, wp);
  float acc = w0 * b;
  if (wm != 0.f) acc = fmaf(wm, a, acc);
  if (wp != 0.f) acc = fmaf(wp, c, acc);
  return acc;
}

// clamp(x, 0, 255) rounded half-to-even to u8 in one instruction (NaN -> 0)
__device__ __forceinline__ uint8_t f2u8_rn_sat(float x) {
  uint32_t r;
  asm("cvt.rni.sat.u8.f32 %0, %1;" : "=r"(r) : "f"(x));
  return (uint8_t)r;
}

// Bicubic skip variant (reading R23: Keys, A = -0.75, half-pixel centres without clamping the source coordinate,
// clamped taps = PyTorch bicubic align_corners=False).  Phase ph of S: source offset d = (ph + 1/2)/S - 1/2;
// d < 0 -> taps rows -2..+1 with t = 1 + d, else rows -1..+2 with t = d.  w[0..4] are the weights of rows -2..+2.
__device__ __forceinline__ float cubic_w(float x) {
  const float A = -0.75f;
  x = fabsf(x);
  return x <= 1.f ? ((A + 2.f) * x - (A + 3.f)) * x * x + 1.f
                  : (x < 2.f ? ((A * x - 5.f * A) * x + 8.f * A) * x - 4.f * A : 0.f);
}
template <int S>
__device__ __forceinline__ void cubic_phase_w(int ph, float* w) {
  const float d = ((float)ph + 0.5f) / (float)S - 0.5f;
  const bool neg = d < 0.f;
  const float t = neg ? 1.f + d : d;
  const int base = neg ? 0 : 1;  // index of tap k = -1 in rows -2..+2
#pragma unroll
  for (int a = 0; a < 5; ++a) w[a] = 0.f;
#pragma unroll
  for (int k = -1; k <= 2; ++k) w[base + k + 1] = cubic_w((float)k - t);
}

// Tail with the bicubic skip: as epi_tail below, skip = bicubic_S(v) from the 5 x 5 LR neighbourhood.
template <int S, int COUTP, bool TRAIN>
__device__ __noinline__ void epi_tail_bicubic(const EpiParams& ep, const float* sbias, int n, int Y, int X, int H,
                                              int W, float* v, float& lsum, size_t dy_pix) {
  const uint8_t* lr = ep.lr + (size_t)n * H * W * 3;
  float hrow[5][S][3];  // horizontal pass on the five LR rows Y-2..Y+2 (clamped), per output phase j
#pragma unroll
  for (int a = 0; a < 5; ++a) {
    const int yy = min(max(Y + a - 2, 0), H - 1);
    float px[5][3];
#pragma unroll
    for (int b = 0; b < 5; ++b) {
      const int xx = min(max(X + b - 2, 0), W - 1);
      const uint8_t* p = lr + ((size_t)yy * W + xx) * 3;
#pragma unroll
      for (int c = 0; c < 3; ++c) px[b][c] = (float)__ldg(p + c);
    }
#pragma unroll
    for (int j = 0; j < S; ++j) {
      float wx[5];
      cubic_phase_w<S>(j, wx);
#pragma unroll
      for (int c = 0; c < 3; ++c) {
        float acc = 0.f;
#pragma unroll
        for (int b = 0; b < 5; ++b) acc = fmaf(wx[b], px[b][c], acc);
        hrow[a][j][c] = acc;
      }
    }
  }
  const int sH = S * H, sW = S * W;
  float dyv[COUTP];
#pragma unroll
  for (int k = 0; k < COUTP; ++k) dyv[k] = 0.f;
#pragma unroll
  for (int i = 0; i < S; ++i) {
    float wy[5];
    cubic_phase_w<S>(i, wy);
    uint8_t* orow = TRAIN ? nullptr : ep.hr + (((size_t)n * sH + (size_t)S * Y + i) * sW + (size_t)S * X) * 3;
    const uint8_t* trow =
        TRAIN ? ep.hr_ref + (((size_t)n * sH + (size_t)S * Y + i) * sW + (size_t)S * X) * 3 : nullptr;
#pragma unroll
    for (int j = 0; j < S; ++j) {
#pragma unroll
      for (int c = 0; c < 3; ++c) {
        float skip = 0.f;
#pragma unroll
        for (int a = 0; a < 5; ++a) skip = fmaf(wy[a], hrow[a][j][c], skip);
        const int k = c * S * S + i * S + j;
        const float y = v[k] + (sbias ? sbias[k] : 0.f);
        if (TRAIN) {
          const float o = y + skip * (1.f / 255.f);
          const float d = o - (float)__ldg(trow + j * 3 + c) * (1.f / 255.f);
          if (ep.l1) {
            lsum += fabsf(d);
            dyv[k] = d > 0.f ? 1.f : (d < 0.f ? -1.f : 0.f);
          } else {
            lsum += d * d;
            dyv[k] = 2.f * d;
          }
        } else {
          orow[j * 3 + c] = f2u8_rn_sat(fmaf(255.f, y, skip));
        }
      }
    }
  }
  if (TRAIN) store_bf16_row<COUTP>(ep.dy + dy_pix * COUTP, dyv);
}

// Tail: y = acc + b (3 s^2 channels, index c*s^2 + i*s + j = pixel-shuffle phase (i,j) of colour c);
// skip = bilinear_s(v) at HR (sY+i, sX+j).  Inference: u8 = RNE(clamp(255 y + skip, 0, 255)).
// Training: o = y + skip/255, d = o - hr/255 -> loss += d^2, dy[c s^2 + i s + j] = 2 d (L1: |d|, sign(d)).
// (n, Y, X) addresses the LR image / HR target (n-th image of size H x W); dy_pix is the pixel index of this
// output in the conv's own layout (equal to ((n H + Y) W + X) except for the virtual training batch).
template <int S, int COUTP, bool TRAIN>
__device__ __forceinline__ void epi_tail(const EpiParams& ep, const float* sbias, int n, int Y, int X, int H,
                                         int W, float* v, float& lsum, size_t dy_pix) {
  if (ep.bicubic) {  // a copy goes to the non-inlined variant, so v itself never escapes (stays in registers)
    float vb[COUTP];
#pragma unroll
    for (int k = 0; k < COUTP; ++k) vb[k] = v[k];
    epi_tail_bicubic<S, COUTP, TRAIN>(ep, sbias, n, Y, X, H, W, vb, lsum, dy_pix);
    return;
  }
  const uint8_t* lr = ep.lr + (size_t)n * H * W * 3;
  float nb[3][3][3];  // [dy][dx][c] neighbourhood of LR pixel (Y,X), clamped (edge replicate)
#pragma unroll
  for (int a = 0; a < 3; ++a) {
    int yy = min(max(Y + a - 1, 0), H - 1);
#pragma unroll
    for (int b = 0; b < 3; ++b) {
      int xx = min(max(X + b - 1, 0), W - 1);
      const uint8_t* p = lr + ((size_t)yy * W + xx) * 3;
#pragma unroll
      for (int c = 0; c < 3; ++c) nb[a][b][c] = (float)__ldg(p + c);
    }
  }
  float hx[3][S][3];  // horizontal pass per LR row and output column phase
#pragma unroll
  for (int a = 0; a < 3; ++a)
#pragma unroll
    for (int j = 0; j < S; ++j)
#pragma unroll
      for (int c = 0; c < 3; ++c) hx[a][j][c] = bil3<S>(j, nb[a][0][c], nb[a][1][c], nb[a][2][c]);
  const int sH = S * H, sW = S * W;
  float dyv[COUTP];
#pragma unroll
  for (int k = 0; k < COUTP; ++k) dyv[k] = 0.f;
#pragma unroll
  for (int i = 0; i < S; ++i) {
    uint8_t* hrow = TRAIN ? nullptr : ep.hr + (((size_t)n * sH + (size_t)S * Y + i) * sW + (size_t)S * X) * 3;
    const uint8_t* trow =
        TRAIN ? ep.hr_ref + (((size_t)n * sH + (size_t)S * Y + i) * sW + (size_t)S * X) * 3 : nullptr;
#pragma unroll
    for (int j = 0; j < S; ++j) {
#pragma unroll
      for (int c = 0; c < 3; ++c) {
        // horizontal pass on the three LR rows (hx), then vertical
        const float skip = bil3<S>(i, hx[0][j][c], hx[1][j][c], hx[2][j][c]);
        const int k = c * S * S + i * S + j;
        float y = v[k] + (sbias ? sbias[k] : 0.f);
        if (TRAIN) {
          float o = y + skip * (1.f / 255.f);
          float d = o - (float)__ldg(trow + j * 3 + c) * (1.f / 255.f);
          if (ep.l1) {  // L1 variant: |d|, d/d o = sign(d) (0 at 0)
            lsum += fabsf(d);
            dyv[k] = d > 0.f ? 1.f : (d < 0.f ? -1.f : 0.f);
          } else {
            lsum += d * d;
            dyv[k] = 2.f * d;
          }
        } else {
          hrow[j * 3 + c] = f2u8_rn_sat(fmaf(255.f, y, skip));
        }
      }
    }
  }
  if (TRAIN) store_bf16_row<COUTP>(ep.dy + dy_pix * COUTP, dyv);
}

__device__ __forceinline__ float lds_u8f(uint32_t a) {
  uint32_t r;
  asm volatile("ld.shared.u8 %0, [%1];" : "=r"(r) : "r"(a));
  return (float)r;
}
__device__ __forceinline__ void sts_u8(uint32_t a, uint8_t v) {
  asm volatile("st.shared.u8 [%0], %1;" ::"r"(a), "h"((unsigned short)v) : "memory");
}

// Inference tail from an LR neighbourhood in shared memory, result in registers:
//   L: LR rows Y-2 .. Y+2 of the strip (rows outside the image are zero-filled; the clamp below never reads
//      them), lpitch bytes per row, LR pixel p of a row at byte 3 p - lbase (shared-memory state-space address);
//   o[(i S + j) 3 + c] = u8 of HR pixel (S Y + i, S X + j), colour c.
// Arithmetic and its order are those of epi_tail / epi_tail_bicubic (no bias term: the ring held it), so the
// u8 result is bit-identical to the global-memory path.
template <int S>
__device__ __forceinline__ void tail_u8_px(uint32_t L, int lpitch, int lbase, int Y, int X, int H, int W,
                                           const float* v, int bicubic, uint8_t* o) {
  if (bicubic) {
    float hrow[5][S][3];
#pragma unroll
    for (int a = 0; a < 5; ++a) {
      const uint32_t lrow = L + (min(max(Y + a - 2, 0), H - 1) - Y + 2) * lpitch - lbase;
      float px[5][3];
#pragma unroll
      for (int b = 0; b < 5; ++b) {
        const uint32_t p = lrow + 3 * min(max(X + b - 2, 0), W - 1);
#pragma unroll
        for (int c = 0; c < 3; ++c) px[b][c] = lds_u8f(p + c);
      }
#pragma unroll
      for (int j = 0; j < S; ++j) {
        float wx[5];
        cubic_phase_w<S>(j, wx);
#pragma unroll
        for (int c = 0; c < 3; ++c) {
          float acc = 0.f;
#pragma unroll
          for (int b = 0; b < 5; ++b) acc = fmaf(wx[b], px[b][c], acc);
          hrow[a][j][c] = acc;
        }
      }
    }
#pragma unroll
    for (int i = 0; i < S; ++i) {
      float wy[5];
      cubic_phase_w<S>(i, wy);
#pragma unroll
      for (int j = 0; j < S; ++j) {
#pragma unroll
        for (int c = 0; c < 3; ++c) {
          float skip = 0.f;
#pragma unroll
          for (int a = 0; a < 5; ++a) skip = fmaf(wy[a], hrow[a][j][c], skip);
          o[(i * S + j) * 3 + c] = f2u8_rn_sat(fmaf(255.f, v[c * S * S + i * S + j] + 0.f, skip));
        }
      }
    }
    return;
  }
  // the 9 bytes of pixels X-1 .. X+1 of an LR row come from 3 aligned words (one wavefront each, instead of 9
  // byte loads), then edge replication replaces the pixel outside the frame (the slot holds the strip's pixels
  // with a margin, so the words are inside it)
  float nb[3][3][3];
  const uint32_t b0 = 3u * (uint32_t)X - 3u;  // byte of pixel X-1 (wraps at X = 0; that pixel is replaced)
  const bool lclamp = X == 0, rclamp = X + 1 >= W;
#pragma unroll
  for (int a = 0; a < 3; ++a) {
    const uint32_t ad = L + (min(max(Y + a - 1, 0), H - 1) - Y + 2) * lpitch - lbase + b0;
    const uint32_t wa = ad & ~3u, sft = 8u * (ad & 3u);
    uint32_t w0, w1, w2;
    asm volatile("ld.shared.u32 %0, [%1];" : "=r"(w0) : "r"(wa));
    asm volatile("ld.shared.u32 %0, [%1];" : "=r"(w1) : "r"(wa + 4));
    asm volatile("ld.shared.u32 %0, [%1];" : "=r"(w2) : "r"(wa + 8));
    const uint32_t q0 = __funnelshift_r(w0, w1, sft), q1 = __funnelshift_r(w1, w2, sft), q2 = w2 >> sft;
    float px[9];
#pragma unroll
    for (int k = 0; k < 4; ++k) {
      px[k] = (float)((q0 >> (8 * k)) & 0xffu);
      px[4 + k] = (float)((q1 >> (8 * k)) & 0xffu);
    }
    px[8] = (float)(q2 & 0xffu);
#pragma unroll
    for (int c = 0; c < 3; ++c) {
      nb[a][1][c] = px[3 + c];
      nb[a][0][c] = lclamp ? px[3 + c] : px[c];
      nb[a][2][c] = rclamp ? px[3 + c] : px[6 + c];
    }
  }
  float hx[3][S][3];
#pragma unroll
  for (int a = 0; a < 3; ++a)
#pragma unroll
    for (int j = 0; j < S; ++j)
#pragma unroll
      for (int c = 0; c < 3; ++c) hx[a][j][c] = bil3<S>(j, nb[a][0][c], nb[a][1][c], nb[a][2][c]);
#pragma unroll
  for (int i = 0; i < S; ++i)
#pragma unroll
    for (int j = 0; j < S; ++j)
#pragma unroll
      for (int c = 0; c < 3; ++c) {
        const float skip = bil3<S>(i, hx[0][j][c], hx[1][j][c], hx[2][j][c]);
        o[(i * S + j) * 3 + c] = f2u8_rn_sat(fmaf(255.f, v[c * S * S + i * S + j] + 0.f, skip));
      }
}

// The same with the S HR rows written to shared memory: HR pixel (S Y + i, S X + j) at O + i opitch + ox + 3 j.
template <int S>
__device__ __forceinline__ void tail_u8_smem(uint32_t L, int lpitch, int lbase, uint32_t O, int opitch,
                                             int ox, int Y, int X, int H, int W, const float* v, int bicubic) {
  uint8_t o[S * S * 3];
  tail_u8_px<S>(L, lpitch, lbase, Y, X, H, W, v, bicubic, o);
#pragma unroll
  for (int i = 0; i < S; ++i)
#pragma unroll
    for (int k = 0; k < 3 * S; ++k) sts_u8(O + i * opitch + ox + k, o[i * 3 * S + k]);
}

}  // namespace sr

// Memory-bound kernels of the hot path: input packing, weight packing, wgrad reduction, fused Adam,
// recency-weighted sampler + patch gather, integer SSE (PSNR), bilinear-only baseline.
#include <algorithm>
#include "ptx.cuh"
#include "color.cuh"
#include "sr_internal.h"
#include "kernels.h"
#include "launch.cuh"

namespace sr {

// --------------------------------------------------------------- head input: u8 RGB -> bf16 [.., 16]
// x = v / 255 (reading R3), channels 3..15 zero so the head conv runs with K = 9 x 16.
__global__ void k_pack_input(const uint8_t* __restrict__ lr, size_t npix, uint4* __restrict__ x) {
  pdl_enter();
  size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= npix) return;
  const uint8_t* p = lr + i * 3;
  uint4 lo;
  lo.x = pack_bf16x2(p[0] * (1.f / 255.f), p[1] * (1.f / 255.f));
  lo.y = pack_bf16x2(p[2] * (1.f / 255.f), 0.f);
  lo.z = 0u;
  lo.w = 0u;
  x[2 * i] = lo;
  x[2 * i + 1] = make_uint4(0u, 0u, 0u, 0u);
}

void launch_pack_input(const uint8_t* lr, size_t npix, bf16* x, cudaStream_t st) {
  int th = 256;
  launch_k(k_pack_input, dim3((unsigned)((npix + th - 1) / th)), dim3(th), 0, st, lr, npix, reinterpret_cast<uint4*>(x));
}

// ------------------------------------------------------------------ I420 <-> RGB (BT.601 studio swing, reading R21)
// yuv_to_rgb / clip8: color.cuh (shared with the fused I420 head conv)

// one thread per pixel: planes y [n][h][w], u/v [n][h/2][w/2] -> rgb [n][h][w][3]
__global__ void k_i420_to_rgb(const uint8_t* __restrict__ y, const uint8_t* __restrict__ u,
                              const uint8_t* __restrict__ v, int n, int h, int w, uint8_t* __restrict__ rgb) {
  pdl_enter();
  const long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= (long long)n * h * w) return;
  const int x = (int)(i % w);
  const long long r = i / w;
  const int yy = (int)(r % h), f = (int)(r / h);
  const size_t ci = ((size_t)f * (h / 2) + yy / 2) * (w / 2) + x / 2;
  yuv_to_rgb(y[i], u[ci], v[ci], rgb + i * 3);
}

// one thread per 2x2 block: Y per pixel, U/V from the block's rounded mean colour
__global__ void k_rgb_to_i420(const uint8_t* __restrict__ rgb, int n, int h, int w, uint8_t* __restrict__ y,
                              uint8_t* __restrict__ u, uint8_t* __restrict__ v) {
  pdl_enter();
  const int hw = w / 2, hh = h / 2;
  const long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= (long long)n * hh * hw) return;
  const int bx = (int)(i % hw);
  const long long r = i / hw;
  const int by = (int)(r % hh), f = (int)(r / hh);
  int sr = 0, sg = 0, sb = 0;
#pragma unroll
  for (int dy = 0; dy < 2; ++dy)
#pragma unroll
    for (int dx = 0; dx < 2; ++dx) {
      const size_t p = ((size_t)f * h + 2 * by + dy) * w + 2 * bx + dx;
      const int R = rgb[p * 3], G = rgb[p * 3 + 1], B = rgb[p * 3 + 2];
      y[p] = rgb_to_y(R, G, B);
      sr += R; sg += G; sb += B;
    }
  rgb_sums_to_uv(sr, sg, sb, u[i], v[i]);
}

// LR counterparts of arriving HR patches (§5.2): pp x pp RGB crops of decoded frame 0 at LR top-left
// xy[j] = (x, y); grid (n, pp), one thread per pixel of a crop row.  The corners come from the ingest client, i.e.
// they are external input: a crop that does not lie inside the frame is clamped into it (pp <= h, w is checked by
// the host) and counted once in *rejected, so a bad corner can never read outside the planes.
__global__ void k_i420_crop(const uint8_t* __restrict__ y, const uint8_t* __restrict__ u,
                            const uint8_t* __restrict__ v, int h, int w, const int32_t* __restrict__ xy, int pp,
                            uint8_t* __restrict__ out, unsigned long long* __restrict__ rejected) {
  pdl_enter();
  const int j = blockIdx.x, r = blockIdx.y;
  const int xr = xy[2 * j], yr = xy[2 * j + 1];
  const int x0 = min(max(xr, 0), w - pp), y0 = min(max(yr, 0), h - pp);
  if ((x0 != xr || y0 != yr) && r == 0 && threadIdx.x == 0 && rejected) atomicAdd(rejected, 1ull);
  for (int c = threadIdx.x; c < pp; c += blockDim.x) {
    const int X = x0 + c, Y = y0 + r;
    const size_t ci = (size_t)(Y / 2) * (w / 2) + X / 2;
    yuv_to_rgb(y[(size_t)Y * w + X], u[ci], v[ci], out + (((size_t)j * pp + r) * pp + c) * 3);
  }
}

void launch_i420_to_rgb(const uint8_t* y, const uint8_t* u, const uint8_t* v, int n, int h, int w, uint8_t* rgb,
                        cudaStream_t st) {
  const long long tot = (long long)n * h * w;
  launch_k(k_i420_to_rgb, dim3((unsigned)((tot + 255) / 256)), dim3(256), 0, st, y, u, v, n, h, w, rgb);
}
void launch_rgb_to_i420(const uint8_t* rgb, int n, int h, int w, uint8_t* y, uint8_t* u, uint8_t* v,
                        cudaStream_t st) {
  const long long tot = (long long)n * (h / 2) * (w / 2);
  launch_k(k_rgb_to_i420, dim3((unsigned)((tot + 255) / 256)), dim3(256), 0, st, rgb, n, h, w, y, u, v);
}
void launch_i420_crop(const uint8_t* y, const uint8_t* u, const uint8_t* v, int h, int w, const int32_t* xy, int n,
                      int pp, uint8_t* out, unsigned long long* rejected, cudaStream_t st) {
  launch_k(k_i420_crop, dim3(n, pp), dim3(64), 0, st, y, u, v, h, w, xy, pp, out, rejected);
}

// ------------------------------------------------------------------ per-cell integer SSE (patch selection)
// grid (ncx, ncy): block (cx, cy) sums (raw - dec)^2 over the (possibly partial) cell of a [h][w][3] frame.
__global__ void k_cell_sse(const uint8_t* __restrict__ raw, const uint8_t* __restrict__ dec, int h, int w, int cell,
                           unsigned long long* __restrict__ out) {
  pdl_enter();
  const int cx = blockIdx.x, cy = blockIdx.y;
  const int x0 = cx * cell, y0 = cy * cell;
  const int cw = min(cell, w - x0), ch = min(cell, h - y0);
  const int rowb = cw * 3;
  unsigned long long acc = 0;
  for (int i = threadIdx.x; i < ch * rowb; i += blockDim.x) {
    const int r = i / rowb, c = i - r * rowb;
    const size_t o = ((size_t)(y0 + r) * w + x0) * 3 + c;
    const int d = (int)raw[o] - (int)dec[o];
    acc += (unsigned long long)(d * d);
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
  __shared__ unsigned long long part[32];
  if ((threadIdx.x & 31) == 0) part[threadIdx.x >> 5] = acc;
  __syncthreads();
  if (threadIdx.x < 32) {
    unsigned long long t = threadIdx.x < (blockDim.x >> 5) ? part[threadIdx.x] : 0ull;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) t += __shfl_xor_sync(0xffffffffu, t, o);
    if (threadIdx.x == 0) out[(size_t)cy * gridDim.x + cx] = t;
  }
}

void launch_cell_sse(const uint8_t* raw, const uint8_t* dec, int h, int w, int cell, unsigned long long* out,
                     cudaStream_t st) {
  const int nx = (w + cell - 1) / cell, ny = (h + cell - 1) / cell;
  launch_k(k_cell_sse, dim3(nx, ny), dim3(256), 0, st, raw, dec, h, w, cell, out);
}

// Virtual training batch: n patches p x p laid side by side in one p x (n (p+2)) image, patch j at columns
// [j (p+2) + 1, j (p+2) + 1 + p); the separator columns j (p+2) and j (p+2) + p + 1 are zero and act as every
// patch's own zero padding for all the 3x3 convs (which re-zero them in their epilogues).
__global__ void k_pack_input_virtual(const uint8_t* __restrict__ lr, int n, int p, uint4* __restrict__ x) {
  pdl_enter();
  const int Wv = n * (p + 2);
  const size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= (size_t)p * Wv) return;
  const int y = (int)(i / Wv), X = (int)(i % Wv);
  const int j = X / (p + 2), xx = X - j * (p + 2) - 1;
  uint4 lo = make_uint4(0u, 0u, 0u, 0u);
  if (xx >= 0 && xx < p) {
    const uint8_t* q = lr + (((size_t)j * p + y) * p + xx) * 3;
    lo.x = pack_bf16x2(q[0] * (1.f / 255.f), q[1] * (1.f / 255.f));
    lo.y = pack_bf16x2(q[2] * (1.f / 255.f), 0.f);
  }
  x[2 * i] = lo;
  x[2 * i + 1] = make_uint4(0u, 0u, 0u, 0u);
}

void launch_pack_input_virtual(const uint8_t* lr, int n, int p, bf16* x, cudaStream_t st) {
  const size_t tot = (size_t)p * n * (p + 2);
  launch_k(k_pack_input_virtual, dim3((unsigned)((tot + 255) / 256)), dim3(256), 0, st, lr, n, p, reinterpret_cast<uint4*>(x));
}

// --------------------------------------------------------------- weight packing
// fwd:   Wf[t][ci/8][co][ci%8]   = W[co][ci][ky][kx],        t = 3 ky + kx    (B operand, K-major, no swizzle)
// dgrad: Wd[t'][co/8][ci][co%8]  = W[co][ci][2-ky'][2-kx'],  t' = 3 ky' + kx' (180-degree rotation, Cin<->Cout)
// fold:  Wo[kx][ci/8][ky*coutp + co][ci%8] = W[co][ci][ky][kx]  (N = 3 coutp: the rolling dy-fold conv, conv_roll.cu)
// dfold: Wdo[kx'][co/8][ky' cinp + ci][co%8] = W[co][ci][2-ky'][2-kx']  (dy-fold weights of the data-grad conv)
__global__ void k_pack_weights(const float* __restrict__ params, const ConvDesc* __restrict__ convs, int nconv,
                               bf16* __restrict__ wf, bf16* __restrict__ wd, bf16* __restrict__ wo,
                               bf16* __restrict__ wdo, float* __restrict__ bias, long long* __restrict__ bump) {
  pdl_enter();
  // bump (training only): the Adam step counter, advanced here -- after k_adam of this step has read it -- instead
  // of by a separate launch before k_adam
  if (bump && blockIdx.x == 0 && blockIdx.y == 0 && threadIdx.x == 0) ++*bump;
  const int c = blockIdx.y;
  if (c >= nconv) return;
  const ConvDesc d = convs[c];
  const float* W = params + d.w_off;
  const int tot = 9 * d.cinp * d.coutp;
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < tot; i += gridDim.x * blockDim.x) {
    if (wf) {  // fwd element i = ((t * cinp/8 + j) * coutp + co) * 8 + e
      int e = i & 7, r = i >> 3;
      int co = r % d.coutp; r /= d.coutp;
      int j = r % (d.cinp / 8), t = r / (d.cinp / 8);
      int ci = 8 * j + e;
      float v = (ci < d.cin && co < d.cout) ? W[((co * d.cin + ci) * 3 + t / 3) * 3 + t % 3] : 0.f;
      wf[d.pk_off + i] = __float2bfloat16_rn(v);
    }
    if (wd) {  // dgrad element i = ((t' * coutp/8 + j') * cinp + co') * 8 + e'; ci' = fwd co, co' = fwd ci
      int e = i & 7, r = i >> 3;
      int cop = r % d.cinp; r /= d.cinp;
      int j = r % (d.coutp / 8), t = r / (d.coutp / 8);
      int cip = 8 * j + e;
      int ky = 2 - t / 3, kx = 2 - t % 3;
      float v = (cip < d.cout && cop < d.cin) ? W[((cip * d.cin + cop) * 3 + ky) * 3 + kx] : 0.f;
      wd[d.pk_off + i] = __float2bfloat16_rn(v);
    }
    if (wo) {  // fold element i = ((kx * cinp/8 + j) * 3 coutp + ky * coutp + co) * 8 + e
      int e = i & 7, r = i >> 3;
      int n = r % (3 * d.coutp); r /= 3 * d.coutp;
      int j = r % (d.cinp / 8), kx = r / (d.cinp / 8);
      int ky = n / d.coutp, co = n % d.coutp;
      int ci = 8 * j + e;
      float v = (ci < d.cin && co < d.cout) ? W[((co * d.cin + ci) * 3 + ky) * 3 + kx] : 0.f;
      wo[d.pk_off + i] = __float2bfloat16_rn(v);
    }
    if (wdo) {  // dgrad fold element i = ((kx' * coutp/8 + j') * 3 cinp + ky' * cinp + co') * 8 + e'
      int e = i & 7, r = i >> 3;
      int nn = r % (3 * d.cinp); r /= 3 * d.cinp;
      int j = r % (d.coutp / 8), kxp = r / (d.coutp / 8);
      int kyp = nn / d.cinp, cop = nn % d.cinp;  // cop = fwd input channel
      int cip = 8 * j + e;                         // cip = fwd output channel
      float v = (cip < d.cout && cop < d.cin) ? W[((cip * d.cin + cop) * 3 + (2 - kyp)) * 3 + (2 - kxp)] : 0.f;
      wdo[d.pk_off + i] = __float2bfloat16_rn(v);
    }
  }
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < d.coutp; i += gridDim.x * blockDim.x)
    bias[d.b_off + i] = i < d.cout ? params[d.w_off + (size_t)d.cout * d.cin * 9 + i] : 0.f;
}

void launch_pack_weights(const float* params, const ConvDesc* convs_dev, int nconv, int max_elems, bf16* wf,
                         bf16* wd, bf16* wo, bf16* wdo, float* bias, cudaStream_t st, long long* bump) {
  dim3 grid((max_elems + 255) / 256, nconv);
  launch_k(k_pack_weights, grid, dim3(256), 0, st, params, convs_dev, nconv, wf, wd, wo, wdo, bias, bump);
}

// --------------------------------------------------------------- fused Adam (PyTorch semantics)
// m = b1 m + (1-b1) g;  v = b2 v + (1-b2) g^2;  p -= (lr / bc1) * m / (sqrt(v) / sqrt(bc2) + eps),  g = s * grad
// t lives on the device (counters[1]) so the step is replayable from a CUDA graph.

// k_adam computes the bias corrections itself from the device step counter: t = counters[1] + 1 (the counter is
// advanced by the TRAIN repack that follows, k_pack_weights' bump) -- one launch less per training iteration.
// HBM-bound (28 B per parameter): 16-B vector accesses for the 4-aligned body (the buffers are cudaMalloc'd), the
// n % 4 tail by the first threads; grid = enough blocks for ~8 per SM, grid-strided.
__device__ __forceinline__ float adam1(float& p, float& m, float& v, float g, float b1, float b2, float lr_bc1,
                                       float inv_sqrt_bc2, float eps) {
  m = fmaf(b1, m, (1.f - b1) * g);
  v = fmaf(b2, v, (1.f - b2) * g * g);
  p -= lr_bc1 * m / (sqrtf(v) * inv_sqrt_bc2 + eps);
  return p;
}

__global__ void k_adam(float* __restrict__ p, float* __restrict__ m, float* __restrict__ v,
                       const float* __restrict__ grad, size_t n, const float* __restrict__ gscale_dev, float gscale,
                       const long long* __restrict__ counters, double lr, float b1, float b2, float eps) {
  pdl_enter();
  __shared__ float s_bc[2];
  if (threadIdx.x == 0) {
    const double t = (double)(counters[1] + 1);
    s_bc[0] = (float)(lr / (1.0 - pow((double)b1, t)));
    s_bc[1] = (float)(1.0 / sqrt(1.0 - pow((double)b2, t)));
  }
  __syncthreads();
  const float gs = gscale * (gscale_dev ? *gscale_dev : 1.f);
  const float lr_bc1 = s_bc[0], inv_sqrt_bc2 = s_bc[1];
  const size_t n4 = n / 4;
  float4* p4 = reinterpret_cast<float4*>(p);
  float4* m4 = reinterpret_cast<float4*>(m);
  float4* v4 = reinterpret_cast<float4*>(v);
  const float4* g4 = reinterpret_cast<const float4*>(grad);
  const size_t stride = (size_t)gridDim.x * blockDim.x;
  for (size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x; i < n4; i += stride) {
    float4 pp = p4[i], mm = m4[i], vv = v4[i];
    const float4 gg = __ldg(g4 + i);
    adam1(pp.x, mm.x, vv.x, gg.x * gs, b1, b2, lr_bc1, inv_sqrt_bc2, eps);
    adam1(pp.y, mm.y, vv.y, gg.y * gs, b1, b2, lr_bc1, inv_sqrt_bc2, eps);
    adam1(pp.z, mm.z, vv.z, gg.z * gs, b1, b2, lr_bc1, inv_sqrt_bc2, eps);
    adam1(pp.w, mm.w, vv.w, gg.w * gs, b1, b2, lr_bc1, inv_sqrt_bc2, eps);
    p4[i] = pp;
    m4[i] = mm;
    v4[i] = vv;
  }
  const size_t i = 4 * n4 + (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) adam1(p[i], m[i], v[i], grad[i] * gs, b1, b2, lr_bc1, inv_sqrt_bc2, eps);
}

void launch_adam(float* p, float* m, float* v, const float* g, size_t n, const float* gscale_dev, float gscale,
                 const long long* counters, double lr, float b1, float b2, float eps, cudaStream_t st) {
  int th = 256;
  long long blocks = (long long)((n / 4 + th - 1) / th);
  blocks = std::max<long long>(1, std::min<long long>(blocks, 8LL * num_sms()));
  launch_k(k_adam, dim3((unsigned)blocks), dim3(th), 0, st, p, m, v, g, n, gscale_dev, gscale, counters, lr, b1, b2,
           eps);
}

__global__ void k_counter_add(long long* c, long long d) {
  pdl_enter();
  *c += d;
}
void launch_counter_add(long long* counter, long long delta, cudaStream_t st) {
  launch_k(k_counter_add, dim3(1), dim3(1), 0, st, counter, delta);
}

// --------------------------------------------------------------- sampler + gather (reading R10)
// u_k = mix64(seed + GAMMA * ((((t G + r) << 20) + j) * 4 + k + 1)); K' = min(K, n); W = w K' + n - K';
// q = umulhi(u_0, W); idx = q < w K' ? n-1-q/w : q - w K'; o = umulhi(u_k, Pp - P + 1).
__device__ __forceinline__ uint64_t mix64(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

__global__ void k_sample_gather(SampleArgs a) {
  pdl_enter();
  // grid (batch, kGatherSplit): block (j, part) computes draw j (cheap, redundant per part) and copies the crop
  // rows r = part, part + kGatherSplit, ...
  const int j = blockIdx.x;
  __shared__ int s_slot, s_oy, s_ox;
  if (threadIdx.x == 0) {
    const uint64_t GAMMA = 0x9E3779B97F4A7C15ull;
    const long long step = a.step >= 0 ? a.step : *a.step_dev;
    const uint64_t base = ((((uint64_t)step * a.world + a.rank) << 20) + (uint64_t)j) * 4ull;
    const uint64_t u0 = mix64(a.seed + GAMMA * (base + 1));
    const uint64_t u1 = mix64(a.seed + GAMMA * (base + 2));
    const uint64_t u2 = mix64(a.seed + GAMMA * (base + 3));
    long long n_view = a.n_view, view_base = a.view_base;
    if (a.pool_total_dev) {  // the rank's arrival-order chunk of the pool as it is now (stream-ordered with pushes)
      const long long tot = *a.pool_total_dev;
      const long long avail = tot < a.capacity ? tot : a.capacity;
      const long long lo = avail * a.rank / a.world, hi = avail * (a.rank + 1) / a.world;
      n_view = hi - lo;
      view_base = tot - avail + lo;
    }
    const uint64_t n = n_view > 0 ? (uint64_t)n_view : 1ull;
    const uint64_t kp = n < (uint64_t)a.recent_k ? n : (uint64_t)a.recent_k;
    const uint64_t Wt = (uint64_t)a.recent_w * kp + (n - kp);
    const uint64_t q = __umul64hi(u0, Wt);
    const uint64_t idx = q < (uint64_t)a.recent_w * kp ? n - 1 - q / (uint64_t)a.recent_w : q - (uint64_t)a.recent_w * kp;
    const uint64_t span = (uint64_t)(a.pp - a.p + 1);
    s_oy = (int)__umul64hi(u1, span);
    s_ox = (int)__umul64hi(u2, span);
    const int64_t arrival = view_base + (int64_t)idx;
    s_slot = n_view > 0 ? (int)(arrival % a.capacity) : -1;  // empty view: zero patches, index -1
    if (a.idx_out && blockIdx.y == 0) a.idx_out[j] = n_view > 0 ? (int32_t)idx : -1;
  }
  __syncthreads();
  const int slot = s_slot, oy = s_oy, ox = s_ox;
  const int p = a.p, pp = a.pp, s = a.scale;
  // Crop copies: one warp per crop row (rows r = part, part + gridDim.y, ... of this block, warps round-robin);
  // the lanes issue all of a row's byte loads (coalesced, up to 16 per lane) before its stores, so the load
  // latencies overlap instead of one load-store round trip per byte.
  auto copy_rows = [&](const uint8_t* __restrict__ src, uint8_t* __restrict__ dst, int rows, int rowb, int src_pitch,
                       int src_x0b, int src_y0) {
    const int lane = threadIdx.x & 31, nw = blockDim.x >> 5;
    for (int r = (int)blockIdx.y + (int)(threadIdx.x >> 5) * (int)gridDim.y; r < rows; r += nw * (int)gridDim.y) {
      const uint8_t* __restrict__ sr = src + (size_t)(src_y0 + r) * src_pitch + src_x0b;
      uint8_t* __restrict__ dr = dst + (size_t)r * rowb;
      for (int c0 = 0; c0 < rowb; c0 += 32 * 16) {
        uint8_t v[16];
#pragma unroll
        for (int k = 0; k < 16; ++k) {
          const int c = c0 + 32 * k + lane;
          if (c < rowb) v[k] = __ldg(sr + c);
        }
#pragma unroll
        for (int k = 0; k < 16; ++k) {
          const int c = c0 + 32 * k + lane;
          if (c < rowb) dr[c] = v[k];
        }
      }
    }
  };
  const int sp = s * p, spp = s * pp;
  if (slot >= 0) {
    copy_rows(a.lr_pool + (size_t)slot * pp * pp * 3, a.lr_out + (size_t)j * p * p * 3, p, 3 * p, 3 * pp, 3 * ox, oy);
    copy_rows(a.hr_pool + (size_t)slot * spp * spp * 3, a.hr_out + (size_t)j * sp * sp * 3, sp, 3 * sp, 3 * spp,
              3 * s * ox, s * oy);
  } else {
    for (int i = threadIdx.x + blockIdx.y * blockDim.x; i < 3 * p * p; i += blockDim.x * gridDim.y)
      a.lr_out[(size_t)j * p * p * 3 + i] = 0;
    for (int i = threadIdx.x + blockIdx.y * blockDim.x; i < 3 * sp * sp; i += blockDim.x * gridDim.y)
      a.hr_out[(size_t)j * sp * sp * 3 + i] = 0;
  }
  if (a.step_bump) {  // every block read the step before arriving: the last arrival advances it for the next draw
    __syncthreads();
    if (threadIdx.x == 0) {
      __threadfence();
      const unsigned nb = gridDim.x * gridDim.y;
      if (atomicAdd(a.done, 1u) == nb - 1) {
        *a.step_bump += 1;
        *a.done = 0u;
        __threadfence();
      }
    }
  }
}

void launch_sample_gather(const SampleArgs& a, int batch, cudaStream_t st) {
  launch_k(k_sample_gather, dim3(batch, 16), dim3(128), 0, st, a);
}

// --------------------------------------------------------------- integer SSE per item (warp-shuffle reduction)
// out[i] = sum over item i's `elems` bytes of (a - b)^2, exactly (Q1: PSNR, reading R13).  Grid (n, parts): block
// (i, part) reduces one chunk of item i -- 16-B loads, |a - b| per byte by __vabsdiffu4 and the squares summed by
// __dp4a -- then a warp-shuffle + shared-memory reduction and one 64-bit atomicAdd into out[i] (zeroed by the
// launcher), so a whole 4K frame pair streams at HBM rate instead of through one block.
__device__ __forceinline__ unsigned sse4(unsigned x, unsigned y) {
  const unsigned d = __vabsdiffu4(x, y);
  return __dp4a(d, d, 0u);
}

__global__ void k_sse_u8(const uint8_t* __restrict__ a, const uint8_t* __restrict__ b, int64_t elems, int64_t chunk,
                         unsigned long long* __restrict__ out) {
  pdl_enter();
  const uint8_t* pa = a + (size_t)blockIdx.x * elems;
  const uint8_t* pb = b + (size_t)blockIdx.x * elems;
  const int64_t lo = (int64_t)blockIdx.y * chunk;
  const int64_t hi = min(elems, lo + chunk);
  unsigned long long s = 0;
  if (lo < hi) {
    // 16-B vector body when both items share their alignment; bytes before / after it (and everything otherwise)
    // one per thread
    const uintptr_t ma = reinterpret_cast<uintptr_t>(pa + lo) & 15, mb = reinterpret_cast<uintptr_t>(pb + lo) & 15;
    int64_t v0 = hi, v1 = hi;
    if (ma == mb) {
      v0 = min(hi, lo + (int64_t)((16 - ma) & 15));
      v1 = v0 + ((hi - v0) & ~(int64_t)15);
    }
    for (int64_t i = lo + threadIdx.x; i < v0; i += blockDim.x) {
      const int d = (int)pa[i] - (int)pb[i];
      s += (unsigned long long)(d * d);
    }
    const uint4* va = reinterpret_cast<const uint4*>(pa + v0);
    const uint4* vb = reinterpret_cast<const uint4*>(pb + v0);
    const int64_t nv = (v1 - v0) >> 4;
    for (int64_t i = threadIdx.x; i < nv; i += blockDim.x) {
      const uint4 x = __ldg(va + i), y = __ldg(vb + i);
      s += (unsigned long long)(sse4(x.x, y.x) + sse4(x.y, y.y)) + (unsigned long long)(sse4(x.z, y.z) + sse4(x.w, y.w));
    }
    for (int64_t i = v1 + threadIdx.x; i < hi; i += blockDim.x) {
      const int d = (int)pa[i] - (int)pb[i];
      s += (unsigned long long)(d * d);
    }
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
  __shared__ unsigned long long part[32];
  if ((threadIdx.x & 31) == 0) part[threadIdx.x >> 5] = s;
  __syncthreads();
  if (threadIdx.x < 32) {
    unsigned long long t = threadIdx.x < (blockDim.x >> 5) ? part[threadIdx.x] : 0ull;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) t += __shfl_xor_sync(0xffffffffu, t, o);
    if (threadIdx.x == 0 && t) atomicAdd(out + blockIdx.x, t);
  }
}

void launch_sse_u8(const uint8_t* a, const uint8_t* b, int n, int64_t elems, unsigned long long* out,
                   cudaStream_t st) {
  // chunks of 64 KiB per block (256 threads x 16 B x 16), at least enough blocks to cover every SM 4 times
  int64_t chunk = 64 * 1024;
  const int64_t want_blocks = 4LL * num_sms();
  if ((int64_t)n * ((elems + chunk - 1) / chunk) < want_blocks)
    chunk = std::max<int64_t>(4096, ((elems * n + want_blocks - 1) / want_blocks + 15) & ~(int64_t)15);
  const int64_t parts = (elems + chunk - 1) / chunk;
  cudaMemsetAsync(out, 0, (size_t)n * sizeof(unsigned long long), st);
  launch_k(k_sse_u8, dim3(n, (unsigned)parts), dim3(256), 0, st, a, b, elems, chunk, out);
}

__global__ void k_loss_finalize(const double* sum, double inv_n, float* out) {
  pdl_enter();
  *out = (float)(*sum * inv_n);
}
void launch_loss_finalize(const double* sum, double inv_n, float* out, cudaStream_t st) {
  launch_k(k_loss_finalize, dim3(1), dim3(1), 0, st, sum, inv_n, out);
}

}  // namespace sr

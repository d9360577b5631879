// Launchers of the memory-bound kernels (kernels.cu) and of the bilinear-only baseline (conv.cu).
#pragma once
#include "sr_internal.h"

namespace sr {

struct ConvDesc {
  int cin, cout, cinp, coutp;
  long long w_off;   // float offset of W in the flat canonical parameter vector (b follows W)
  long long pk_off;  // bf16 element offset in the packed fwd / dgrad buffers
  long long b_off;   // float offset in the packed bias buffer
};

struct SampleArgs {
  uint64_t seed;
  long long step;           // < 0: read the step from *step_dev (graph-replayable sampling)
  const long long* step_dev;
  int world, rank;
  long long n_view, view_base, capacity;
  // non-null: the pool size is read on the device (arrivals counted by sr_pool_push's k_counter_add), and the rank's
  // view [lo, hi) of the min(total, capacity) pooled patches is derived from it -- a captured graph then keeps seeing
  // new arrivals; n_view / view_base are ignored
  const long long* pool_total_dev;
  int recent_k, recent_w;
  int p, pp, scale;
  const uint8_t* lr_pool;
  const uint8_t* hr_pool;
  uint8_t* lr_out;
  uint8_t* hr_out;
  int32_t* idx_out;
  // device step mode: the last block to finish advances *step_dev (done = its block counter, reset by that block)
  long long* step_bump;
  unsigned* done;
};

void launch_pack_input(const uint8_t* lr, size_t npix, bf16* x, cudaStream_t st);
void launch_pack_weights(const float* params, const ConvDesc* convs_dev, int nconv, int max_elems, bf16* wf,
                         bf16* wd, bf16* wo, bf16* wdo, float* bias, cudaStream_t st,
                         long long* bump = nullptr);
void launch_pack_input_virtual(const uint8_t* lr, int n, int p, bf16* x, cudaStream_t st);
bool roll_supported(int cinp, int coutp, int W);
cudaError_t launch_conv_roll(int cinp, int coutp, const void* in, const bf16* wfold, const float* bias,
                             const bf16* res, int relu, bf16* out, int N, int H, int W, cudaStream_t st, int w_early = 0);
// general rolling conv: + res1 + res2, ReLU, x 1[mask > 0], zero-forced separator columns (sep > 0)
cudaError_t launch_conv_roll_ex(int cinp, int coutp, const void* in, const bf16* wfold, const float* bias,
                                const bf16* res1, const bf16* res2, const bf16* mask, int relu, int sep, bf16* out,
                                int N, int H, int W, cudaStream_t st, long long* dbg = nullptr, int w_early = 0);
// rolling up conv + tail (pixel shuffle + skip + clamp + RNE u8 into hr rows of LR rows [hr_row0, hr_row1))
cudaError_t launch_conv_roll_tail(int cinp, int coutp, int s, const void* in, const bf16* wfold, const float* bias,
                                  const uint8_t* lr, uint8_t* hr, int hr_row0, int hr_row1, int bicubic, int N, int H,
                                  int W, cudaStream_t st, int tail_tma_ok = 1, long long* dbg = nullptr,
                                  int w_early = 0);
// fused body conv (+ f0) + up conv + tail (g kept in shared memory); needs W % 16 == 0 and a 16-B aligned LR frame
bool bodytail_supported(int cp, int s, int W, const void* lr, const void* hr);
void set_block_gen(int g);  // benchmarking only
cudaError_t launch_bodytail(int cp, int s, const bf16* f, const bf16* f0, const bf16* w1fold, const bf16* w2fold,
                            const float* b1, const float* b2, const uint8_t* lr, uint8_t* hr, int hr_row0,
                            int hr_row1, int bicubic, int N, int H, int W, cudaStream_t st,
                            long long* dbg = nullptr, uint8_t* hy = nullptr, uint8_t* hu = nullptr,
                            uint8_t* hv = nullptr);
// head conv straight from the u8 frame (k_pack_input fused in); needs W % 16 == 0 and a 16-B aligned frame
bool roll_head_u8_supported(int coutp, int W, const void* lr);
cudaError_t launch_conv_roll_head_u8(int coutp, const uint8_t* lr, const bf16* wfold, const float* bias, bf16* out,
                                     int N, int H, int W, cudaStream_t st, int w_early);
// head conv straight from an I420 frame (Y rows by TMA, U / V read directly, BT.601 integer conversion fused into the
// u8 expansion; also writes the frame's RGB copy rgb_out for the tail); needs W % 32 == 0, even H, 16-B aligned planes
bool roll_head_yuv_supported(int coutp, int W, const void* y, const void* u, const void* v);
cudaError_t launch_conv_roll_head_yuv(int coutp, const uint8_t* y, const uint8_t* u, const uint8_t* v,
                                      uint8_t* rgb_out, const bf16* wfold, const float* bias, bf16* out, int N, int H,
                                      int W, cudaStream_t st, int w_early);
// rolling up conv + training tail (loss partial into *loss_sum, dy rows; vsep > 0: virtual patch batch)
cudaError_t launch_conv_roll_tail_train(int cinp, int coutp, int s, const void* in, const bf16* wfold,
                                        const float* bias, const uint8_t* lr, const uint8_t* hr_ref, bf16* dy,
                                        double* loss_sum, int vsep, int vp, int l1, int bicubic, int N, int H, int W,
                                        cudaStream_t st, int w_early);
// a chain of C -> C rolling convs in one persistent cooperative launch (k_conv_chain, conv_roll.cu); each layer is
// k_conv_roll's conv with the same epilogue variants; aux_dep: index of the earlier layer of the chain whose output
// res1 is (-1: written by an earlier kernel); sync: chain_sync_words() zero-initialised words owned by the caller
struct ChainLayerDesc {
  const void* in;
  bf16* out;
  const bf16* w;
  const float* bias;
  const bf16* res1;
  const bf16* res2;
  const bf16* mask;
  int relu;
  int aux_dep;
};
bool chain_supported(int cp, int W, int nl);
void set_chain_dbg(void* p);  // benchmarking only: globaltimer stamps of k_conv_chain
size_t chain_sync_words(int N, int H, int W);
cudaError_t launch_conv_chain(int cp, const ChainLayerDesc* layers, int nl, int sep, int N, int H, int W,
                              unsigned* sync, cudaStream_t st);
bool resblock_supported(int cp, int W);
// the residual block on CTA pairs (conv_block2.cu, tcgen05 cta_group::2; inference only, bit-identical output)
bool resblock2_supported(int cp, int W);
bool resblock_split_supported(int cp, int W);
cudaError_t launch_resblock_split(int cp, const bf16* f, const bf16* w1fold, const bf16* w2fold, const float* b1,
                                  const float* b2, bf16* out, int N, int H, int W, cudaStream_t st,
                                  long long* dbg = nullptr);
cudaError_t launch_resblock2(int cp, const bf16* f, const bf16* w1fold, const bf16* w2fold, const float* b1,
                             const float* b2, bf16* out, int N, int H, int W, cudaStream_t st);
cudaError_t launch_resblock(int cp, const bf16* f, const bf16* w1fold, const bf16* w2fold, const float* b1,
                            const float* b2, bf16* out, int N, int H, int W, cudaStream_t st,
                            long long* dbg = nullptr, bf16* tsave = nullptr, int sep = 0, int exp = 0,
                            const bf16* mask = nullptr, const bf16* res2 = nullptr);
// Device-side step counters (so a training iteration can be captured once in a CUDA graph and replayed):
// counters[0] = sampler step, counters[1] = Adam step t; scal[0] = lr / (1 - b1^t), scal[1] = 1/sqrt(1 - b2^t).
void launch_adam(float* p, float* m, float* v, const float* g, size_t n, const float* gscale_dev, float gscale,
                 const long long* counters, double lr, float b1, float b2, float eps, cudaStream_t st);
void launch_counter_add(long long* counter, long long delta, cudaStream_t st);
void launch_sample_gather(const SampleArgs& a, int batch, cudaStream_t st);
void launch_sse_u8(const uint8_t* a, const uint8_t* b, int n, int64_t elems, unsigned long long* out,
                   cudaStream_t st);
void launch_loss_finalize(const double* sum, double inv_n, float* out, cudaStream_t st);
void launch_i420_to_rgb(const uint8_t* y, const uint8_t* u, const uint8_t* v, int n, int h, int w, uint8_t* rgb,
                        cudaStream_t st);
void launch_rgb_to_i420(const uint8_t* rgb, int n, int h, int w, uint8_t* y, uint8_t* u, uint8_t* v, cudaStream_t st);
// out-of-frame corners are clamped into the frame (no out-of-bounds reads) and counted in *rejected
void launch_i420_crop(const uint8_t* y, const uint8_t* u, const uint8_t* v, int h, int w, const int32_t* xy, int n,
                      int pp, uint8_t* out, unsigned long long* rejected, cudaStream_t st);
void launch_cell_sse(const uint8_t* raw, const uint8_t* dec, int h, int w, int cell, unsigned long long* out,
                     cudaStream_t st);
cudaError_t launch_bilinear_u8(const uint8_t* lr, int n, int h, int w, int s, uint8_t* hr, cudaStream_t st);

}  // namespace sr

// libsr runtime: context, weight snapshots, workspaces, the forward / backward / Adam orchestration and the
// C ABI declared in include/sr.h.  All arithmetic of the hot path runs in the kernels of conv.cu and
// kernels.cu; this file only sequences launches on the caller's stream.
#include <cmath>
#include <cstdio>
#include <cstring>
#include <string>
#include <vector>
#include <algorithm>
#include <dlfcn.h>
#include <mutex>
#include <atomic>
#include <cuda.h>  // green-context types (driver entry points resolved through the runtime)
#include <nccl.h>  // types only: libnccl is dlopen'ed at sr_create when world > 1 (libsr.so loads without it)
#include "sr_internal.h"
#include "kernels.h"

using namespace sr;

// Streams of the green-context SM partitions (sr_sm_partition).  The synchronous calls below wait for them too:
// a device-wide synchronize of the primary context is not documented to cover work on green-context streams.
static std::vector<cudaStream_t> g_part_streams;
static std::mutex g_part_mu;
static cudaError_t sync_all() {
  cudaError_t e = cudaDeviceSynchronize();
  std::lock_guard<std::mutex> lk(g_part_mu);
  for (cudaStream_t s : g_part_streams) {
    const cudaError_t e2 = cudaStreamSynchronize(s);
    if (e == cudaSuccess) e = e2;
  }
  return e;
}

// ---------------------------------------------------------------------------------- NCCL (T5)
// The data-parallel gradient exchange is one sum-allreduce of the flat fp32 gradient over NVLink/NVSwitch.  libnccl
// is resolved at run time (SR_NCCL_LIB, else the soname "libnccl.so.2": the copy torch already loaded if any, else the
// system one), so the library itself carries no link-time NCCL dependency.
namespace {
struct NcclApi {
  bool tried = false, ok = false;
  std::string why;
  decltype(&ncclGetUniqueId) get_id = nullptr;
  decltype(&ncclCommInitRank) init_rank = nullptr;
  decltype(&ncclAllReduce) all_reduce = nullptr;
  decltype(&ncclCommDestroy) destroy = nullptr;
  decltype(&ncclGetErrorString) err = nullptr;
};
NcclApi& nccl() {
  static NcclApi a;
  if (a.tried) return a;
  a.tried = true;
  const char* path = std::getenv("SR_NCCL_LIB");
  void* h = dlopen(path && path[0] ? path : "libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
  if (!h) { a.why = std::string("dlopen libnccl: ") + dlerror(); return a; }
  a.get_id = (decltype(a.get_id))dlsym(h, "ncclGetUniqueId");
  a.init_rank = (decltype(a.init_rank))dlsym(h, "ncclCommInitRank");
  a.all_reduce = (decltype(a.all_reduce))dlsym(h, "ncclAllReduce");
  a.destroy = (decltype(a.destroy))dlsym(h, "ncclCommDestroy");
  a.err = (decltype(a.err))dlsym(h, "ncclGetErrorString");
  a.ok = a.get_id && a.init_rank && a.all_reduce && a.destroy && a.err;
  if (!a.ok) a.why = "libnccl lacks ncclGetUniqueId/ncclCommInitRank/ncclAllReduce/ncclCommDestroy";
  return a;
}
}  // namespace

struct Snapshot {
  bf16* wf = nullptr;    // packed fwd weights (all convs)
  bf16* wo = nullptr;    // packed dy-fold weights (rolling conv for wide frames)
  float* bias = nullptr; // packed fp32 biases
};

// Activation workspace of one inference path (grown on the first call of a larger shape).  A ctx has two: frames
// (the sr_infer family) and quality evaluation (sr_psnr_gain / sr_controller_step, issued from the training side),
// so the two may run concurrently on different streams without sharing buffers.
struct InferWS {
  size_t pix = 0;
  bf16 *x16 = nullptr, *f0 = nullptr, *fa = nullptr, *fb = nullptr, *tt = nullptr;
};

struct sr_ctx {
  int s = 2, B = 0, C = 0, Cp = 16, OUTP = 16, nconv = 0;
  sr_options opt{};
  std::vector<ConvDesc> convs;
  ConvDesc* convs_dev = nullptr;
  size_t nparams = 0, pk_total = 0, b_total = 0;
  int max_pk = 0;
  float *params = nullptr, *m = nullptr, *v = nullptr, *grad = nullptr;
  long long t = 0;  // Adam step counter
  Snapshot snap[4];
  bf16* wd_train = nullptr;  // dgrad-packed TRAIN weights
  bf16* wdo_train = nullptr; // dgrad weights in dy-fold layout (rolling data-grad convs)
  bool virtual_train = true; // training on the virtual wide batch with the rolling kernels
  // inference workspaces: frames, quality evaluation
  InferWS iws, qws;
  // sr_infer_host(_async): two staging sets used alternately, so two calls can be in flight (call k+1's H2D and
  // compute queue behind call k's while its D2H drains); a call waits only for the call that last used its set
  uint8_t *stage_lr[2] = {nullptr, nullptr}, *stage_hr[2] = {nullptr, nullptr};
  cudaStream_t copy_st = nullptr, h2d_st = nullptr;  // sr_infer_host: PCIe copies overlapped with the tensor work
  std::vector<cudaEvent_t> chunk_ev[2];
  cudaEvent_t host_done[2] = {nullptr, nullptr};  // last D2H of the call that used the set
  cudaEvent_t set_read[2] = {nullptr, nullptr};   // last inference chunk of the call that used the set (its LR read)
  bool set_used[2] = {false, false};
  bool host_busy[2] = {false, false};
  unsigned long long host_calls = 0;
  size_t stage_lr_bytes[2] = {0, 0}, stage_hr_bytes[2] = {0, 0};
  // training workspace
  size_t tr_pix = 0;
  bf16 *tx16 = nullptr, *tg = nullptr, *tdy = nullptr, *tdg = nullptr, *tdfa = nullptr, *tdfb = nullptr,
       *tdt = nullptr;
  std::vector<bf16*> tf, tts;
  std::vector<bf16*> tdf, tdtb;  // virtual training path: every block's df_b (B+1) and dt_b (B), kept for the
                                 // batched wgrad at the end of the backward pass
  float* ws_w = nullptr;       // wgrad split-K partials [grid][9 cinp coutp + coutp]
  size_t ws_w_elems = 0;
  unsigned* wg_sync = nullptr; // wgrad grid barrier {count, generation}
  double* loss_sum = nullptr;
  long long* counters = nullptr;  // device: [0] sampler step (graph mode), [1] Adam t, [2] gather block counter,
                                  // [3] pooled patches (arrivals), [4] i420 crops clamped into the frame
  float* zero_bias = nullptr;     // device: 64 zeros (the bias of the data-gradient convs)
  // patch pool (device ring)
  uint8_t *pool_lr = nullptr, *pool_hr = nullptr;
  long long pool_total = 0, pool_cap = 0;
  int pool_pp = 0;
  uint8_t *batch_lr = nullptr, *batch_hr = nullptr;
  size_t batch_bytes_lr = 0, batch_bytes_hr = 0;
  long long sample_step = 0;
  // psnr
  uint8_t* val_a = nullptr;  // one model's SR output of the validation patches
  uint8_t *yuv_lr = nullptr, *yuv_hr = nullptr, *crop_buf = nullptr;  // I420 boundary staging (RGB)
  size_t yuv_lr_bytes = 0, yuv_hr_bytes = 0, crop_bytes = 0;
  unsigned long long* cell_sse = nullptr;  // patch selection
  int cell_n = 0;
  size_t val_bytes = 0;
  unsigned long long* sse = nullptr;
  int sse_n = 0;
  cudaEvent_t publish_ev = nullptr;
  // CUDA graph of one sampled training iteration (sample -> fwd/bwd -> [allreduce] -> Adam), per (batch, p); re-captured
  // when the loss pointer or any workspace it references changes (ws_gen counts training-workspace reallocations)
  cudaGraphExec_t train_graph = nullptr;
  int graph_batch = 0, graph_p = 0;
  float* graph_loss = nullptr;
  unsigned long long graph_kernels = 0;  // our kernels in one captured iteration
  int graph_sm = 0;                      // sm_train (grid sizes) the graph was captured with
  unsigned long long ws_gen = 0, graph_gen = 0;
  // data parallelism (T5): NCCL communicator owned by the ctx (created from sr_options.nccl_id), sum of the ranks'
  // gradient weights (allreduced once at sr_create)
  ncclComm_t comm = nullptr;
  double sum_w = 1.0;
  int device = 0;
  // inference calls in flight per stream (sr_publish makes its snapshot copies wait for them)
  std::vector<std::pair<cudaStream_t, cudaEvent_t>> infer_evs;
  std::mutex ev_mu;  // infer_evs is touched by the inference side (note_infer) and the training side (sr_publish)
  std::atomic<unsigned long long> launches{0};  // kernels launched (inference and training threads)
  // optional per-kernel-class CUDA-event timing (sr_kernel_timing)
  bool timing = false;
  bool fuse_blocks = true;  // fused residual-block kernel for wide frames (sr_set_option)
  bool roll_tail = true;    // rolling up conv with the tail epilogue for wide frames (sr_set_fusion bit 2 clears)
  bool fuse_bwd = false;    // fused data-gradient residual blocks (sr_set_fusion bit 3; slower at the training shape)
  bool tail_tma = true;     // TMA-staged LR/HR rows in the rolling tail (sr_set_fusion bit 4 clears)
  bool fuse_bodytail = true;  // body conv + up conv + tail as one kernel, g in smem (sr_set_fusion bit 5 clears)
  bool fuse_head = true;      // head conv reads the u8 frame directly (sr_set_fusion bit 6 clears)
  bool pair_blocks = true;    // residual blocks of wide frames on CTA pairs, cta_group::2 (sr_set_fusion bit 7 clears)
  bool split_blocks = false;  // inference residual blocks on CTA pairs split by conv (sr_set_fusion bit 8 sets)
  bool chain = false;         // training: block convs + body conv (forward) and the data-gradient chain as one
                              // persistent launch each (k_conv_chain; sr_set_fusion bit 9 or SR_CHAIN=1 sets)
  unsigned* chain_sync[2] = {nullptr, nullptr};  // k_conv_chain generation + row flags (forward, backward)
  int sm_train = 0;           // sr_set_sm_split: SMs given to the training kernels (0 = all SMs to every call)
  bool train_fold_only = false;  // TRAIN's tiled layouts (wf, wd) may be stale: rebuild before reading them
  int sm_total = 0;
  struct TRec { std::string cls; cudaEvent_t a, b; double flops, bytes; };
  std::vector<TRec> trec;
  size_t tnext = 0;
  std::string err;
  bool poisoned = false;
};

// ------------------------------------------------------------------------------------------ helpers
static bool env_chain() {  // SR_CHAIN=1: training conv chains as persistent k_conv_chain launches (A/B switch)
  const char* e = std::getenv("SR_CHAIN");
  return e && e[0] == '1';
}
static sr_status fail(sr_ctx* c, sr_status st, const std::string& msg) {
  if (c) {
    c->err = msg;
    if (st == SR_E_CUDA) c->poisoned = true;
  }
  return st;
}
#define CK(call)                                                                                       \
  do {                                                                                                 \
    cudaError_t e_ = (call);                                                                           \
    if (e_ != cudaSuccess) return fail(ctx, SR_E_CUDA, std::string(#call) + ": " + cudaGetErrorString(e_)); \
  } while (0)
#define CKL() CK(cudaGetLastError())

template <class T>
static cudaError_t dalloc(T** p, size_t count) {
  if (*p) cudaFree(*p);
  *p = nullptr;
  if (count == 0) return cudaSuccess;
  return cudaMalloc(reinterpret_cast<void**>(p), count * sizeof(T));
}
static int rup16(int c) { return (c + 15) / 16 * 16; }
#define TRY_(x)                  \
  do {                           \
    sr_status s_ = (x);          \
    if (s_ != SR_OK) return s_;  \
  } while (0)

static uint64_t mix64h(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

static sr_status repack(sr_ctx* ctx, int which, bool with_dgrad, cudaStream_t st, long long* bump = nullptr,
                        bool fold_only = false) {
  launch_pack_weights(ctx->params, ctx->convs_dev, ctx->nconv, ctx->max_pk, fold_only ? nullptr : ctx->snap[which].wf,
                      (with_dgrad && !fold_only) ? ctx->wd_train : nullptr, ctx->snap[which].wo,
                      with_dgrad ? ctx->wdo_train : nullptr, ctx->snap[which].bias, st, bump);
  ctx->launches++;
  CKL();
  return SR_OK;
}

static sr_status ensure_full_train_pack(sr_ctx* ctx, cudaStream_t st) {
  if (ctx->train_fold_only) return repack(ctx, SR_TRAIN, true, st);
  return SR_OK;
}

// event pair around one launch when timing is enabled (records reused across resets)
static void tmark_begin(sr_ctx* ctx, const std::string& cls, double flops, double bytes, cudaStream_t st) {
  if (!ctx->timing) return;
  if (ctx->tnext == ctx->trec.size()) {
    sr_ctx::TRec r;
    cudaEventCreate(&r.a);
    cudaEventCreate(&r.b);
    ctx->trec.push_back(r);
  }
  auto& r = ctx->trec[ctx->tnext];
  r.cls = cls;
  r.flops = flops;
  r.bytes = bytes;
  cudaEventRecord(r.a, st);
}
static void tmark_end(sr_ctx* ctx, cudaStream_t st) {
  if (!ctx->timing) return;
  cudaEventRecord(ctx->trec[ctx->tnext].b, st);
  ctx->tnext++;
}

// one conv launch (conv index ci of the network) with given packed weights
static sr_status conv(sr_ctx* ctx, int cinp, int coutp, int epi, const void* in, const bf16* wpk, int N, int H,
                      int W, const EpiParams& ep, cudaStream_t st) {
  size_t smem = 0;
  ConvGeom g = make_geom(N, H, W, cinp, coutp, &smem);
  int grid = std::min(g.units, num_sms());
  if (ctx->timing) {
    // algorithmic work: 2 * 9 * Cin * Cout FLOP per output pixel (padded channels as launched)
    const double px = (double)N * H * W;
    const char* kind = epi == EPI_ACT ? (ep.mask || (!ep.bias && !ep.relu) ? "dgrad" : "fwd") : (epi == EPI_TAIL_U8 ? "tail_u8" : "tail_train");
    tmark_begin(ctx, std::string("conv_") + kind + "_" + std::to_string(cinp) + "x" + std::to_string(coutp),
                2.0 * 9 * cinp * coutp * px, px * 2.0 * (cinp + coutp), st);
  }
  cudaError_t e = launch_conv(cinp, coutp, epi, in, wpk, g, ep, smem, grid, st);
  tmark_end(ctx, st);
  ctx->launches++;
  if (e != cudaSuccess)
    return fail(ctx, e == cudaErrorNotSupported ? SR_E_UNSUPPORTED : SR_E_CUDA,
                std::string("conv launch: ") + cudaGetErrorString(e));
  return SR_OK;
}

// forward conv with the fastest kernel for the shape: the rolling dy-fold kernel for wide frames (EPI_ACT
// without mask / second residual), otherwise the general tiled kernel.
static sr_status conv_fwd(sr_ctx* ctx, int cinp, int coutp, const void* in, const Snapshot& sn, int ci, int N, int H,
                          int W, const EpiParams& ep, cudaStream_t st) {
  if (roll_supported(cinp, coutp, W) && !ep.mask && !ep.res2) {
    if (ctx->timing) {
      const double px = (double)N * H * W;
      tmark_begin(ctx, std::string("conv_roll_") + std::to_string(cinp) + "x" + std::to_string(coutp),
                  2.0 * 9 * cinp * coutp * px, px * 2.0 * (cinp + coutp), st);
    }
    cudaError_t e = launch_conv_roll(cinp, coutp, in, sn.wo + ctx->convs[ci].pk_off, ep.bias, ep.res1, ep.relu,
                                     ep.out, N, H, W, st, 1);  // inside a chain that starts with k_pack_input
    tmark_end(ctx, st);
    ctx->launches++;
    if (e != cudaSuccess) return fail(ctx, SR_E_CUDA, std::string("conv_roll launch: ") + cudaGetErrorString(e));
    return SR_OK;
  }
  return conv(ctx, cinp, coutp, EPI_ACT, in, sn.wf + ctx->convs[ci].pk_off, N, H, W, ep, st);
}

// general rolling conv launch (training / dgrad variants), timed as one class
static sr_status roll_ex(sr_ctx* ctx, const char* cls, int cinp, int coutp, const void* in, const bf16* wfold,
                         const float* bias, const bf16* res1, const bf16* res2, const bf16* mask, int relu, int sep,
                         bf16* out, int N, int H, int W, cudaStream_t st) {
  if (ctx->timing) {
    const double px = (double)N * H * W;
    tmark_begin(ctx, std::string(cls) + "_" + std::to_string(cinp) + "x" + std::to_string(coutp),
                2.0 * 9 * cinp * coutp * px, px * 2.0 * (cinp + coutp), st);
  }
  // w_early: every roll_ex launch sits inside a forward / backward chain that starts with a packing kernel, so its
  // weights were written >= 2 kernels upstream (see k_conv_roll's prologue)
  cudaError_t e = launch_conv_roll_ex(cinp, coutp, in, wfold, bias, res1, res2, mask, relu, sep, out, N, H, W, st,
                                      nullptr, 1);
  tmark_end(ctx, st);
  ctx->launches++;
  if (e != cudaSuccess) return fail(ctx, SR_E_CUDA, std::string("roll launch: ") + cudaGetErrorString(e));
  return SR_OK;
}

// a chain of C -> C training convs as one persistent launch (k_conv_chain), timed as one class
static sr_status chain_launch(sr_ctx* ctx, const char* cls, const std::vector<ChainLayerDesc>& L, int sep, int H,
                              int W, unsigned* sync, cudaStream_t st) {
  const int Cp = ctx->Cp;
  if (ctx->timing) {
    const double px = (double)H * W * L.size();
    tmark_begin(ctx, std::string(cls) + "_" + std::to_string(Cp), 2.0 * 9 * Cp * Cp * px, px * 2.0 * 2 * Cp, st);
  }
  cudaError_t e = launch_conv_chain(Cp, L.data(), (int)L.size(), sep, 1, H, W, sync, st);
  tmark_end(ctx, st);
  ctx->launches++;
  if (e != cudaSuccess) return fail(ctx, SR_E_CUDA, std::string("chain launch: ") + cudaGetErrorString(e));
  return SR_OK;
}

static WgradJob wjob(sr_ctx* ctx, int ci, const bf16* x, const bf16* dy) {
  const ConvDesc& d = ctx->convs[ci];
  float* gW = ctx->grad + d.w_off;
  return WgradJob{x, dy, d.cinp, d.coutp, d.cin, d.cout, gW, gW + (size_t)d.cout * d.cin * 9};
}

static sr_status ensure_wg(sr_ctx* ctx, size_t elems, cudaStream_t st) {
  if (elems > ctx->ws_w_elems) { CK(dalloc(&ctx->ws_w, elems)); ctx->ws_w_elems = elems; ctx->ws_gen++; }
  if (!ctx->wg_sync) {
    CK(dalloc(&ctx->wg_sync, 2));
    CK(cudaMemsetAsync(ctx->wg_sync, 0, 2 * sizeof(unsigned), st));
  }
  return SR_OK;
}

// Weight (+ bias) gradients of a list of convs whose inputs share one shape: grad <- scale * dL/dW.  Wide images: the
// batched rolling kernel (one launch per kWgradMaxJobs convs); otherwise the tiled kernel, one launch per conv.
static sr_status wgrad_jobs(sr_ctx* ctx, const WgradJob* jobs, int J, int N, int H, int W, float scale,
                            cudaStream_t st) {
  for (int k0 = 0; k0 < J; k0 += kWgradMaxJobs) {
    const int nj = std::min(kWgradMaxJobs, J - k0);
    const WgradJob* jb = jobs + k0;
    if (!wgrad_multi_supported(jb, nj, W)) break;
    const int grid = wgrad_multi_grid(nj, N, H, W);
    TRY_(ensure_wg(ctx, wgrad_multi_ws_floats(jb, nj, grid), st));
    if (ctx->timing) {
      double fl = 0, by = 0;
      const double px = (double)N * H * W;
      for (int k = 0; k < nj; ++k) {
        fl += 2.0 * 9 * jb[k].cinp * jb[k].coutp * px;
        by += px * 2.0 * (jb[k].cinp + jb[k].coutp);
      }
      tmark_begin(ctx, nj > 1 ? "wgrad_batch" : "wgrad_" + std::to_string(jb[0].cinp) + "x" +
                                                    std::to_string(jb[0].coutp), fl, by, st);
    }
    cudaError_t e = launch_wgrad_multi(jb, nj, N, H, W, scale, ctx->ws_w, ctx->wg_sync, grid, nullptr, st);
    tmark_end(ctx, st);
    ctx->launches++;
    if (e != cudaSuccess) return fail(ctx, SR_E_CUDA, std::string("wgrad launch: ") + cudaGetErrorString(e));
    if (k0 + nj == J) return SR_OK;
  }
  for (int k = 0; k < J; ++k) {  // tiled kernel
    const WgradJob& j = jobs[k];
    size_t smem = 0;
    WgradGeom g = make_wgrad_geom(N, H, W, j.cinp, j.coutp, &smem);
    const int grid = std::min(g.units, num_sms());
    TRY_(ensure_wg(ctx, (size_t)grid * (9 * j.cinp * j.coutp + j.coutp), st));
    if (ctx->timing) {
      const double px = (double)N * H * W;
      tmark_begin(ctx, "wgrad_" + std::to_string(j.cinp) + "x" + std::to_string(j.coutp),
                  2.0 * 9 * j.cinp * j.coutp * px, px * 2.0 * (j.cinp + j.coutp), st);
    }
    WgradOut o{ctx->ws_w, ctx->wg_sync, j.gW, j.gb, j.cin, j.cout, scale};
    cudaError_t e = launch_wgrad(j.cinp, j.coutp, j.x, j.dy, g, o, smem, grid, st);
    tmark_end(ctx, st);
    ctx->launches++;
    if (e != cudaSuccess) return fail(ctx, SR_E_CUDA, std::string("wgrad launch: ") + cudaGetErrorString(e));
  }
  return SR_OK;
}

static sr_status wgrad(sr_ctx* ctx, int ci, const bf16* x, const bf16* dy, int N, int H, int W, float scale,
                       cudaStream_t st) {
  const WgradJob j = wjob(ctx, ci, x, dy);
  return wgrad_jobs(ctx, &j, 1, N, H, W, scale, st);
}

#define TRY(x)                   \
  do {                           \
    sr_status s_ = (x);          \
    if (s_ != SR_OK) return s_;  \
  } while (0)

static sr_status ensure_infer_ws(sr_ctx* ctx, InferWS& ws, size_t pix) {
  if (pix <= ws.pix) return SR_OK;
  CK(dalloc(&ws.x16, pix * 16));
  CK(dalloc(&ws.f0, pix * ctx->Cp));
  CK(dalloc(&ws.fa, pix * ctx->Cp));
  CK(dalloc(&ws.fb, pix * ctx->Cp));
  CK(dalloc(&ws.tt, pix * ctx->Cp));
  ws.pix = pix;
  return SR_OK;
}

// Inference forward (reading R1): x = v/255; f0 = head(x); f <- f + conv2(relu(conv1(f))) x B;
// g = f0 + body(f); tail(up(g)) -> u8 with pixel shuffle + bilinear skip + clamp + RNE.
struct YuvIn {  // an I420 LR frame batch: planes y [n][h][w], u / v [n][h/2][w/2]
  const uint8_t *y, *u, *v;
};
struct YuvOut {  // the I420 HR output planes: y [n][sh][sw], u / v [n][sh/2][sw/2]
  uint8_t *y, *u, *v;
};

// yuv (optional): the LR frames arrive as I420; the head conv converts them itself (the I420 -> RGB conversion fused
// into its u8 expansion) and writes the RGB copy into `lr` (a ctx buffer) for the tail's skip.
// yo (optional, s = 2 or 4): the fused body + tail kernel writes the HR frames as I420 planes instead of RGB into hr
// (a lane's s x s HR block holds whole 2x2 chroma blocks); *yo_done says whether it did (else hr holds RGB).
static sr_status forward_infer(sr_ctx* ctx, InferWS& ws, const Snapshot& sn, const uint8_t* lr, int n, int h, int w,
                               uint8_t* hr, int row0, int row1, cudaStream_t st, const YuvIn* yuv = nullptr,
                               const YuvOut* yo = nullptr, bool* yo_done = nullptr) {
  if (yo_done) *yo_done = false;
  if (&sn == &ctx->snap[SR_TRAIN]) TRY(ensure_full_train_pack(ctx, st));
  const size_t pix = (size_t)n * h * w;
  TRY(ensure_infer_ws(ctx, ws, pix));
  const int Cp = ctx->Cp;
  auto W = [&](int ci) { return sn.wf + ctx->convs[ci].pk_off; };
  auto Bv = [&](int ci) { return sn.bias + ctx->convs[ci].b_off; };
  if (yuv) {
    if (ctx->timing) {
      const double px = (double)n * h * w;
      tmark_begin(ctx, "conv_roll_yuv_16x" + std::to_string(Cp), 2.0 * 9 * 16 * Cp * px, px * (1.5 + 3.0 + 2.0 * Cp), st);
    }
    cudaError_t e = launch_conv_roll_head_yuv(Cp, yuv->y, yuv->u, yuv->v, const_cast<uint8_t*>(lr),
                                              sn.wo + ctx->convs[0].pk_off, Bv(0), ws.f0, n, h, w, st, 1);
    tmark_end(ctx, st);
    ctx->launches++;
    if (e != cudaSuccess) return fail(ctx, SR_E_CUDA, std::string("I420 head launch: ") + cudaGetErrorString(e));
  } else if (ctx->fuse_head && roll_supported(16, Cp, w) && roll_head_u8_supported(Cp, w, lr)) {
    // head conv straight from the u8 frame (x = v/255 expanded in shared memory; no k_pack_input pass)
    if (ctx->timing) {
      const double px = (double)n * h * w;
      tmark_begin(ctx, "conv_roll_16x" + std::to_string(Cp), 2.0 * 9 * 16 * Cp * px, px * (3.0 + 2.0 * Cp), st);
    }
    cudaError_t e = launch_conv_roll_head_u8(Cp, lr, sn.wo + ctx->convs[0].pk_off, Bv(0), ws.f0, n, h, w, st, 1);
    tmark_end(ctx, st);
    ctx->launches++;
    if (e != cudaSuccess) return fail(ctx, SR_E_CUDA, std::string("u8 head launch: ") + cudaGetErrorString(e));
  } else {
    launch_pack_input(lr, pix, ws.x16, st);
    ctx->launches++;
    CKL();
    EpiParams ep{};
    ep.bias = Bv(0);
    ep.out = ws.f0;
    TRY(conv_fwd(ctx, 16, Cp, ws.x16, sn, 0, n, h, w, ep, st));
  }
  bf16* cur = ws.f0;
  for (int b = 0; b < ctx->B; ++b) {
    bf16* nxt = (cur == ws.fa) ? ws.fb : ws.fa;
    if (ctx->fuse_blocks && resblock_supported(Cp, w)) {  // fused block: t stays in shared memory
      if (ctx->timing) {
        const double px = (double)n * h * w;
        tmark_begin(ctx, "resblock_" + std::to_string(Cp), 2 * 2.0 * 9 * Cp * Cp * px, px * 2.0 * 2 * Cp, st);
      }
      cudaError_t e =
          ctx->split_blocks && resblock_split_supported(Cp, w)
              ? launch_resblock_split(Cp, cur, sn.wo + ctx->convs[1 + 2 * b].pk_off,
                                      sn.wo + ctx->convs[2 + 2 * b].pk_off, Bv(1 + 2 * b), Bv(2 + 2 * b), nxt, n, h, w,
                                      st)
          : ctx->pair_blocks && resblock2_supported(Cp, w)
              ? launch_resblock2(Cp, cur, sn.wo + ctx->convs[1 + 2 * b].pk_off, sn.wo + ctx->convs[2 + 2 * b].pk_off,
                                 Bv(1 + 2 * b), Bv(2 + 2 * b), nxt, n, h, w, st)
              : launch_resblock(Cp, cur, sn.wo + ctx->convs[1 + 2 * b].pk_off, sn.wo + ctx->convs[2 + 2 * b].pk_off,
                                Bv(1 + 2 * b), Bv(2 + 2 * b), nxt, n, h, w, st);
      tmark_end(ctx, st);
      ctx->launches++;
      if (e != cudaSuccess) return fail(ctx, SR_E_CUDA, std::string("resblock launch: ") + cudaGetErrorString(e));
      cur = nxt;
      continue;
    }
    EpiParams e1{};
    e1.bias = Bv(1 + 2 * b);
    e1.relu = 1;
    e1.out = ws.tt;
    TRY(conv_fwd(ctx, Cp, Cp, cur, sn, 1 + 2 * b, n, h, w, e1, st));
    EpiParams e2{};
    e2.bias = Bv(2 + 2 * b);
    e2.res1 = cur;
    e2.out = nxt;
    TRY(conv_fwd(ctx, Cp, Cp, ws.tt, sn, 2 + 2 * b, n, h, w, e2, st));
    cur = nxt;
  }
  const int cb = 1 + 2 * ctx->B, cu = cb + 1;
  if (ctx->fuse_bodytail && ctx->roll_tail && ctx->OUTP == (ctx->s == 2 ? 16 : ctx->s == 3 ? 32 : 48) &&
      bodytail_supported(Cp, ctx->s, w, lr, hr)) {  // g = f0 + body(f) stays in shared memory
    if (ctx->timing) {
      const double px = (double)n * h * w;
      tmark_begin(ctx, "bodytail_" + std::to_string(Cp) + "x" + std::to_string(ctx->OUTP),
                  2.0 * 9 * Cp * (Cp + ctx->OUTP) * px, px * (4.0 * Cp + 3.0 * (1 + ctx->s * ctx->s)), st);
    }
    const bool i420 = yo && ctx->s % 2 == 0;
    cudaError_t e = launch_bodytail(Cp, ctx->s, cur, ws.f0, sn.wo + ctx->convs[cb].pk_off,
                                    sn.wo + ctx->convs[cu].pk_off, Bv(cb), Bv(cu), lr, hr, row0, row1,
                                    ctx->opt.skip == 1, n, h, w, st, nullptr, i420 ? yo->y : nullptr,
                                    i420 ? yo->u : nullptr, i420 ? yo->v : nullptr);
    tmark_end(ctx, st);
    ctx->launches++;
    if (e != cudaSuccess) return fail(ctx, SR_E_CUDA, std::string("bodytail launch: ") + cudaGetErrorString(e));
    if (yo_done) *yo_done = i420;
    return SR_OK;
  }
  bf16* gbuf = (cur == ws.fa) ? ws.fb : ws.fa;
  EpiParams eb{};
  eb.bias = Bv(cb);
  eb.res1 = ws.f0;
  eb.out = gbuf;
  TRY(conv_fwd(ctx, Cp, Cp, cur, sn, cb, n, h, w, eb, st));
  if (roll_supported(Cp, ctx->OUTP, w) && ctx->roll_tail) {  // rolling up conv with the tail in its epilogue
    if (ctx->timing) {
      const double px = (double)n * h * w;
      tmark_begin(ctx, "conv_tail_roll_" + std::to_string(Cp) + "x" + std::to_string(ctx->OUTP),
                  2.0 * 9 * Cp * ctx->OUTP * px, px * (2.0 * Cp + 3.0 * (1 + ctx->s * ctx->s)), st);
    }
    cudaError_t e = launch_conv_roll_tail(Cp, ctx->OUTP, ctx->s, gbuf, sn.wo + ctx->convs[cu].pk_off, Bv(cu), lr, hr,
                                          row0, row1, ctx->opt.skip == 1, n, h, w, st, ctx->tail_tma, nullptr, 1);
    tmark_end(ctx, st);
    ctx->launches++;
    if (e != cudaSuccess) return fail(ctx, SR_E_CUDA, std::string("roll tail launch: ") + cudaGetErrorString(e));
    return SR_OK;
  }
  EpiParams et{};
  et.bias = Bv(cu);
  et.scale = ctx->s;
  et.bicubic = ctx->opt.skip == 1;
  et.lr = lr;
  et.hr = hr;
  et.hr_row0 = row0;
  et.hr_row1 = row1;
  TRY(conv(ctx, Cp, ctx->OUTP, EPI_TAIL_U8, gbuf, W(cu), n, h, w, et, st));
  return SR_OK;
}

// Batches of small square images (the validation patches of sr_psnr_gain / sr_controller_step): too narrow for
// the wide kernels one by one, so they run as ONE virtual wide image, side by side with zero separator columns
// (re-zeroed by every conv epilogue = each image's own zero padding), exactly like the training batch.  Same
// math as forward_infer.
static bool use_virtual_infer(const sr_ctx* ctx, int n, int h, int w) {
  const int Wv = n * (w + 2);
  return n > 1 && h == w && !roll_supported(16, ctx->Cp, w) && roll_supported(16, ctx->Cp, Wv) &&
         roll_supported(ctx->Cp, ctx->Cp, Wv);
}

static sr_status forward_infer_virtual(sr_ctx* ctx, InferWS& ws, const Snapshot& sn, const uint8_t* lr, int n, int p,
                                       uint8_t* hr, cudaStream_t st) {
  if (&sn == &ctx->snap[SR_TRAIN]) TRY(ensure_full_train_pack(ctx, st));
  const int Hv = p, Wv = n * (p + 2), sep = p + 2;
  TRY(ensure_infer_ws(ctx, ws, (size_t)Hv * Wv));
  const int Cp = ctx->Cp;
  auto WO = [&](int ci) { return sn.wo + ctx->convs[ci].pk_off; };
  auto Bv = [&](int ci) { return sn.bias + ctx->convs[ci].b_off; };
  launch_pack_input_virtual(lr, n, p, ws.x16, st);
  ctx->launches++;
  CKL();
  TRY(roll_ex(ctx, "infer_v", 16, Cp, ws.x16, WO(0), Bv(0), nullptr, nullptr, nullptr, 0, sep, ws.f0, 1, Hv, Wv,
              st));
  bf16* cur = ws.f0;
  for (int b = 0; b < ctx->B; ++b) {
    bf16* nxt = (cur == ws.fa) ? ws.fb : ws.fa;
    if (ctx->fuse_blocks && resblock_supported(Cp, Wv)) {
      cudaError_t e = launch_resblock(Cp, cur, WO(1 + 2 * b), WO(2 + 2 * b), Bv(1 + 2 * b), Bv(2 + 2 * b), nxt, 1, Hv,
                                      Wv, st, nullptr, nullptr, sep);
      ctx->launches++;
      if (e != cudaSuccess) return fail(ctx, SR_E_CUDA, std::string("resblock launch: ") + cudaGetErrorString(e));
    } else {
      TRY(roll_ex(ctx, "infer_v", Cp, Cp, cur, WO(1 + 2 * b), Bv(1 + 2 * b), nullptr, nullptr, nullptr, 1, sep, ws.tt,
                  1, Hv, Wv, st));
      TRY(roll_ex(ctx, "infer_v", Cp, Cp, ws.tt, WO(2 + 2 * b), Bv(2 + 2 * b), cur, nullptr, nullptr, 0, sep, nxt, 1,
                  Hv, Wv, st));
    }
    cur = nxt;
  }
  const int cb = 1 + 2 * ctx->B, cu = cb + 1;
  bf16* gbuf = (cur == ws.fa) ? ws.fb : ws.fa;
  TRY(roll_ex(ctx, "infer_v", Cp, Cp, cur, WO(cb), Bv(cb), ws.f0, nullptr, nullptr, 0, sep, gbuf, 1, Hv, Wv, st));
  EpiParams et{};
  et.bias = Bv(cu);
  et.scale = ctx->s;
  et.bicubic = ctx->opt.skip == 1;
  et.lr = lr;
  et.hr = hr;
  et.vsep = sep;
  et.vp = p;
  TRY(conv(ctx, Cp, ctx->OUTP, EPI_TAIL_U8, gbuf, sn.wf + ctx->convs[cu].pk_off, 1, Hv, Wv, et, st));
  return SR_OK;
}

static sr_status ensure_train_ws(sr_ctx* ctx, size_t pix) {
  if (pix <= ctx->tr_pix) return SR_OK;
  ctx->ws_gen++;
  const int Cp = ctx->Cp;
  CK(dalloc(&ctx->tx16, pix * 16));
  for (auto& p : ctx->tf) CK(dalloc(&p, pix * Cp));
  for (auto& p : ctx->tts) CK(dalloc(&p, pix * Cp));
  CK(dalloc(&ctx->tg, pix * Cp));
  CK(dalloc(&ctx->tdy, pix * ctx->OUTP));
  CK(dalloc(&ctx->tdg, pix * Cp));
  CK(dalloc(&ctx->tdfa, pix * Cp));
  CK(dalloc(&ctx->tdfb, pix * Cp));
  CK(dalloc(&ctx->tdt, pix * Cp));
  for (auto& p : ctx->tdf) CK(dalloc(&p, pix * Cp));
  for (auto& p : ctx->tdtb) CK(dalloc(&p, pix * Cp));
  for (auto& p : ctx->chain_sync) {  // >= chain_sync_words(1, H, W) for any H x W = pix with W >= 96
    const size_t words = 66 + pix / 48;
    CK(dalloc(&p, words));
    CK(cudaMemset(p, 0, words * sizeof(unsigned)));
  }
  ctx->tr_pix = pix;
  return SR_OK;
}

// Training step on the virtual wide batch: the n patches (p x p) sit side by side in one p x n(p+2) image with
// zero separator columns, so every conv of the forward and of the data-gradient pass runs on the rolling wide
// kernels (separators re-zeroed in their epilogues = each patch's own zero padding), and wgrad sums over the
// whole image (separators contribute zero).  Same math as the per-patch path below.
static sr_status train_grad_virtual(sr_ctx* ctx, const uint8_t* lr, const uint8_t* hr, int n, int p,
                                    float* loss_dev, cudaStream_t st) {
  const int Hv = p, Wv = n * (p + 2), sep = p + 2;
  const size_t pix = (size_t)Hv * Wv;
  TRY(ensure_train_ws(ctx, pix));
  const int Cp = ctx->Cp, B = ctx->B, OUTP = ctx->OUTP;
  const Snapshot& sn = ctx->snap[SR_TRAIN];
  auto WO = [&](int ci) { return sn.wo + ctx->convs[ci].pk_off; };
  auto WDO = [&](int ci) { return ctx->wdo_train + ctx->convs[ci].pk_off; };
  auto Bv = [&](int ci) { return sn.bias + ctx->convs[ci].b_off; };
  launch_pack_input_virtual(lr, n, p, ctx->tx16, st);
  ctx->launches++;
  CK(cudaMemsetAsync(ctx->loss_sum, 0, sizeof(double), st));
  // ---- forward (saving f_0..f_B, t_1..t_B, g)
  TRY(roll_ex(ctx, "train_fwd", 16, Cp, ctx->tx16, WO(0), Bv(0), nullptr, nullptr, nullptr, 0, sep, ctx->tf[0], 1,
              Hv, Wv, st));
  const int cb = 1 + 2 * B, cu = cb + 1;
  const bool use_chain = ctx->chain && chain_supported(Cp, Wv, 2 * B + 1) &&
                         chain_sync_words(1, Hv, Wv) <= 66 + pix / 48;
  if (use_chain) {  // the B blocks (conv1 ReLU -> t_b, conv2 + f_b -> f_b+1) and the body conv (+ f_0) in one launch
    std::vector<ChainLayerDesc> L;
    for (int b = 0; b < B; ++b) {
      L.push_back({ctx->tf[b], ctx->tts[b], WO(1 + 2 * b), Bv(1 + 2 * b), nullptr, nullptr, nullptr, 1, -1});
      L.push_back({ctx->tts[b], ctx->tf[b + 1], WO(2 + 2 * b), Bv(2 + 2 * b), ctx->tf[b], nullptr, nullptr, 0,
                   b == 0 ? -1 : 2 * b - 1});
    }
    L.push_back({ctx->tf[B], ctx->tg, WO(cb), Bv(cb), ctx->tf[0], nullptr, nullptr, 0, -1});
    TRY(chain_launch(ctx, "train_fwd_chain", L, sep, Hv, Wv, ctx->chain_sync[0], st));
  }
  for (int b = 0; b < B && !use_chain; ++b) {
    if (ctx->fuse_blocks && resblock_supported(Cp, Wv)) {  // fused block, t also saved for the backward pass
      if (ctx->timing) {
        const double px = (double)Hv * Wv;
        tmark_begin(ctx, "train_resblock_" + std::to_string(Cp), 2 * 2.0 * 9 * Cp * Cp * px, px * 2.0 * 3 * Cp, st);
      }
      cudaError_t e = launch_resblock(Cp, ctx->tf[b], WO(1 + 2 * b), WO(2 + 2 * b), Bv(1 + 2 * b), Bv(2 + 2 * b),
                                      ctx->tf[b + 1], 1, Hv, Wv, st, nullptr, ctx->tts[b], sep);
      tmark_end(ctx, st);
      ctx->launches++;
      if (e != cudaSuccess) return fail(ctx, SR_E_CUDA, std::string("resblock launch: ") + cudaGetErrorString(e));
      continue;
    }
    TRY(roll_ex(ctx, "train_fwd", Cp, Cp, ctx->tf[b], WO(1 + 2 * b), Bv(1 + 2 * b), nullptr, nullptr, nullptr, 1,
                sep, ctx->tts[b], 1, Hv, Wv, st));
    TRY(roll_ex(ctx, "train_fwd", Cp, Cp, ctx->tts[b], WO(2 + 2 * b), Bv(2 + 2 * b), ctx->tf[b], nullptr, nullptr, 0,
                sep, ctx->tf[b + 1], 1, Hv, Wv, st));
  }
  if (!use_chain)
    TRY(roll_ex(ctx, "train_fwd", Cp, Cp, ctx->tf[B], WO(cb), Bv(cb), ctx->tf[0], nullptr, nullptr, 0, sep, ctx->tg, 1,
                Hv, Wv, st));
  {
    EpiParams e{};
    e.bias = Bv(cu);
    e.scale = ctx->s;
    e.lr = lr;
    e.hr_ref = hr;
    e.dy = ctx->tdy;
    e.loss_sum = ctx->loss_sum;
    e.l1 = ctx->opt.loss == 1;
    e.bicubic = ctx->opt.skip == 1;
    e.vsep = sep;
    e.vp = p;
    if (ctx->roll_tail && roll_supported(Cp, OUTP, Wv)) {  // rolling up conv with the training tail epilogue
      if (ctx->timing) {
        const double px = (double)Hv * Wv;
        tmark_begin(ctx, "conv_tail_train_roll_" + std::to_string(Cp) + "x" + std::to_string(OUTP),
                    2.0 * 9 * Cp * OUTP * px, px * (2.0 * Cp + 2.0 * OUTP), st);
      }
      cudaError_t er = launch_conv_roll_tail_train(Cp, OUTP, ctx->s, ctx->tg, WO(cu), Bv(cu), lr, hr, ctx->tdy,
                                                   ctx->loss_sum, sep, p, e.l1, e.bicubic, 1, Hv, Wv, st, 1);
      tmark_end(ctx, st);
      ctx->launches++;
      if (er != cudaSuccess) return fail(ctx, SR_E_CUDA, std::string("roll train tail: ") + cudaGetErrorString(er));
    } else {
      TRY(ensure_full_train_pack(ctx, st));  // the tiled tail reads TRAIN's tiled layout
      TRY(conv(ctx, Cp, OUTP, EPI_TAIL_TRAIN, ctx->tg, sn.wf + ctx->convs[cu].pk_off, 1, Hv, Wv, e, st));
    }
  }
  const double n_el = (double)n * p * p * ctx->s * ctx->s * 3;
  if (loss_dev) {
    launch_loss_finalize(ctx->loss_sum, 1.0 / n_el, loss_dev, st);
    ctx->launches++;
  }
  const float gscale = (float)((ctx->opt.dp_weight > 0 ? ctx->opt.dp_weight : 1.0f) / n_el);
  // ---- backward: the data-gradient chain (every df_b, dt_b kept), then all weight gradients in one batched launch
  TRY(roll_ex(ctx, "train_dgrad", OUTP, Cp, ctx->tdy, WDO(cu), nullptr, nullptr, nullptr, nullptr, 0, sep, ctx->tdg, 1,
              Hv, Wv, st));
  if (use_chain) {  // body dgrad, then per block (last first): dt_b = dgrad_conv2(df_b+1) x 1[t_b > 0] and
                    // df_b = dgrad_conv1(dt_b) + df_b+1 (+ dg at b = 0), in one launch
    std::vector<ChainLayerDesc> L;
    L.push_back({ctx->tdg, ctx->tdf[B], WDO(cb), nullptr, B == 0 ? ctx->tdg : nullptr, nullptr, nullptr, 0, -1});
    for (int b = B - 1; b >= 0; --b) {
      const int l2 = (int)L.size();
      L.push_back({ctx->tdf[b + 1], ctx->tdtb[b], WDO(2 + 2 * b), nullptr, nullptr, nullptr, ctx->tts[b], 0, -1});
      L.push_back({ctx->tdtb[b], ctx->tdf[b], WDO(1 + 2 * b), nullptr, ctx->tdf[b + 1], b == 0 ? ctx->tdg : nullptr,
                   nullptr, 0, l2 - 1});
    }
    TRY(chain_launch(ctx, "train_dgrad_chain", L, sep, Hv, Wv, ctx->chain_sync[1], st));
  } else {
    TRY(roll_ex(ctx, "train_dgrad", Cp, Cp, ctx->tdg, WDO(cb), nullptr, B == 0 ? ctx->tdg : nullptr, nullptr, nullptr,
                0, sep, ctx->tdf[B], 1, Hv, Wv, st));
  }
  for (int b = B - 1; b >= 0 && !use_chain; --b) {
    if (ctx->fuse_blocks && ctx->fuse_bwd && resblock_supported(Cp, Wv)) {
      // the block's data gradient in one fused kernel (k_resblock in mask mode): dt = dgrad_conv2(df) * 1[t > 0]
      // stays in shared memory (and is saved for the wgrad), df' = df + dgrad_conv1(dt) (+ dg into f0 at b = 0)
      if (ctx->timing) {
        const double px = (double)Hv * Wv;
        tmark_begin(ctx, "train_dgrad_block_" + std::to_string(Cp), 2 * 2.0 * 9 * Cp * Cp * px, px * 2.0 * 4 * Cp, st);
      }
      cudaError_t e = launch_resblock(Cp, ctx->tdf[b + 1], WDO(2 + 2 * b), WDO(1 + 2 * b), ctx->zero_bias,
                                      ctx->zero_bias, ctx->tdf[b], 1, Hv, Wv, st, nullptr, ctx->tdtb[b], sep, 0,
                                      ctx->tts[b], b == 0 ? ctx->tdg : nullptr);
      tmark_end(ctx, st);
      ctx->launches++;
      if (e != cudaSuccess) return fail(ctx, SR_E_CUDA, std::string("dgrad block launch: ") + cudaGetErrorString(e));
      continue;
    }
    TRY(roll_ex(ctx, "train_dgrad", Cp, Cp, ctx->tdf[b + 1], WDO(2 + 2 * b), nullptr, nullptr, nullptr, ctx->tts[b],
                0, sep, ctx->tdtb[b], 1, Hv, Wv, st));
    TRY(roll_ex(ctx, "train_dgrad", Cp, Cp, ctx->tdtb[b], WDO(1 + 2 * b), nullptr, ctx->tdf[b + 1],
                b == 0 ? ctx->tdg : nullptr, nullptr, 0, sep, ctx->tdf[b], 1, Hv, Wv, st));
  }
  // jobs in reverse production order of their dY (the most recent dY is the likeliest to still sit in L2)
  std::vector<WgradJob> jobs;
  jobs.push_back(wjob(ctx, 0, ctx->tx16, ctx->tdf[0]));
  for (int b = 0; b < B; ++b) {
    jobs.push_back(wjob(ctx, 1 + 2 * b, ctx->tf[b], ctx->tdtb[b]));
    jobs.push_back(wjob(ctx, 2 + 2 * b, ctx->tts[b], ctx->tdf[b + 1]));
  }
  jobs.push_back(wjob(ctx, cb, ctx->tf[B], ctx->tdg));
  jobs.push_back(wjob(ctx, cu, ctx->tg, ctx->tdy));
  return wgrad_jobs(ctx, jobs.data(), (int)jobs.size(), 1, Hv, Wv, gscale, st);
}

// Forward with saved activations, MSE loss + gradient fused into the tail, backward (dgrad = the fwd conv
// kernel on 180-degree-rotated / transposed weights with ReLU-mask and residual epilogues; wgrad =
// tcgen05 split-K + deterministic reduce).  grad <- w_r * dL/dtheta.
static sr_status train_grad(sr_ctx* ctx, const uint8_t* lr, const uint8_t* hr, int n, int p, float* loss_dev,
                            cudaStream_t st) {
  if (ctx->virtual_train && roll_supported(ctx->OUTP, ctx->Cp, n * (p + 2)) && roll_supported(16, ctx->Cp, n * (p + 2)))
    return train_grad_virtual(ctx, lr, hr, n, p, loss_dev, st);
  TRY(ensure_full_train_pack(ctx, st));
  const size_t pix = (size_t)n * p * p;
  TRY(ensure_train_ws(ctx, pix));
  const int Cp = ctx->Cp, B = ctx->B, OUTP = ctx->OUTP;
  const Snapshot& sn = ctx->snap[SR_TRAIN];
  auto W = [&](int ci) { return sn.wf + ctx->convs[ci].pk_off; };
  auto WD = [&](int ci) { return ctx->wd_train + ctx->convs[ci].pk_off; };
  auto Bv = [&](int ci) { return sn.bias + ctx->convs[ci].b_off; };
  launch_pack_input(lr, pix, ctx->tx16, st);
  ctx->launches++;
  CK(cudaMemsetAsync(ctx->loss_sum, 0, sizeof(double), st));
  // ---- forward, saving f_0..f_B and t_1..t_B
  {
    EpiParams e{};
    e.bias = Bv(0);
    e.out = ctx->tf[0];
    TRY(conv(ctx, 16, Cp, EPI_ACT, ctx->tx16, W(0), n, p, p, e, st));
  }
  for (int b = 0; b < B; ++b) {
    EpiParams e1{};
    e1.bias = Bv(1 + 2 * b);
    e1.relu = 1;
    e1.out = ctx->tts[b];
    TRY(conv(ctx, Cp, Cp, EPI_ACT, ctx->tf[b], W(1 + 2 * b), n, p, p, e1, st));
    EpiParams e2{};
    e2.bias = Bv(2 + 2 * b);
    e2.res1 = ctx->tf[b];
    e2.out = ctx->tf[b + 1];
    TRY(conv(ctx, Cp, Cp, EPI_ACT, ctx->tts[b], W(2 + 2 * b), n, p, p, e2, st));
  }
  const int cb = 1 + 2 * B, cu = cb + 1;
  {
    EpiParams e{};
    e.bias = Bv(cb);
    e.res1 = ctx->tf[0];
    e.out = ctx->tg;
    TRY(conv(ctx, Cp, Cp, EPI_ACT, ctx->tf[B], W(cb), n, p, p, e, st));
  }
  {
    EpiParams e{};
    e.bias = Bv(cu);
    e.scale = ctx->s;
    e.lr = lr;
    e.hr_ref = hr;
    e.dy = ctx->tdy;
    e.loss_sum = ctx->loss_sum;
    e.l1 = ctx->opt.loss == 1;
    e.bicubic = ctx->opt.skip == 1;
    TRY(conv(ctx, Cp, OUTP, EPI_TAIL_TRAIN, ctx->tg, W(cu), n, p, p, e, st));
  }
  const double n_el = (double)pix * ctx->s * ctx->s * 3;
  if (loss_dev) {
    launch_loss_finalize(ctx->loss_sum, 1.0 / n_el, loss_dev, st);
    ctx->launches++;
  }
  // dy holds 2 (o - t); the mean's 1/n_el and the DP weight are applied once in the wgrad reduction
  const float gscale = (float)((ctx->opt.dp_weight > 0 ? ctx->opt.dp_weight : 1.0f) / n_el);
  // ---- backward
  TRY(wgrad(ctx, cu, ctx->tg, ctx->tdy, n, p, p, gscale, st));
  {
    EpiParams e{};
    e.out = ctx->tdg;  // dg = dgrad_up(dy)
    TRY(conv(ctx, OUTP, Cp, EPI_ACT, ctx->tdy, WD(cu), n, p, p, e, st));
  }
  TRY(wgrad(ctx, cb, ctx->tf[B], ctx->tdg, n, p, p, gscale, st));
  bf16* df = ctx->tdfa;
  {
    EpiParams e{};
    e.out = df;                    // df_B = dgrad_body(dg)   (B == 0: + dg, since f_B = f0)
    if (B == 0) e.res1 = ctx->tdg;
    TRY(conv(ctx, Cp, Cp, EPI_ACT, ctx->tdg, WD(cb), n, p, p, e, st));
  }
  for (int b = B - 1; b >= 0; --b) {
    TRY(wgrad(ctx, 2 + 2 * b, ctx->tts[b], df, n, p, p, gscale, st));
    {
      EpiParams e{};
      e.mask = ctx->tts[b];        // ReLU' = 1[t > 0]
      e.out = ctx->tdt;
      TRY(conv(ctx, Cp, Cp, EPI_ACT, df, WD(2 + 2 * b), n, p, p, e, st));
    }
    TRY(wgrad(ctx, 1 + 2 * b, ctx->tf[b], ctx->tdt, n, p, p, gscale, st));
    bf16* dfn = (df == ctx->tdfa) ? ctx->tdfb : ctx->tdfa;
    {
      EpiParams e{};
      e.res1 = df;                 // residual path
      if (b == 0) e.res2 = ctx->tdg;  // global skip into f0
      e.out = dfn;
      TRY(conv(ctx, Cp, Cp, EPI_ACT, ctx->tdt, WD(1 + 2 * b), n, p, p, e, st));
    }
    df = dfn;
  }
  TRY(wgrad(ctx, 0, ctx->tx16, df, n, p, p, gscale, st));
  return SR_OK;
}

static sr_status train_apply(sr_ctx* ctx, float grad_scale, const float* grad_scale_dev, cudaStream_t st) {
  ctx->t += 1;  // host mirror only; the kernels use the device counter (graph-replayable)
  launch_adam(ctx->params, ctx->m, ctx->v, ctx->grad, ctx->nparams, grad_scale_dev, grad_scale, ctx->counters,
              ctx->opt.lr, ctx->opt.beta1, ctx->opt.beta2, ctx->opt.eps, st);
  ctx->launches += 1;
  CKL();
  // The per-step repack writes only the dy-fold layouts the wide (virtual-batch) path reads; the tiled layouts of
  // TRAIN are rebuilt on demand (ensure_full_train_pack) by the calls that read them.  The flag is sticky: graph
  // replays of this step do not pass through the host.
  if (ctx->virtual_train) ctx->train_fold_only = true;
  return repack(ctx, SR_TRAIN, true, st, ctx->counters + 1, ctx->virtual_train);  // + Adam step counter
}

static bool valid_model(sr_model m) { return m >= SR_TRAIN && m <= SR_INIT; }

#define NCK(call)                                                                                           \
  do {                                                                                                      \
    ncclResult_t r_ = (call);                                                                               \
    if (r_ != ncclSuccess) return fail(ctx, SR_E_NCCL, std::string(#call) + ": " + nccl().err(r_));        \
  } while (0)

// Communicator of the DP group from the caller's ncclUniqueId (collective over the ranks: every rank calls sr_create
// with the same id), then sum_r w_r of the ranks' gradient weights, once (the weights are fixed per ctx).
static sr_status comm_init(sr_ctx* ctx) {
  NcclApi& a = nccl();
  if (!a.ok) return fail(ctx, SR_E_NCCL, a.why);
  ncclUniqueId id;
  memcpy(&id, ctx->opt.nccl_id, sizeof(id));
  NCK(a.init_rank(&ctx->comm, ctx->opt.world, id, ctx->opt.rank));
  float* w = nullptr;
  CK(cudaMalloc(&w, sizeof(float)));
  const float mine = ctx->opt.dp_weight;
  CK(cudaMemcpy(w, &mine, sizeof(float), cudaMemcpyHostToDevice));
  ncclResult_t r = a.all_reduce(w, w, 1, ncclFloat32, ncclSum, ctx->comm, 0);
  float tot = 0.f;
  cudaError_t e = cudaMemcpy(&tot, w, sizeof(float), cudaMemcpyDeviceToHost);
  cudaFree(w);
  if (r != ncclSuccess) return fail(ctx, SR_E_NCCL, std::string("ncclAllReduce(weights): ") + a.err(r));
  CK(e);
  if (!(tot > 0.f)) return fail(ctx, SR_E_INVAL, "sum of dp_weight over ranks must be > 0");
  ctx->sum_w = tot;
  return SR_OK;
}

// T5 exchange: grad <- sum_r (w_r g_r) over the DP group, in place, stream-ordered (graph-capturable).
static sr_status grad_exchange(sr_ctx* ctx, cudaStream_t st) {
  if (!ctx->comm) {
    if (ctx->opt.world > 1)
      return fail(ctx, SR_E_STATE, "world > 1 without sr_options.nccl_id: exchange the gradient yourself "
                                   "(sr_grad_buffer) and call sr_train_apply");
    return SR_OK;
  }
  NCK(nccl().all_reduce(ctx->grad, ctx->grad, ctx->nparams, ncclFloat32, ncclSum, ctx->comm, st));
  return SR_OK;  // (NCCL's kernel, not counted in sr_launch_count)
}

// the stream's last inference call (sr_publish orders its snapshot copies after it)
static sr_status note_infer(sr_ctx* ctx, cudaStream_t st) {
  cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
  CK(cudaStreamIsCapturing(st, &cs));
  if (cs != cudaStreamCaptureStatusNone) return SR_OK;  // inside a caller's graph capture: the caller orders it
  std::lock_guard<std::mutex> lk(ctx->ev_mu);
  for (auto& pe : ctx->infer_evs)
    if (pe.first == st) { CK(cudaEventRecord(pe.second, st)); return SR_OK; }
  cudaEvent_t e;
  CK(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
  ctx->infer_evs.push_back({st, e});
  CK(cudaEventRecord(e, st));
  return SR_OK;
}

// ------------------------------------------------------------------------------------------ C ABI
extern "C" {

sr_status sr_create(int scale, int blocks, int channels, const sr_options* opt, sr_ctx** out) {
  if (!out) return SR_E_INVAL;
  *out = nullptr;
  if ((scale < 2 || scale > 4) || blocks < 0 || channels < 1 || channels > 64) return SR_E_INVAL;
  sr_ctx* ctx = new sr_ctx();
  ctx->chain = env_chain();
  ctx->s = scale;
  ctx->B = blocks;
  ctx->C = channels;
  ctx->Cp = rup16(channels);
  if (ctx->Cp == 16 && channels > 16) ctx->Cp = 32;
  ctx->OUTP = rup16(3 * scale * scale);
  if (opt) ctx->opt = *opt;
  if (ctx->opt.lr == 0.f) ctx->opt.lr = 1e-4f;
  if (ctx->opt.beta1 == 0.f) ctx->opt.beta1 = 0.9f;
  if (ctx->opt.beta2 == 0.f) ctx->opt.beta2 = 0.999f;
  if (ctx->opt.eps == 0.f) ctx->opt.eps = 1e-8f;
  if (ctx->opt.recent_k == 0) ctx->opt.recent_k = 150;
  if (ctx->opt.recent_w == 0) ctx->opt.recent_w = 4;
  if (ctx->opt.world <= 0) ctx->opt.world = 1;
  if (ctx->opt.dp_weight == 0.f) ctx->opt.dp_weight = 1.f;
  if (ctx->opt.pool_capacity <= 0) ctx->opt.pool_capacity = 8192;
  if (ctx->opt.rank < 0 || ctx->opt.rank >= ctx->opt.world) { delete ctx; return SR_E_INVAL; }
  if (opt && opt->device >= 0) {
    if (cudaSetDevice(opt->device) != cudaSuccess) { delete ctx; return SR_E_INVAL; }
  }
  if (cudaGetDevice(&ctx->device) != cudaSuccess) { delete ctx; return SR_E_CUDA; }
  if (ctx->opt.loss < 0 || ctx->opt.loss > 1 || ctx->opt.skip < 0 || ctx->opt.skip > 1) { delete ctx; return SR_E_INVAL; }
  // conv table in canonical order: head, (b.conv1, b.conv2) x B, body, up
  std::vector<std::pair<int, int>> shp;  // (cout, cin)
  shp.push_back({channels, 3});
  for (int b = 0; b < blocks; ++b) { shp.push_back({channels, channels}); shp.push_back({channels, channels}); }
  shp.push_back({channels, channels});
  shp.push_back({3 * scale * scale, channels});
  long long woff = 0, pk = 0, bo = 0;
  for (auto& sc : shp) {
    ConvDesc d{};
    d.cout = sc.first;
    d.cin = sc.second;
    d.cinp = d.cin == 3 ? 16 : ctx->Cp;
    d.coutp = d.cout == 3 * scale * scale ? ctx->OUTP : ctx->Cp;
    d.w_off = woff;
    d.pk_off = pk;
    d.b_off = bo;
    woff += (long long)d.cout * d.cin * 9 + d.cout;
    pk += 9LL * d.cinp * d.coutp;
    bo += d.coutp;
    ctx->max_pk = std::max(ctx->max_pk, 9 * d.cinp * d.coutp);
    ctx->convs.push_back(d);
  }
  ctx->nconv = (int)ctx->convs.size();
  ctx->nparams = (size_t)woff;
  ctx->pk_total = (size_t)pk;
  ctx->b_total = (size_t)bo;
  sr_status st = SR_OK;
  auto al = [&](auto** p, size_t n) {
    if (st == SR_OK && dalloc(p, n) != cudaSuccess) st = SR_E_NOMEM;
  };
  al(&ctx->convs_dev, ctx->convs.size());
  al(&ctx->params, ctx->nparams);
  al(&ctx->m, ctx->nparams);
  al(&ctx->v, ctx->nparams);
  al(&ctx->grad, ctx->nparams);
  for (int k = 0; k < 4; ++k) {
    al(&ctx->snap[k].wf, ctx->pk_total);
    al(&ctx->snap[k].wo, ctx->pk_total);
    al(&ctx->snap[k].bias, ctx->b_total);
  }
  al(&ctx->wd_train, ctx->pk_total);
  al(&ctx->wdo_train, ctx->pk_total);
  al(&ctx->loss_sum, 1);
  al(&ctx->counters, 5);  // [0] sampler step, [1] Adam t, [2] gather block counter, [3] pool arrivals, [4] clamped crops
  al(&ctx->zero_bias, 64);
  if (st == SR_OK && cudaMemset(ctx->zero_bias, 0, 64 * sizeof(float)) != cudaSuccess) st = SR_E_CUDA;
  if (st == SR_OK && cudaMemset(ctx->counters, 0, 5 * sizeof(long long)) != cudaSuccess) st = SR_E_CUDA;
  ctx->tf.assign(blocks + 1, nullptr);
  ctx->tts.assign(blocks, nullptr);
  ctx->tdf.assign(blocks + 1, nullptr);
  ctx->tdtb.assign(blocks, nullptr);
  if (st != SR_OK) { sr_destroy(ctx); return st; }
  if (cudaMemcpy(ctx->convs_dev, ctx->convs.data(), ctx->convs.size() * sizeof(ConvDesc),
                 cudaMemcpyHostToDevice) != cudaSuccess ||
      cudaEventCreateWithFlags(&ctx->publish_ev, cudaEventDisableTiming) != cudaSuccess) {
    sr_destroy(ctx);
    return SR_E_CUDA;
  }
  // seeded init: SplitMix64 stream, u = (z >> 40) 2^-24, w = fp32((2u - 1) / sqrt(9 Cin)), per conv W then b
  std::vector<float> h(ctx->nparams);
  uint64_t state = ctx->opt.seed;
  size_t i = 0;
  for (auto& d : ctx->convs) {
    const double bound = 1.0 / std::sqrt(9.0 * d.cin);
    const size_t cnt = (size_t)d.cout * d.cin * 9 + d.cout;
    for (size_t k = 0; k < cnt; ++k, ++i) {
      state += 0x9E3779B97F4A7C15ull;
      const double u = (double)(mix64h(state) >> 40) * (1.0 / 16777216.0);
      h[i] = (float)((2.0 * u - 1.0) * bound);
    }
  }
  st = sr_set_params(ctx, h.data(), h.size());
  if (st != SR_OK) { sr_destroy(ctx); return st; }
  if (ctx->opt.nccl_id) {  // T5: the ctx owns the NCCL communicator of the data-parallel group
    st = comm_init(ctx);
    if (st != SR_OK) {
      std::string msg = ctx->err;
      sr_destroy(ctx);
      fprintf(stderr, "sr_create: %s\n", msg.c_str());
      return st;
    }
  } else {
    // world 1: the rank's own weight; world > 1 without a communicator: external exchange (the caller allreduces
    // sr_grad_buffer and passes 1 / sum_r w_r to sr_train_apply), sum unknown here
    ctx->sum_w = ctx->opt.world > 1 ? 0.0 : ctx->opt.dp_weight;
  }
  *out = ctx;
  return SR_OK;
}

void sr_destroy(sr_ctx* ctx) {
  if (!ctx) return;
  sync_all();
  for (InferWS* ws : {&ctx->iws, &ctx->qws})
    for (bf16* q : {ws->x16, ws->f0, ws->fa, ws->fb, ws->tt})
      if (q) cudaFree(q);
  for (int k = 0; k < 2; ++k) {
    if (ctx->stage_lr[k]) cudaFree(ctx->stage_lr[k]);
    if (ctx->stage_hr[k]) cudaFree(ctx->stage_hr[k]);
    for (auto e : ctx->chunk_ev[k]) if (e) cudaEventDestroy(e);
    if (ctx->host_done[k]) cudaEventDestroy(ctx->host_done[k]);
    if (ctx->set_read[k]) cudaEventDestroy(ctx->set_read[k]);
  }
  void* ptrs[] = {ctx->convs_dev, ctx->params, ctx->m, ctx->v, ctx->grad, ctx->wd_train, ctx->wdo_train, ctx->tx16, ctx->tg, ctx->tdy,
                  ctx->tdg, ctx->tdfa, ctx->tdfb, ctx->tdt, ctx->ws_w, ctx->wg_sync, ctx->loss_sum, ctx->counters,
                  ctx->zero_bias, ctx->pool_lr,
                  ctx->pool_hr, ctx->batch_lr, ctx->batch_hr, ctx->val_a, ctx->sse, ctx->yuv_lr, ctx->yuv_hr, ctx->crop_buf, ctx->cell_sse};
  for (void* p : ptrs)
    if (p) cudaFree(p);
  for (int k = 0; k < 4; ++k) { cudaFree(ctx->snap[k].wf); cudaFree(ctx->snap[k].wo); cudaFree(ctx->snap[k].bias); }
  for (auto p : ctx->tf) if (p) cudaFree(p);
  for (auto p : ctx->tts) if (p) cudaFree(p);
  for (auto p : ctx->tdf) if (p) cudaFree(p);
  for (auto p : ctx->tdtb) if (p) cudaFree(p);
  for (auto p : ctx->chain_sync) if (p) cudaFree(p);
  if (ctx->publish_ev) cudaEventDestroy(ctx->publish_ev);
  for (auto& pe : ctx->infer_evs) cudaEventDestroy(pe.second);
  if (ctx->comm) nccl().destroy(ctx->comm);
  if (ctx->train_graph) cudaGraphExecDestroy(ctx->train_graph);
  if (ctx->copy_st) cudaStreamDestroy(ctx->copy_st);
  if (ctx->h2d_st) cudaStreamDestroy(ctx->h2d_st);
  for (auto& r : ctx->trec) { cudaEventDestroy(r.a); cudaEventDestroy(r.b); }
  delete ctx;
}

sr_status sr_set_fusion(sr_ctx* ctx, int fuse_blocks) {
  if (!ctx) return SR_E_INVAL;
  ctx->fuse_blocks = (fuse_blocks & 1) != 0;
  ctx->virtual_train = (fuse_blocks & 2) == 0;  // bit 1 set: per-patch (narrow tile) training path
  ctx->roll_tail = (fuse_blocks & 4) == 0;      // bit 2 set: tiled up conv + tail instead of the rolling one
  ctx->fuse_bwd = (fuse_blocks & 8) != 0;       // bit 3 set: fused data-gradient blocks in training
  ctx->tail_tma = (fuse_blocks & 16) == 0;      // bit 4 set: rolling tail reads/writes u8 pixels per lane
  ctx->fuse_bodytail = (fuse_blocks & 32) == 0; // bit 5 set: body conv and up conv + tail as two kernels
  ctx->fuse_head = (fuse_blocks & 64) == 0;     // bit 6 set: k_pack_input + head conv on the bf16 copy
  ctx->pair_blocks = (fuse_blocks & 128) == 0;  // bit 7 set: single-CTA residual blocks instead of CTA pairs
  ctx->split_blocks = (fuse_blocks & 256) != 0; // bit 8 set: inference blocks on conv-split CTA pairs
  ctx->chain = (fuse_blocks & 512) != 0 || env_chain();  // bit 9 set: training conv chains as k_conv_chain
  return SR_OK;
}

sr_status sr_set_sm_split(sr_ctx* ctx, int train_sms) {
  if (!ctx) return SR_E_INVAL;
  set_grid_cap(0);
  const int n = num_sms();
  if (train_sms < 0 || train_sms >= n) return fail(ctx, SR_E_INVAL, "sr_set_sm_split: need 0 <= train_sms < #SMs");
  ctx->sm_total = n;
  ctx->sm_train = train_sms;
  return SR_OK;
}

sr_status sr_kernel_timing(sr_ctx* ctx, int enable) {
  if (!ctx) return SR_E_INVAL;
  ctx->timing = enable != 0;
  ctx->tnext = 0;
  return SR_OK;
}

int sr_kernel_stats(sr_ctx* ctx, char* buf, size_t cap) {
  if (!ctx || !buf || cap == 0) return SR_E_INVAL;
  if (sync_all() != cudaSuccess) return SR_E_CUDA;
  struct Acc { long long n = 0; double ms = 0, flops = 0, bytes = 0; };
  std::vector<std::pair<std::string, Acc>> acc;
  for (size_t i = 0; i < ctx->tnext; ++i) {
    auto& r = ctx->trec[i];
    float ms = 0.f;
    cudaEventElapsedTime(&ms, r.a, r.b);
    auto it = std::find_if(acc.begin(), acc.end(), [&](auto& kv) { return kv.first == r.cls; });
    if (it == acc.end()) { acc.push_back({r.cls, Acc{}}); it = acc.end() - 1; }
    it->second.n++;
    it->second.ms += ms;
    it->second.flops += r.flops;
    it->second.bytes += r.bytes;
  }
  std::string out = "{";
  for (size_t i = 0; i < acc.size(); ++i) {
    char tmp[512];
    snprintf(tmp, sizeof tmp, "%s\"%s\": {\"launches\": %lld, \"ms\": %.6f, \"flops\": %.6e, \"bytes\": %.6e}",
             i ? ", " : "", acc[i].first.c_str(), acc[i].second.n, acc[i].second.ms, acc[i].second.flops,
             acc[i].second.bytes);
    out += tmp;
  }
  out += "}";
  snprintf(buf, cap, "%s", out.c_str());
  return (int)out.size();
}

const char* sr_last_error(const sr_ctx* ctx) { return ctx ? ctx->err.c_str() : "null ctx"; }
size_t sr_num_params(const sr_ctx* ctx) { return ctx ? ctx->nparams : 0; }
uint64_t sr_launch_count(const sr_ctx* ctx) { return ctx ? ctx->launches.load() : 0ull; }
float* sr_grad_buffer(sr_ctx* ctx) { return ctx ? ctx->grad : nullptr; }

// Every call runs on the ctx's device (restored on return), so one process may drive ctxs on several GPUs.
struct DeviceScope {
  int prev = -1;
  explicit DeviceScope(const sr_ctx* ctx) {
    if (ctx && cudaGetDevice(&prev) == cudaSuccess && prev != ctx->device) cudaSetDevice(ctx->device);
    else prev = -1;
  }
  ~DeviceScope() { if (prev >= 0) cudaSetDevice(prev); }
};
#define GUARD()                                                                  \
  if (!ctx) return SR_E_INVAL;                                                   \
  DeviceScope dev_scope_(ctx);                                                   \
  if (ctx->poisoned) return fail(ctx, SR_E_STATE, "ctx poisoned: " + ctx->err)

// SM share of an API entry (restored on return): inference-side calls get sm_total - sm_train SMs, training-side
// calls sm_train, when a split is set.
struct GridCapScope {
  int prev;
  GridCapScope(const sr_ctx* ctx, bool train) : prev(grid_cap()) {
    if (ctx && ctx->sm_train > 0) set_grid_cap(train ? ctx->sm_train : ctx->sm_total - ctx->sm_train);
  }
  ~GridCapScope() { set_grid_cap(prev); }
};
#define CAP_INFER() GridCapScope cap_scope_(ctx, false)
#define CAP_TRAIN() GridCapScope cap_scope_(ctx, true)

sr_status sr_set_params(sr_ctx* ctx, const float* host_in, size_t n) {
  GUARD();
  if (!host_in || n != ctx->nparams) return fail(ctx, SR_E_INVAL, "sr_set_params: size mismatch");
  CK(cudaMemcpy(ctx->params, host_in, n * sizeof(float), cudaMemcpyHostToDevice));
  CK(cudaMemset(ctx->m, 0, n * sizeof(float)));
  CK(cudaMemset(ctx->v, 0, n * sizeof(float)));
  CK(cudaMemset(ctx->grad, 0, n * sizeof(float)));
  CK(cudaMemset(ctx->counters, 0, 3 * sizeof(long long)));
  ctx->t = 0;
  TRY(repack(ctx, SR_TRAIN, true, 0));
  for (int k = 1; k < 4; ++k) {
    CK(cudaMemcpy(ctx->snap[k].wf, ctx->snap[SR_TRAIN].wf, ctx->pk_total * sizeof(bf16), cudaMemcpyDeviceToDevice));
    CK(cudaMemcpy(ctx->snap[k].wo, ctx->snap[SR_TRAIN].wo, ctx->pk_total * sizeof(bf16), cudaMemcpyDeviceToDevice));
    CK(cudaMemcpy(ctx->snap[k].bias, ctx->snap[SR_TRAIN].bias, ctx->b_total * sizeof(float),
                  cudaMemcpyDeviceToDevice));
  }
  CK(sync_all());
  return SR_OK;
}

sr_status sr_get_params(sr_ctx* ctx, sr_model which, float* host_out, size_t n) {
  GUARD();
  if (!host_out || n != ctx->nparams || !valid_model(which)) return fail(ctx, SR_E_INVAL, "sr_get_params: bad args");
  CK(sync_all());
  if (which == SR_TRAIN) {
    CK(cudaMemcpy(host_out, ctx->params, n * sizeof(float), cudaMemcpyDeviceToHost));
    return SR_OK;
  }
  std::vector<bf16> wf(ctx->pk_total);
  std::vector<float> bias(ctx->b_total);
  CK(cudaMemcpy(wf.data(), ctx->snap[which].wf, wf.size() * sizeof(bf16), cudaMemcpyDeviceToHost));
  CK(cudaMemcpy(bias.data(), ctx->snap[which].bias, bias.size() * sizeof(float), cudaMemcpyDeviceToHost));
  for (auto& d : ctx->convs) {
    float* W = host_out + d.w_off;
    for (int co = 0; co < d.cout; ++co)
      for (int ci = 0; ci < d.cin; ++ci)
        for (int t = 0; t < 9; ++t)
          W[(co * d.cin + ci) * 9 + t] =
              __bfloat162float(wf[d.pk_off + ((size_t)(t * d.cinp / 8 + ci / 8) * d.coutp + co) * 8 + ci % 8]);
    for (int co = 0; co < d.cout; ++co) W[(size_t)d.cout * d.cin * 9 + co] = bias[d.b_off + co];
  }
  return SR_OK;
}

// inference of n frames (or a batch of small square images) with snapshot `which` on workspace ws
static sr_status infer_ws(sr_ctx* ctx, InferWS& ws, sr_model which, const uint8_t* lr_dev, int n, int h, int w,
                          uint8_t* hr_dev, cudaStream_t st) {
  if (which == SR_BILINEAR) {
    cudaError_t e = launch_bilinear_u8(lr_dev, n, h, w, ctx->s, hr_dev, st);
    ctx->launches++;
    if (e != cudaSuccess) return fail(ctx, SR_E_CUDA, cudaGetErrorString(e));
    return SR_OK;
  }
  CK(cudaStreamWaitEvent(st, ctx->publish_ev, 0));
  if (use_virtual_infer(ctx, n, h, w) && ctx->virtual_train)
    TRY(forward_infer_virtual(ctx, ws, ctx->snap[which], lr_dev, n, h, hr_dev, st));
  else
    TRY(forward_infer(ctx, ws, ctx->snap[which], lr_dev, n, h, w, hr_dev, 0, h, st));
  return note_infer(ctx, st);
}

sr_status sr_infer(sr_ctx* ctx, sr_model which, const uint8_t* lr_dev, int n, int h, int w, uint8_t* hr_dev,
                   sr_stream stream) {
  GUARD();
  CAP_INFER();
  if (!lr_dev || !hr_dev || n < 1 || h < 1 || w < 1) return fail(ctx, SR_E_INVAL, "sr_infer: bad args");
  cudaStream_t st = (cudaStream_t)stream;
  if (which == SR_BILINEAR) {
    cudaError_t e = launch_bilinear_u8(lr_dev, n, h, w, ctx->s, hr_dev, st);
    ctx->launches++;
    if (e != cudaSuccess) return fail(ctx, SR_E_CUDA, cudaGetErrorString(e));
    return SR_OK;
  }
  if (!valid_model(which)) return fail(ctx, SR_E_INVAL, "sr_infer: bad model");
  return infer_ws(ctx, ctx->iws, which, lr_dev, n, h, w, hr_dev, st);
}

sr_status sr_infer_i420(sr_ctx* ctx, sr_model which, const uint8_t* y_dev, const uint8_t* u_dev,
                        const uint8_t* v_dev, int n, int h, int w, uint8_t* hy_dev, uint8_t* hu_dev, uint8_t* hv_dev,
                        sr_stream stream) {
  GUARD();
  CAP_INFER();
  if (!y_dev || !u_dev || !v_dev || !hy_dev || !hu_dev || !hv_dev || n < 1 || h < 2 || w < 2 || (h | w) & 1)
    return fail(ctx, SR_E_INVAL, "sr_infer_i420: bad args (h, w must be even)");
  cudaStream_t st = (cudaStream_t)stream;
  const int s = ctx->s;
  const size_t lb = (size_t)n * h * w * 3, hb = lb * s * s;
  if (lb > ctx->yuv_lr_bytes) { CK(dalloc(&ctx->yuv_lr, lb)); ctx->yuv_lr_bytes = lb; }
  if (hb > ctx->yuv_hr_bytes) { CK(dalloc(&ctx->yuv_hr, hb)); ctx->yuv_hr_bytes = hb; }
  // Frames on the rolling / fused path (a DNN model, not a small-image batch): the I420 -> RGB conversion runs inside
  // the head conv when it can (W % 32 == 0; it also leaves the RGB copy for the tail) and, at s = 2 / 4, the fused
  // body + tail kernel writes the I420 planes itself; whatever is not fused runs as a separate conversion pass.
  const bool direct = valid_model(which) && which != SR_BILINEAR && !(use_virtual_infer(ctx, n, h, w) && ctx->virtual_train);
  bool yo_done = false;
  if (direct) {
    const bool fused_in = ctx->fuse_head && roll_supported(16, ctx->Cp, w) &&
                          roll_head_yuv_supported(ctx->Cp, w, y_dev, u_dev, v_dev);
    if (!fused_in) {
      launch_i420_to_rgb(y_dev, u_dev, v_dev, n, h, w, ctx->yuv_lr, st);
      ctx->launches++;
      CKL();
    }
    const YuvIn yin{y_dev, u_dev, v_dev};
    const YuvOut yout{hy_dev, hu_dev, hv_dev};
    CK(cudaStreamWaitEvent(st, ctx->publish_ev, 0));
    TRY(forward_infer(ctx, ctx->iws, ctx->snap[which], ctx->yuv_lr, n, h, w, ctx->yuv_hr, 0, h, st,
                      fused_in ? &yin : nullptr, &yout, &yo_done));
    TRY(note_infer(ctx, st));
  } else {
    launch_i420_to_rgb(y_dev, u_dev, v_dev, n, h, w, ctx->yuv_lr, st);
    ctx->launches++;
    CKL();
    TRY(sr_infer(ctx, which, ctx->yuv_lr, n, h, w, ctx->yuv_hr, stream));
  }
  if (!yo_done) {
    launch_rgb_to_i420(ctx->yuv_hr, n, s * h, s * w, hy_dev, hu_dev, hv_dev, st);
    ctx->launches++;
    CKL();
  }
  return SR_OK;
}

static sr_status infer_host_impl(sr_ctx* ctx, sr_model which, const uint8_t* lr_host, int n, int h, int w,
                                 uint8_t* hr_host, sr_stream stream, bool sync) {
  CAP_INFER();
  if (!lr_host || !hr_host || n < 1 || h < 1 || w < 1) return fail(ctx, SR_E_INVAL, "sr_infer_host: bad args");
  const int set = (int)(ctx->host_calls & 1);
  if (ctx->host_busy[set]) {  // the call two back used this staging set: its D2H copies must have drained
    CK(cudaEventSynchronize(ctx->host_done[set]));
    ctx->host_busy[set] = false;
  }
  cudaStream_t st = (cudaStream_t)stream;
  const size_t fl = (size_t)h * w * 3, fh = fl * ctx->s * ctx->s;
  const size_t lb = (size_t)n * fl, hb = (size_t)n * fh;
  if (lb > ctx->stage_lr_bytes[set]) { CK(dalloc(&ctx->stage_lr[set], lb)); ctx->stage_lr_bytes[set] = lb; }
  if (hb > ctx->stage_hr_bytes[set]) { CK(dalloc(&ctx->stage_hr[set], hb)); ctx->stage_hr_bytes[set] = hb; }
  uint8_t* const stage_lr = ctx->stage_lr[set];
  uint8_t* const stage_hr = ctx->stage_hr[set];
  if (!ctx->copy_st) {
    CK(cudaStreamCreateWithFlags(&ctx->copy_st, cudaStreamNonBlocking));
    CK(cudaStreamCreateWithFlags(&ctx->h2d_st, cudaStreamNonBlocking));
    CK(cudaEventCreateWithFlags(&ctx->host_done[0], cudaEventDisableTiming));
    CK(cudaEventCreateWithFlags(&ctx->host_done[1], cudaEventDisableTiming));
    CK(cudaEventCreateWithFlags(&ctx->set_read[0], cudaEventDisableTiming));
    CK(cudaEventCreateWithFlags(&ctx->set_read[1], cudaEventDisableTiming));
  }
  // Chunked pipeline: all H2D copies go first on their own stream (per-chunk events), chunk k is super-resolved
  // on `stream` as soon as its frames landed, and its D2H runs on a third stream while chunk k+1 computes.
  // PCIe (55 GB/s measured) then hides behind the tensor work; only the last chunk's D2H is exposed.
  // Chunk sizes: ~240 MB of HR output per chunk (fewer, larger inference launches; with two calls in flight the
  // other call's work hides the longer exposed copies), except a one-frame first chunk (compute starts after one
  // frame's H2D) and a one-frame last chunk (only one frame's D2H is left exposed after the last kernel).
  const int F = std::max(1, std::min(n, (int)std::max<size_t>(1, (size_t)(240u << 20) / std::max<size_t>(fh, 1))));
  std::vector<int> c0s;  // first frame of each chunk (+ n at the end)
  if (!sync && n >= 2) {
    // two calls in flight: this call's H2D overlaps the previous call's compute and its D2H the next call's, so
    // the batch goes as two chunks (fewer, larger inference launches)
    c0s = {0, (n + 1) / 2, n};
  } else {
    int f = 0;
    c0s.push_back(0);
    if (n >= 3 && F > 1) { f = 1; c0s.push_back(f); }
    while (f < n) {
      const int left = n - f;
      int take = std::min(F, left);
      if (F > 1 && left > 1 && take == left) take = left - 1;  // keep the final frame as its own chunk
      f += take;
      c0s.push_back(f);
    }
  }
  const int nch = (int)c0s.size() - 1;
  (void)F;
  while ((int)ctx->chunk_ev[set].size() < 2 * nch + 1) {
    cudaEvent_t e;
    CK(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
    ctx->chunk_ev[set].push_back(e);
  }
  cudaEvent_t* ev = ctx->chunk_ev[set].data();  // [0] start, [1 + c] chunk c landed, [1 + nch + c] chunk c done
  // the H2D into this staging set waits only for the inference that last read it (two calls back), not for all
  // earlier work on `stream`: it overlaps the previous call's compute
  if (ctx->set_used[set]) CK(cudaStreamWaitEvent(ctx->h2d_st, ctx->set_read[set], 0));
  for (int c = 0; c < nch; ++c) {
    const int f0 = c0s[c], fn = c0s[c + 1] - c0s[c];
    CK(cudaMemcpyAsync(stage_lr + f0 * fl, lr_host + f0 * fl, fn * fl, cudaMemcpyHostToDevice, ctx->h2d_st));
    CK(cudaEventRecord(ev[1 + c], ctx->h2d_st));
  }
  for (int c = 0; c < nch; ++c) {
    const int f0 = c0s[c], fn = c0s[c + 1] - c0s[c];
    CK(cudaStreamWaitEvent(st, ev[1 + c], 0));
    TRY(sr_infer(ctx, which, stage_lr + f0 * fl, fn, h, w, stage_hr + f0 * fh, stream));
    CK(cudaEventRecord(ev[1 + nch + c], st));
    if (c == nch - 1) {
      CK(cudaEventRecord(ctx->set_read[set], st));
      ctx->set_used[set] = true;
    }
    CK(cudaStreamWaitEvent(ctx->copy_st, ev[1 + nch + c], 0));
    CK(cudaMemcpyAsync(hr_host + f0 * fh, stage_hr + f0 * fh, fn * fh, cudaMemcpyDeviceToHost, ctx->copy_st));
  }
  CK(cudaEventRecord(ctx->host_done[set], ctx->copy_st));
  ctx->host_calls++;
  if (sync) {
    CK(cudaEventSynchronize(ctx->host_done[set]));
  } else {
    ctx->host_busy[set] = true;
  }
  return SR_OK;
}

sr_status sr_infer_host(sr_ctx* ctx, sr_model which, const uint8_t* lr_host, int n, int h, int w,
                        uint8_t* hr_host, sr_stream stream) {
  GUARD();
  return infer_host_impl(ctx, which, lr_host, n, h, w, hr_host, stream, true);
}

sr_status sr_infer_host_async(sr_ctx* ctx, sr_model which, const uint8_t* lr_host, int n, int h, int w,
                              uint8_t* hr_host, sr_stream stream) {
  GUARD();
  return infer_host_impl(ctx, which, lr_host, n, h, w, hr_host, stream, false);
}

sr_status sr_infer_host_wait(sr_ctx* ctx) {
  GUARD();
  for (int k = 0; k < 2; ++k)
    if (ctx->host_busy[k]) {
      CK(cudaEventSynchronize(ctx->host_done[k]));
      ctx->host_busy[k] = false;
    }
  return SR_OK;
}

sr_status sr_infer_rows(sr_ctx* ctx, sr_model which, const uint8_t* lr_full_dev, int h, int w, int row0, int row1,
                        uint8_t* hr_full_dev, sr_stream stream) {
  GUARD();
  CAP_INFER();
  if (!lr_full_dev || !hr_full_dev || h < 1 || w < 1 || row0 < 0 || row1 > h || row0 >= row1)
    return fail(ctx, SR_E_INVAL, "sr_infer_rows: bad args");
  if (!valid_model(which)) return fail(ctx, SR_E_INVAL, "sr_infer_rows: bad model");
  cudaStream_t st = (cudaStream_t)stream;
  const int halo = 2 * ctx->B + 4;  // receptive field of the 2B+3 convs (+1 margin)
  const int lo = std::max(0, row0 - halo), hi = std::min(h, row1 + halo);
  const int s = ctx->s;
  CK(cudaStreamWaitEvent(st, ctx->publish_ev, 0));
  TRY(forward_infer(ctx, ctx->iws, ctx->snap[which], lr_full_dev + (size_t)lo * w * 3, 1, hi - lo, w,
                    hr_full_dev + (size_t)lo * s * (size_t)s * w * 3, row0 - lo, row1 - lo, st));
  return note_infer(ctx, st);
}

sr_status sr_train_grad(sr_ctx* ctx, const uint8_t* lr_dev, const uint8_t* hr_dev, int n, int p, float* loss_dev,
                        sr_stream stream) {
  GUARD();
  CAP_TRAIN();
  if (!lr_dev || !hr_dev || n < 1 || p < 1) return fail(ctx, SR_E_INVAL, "sr_train_grad: bad args");
  return train_grad(ctx, lr_dev, hr_dev, n, p, loss_dev, (cudaStream_t)stream);
}

sr_status sr_train_apply(sr_ctx* ctx, float grad_scale, sr_stream stream) {
  GUARD();
  CAP_TRAIN();
  return train_apply(ctx, grad_scale, nullptr, (cudaStream_t)stream);
}

sr_status sr_train_apply_dev(sr_ctx* ctx, const float* grad_scale_dev, sr_stream stream) {
  GUARD();
  CAP_TRAIN();
  if (!grad_scale_dev) return fail(ctx, SR_E_INVAL, "sr_train_apply_dev: null scale");
  return train_apply(ctx, 1.0f, grad_scale_dev, (cudaStream_t)stream);
}

sr_status sr_train_step(sr_ctx* ctx, const uint8_t* lr_dev, const uint8_t* hr_dev, int n, int p, float* loss_dev,
                        sr_stream stream) {
  GUARD();
  CAP_TRAIN();
  if (ctx->opt.world > 1 && !ctx->comm)
    return fail(ctx, SR_E_STATE, "sr_train_step: world > 1 needs sr_options.nccl_id (or sr_train_grad + your "
                                 "allreduce + sr_train_apply)");
  TRY(sr_train_grad(ctx, lr_dev, hr_dev, n, p, loss_dev, stream));
  TRY(grad_exchange(ctx, (cudaStream_t)stream));  // T5: sum_r w_r g_r over the DP group (no-op at world 1)
  return train_apply(ctx, (float)(1.0 / ctx->sum_w), nullptr, (cudaStream_t)stream);
}

sr_status sr_train_allreduce(sr_ctx* ctx, sr_stream stream) {
  GUARD();
  return grad_exchange(ctx, (cudaStream_t)stream);
}

double sr_dp_weight_sum(const sr_ctx* ctx) { return ctx ? ctx->sum_w : 0.0; }

sr_status sr_pool_push(sr_ctx* ctx, const uint8_t* lr_dev, const uint8_t* hr_dev, int n, int pp,
                       const int64_t* arrival_ts, sr_stream stream) {
  (void)arrival_ts;
  GUARD();
  CAP_TRAIN();
  if (!lr_dev || !hr_dev || n < 1 || pp < 1) return fail(ctx, SR_E_INVAL, "sr_pool_push: bad args");
  cudaStream_t st = (cudaStream_t)stream;
  const int s = ctx->s;
  if (!ctx->pool_lr) {
    ctx->pool_pp = pp;
    ctx->pool_cap = ctx->opt.pool_capacity;
    CK(dalloc(&ctx->pool_lr, (size_t)ctx->pool_cap * pp * pp * 3));
    CK(dalloc(&ctx->pool_hr, (size_t)ctx->pool_cap * s * s * pp * pp * 3));
  } else if (pp != ctx->pool_pp) {
    return fail(ctx, SR_E_INVAL, "sr_pool_push: patch size differs from the first push");
  }
  const size_t lb = (size_t)pp * pp * 3, hb = lb * s * s;
  for (int i = 0; i < n;) {  // arrival order into the ring: at most two contiguous runs per call (wrap)
    const long long slot = (ctx->pool_total + i) % ctx->pool_cap;
    const int run = (int)std::min<long long>(n - i, ctx->pool_cap - slot);
    CK(cudaMemcpyAsync(ctx->pool_lr + slot * lb, lr_dev + i * lb, run * lb, cudaMemcpyDeviceToDevice, st));
    CK(cudaMemcpyAsync(ctx->pool_hr + slot * hb, hr_dev + i * hb, run * hb, cudaMemcpyDeviceToDevice, st));
    i += run;
  }
  ctx->pool_total += n;
  launch_counter_add(ctx->counters + 3, n, st);  // the device-side arrival count the sampler reads (graph replays)
  ctx->launches++;
  CKL();
  return SR_OK;
}

sr_status sr_pool_push_i420(sr_ctx* ctx, const uint8_t* y_dev, const uint8_t* u_dev, const uint8_t* v_dev, int h,
                            int w, const uint8_t* hr_dev, const int32_t* xy_dev, int n, int pp,
                            const int64_t* arrival_ts, sr_stream stream) {
  GUARD();
  CAP_TRAIN();
  if (!y_dev || !u_dev || !v_dev || !hr_dev || !xy_dev || n < 1 || pp < 1 || h < 2 || w < 2 || (h | w) & 1 ||
      pp > h || pp > w)
    return fail(ctx, SR_E_INVAL, "sr_pool_push_i420: bad args (even h, w >= pp)");
  cudaStream_t st = (cudaStream_t)stream;
  const size_t need = (size_t)n * pp * pp * 3;
  if (need > ctx->crop_bytes) { CK(dalloc(&ctx->crop_buf, need)); ctx->crop_bytes = need; }
  launch_i420_crop(y_dev, u_dev, v_dev, h, w, xy_dev, n, pp, ctx->crop_buf,
                   reinterpret_cast<unsigned long long*>(ctx->counters + 4), st);
  ctx->launches++;
  CKL();
  return sr_pool_push(ctx, ctx->crop_buf, hr_dev, n, pp, arrival_ts, stream);
}

size_t sr_pool_size(const sr_ctx* ctx) {
  if (!ctx) return 0;
  return (size_t)std::min(ctx->pool_total, ctx->pool_cap);
}

sr_status sr_pool_stats(sr_ctx* ctx, int64_t* arrivals, int64_t* clamped) {
  GUARD();
  long long h[2] = {0, 0};
  CK(sync_all());
  CK(cudaMemcpy(h, ctx->counters + 3, sizeof h, cudaMemcpyDeviceToHost));
  if (arrivals) *arrivals = h[0];
  if (clamped) *clamped = h[1];
  return SR_OK;
}

sr_status sr_sample_batch(sr_ctx* ctx, int64_t step, int batch, int p, uint8_t* lr_out_dev, uint8_t* hr_out_dev,
                          int32_t* idx_out_dev, sr_stream stream) {
  GUARD();
  CAP_TRAIN();
  if (!lr_out_dev || !hr_out_dev || batch < 1 || p < 1) return fail(ctx, SR_E_INVAL, "sr_sample_batch: bad args");
  if (ctx->pool_total == 0) return fail(ctx, SR_E_STATE, "sr_sample_batch: empty pool");
  if (p > ctx->pool_pp) return fail(ctx, SR_E_INVAL, "sr_sample_batch: p larger than pool patch");
  const long long avail = std::min(ctx->pool_total, ctx->pool_cap);
  const int G = ctx->opt.world, r = ctx->opt.rank;
  const long long lo = avail * r / G, hi = avail * (r + 1) / G;
  if (hi <= lo) return fail(ctx, SR_E_STATE, "sr_sample_batch: empty rank view");
  SampleArgs a{};
  a.seed = ctx->opt.seed;
  a.step = step;
  a.step_dev = ctx->counters;
  a.world = G;
  a.rank = r;
  a.n_view = hi - lo;
  a.view_base = ctx->pool_total - avail + lo;
  a.pool_total_dev = ctx->counters + 3;  // the same view, derived on the device (stays current in graph replays)
  a.capacity = ctx->pool_cap;
  a.recent_k = ctx->opt.recent_k;
  a.recent_w = ctx->opt.recent_w;
  a.p = p;
  a.pp = ctx->pool_pp;
  a.scale = ctx->s;
  a.lr_pool = ctx->pool_lr;
  a.hr_pool = ctx->pool_hr;
  a.lr_out = lr_out_dev;
  a.hr_out = hr_out_dev;
  a.idx_out = idx_out_dev;
  if (step < 0) {  // graph mode: the gather's last block advances the device-side sampler step
    a.step_bump = ctx->counters;
    a.done = reinterpret_cast<unsigned*>(ctx->counters + 2);
  }
  launch_sample_gather(a, batch, (cudaStream_t)stream);
  ctx->launches++;
  CKL();
  return SR_OK;
}

sr_status sr_train_sampled(sr_ctx* ctx, int iters, int batch, int p, float* loss_dev, sr_stream stream) {
  GUARD();
  CAP_TRAIN();
  if (iters < 1 || batch < 1 || p < 1) return fail(ctx, SR_E_INVAL, "sr_train_sampled: bad args");
  if (ctx->opt.world > 1 && !ctx->comm)
    return fail(ctx, SR_E_STATE, "sr_train_sampled: world > 1 needs sr_options.nccl_id (the ctx's communicator)");
  cudaStream_t st = (cudaStream_t)stream;
  const size_t lb = (size_t)batch * p * p * 3, hb = lb * ctx->s * ctx->s;
  // one iteration: sample + gather from the device-side pool view and step counter (T1), forward / loss / backward
  // (T2-T4), sum-allreduce of w_r g_r over the DP group (T5, world > 1), Adam with 1 / sum_r w_r (T6)
  auto one_iter = [&]() -> sr_status {
    TRY(sr_sample_batch(ctx, -1, batch, p, ctx->batch_lr, ctx->batch_hr, nullptr, stream));  // device step counter
    TRY(train_grad(ctx, ctx->batch_lr, ctx->batch_hr, batch, p, loss_dev, st));
    TRY(grad_exchange(ctx, st));
    return train_apply(ctx, (float)(1.0 / ctx->sum_w), nullptr, st);
  };
  // the captured graph bakes in the loss pointer and every workspace address: re-capture when any of them changed
  const bool stale = !ctx->train_graph || ctx->graph_batch != batch || ctx->graph_p != p ||
                     ctx->graph_loss != loss_dev || ctx->graph_gen != ctx->ws_gen || ctx->graph_sm != ctx->sm_train;
  if (stale || st == nullptr) {
    if (lb > ctx->batch_bytes_lr) { CK(dalloc(&ctx->batch_lr, lb)); ctx->batch_bytes_lr = lb; ctx->ws_gen++; }
    if (hb > ctx->batch_bytes_hr) { CK(dalloc(&ctx->batch_hr, hb)); ctx->batch_bytes_hr = hb; ctx->ws_gen++; }
    TRY(one_iter());  // eager iteration: grows the workspaces, configures the kernels
    --iters;
    if (st != nullptr) {  // capture one iteration (the legacy default stream cannot be captured)
      if (ctx->train_graph) { cudaGraphExecDestroy(ctx->train_graph); ctx->train_graph = nullptr; }
      const bool timing = ctx->timing;
      ctx->timing = false;
      cudaGraph_t g = nullptr;
      const unsigned long long l0 = ctx->launches;
      CK(cudaStreamBeginCapture(st, cudaStreamCaptureModeThreadLocal));
      sr_status cs = one_iter();
      cudaError_t ce = cudaStreamEndCapture(st, &g);
      ctx->graph_kernels = ctx->launches - l0;  // captured, not run: counted per replay below
      ctx->launches = l0;
      ctx->timing = timing;
      TRY(cs);
      CK(ce);
      CK(cudaGraphInstantiate(&ctx->train_graph, g, 0));
      cudaGraphDestroy(g);
      ctx->graph_batch = batch;
      ctx->graph_p = p;
      ctx->graph_loss = loss_dev;
      ctx->graph_gen = ctx->ws_gen;
      ctx->graph_sm = ctx->sm_train;
    }
  }
  for (int it = 0; it < iters; ++it) {
    if (ctx->train_graph && st != nullptr) {
      CK(cudaGraphLaunch(ctx->train_graph, st));
      ctx->launches += ctx->graph_kernels;
    } else {
      TRY(one_iter());
    }
  }
  return SR_OK;
}

sr_status sr_publish(sr_ctx* ctx, sr_stream stream) {
  GUARD();
  CAP_TRAIN();
  cudaStream_t st = (cudaStream_t)stream;
  // inference reading SERVE / PREV may be in flight on other streams: the snapshot copies wait for it (a frame is
  // never computed with a mix of old and new layer weights; the paper syncs inference at the epoch end, L1252-1253)
  {
    std::lock_guard<std::mutex> lk(ctx->ev_mu);
    for (auto& pe : ctx->infer_evs)
      if (pe.first != st) CK(cudaStreamWaitEvent(st, pe.second, 0));
  }
  TRY(ensure_full_train_pack(ctx, st));
  CK(cudaMemcpyAsync(ctx->snap[SR_PREV].wf, ctx->snap[SR_SERVE].wf, ctx->pk_total * sizeof(bf16),
                     cudaMemcpyDeviceToDevice, st));
  CK(cudaMemcpyAsync(ctx->snap[SR_PREV].bias, ctx->snap[SR_SERVE].bias, ctx->b_total * sizeof(float),
                     cudaMemcpyDeviceToDevice, st));
  CK(cudaMemcpyAsync(ctx->snap[SR_PREV].wo, ctx->snap[SR_SERVE].wo, ctx->pk_total * sizeof(bf16),
                     cudaMemcpyDeviceToDevice, st));
  CK(cudaMemcpyAsync(ctx->snap[SR_SERVE].wo, ctx->snap[SR_TRAIN].wo, ctx->pk_total * sizeof(bf16),
                     cudaMemcpyDeviceToDevice, st));
  CK(cudaMemcpyAsync(ctx->snap[SR_SERVE].wf, ctx->snap[SR_TRAIN].wf, ctx->pk_total * sizeof(bf16),
                     cudaMemcpyDeviceToDevice, st));
  CK(cudaMemcpyAsync(ctx->snap[SR_SERVE].bias, ctx->snap[SR_TRAIN].bias, ctx->b_total * sizeof(float),
                     cudaMemcpyDeviceToDevice, st));
  CK(cudaEventRecord(ctx->publish_ev, st));
  return SR_OK;
}

sr_status sr_sse_u8(const uint8_t* a_dev, const uint8_t* b_dev, int n, int64_t elems, uint64_t* out_dev,
                    sr_stream stream) {
  if (!a_dev || !b_dev || !out_dev || n < 1 || elems < 1) return SR_E_INVAL;
  launch_sse_u8(a_dev, b_dev, n, elems, reinterpret_cast<unsigned long long*>(out_dev), (cudaStream_t)stream);
  return cudaGetLastError() == cudaSuccess ? SR_OK : SR_E_CUDA;
}

// Mean per-patch PSNR of k models on the same validation patches (one sync).  Per patch: integer SSE (K9) ->
// 10 log10(255^2 count / SSE), capped at 100 dB for SSE = 0.
static sr_status mean_psnr(sr_ctx* ctx, const sr_model* models, int k, const uint8_t* lr_dev, const uint8_t* hr_dev,
                           int n, int p, double* out, cudaStream_t st) {
  const int s = ctx->s;
  const size_t per = (size_t)s * p * s * p * 3, tot = per * n;
  if (tot > ctx->val_bytes) {
    CK(dalloc(&ctx->val_a, tot));
    ctx->val_bytes = tot;
  }
  if ((size_t)k * n > (size_t)ctx->sse_n) { CK(dalloc(&ctx->sse, (size_t)k * n)); ctx->sse_n = k * n; }
  for (int m = 0; m < k; ++m) {
    // sse of model m is launched on st right after its inference, so val_a can be reused (stream order)
    if (!(valid_model(models[m]) || models[m] == SR_BILINEAR)) return fail(ctx, SR_E_INVAL, "bad model");
    TRY(infer_ws(ctx, ctx->qws, models[m], lr_dev, n, p, p, ctx->val_a, st));  // own workspace (training side)
    launch_sse_u8(ctx->val_a, hr_dev, n, (int64_t)per, ctx->sse + (size_t)m * n, st);
    ctx->launches++;
    CKL();
  }
  std::vector<unsigned long long> h((size_t)k * n);
  CK(cudaMemcpyAsync(h.data(), ctx->sse, h.size() * sizeof(unsigned long long), cudaMemcpyDeviceToHost, st));
  CK(cudaStreamSynchronize(st));
  for (int m = 0; m < k; ++m) {
    double acc = 0;
    for (int i = 0; i < n; ++i) {
      const unsigned long long e = h[(size_t)m * n + i];
      acc += e == 0 ? 100.0 : 10.0 * std::log10(255.0 * 255.0 * (double)per / (double)e);
    }
    out[m] = acc / n;
  }
  return SR_OK;
}

sr_status sr_psnr_gain(sr_ctx* ctx, sr_model a, sr_model b, const uint8_t* lr_dev, const uint8_t* hr_dev, int n,
                       int p, sr_quality* out_host, sr_stream stream) {
  GUARD();
  CAP_INFER();
  if (!lr_dev || !hr_dev || !out_host || n < 1 || p < 1) return fail(ctx, SR_E_INVAL, "sr_psnr_gain: bad args");
  const sr_model ms[2] = {a, b};
  double q[2];
  TRY(mean_psnr(ctx, ms, 2, lr_dev, hr_dev, n, p, q, (cudaStream_t)stream));
  out_host->psnr_a = q[0];
  out_host->psnr_b = q[1];
  out_host->gain = q[0] - q[1];
  return SR_OK;
}

// ---- client-side patch selection (§5.2; reading R22)
sr_status sr_patch_select(sr_ctx* ctx, const uint8_t* raw_dev, const uint8_t* dec_dev, int h, int w, int cell,
                          int max_sel, uint64_t seed, int64_t step, int32_t* xy_host, int* n_sel, sr_stream stream) {
  GUARD();
  CAP_INFER();
  if (!raw_dev || !dec_dev || !xy_host || !n_sel || h < 1 || w < 1 || cell < 1 || max_sel < 0)
    return fail(ctx, SR_E_INVAL, "sr_patch_select: bad args");
  cudaStream_t st = (cudaStream_t)stream;
  const int nx = (w + cell - 1) / cell, ny = (h + cell - 1) / cell;
  if (nx * ny > ctx->cell_n) { CK(dalloc(&ctx->cell_sse, (size_t)nx * ny)); ctx->cell_n = nx * ny; }
  launch_cell_sse(raw_dev, dec_dev, h, w, cell, ctx->cell_sse, st);
  ctx->launches++;
  CKL();
  std::vector<unsigned long long> sse((size_t)nx * ny);
  CK(cudaMemcpyAsync(sse.data(), ctx->cell_sse, sse.size() * 8, cudaMemcpyDeviceToHost, st));
  CK(cudaStreamSynchronize(st));
  unsigned long long s_frame = 0;
  for (auto v : sse) s_frame += v;
  const unsigned long long n_frame = (unsigned long long)h * w * 3;
  const int gx = w / cell, gy = h / cell, n = gx * gy;  // whole cells are the candidates
  std::vector<int> perm(n);
  for (int k = 0; k < n; ++k) perm[k] = k;
  for (int k = 0; k < n; ++k) {  // Fisher-Yates on the counter-based SplitMix64 stream
    const uint64_t u = mix64h(seed + 0x9E3779B97F4A7C15ull * (((uint64_t)step << 32) + k + 1));
    const int j = k + (int)(((unsigned __int128)u * (uint64_t)(n - k)) >> 64);
    std::swap(perm[k], perm[j]);
  }
  int cnt = 0;
  const unsigned long long n_cell = (unsigned long long)cell * cell * 3;
  for (int i = 0; i < n && cnt < max_sel; ++i) {
    const int cy = perm[i] / gx, cx = perm[i] % gx;
    // PSNR(cell) < PSNR(frame)  <=>  SSE_cell * n_frame > SSE_frame * n_cell  (exact, 128-bit)
    if ((unsigned __int128)sse[(size_t)cy * nx + cx] * n_frame > (unsigned __int128)s_frame * n_cell) {
      xy_host[2 * cnt] = cx * cell;
      xy_host[2 * cnt + 1] = cy * cell;
      ++cnt;
    }
  }
  *n_sel = cnt;
  return SR_OK;
}

// ---- Algorithm 1 (App. A), written in the paper's line order
sr_status sr_controller_init(sr_controller* c, double thresh_sat, int count_sat, double thresh_online,
                             int count_online) {
  if (!c || count_sat < 0 || count_online < 0) return SR_E_INVAL;
  c->thresh_sat = thresh_sat;
  c->count_sat = count_sat;
  c->thresh_online = thresh_online;
  c->count_online = count_online;
  c->state = SR_TRAINING;  // line 1
  c->patience = 0;
  return SR_OK;
}

sr_status sr_controller_update(sr_controller* c, double diff, int* event_out) {
  if (!c || (c->state != SR_TRAINING && c->state != SR_SUSPENDED)) return SR_E_INVAL;
  int ev = SR_EV_NONE;
  if (c->state == SR_TRAINING) {       // lines 4-14: one training epoch
    if (diff < c->thresh_sat) {        // line 7
      c->patience += 1;                // line 8
      if (c->patience > c->count_sat) {  // line 9
        ev = SR_EV_SUSPEND;            // line 10
        c->state = SR_SUSPENDED;       // line 11
        c->patience = 0;               // line 12
      }
    } else {
      c->patience = 0;                 // line 14
    }
  } else {                             // lines 15-25: one validation period
    if (diff < c->thresh_online) {     // line 18
      c->patience += 1;                // line 19
      if (c->patience > c->count_online) {  // line 20
        ev = SR_EV_RESUME;             // line 21
        c->state = SR_TRAINING;        // line 22
        c->patience = 0;               // line 23
      }
    } else {
      c->patience = 0;                 // line 25
    }
  }
  if (event_out) *event_out = ev;
  return SR_OK;
}

sr_status sr_controller_step(sr_ctx* ctx, sr_controller* c, const uint8_t* lr_dev, const uint8_t* hr_dev, int n,
                             int p, sr_epoch_report* out_host, sr_stream stream) {
  GUARD();
  CAP_INFER();
  if (!c || !lr_dev || !hr_dev || !out_host || n < 1 || p < 1)
    return fail(ctx, SR_E_INVAL, "sr_controller_step: bad args");
  if (c->state != SR_TRAINING && c->state != SR_SUSPENDED)
    return fail(ctx, SR_E_INVAL, "sr_controller_step: controller not initialised");
  const sr_model ms[4] = {SR_SERVE, SR_PREV, SR_INIT, SR_BILINEAR};
  double q[4];
  TRY(mean_psnr(ctx, ms, 4, lr_dev, hr_dev, n, p, q, (cudaStream_t)stream));
  sr_epoch_report r{};
  r.psnr_serve = q[0];
  r.psnr_prev = q[1];
  r.psnr_init = q[2];
  r.psnr_bilinear = q[3];
  r.q_dnn = q[0] - q[3];
  r.q_dnn_prev = q[1] - q[3];
  r.state_before = c->state;
  r.diff = c->state == SR_TRAINING ? q[0] - q[1] : q[0] - q[2];  // line 6 / line 17
  int ev = SR_EV_NONE;
  sr_status st = sr_controller_update(c, r.diff, &ev);
  if (st != SR_OK) return fail(ctx, st, "sr_controller_step: update failed");
  r.event = ev;
  r.state_after = c->state;
  *out_host = r;
  return SR_OK;
}

// ---- disjoint SM partitions for concurrent inference + training (green contexts; §7: the server runs
// inference and online training side by side)
}  // extern "C"
namespace {
struct GreenApi {
  bool ok = false;
  CUresult (*dev_get)(CUdevice*, int) = nullptr;
  CUresult (*get_res)(CUdevice, CUdevResource*, CUdevResourceType) = nullptr;
  CUresult (*split)(CUdevResource*, unsigned*, const CUdevResource*, CUdevResource*, unsigned, unsigned) = nullptr;
  CUresult (*gen_desc)(CUdevResourceDesc*, CUdevResource*, unsigned) = nullptr;
  CUresult (*create)(CUgreenCtx*, CUdevResourceDesc, CUdevice, unsigned) = nullptr;
  CUresult (*to_ctx)(CUcontext*, CUgreenCtx) = nullptr;
  CUresult (*stream)(CUstream*, CUgreenCtx, unsigned, int) = nullptr;
  CUresult (*destroy)(CUgreenCtx) = nullptr;
};
template <class F>
static bool entry(const char* name, F* fn) {
  void* p = nullptr;
  cudaDriverEntryPointQueryResult q;
  if (cudaGetDriverEntryPoint(name, &p, cudaEnableDefault, &q) != cudaSuccess || !p) return false;
  *fn = reinterpret_cast<F>(p);
  return true;
}
GreenApi& green() {
  static GreenApi g;
  static bool tried = false;
  if (!tried) {
    tried = true;
    g.ok = entry("cuDeviceGet", &g.dev_get) && entry("cuDeviceGetDevResource", &g.get_res) &&
           entry("cuDevSmResourceSplitByCount", &g.split) && entry("cuDevResourceGenerateDesc", &g.gen_desc) &&
           entry("cuGreenCtxCreate", &g.create) && entry("cuCtxFromGreenCtx", &g.to_ctx) &&
           entry("cuGreenCtxStreamCreate", &g.stream) && entry("cuGreenCtxDestroy", &g.destroy);
  }
  return g;
}
std::vector<CUgreenCtx> g_green;  // green contexts created by sr_sm_partition (destroyed by sr_sm_partition_release)
std::mutex g_green_mu;
}  // namespace
extern "C" {

sr_status sr_sm_partition(int train_sms, sr_stream* infer_stream, sr_stream* train_stream, int* infer_sms,
                          int* train_sms_out) {
  if (!infer_stream || !train_stream || train_sms < 1) return SR_E_INVAL;
  GreenApi& g = green();
  if (!g.ok) return SR_E_UNSUPPORTED;
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess || cudaFree(nullptr) != cudaSuccess) return SR_E_CUDA;  // primary ctx up
  CUdevice cd;
  CUdevResource all{}, grp[1]{}, rest{};
  unsigned nb = 1;
  if (g.dev_get(&cd, dev) != CUDA_SUCCESS || g.get_res(cd, &all, CU_DEV_RESOURCE_TYPE_SM) != CUDA_SUCCESS)
    return SR_E_CUDA;
  if (train_sms >= (int)all.sm.smCount) return SR_E_INVAL;
  if (g.split(grp, &nb, &all, &rest, 0, (unsigned)train_sms) != CUDA_SUCCESS || nb != 1 || rest.sm.smCount == 0)
    return SR_E_INVAL;  // (sm_90+: partitions are multiples of 8 SMs, >= 8)
  CUdevResourceDesc dt, di;
  CUgreenCtx gt, gi;
  CUcontext ct, ci;
  CUstream st_t, st_i;
  int lo = 0, hi = 0;
  cudaDeviceGetStreamPriorityRange(&lo, &hi);
  if (g.gen_desc(&dt, grp, 1) != CUDA_SUCCESS || g.gen_desc(&di, &rest, 1) != CUDA_SUCCESS) return SR_E_CUDA;
  if (g.create(&gt, dt, cd, CU_GREEN_CTX_DEFAULT_STREAM) != CUDA_SUCCESS) return SR_E_CUDA;
  if (g.create(&gi, di, cd, CU_GREEN_CTX_DEFAULT_STREAM) != CUDA_SUCCESS) { g.destroy(gt); return SR_E_CUDA; }
  if (g.to_ctx(&ct, gt) != CUDA_SUCCESS || g.to_ctx(&ci, gi) != CUDA_SUCCESS ||
      g.stream(&st_t, gt, CU_STREAM_NON_BLOCKING, lo) != CUDA_SUCCESS ||
      g.stream(&st_i, gi, CU_STREAM_NON_BLOCKING, hi) != CUDA_SUCCESS) {
    g.destroy(gt);
    g.destroy(gi);
    return SR_E_CUDA;
  }
  {
    std::lock_guard<std::mutex> lk(g_green_mu);
    g_green.push_back(gt);
    g_green.push_back(gi);
  }
  {
    std::lock_guard<std::mutex> lk(g_part_mu);
    g_part_streams.push_back(reinterpret_cast<cudaStream_t>(st_t));
    g_part_streams.push_back(reinterpret_cast<cudaStream_t>(st_i));
  }
  *train_stream = reinterpret_cast<sr_stream>(st_t);
  *infer_stream = reinterpret_cast<sr_stream>(st_i);
  if (train_sms_out) *train_sms_out = (int)grp[0].sm.smCount;
  if (infer_sms) *infer_sms = (int)rest.sm.smCount;
  return SR_OK;
}

sr_status sr_sm_partition_release(void) {
  sync_all();
  {
    std::lock_guard<std::mutex> lk(g_part_mu);
    g_part_streams.clear();
  }
  std::lock_guard<std::mutex> lk(g_green_mu);
  GreenApi& g = green();
  for (CUgreenCtx c : g_green) g.destroy(c);
  g_green.clear();
  return SR_OK;
}

sr_status sr_get_adam_state(sr_ctx* ctx, float* m_host, float* v_host, size_t n, int64_t* t_host) {
  GUARD();
  if (n != ctx->nparams) return fail(ctx, SR_E_INVAL, "sr_get_adam_state: size mismatch");
  CK(sync_all());
  if (m_host) CK(cudaMemcpy(m_host, ctx->m, n * sizeof(float), cudaMemcpyDeviceToHost));
  if (v_host) CK(cudaMemcpy(v_host, ctx->v, n * sizeof(float), cudaMemcpyDeviceToHost));
  if (t_host) {
    long long t = 0;
    CK(cudaMemcpy(&t, ctx->counters + 1, sizeof t, cudaMemcpyDeviceToHost));
    *t_host = t;
  }
  return SR_OK;
}

sr_status sr_nccl_unique_id(void* id_out, size_t cap) {
  if (!id_out || cap < sizeof(ncclUniqueId)) return SR_E_INVAL;
  NcclApi& a = nccl();
  if (!a.ok) {
    fprintf(stderr, "sr_nccl_unique_id: %s\n", a.why.c_str());
    return SR_E_NCCL;
  }
  ncclUniqueId id;
  if (a.get_id(&id) != ncclSuccess) return SR_E_NCCL;
  memcpy(id_out, &id, sizeof id);
  return SR_OK;
}

// ---- test-only exports
sr_status sr_test_pack_input(const uint8_t* lr_dev, int n, int h, int w, void* x_dev, sr_stream stream) {
  if (!lr_dev || !x_dev) return SR_E_INVAL;
  launch_pack_input(lr_dev, (size_t)n * h * w, (bf16*)x_dev, (cudaStream_t)stream);
  return cudaGetLastError() == cudaSuccess ? SR_OK : SR_E_CUDA;
}

sr_status sr_test_conv(const void* x_dev, int n, int h, int w, int cin, int cout, const float* w_host,
                       const float* b_host, const void* res_dev, const void* mask_dev, int relu, int dgrad,
                       void* out_dev, sr_stream stream) {
  if (!x_dev || !w_host || !out_dev) return SR_E_INVAL;
  cudaStream_t st = (cudaStream_t)stream;
  const int cinp = rup16(cin), coutp = rup16(cout);
  ConvDesc d{};
  d.cin = cin; d.cout = cout; d.cinp = cinp; d.coutp = coutp;
  const size_t np = (size_t)cout * cin * 9 + cout;
  std::vector<float> hp(np, 0.f);
  memcpy(hp.data(), w_host, (size_t)cout * cin * 9 * sizeof(float));
  if (b_host) memcpy(hp.data() + (size_t)cout * cin * 9, b_host, cout * sizeof(float));
  float *pd = nullptr, *bias = nullptr;
  bf16 *wf = nullptr, *wd = nullptr;
  ConvDesc* dd = nullptr;
  const size_t pk = 9 * (size_t)cinp * coutp;
  if (cudaMalloc(&pd, np * 4) || cudaMalloc(&bias, coutp * 4) || cudaMalloc(&wf, pk * 2) ||
      cudaMalloc(&wd, pk * 2) || cudaMalloc(&dd, sizeof(ConvDesc)))
    return SR_E_NOMEM;
  cudaMemcpy(pd, hp.data(), np * 4, cudaMemcpyHostToDevice);
  cudaMemcpy(dd, &d, sizeof(ConvDesc), cudaMemcpyHostToDevice);
  bf16 *wo = nullptr, *wdo = nullptr;
  if (cudaMalloc(&wo, pk * 2) || cudaMalloc(&wdo, pk * 2)) return SR_E_NOMEM;
  launch_pack_weights(pd, dd, 1, (int)pk, wf, wd, wo, wdo, bias, st);
  EpiParams ep{};
  ep.bias = (b_host && !dgrad) ? bias : nullptr;
  ep.res1 = (const bf16*)res_dev;
  ep.mask = (const bf16*)mask_dev;
  ep.relu = relu;
  ep.out = (bf16*)out_dev;
  size_t smem = 0;
  const int ci_eff = dgrad ? coutp : cinp, co_eff = dgrad ? cinp : coutp;
  ConvGeom g = make_geom(n, h, w, ci_eff, co_eff, &smem);
  int grid = std::min(g.units, num_sms());
  cudaError_t e;
  if (roll_supported(ci_eff, co_eff, w) && !(res_dev && mask_dev))
    e = launch_conv_roll_ex(ci_eff, co_eff, x_dev, dgrad ? wdo : wo, ep.bias, ep.res1, nullptr, ep.mask, relu, 0,
                            (bf16*)out_dev, n, h, w, st);
  else
    e = launch_conv(ci_eff, co_eff, EPI_ACT, x_dev, dgrad ? wd : wf, g, ep, smem, grid, st);
  cudaError_t e2 = cudaStreamSynchronize(st);
  cudaFree(pd); cudaFree(bias); cudaFree(wf); cudaFree(wd); cudaFree(wo); cudaFree(wdo); cudaFree(dd);
  if (e == cudaErrorNotSupported) return SR_E_UNSUPPORTED;
  return (e == cudaSuccess && e2 == cudaSuccess) ? SR_OK : SR_E_CUDA;
}

sr_status sr_test_adam(float* p_dev, float* m_dev, float* v_dev, const float* g_dev, size_t n, int steps,
                       float lr, sr_stream stream) {
  if (!p_dev || !m_dev || !v_dev || !g_dev || n == 0 || steps < 1) return SR_E_INVAL;
  cudaStream_t st = (cudaStream_t)stream;
  static long long* counters = nullptr;  // test-only step counters, kept for the process
  if (!counters) {
    if (cudaMalloc(&counters, 2 * sizeof(long long)) != cudaSuccess) return SR_E_NOMEM;
    if (cudaMemset(counters, 0, 2 * sizeof(long long)) != cudaSuccess) return SR_E_CUDA;
  }
  for (int k = 0; k < steps; ++k) {
    launch_adam(p_dev, m_dev, v_dev, g_dev, n, nullptr, 1.0f, counters, lr, 0.9f, 0.999f, 1e-8f, st);
    launch_counter_add(counters + 1, 1, st);  // t (the training path advances it in the repack)
  }
  return cudaGetLastError() == cudaSuccess ? SR_OK : SR_E_CUDA;
}

sr_status sr_test_wgrad_batch(int J, const void* const* x_devs, const void* const* dy_devs, int n, int h, int w,
                              const int* cins, const int* couts, float* out_host, sr_stream stream) {
  if (J < 1 || !x_devs || !dy_devs || !cins || !couts || !out_host) return SR_E_INVAL;
  cudaStream_t st = (cudaStream_t)stream;
  std::vector<size_t> off(J + 1, 0);
  for (int k = 0; k < J; ++k) off[k + 1] = off[k] + (size_t)couts[k] * cins[k] * 9 + couts[k];
  float* gout = nullptr;
  if (cudaMalloc(&gout, off[J] * 4)) return SR_E_NOMEM;
  std::vector<WgradJob> jobs(J);
  for (int k = 0; k < J; ++k)
    jobs[k] = WgradJob{(const bf16*)x_devs[k], (const bf16*)dy_devs[k], rup16(cins[k]), rup16(couts[k]), cins[k],
                       couts[k], gout + off[k], gout + off[k] + (size_t)couts[k] * cins[k] * 9};
  sr_ctx tmp;  // workspace holder only (the same batching/fallback logic as training)
  sr_status rc = wgrad_jobs(&tmp, jobs.data(), J, n, h, w, 1.0f, st);
  cudaError_t e2 = cudaStreamSynchronize(st);
  if (rc == SR_OK && e2 == cudaSuccess) cudaMemcpy(out_host, gout, off[J] * 4, cudaMemcpyDeviceToHost);
  cudaFree(gout);
  if (tmp.ws_w) cudaFree(tmp.ws_w);
  if (tmp.wg_sync) cudaFree(tmp.wg_sync);
  return rc != SR_OK ? rc : (e2 == cudaSuccess ? SR_OK : SR_E_CUDA);
}

sr_status sr_test_wgrad(const void* x_dev, const void* dy_dev, int n, int h, int w, int cin, int cout,
                        float* dw_host, float* db_host, sr_stream stream) {
  if (!x_dev || !dy_dev || !dw_host || !db_host) return SR_E_INVAL;
  std::vector<float> h_((size_t)cout * cin * 9 + cout);
  sr_status rc = sr_test_wgrad_batch(1, &x_dev, &dy_dev, n, h, w, &cin, &cout, h_.data(), stream);
  if (rc != SR_OK) return rc;
  memcpy(dw_host, h_.data(), (size_t)cout * cin * 9 * 4);
  memcpy(db_host, h_.data() + (size_t)cout * cin * 9, cout * 4);
  return SR_OK;
}

}  // extern "C"

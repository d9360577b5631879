"""Where the bench step's time goes: inference of 30 frames, 10 graph-replayed training iterations, and the
epoch-end work (publish + Algorithm 1 evaluation), each timed alone with CUDA events (+ host wall for the sync)."""
import os, sys, time
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench as B
from paper_conf_sigcomm_kimjyyh20_b200 import Controller, SRContext
from synth import synth_frames, synth_patch_pool

ctx = SRContext(B.S, B.BLOCKS, B.CH, seed=0)
dev = torch.device("cuda")
lr = torch.from_numpy(synth_frames(B.FRAMES, B.LR_H, B.LR_W, seed=1003)).to(dev)
hr = torch.empty((B.FRAMES, B.S * B.LR_H, B.S * B.LR_W, 3), dtype=torch.uint8, device=dev)
plr, phr, _ = synth_patch_pool(B.POOL_N, B.S, B.S * B.POOL_LR, seed=1004, frame_hw=(1080, 1800))
ctx.pool_push(torch.from_numpy(plr).to(dev), torch.from_numpy(phr).to(dev))
val_lr, val_hr = torch.from_numpy(plr[-64:]).to(dev), torch.from_numpy(phr[-64:]).to(dev)
blr = torch.empty((64, 48, 48, 3), dtype=torch.uint8, device=dev)
bhr = torch.empty((64, 144, 144, 3), dtype=torch.uint8, device=dev)
bidx = torch.empty(64, dtype=torch.int32, device=dev)
loss = torch.zeros(1, device=dev)
def it():
    ctx.sample_batch(-1, 64, 48, out=(blr, bhr, bidx)); ctx.train_grad(blr, bhr, loss); ctx.train_apply(1.0)
it(); torch.cuda.synchronize()
g = torch.cuda.CUDAGraph()
with torch.cuda.graph(g):
    it()
ctrl = Controller(thresh_sat=0.05, count_sat=2, thresh_online=0.5, count_online=2)
def timeit(f, n=5):
    for _ in range(2): f()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    t = time.perf_counter(); a.record()
    for _ in range(n): f()
    b.record(); torch.cuda.synchronize()
    return a.elapsed_time(b) / n, (time.perf_counter() - t) * 1e3 / n
print("infer 30 frames      %.3f ms (wall %.3f)" % timeit(lambda: ctx.infer(lr, "serve", out=hr)))
print("10 train iters       %.3f ms (wall %.3f)" % timeit(lambda: [g.replay() for _ in range(10)]))
print("publish              %.3f ms (wall %.3f)" % timeit(lambda: ctx.publish()))
print("controller_step      %.3f ms (wall %.3f)" % timeit(lambda: ctx.controller_step(ctrl, val_lr, val_hr)))
print("psnr_gain(serve,bil) %.3f ms (wall %.3f)" % timeit(lambda: ctx.psnr_gain(val_lr, val_hr, "serve", "bilinear")))

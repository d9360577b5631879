"""Bench-step A/B: the step of bench.py with and without the per-kernel CUDA-event timing, and its parts."""
import os, sys
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench as B
from paper_conf_sigcomm_kimjyyh20_b200 import SRContext
from synth import synth_frames, synth_patch_pool

ctx = SRContext(B.S, B.BLOCKS, B.CH, seed=0)
dev = torch.device("cuda")
lr = torch.from_numpy(synth_frames(B.FRAMES, B.LR_H, B.LR_W, seed=1003)).to(dev)
hr = torch.empty((B.FRAMES, B.S * B.LR_H, B.S * B.LR_W, 3), dtype=torch.uint8, device=dev)
plr, phr, _ = synth_patch_pool(B.POOL_N, B.S, B.S * B.POOL_LR, seed=1004, frame_hw=(1080, 1800))
ctx.pool_push(torch.from_numpy(plr).to(dev), torch.from_numpy(phr).to(dev))
blr = torch.empty((64, 48, 48, 3), dtype=torch.uint8, device=dev)
bhr = torch.empty((64, 144, 144, 3), dtype=torch.uint8, device=dev)
bidx = torch.empty(64, dtype=torch.int32, device=dev)
loss = torch.zeros(1, device=dev)
inv_w = torch.ones(1, device=dev)
def it():
    ctx.sample_batch(-1, 64, 48, out=(blr, bhr, bidx)); ctx.train_grad(blr, bhr, loss); ctx.train_apply_dev(inv_w)
it(); torch.cuda.synchronize()
g = torch.cuda.CUDAGraph()
with torch.cuda.graph(g):
    it()
def step():
    ctx.infer(lr, "serve", out=hr)
    for _ in range(10):
        g.replay()
def timeit(f, n=10):
    for _ in range(3): f()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(n): f()
    b.record(); torch.cuda.synchronize()
    return a.elapsed_time(b) / n
for rep in range(2):
    ctx.kernel_timing(False)
    t0 = timeit(step)
    ctx.kernel_timing(True)
    t1 = timeit(step)
    ctx.kernel_timing(False)
    ti = timeit(lambda: ctx.infer(lr, "serve", out=hr))
    tt = timeit(lambda: [g.replay() for _ in range(10)])
    print(f"step {t0:.3f} ms (timing on {t1:.3f}); infer alone {ti:.3f}; 10 train iters alone {tt:.3f}; "
          f"sum {ti + tt:.3f}", flush=True)

"""Concurrent inference + training on disjoint SM sets (sr_set_sm_split) vs the sequential step: 30 720p frames
x3 + 10 training iterations per step; K = SMs given to training (0 = sequential on one stream)."""
import os, sys
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench as B
from paper_conf_sigcomm_kimjyyh20_b200 import SRContext
from synth import synth_frames, synth_patch_pool

dev = torch.device("cuda")
lr = torch.from_numpy(synth_frames(B.FRAMES, B.LR_H, B.LR_W, seed=1003)).to(dev)
hr = torch.empty((B.FRAMES, B.S * B.LR_H, B.S * B.LR_W, 3), dtype=torch.uint8, device=dev)
plr, phr, _ = synth_patch_pool(B.POOL_N, B.S, B.S * B.POOL_LR, seed=1004, frame_hw=(1080, 1800))

def run(K, steps=8):
    ctx = SRContext(B.S, B.BLOCKS, B.CH, seed=0)
    ctx.set_sm_split(K)
    ctx.pool_push(torch.from_numpy(plr).to(dev), torch.from_numpy(phr).to(dev))
    blr = torch.empty((64, 48, 48, 3), dtype=torch.uint8, device=dev)
    bhr = torch.empty((64, 144, 144, 3), dtype=torch.uint8, device=dev)
    bidx = torch.empty(64, dtype=torch.int32, device=dev)
    loss = torch.zeros(1, device=dev)
    inv_w = torch.ones(1, device=dev)
    def it():
        ctx.sample_batch(-1, 64, 48, out=(blr, bhr, bidx)); ctx.train_grad(blr, bhr, loss)
        ctx.train_apply_dev(inv_w)
    it(); torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        it()
    sa = torch.cuda.Stream()  # non-default streams: the legacy default stream would serialize with the other
    sb = torch.cuda.Stream() if K > 0 else sa
    def step():
        with torch.cuda.stream(sa):
            ctx.infer(lr, "serve", out=hr)
        with torch.cuda.stream(sb):
            for _ in range(10):
                g.replay()
    for _ in range(2): step()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(sa)
    sb.wait_stream(sa)
    for _ in range(steps): step()
    if K > 0:
        sa.wait_stream(sb)
    b.record(sa)
    torch.cuda.synchronize()
    ms = a.elapsed_time(b) / steps
    # parts alone under the split
    t0 = torch.cuda.Event(enable_timing=True); t1 = torch.cuda.Event(enable_timing=True)
    t0.record(); ctx.infer(lr, "serve", out=hr); t1.record(); torch.cuda.synchronize(); ti = t0.elapsed_time(t1)
    t0.record(); [g.replay() for _ in range(10)]; t1.record(); torch.cuda.synchronize(); tt = t0.elapsed_time(t1)
    print(f"K={K:3d}: step {ms:7.3f} ms ({30 / ms * 1e3:6.1f} frames/s); infer alone {ti:7.3f}, 10 iters alone {tt:7.3f}",
          flush=True)

for K in [int(x) for x in sys.argv[1:]] or [0, 16, 20, 24, 28]:
    run(K)

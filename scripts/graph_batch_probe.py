"""Does capturing several training iterations per CUDA graph (fewer graph launches) speed up the replay?  One
iteration per graph (sr_train_sampled) vs a caller-captured graph of 10 iterations of the split API."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sigcomm_kimjyyh20_b200 import SRContext  # noqa: E402
from synth import synth_patch_pool  # noqa: E402

plr, phr, _ = synth_patch_pool(512, 3, 180, seed=1004, frame_hw=(1080, 1800))
ctx = SRContext(3, 8, 48, seed=0)
ctx.pool_push(torch.from_numpy(plr).cuda(), torch.from_numpy(phr).cuda())
loss = torch.zeros(1, device="cuda")
st = torch.cuda.Stream()
blr = torch.empty((64, 48, 48, 3), dtype=torch.uint8, device="cuda")
bhr = torch.empty((64, 144, 144, 3), dtype=torch.uint8, device="cuda")
scale = torch.ones(1, device="cuda")


def it():
    ctx.sample_batch(-1, 64, 48, out=(blr, bhr, None))
    ctx.train_grad(blr, bhr, loss)
    ctx.train_apply_dev(scale)


with torch.cuda.stream(st):
    it()
torch.cuda.synchronize()
g = torch.cuda.CUDAGraph()
with torch.cuda.graph(g):
    for _ in range(10):
        it()
for rep in range(3):
    with torch.cuda.stream(st):
        ctx.train_sampled(5, 64, 48, loss)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        ctx.train_sampled(100, 64, 48, loss)
        e1.record()
    torch.cuda.synchronize()
    a = e0.elapsed_time(e1) / 100
    with torch.cuda.stream(st):
        g.replay()
        e2, e3 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e2.record()
        for _ in range(10):
            g.replay()
        e3.record()
    torch.cuda.synchronize()
    b = e2.elapsed_time(e3) / 100
    print(f"1-iteration graphs {a:.4f} ms/iter   10-iteration graph {b:.4f} ms/iter", flush=True)

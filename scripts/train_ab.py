"""Training iteration time (graph replay) with the default kernels vs set_fusion variants given on the command line."""
import os, sys
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sigcomm_kimjyyh20_b200 import SRContext
from synth import synth_patch_pool

def run(fusion):
    ctx = SRContext(3, 8, 48, seed=0)
    ctx.set_fusion(fusion)
    dev = torch.device("cuda")
    plr, phr, _ = synth_patch_pool(512, 3, 180, seed=1004, frame_hw=(1080, 1800))
    ctx.pool_push(torch.from_numpy(plr).to(dev), torch.from_numpy(phr).to(dev))
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
    for _ in range(20): g.replay()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(100): g.replay()
    b.record(); torch.cuda.synchronize()
    return a.elapsed_time(b) / 100

for rep in range(2):
    for f in [int(x) for x in sys.argv[1:]] or [1]:
        print(f"fusion={f:3d}: {run(f):.4f} ms/iter")

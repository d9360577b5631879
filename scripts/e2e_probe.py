import os, sys, time
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sigcomm_kimjyyh20_b200 import SRContext
from synth import synth_frames
ctx = SRContext(3, 8, 48, seed=0)
lr_np = synth_frames(30, 720, 1280, seed=1)
lr_d = torch.from_numpy(lr_np).cuda()
hr_d = torch.empty((30, 2160, 3840, 3), dtype=torch.uint8, device="cuda")
lr_h = torch.from_numpy(lr_np).pin_memory()
hr_h = torch.empty((30, 2160, 3840, 3), dtype=torch.uint8).pin_memory()
def t(fn, k=5):
    fn(); torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(k): fn()
    torch.cuda.synchronize()
    return (time.perf_counter() - t0) / k * 1e3
print("D2H 746MB  ms", t(lambda: hr_h.copy_(hr_d, non_blocking=True)), flush=True)
print("H2D 83MB   ms", t(lambda: lr_d.copy_(lr_h, non_blocking=True)), flush=True)
print("infer dev  ms", t(lambda: ctx.infer(lr_d, "serve", out=hr_d)), flush=True)
print("infer host ms", t(lambda: ctx.infer_host(lr_h, hr_h, "serve")), flush=True)
s2 = torch.cuda.Stream()
def both():
    ctx.infer(lr_d, "serve", out=hr_d)
    with torch.cuda.stream(s2):
        hr_h.copy_(hr_d, non_blocking=True)
print("infer + concurrent D2H ms", t(both), flush=True)

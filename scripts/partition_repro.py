"""Repro of the whole-GPU training slowdown seen after partitioned steps in bench.py: alternate partitioned steps
(inference on the 108-SM partition, training on the 40-SM one, + host-pipeline e2e steps) with whole-GPU training
timing on a normal stream, and print every timing."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sigcomm_kimjyyh20_b200 import SRContext  # noqa: E402
from synth import synth_frames, synth_patch_pool  # noqa: E402

ctx = SRContext(3, 8, 48, seed=0)
plr, phr, _ = synth_patch_pool(512, 3, 180, seed=1004, frame_hw=(1080, 1800))
ctx.pool_push(torch.from_numpy(plr).cuda(), torch.from_numpy(phr).cuda())
lr_np = synth_frames(30, 720, 1280, seed=1003)
lr = torch.from_numpy(lr_np).cuda()
hr = torch.empty((30, 2160, 3840, 3), dtype=torch.uint8, device="cuda")
lr_h = torch.from_numpy(lr_np).pin_memory()
hr_h = [torch.empty((30, 2160, 3840, 3), dtype=torch.uint8).pin_memory() for _ in range(2)]
loss = torch.zeros(1, device="cuda")
st = torch.cuda.Stream()
torch.cuda.synchronize()
si, stt, ni, nt = SRContext.sm_partition(40)
mode = os.environ.get("MODE", "all")


def t_train(s, k=50, label=""):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with torch.cuda.stream(s):
        ctx.train_sampled(2, 64, 48, loss)
        e0.record()
        ctx.train_sampled(k, 64, 48, loss)
        e1.record()
    torch.cuda.synchronize()
    print(f"  {label} train {e0.elapsed_time(e1) / k:.4f} ms/iter", flush=True)


for rnd in range(4):
    ctx.set_sm_split(nt)
    for _ in range(10):
        ctx.infer(lr, "serve", out=hr, stream=si)
        ctx.train_sampled(10, 64, 48, loss, stream=stt)
    torch.cuda.synchronize()
    if mode in ("all", "e2e"):
        for k in range(6):
            ctx.infer_host_async(lr_h, hr_h[k & 1], "serve", stream=si)
            ctx.train_sampled(10, 64, 48, loss, stream=stt)
        ctx.infer_host_wait()
        torch.cuda.synchronize()
    ctx.set_sm_split(0)
    t_train(st, label=f"round {rnd} whole-GPU (old stream)")
    t_train(torch.cuda.Stream(), label=f"round {rnd} whole-GPU (new stream)")

"""Small end-to-end run for compute-sanitizer: tiny + mid configs, wide and narrow kernels, training, psnr."""
import os, sys
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sigcomm_kimjyyh20_b200 import SRContext
from synth import synth_frames, synth_patch_pool
for (s, B, C), (h, w) in (((2, 2, 8), (64, 64)), ((3, 2, 48), (37, 260)), ((2, 1, 32), (5, 130)),
                          ((3, 2, 48), (21, 272)), ((4, 1, 16), (9, 400)), ((2, 2, 32), (11, 528))):
    ctx = SRContext(s, B, C, seed=1)
    lr = torch.from_numpy(synth_frames(2, h, w, seed=2)).cuda()
    ctx.infer(lr, "serve")                 # W % 16 == 0: fused body + tail (k_bodytail)
    full = ctx.infer(lr, "serve").clone()
    ctx.set_fusion(1 | 32)                 # body conv + rolling tail with TMA-staged LR/HR rows
    ctx.infer(lr, "serve")
    ctx.set_fusion(1 | 32 | 16)            # rolling tail, per-lane global path
    ctx.infer(lr, "serve")
    ctx.set_fusion(1)
    hr = torch.zeros_like(full[0])
    ctx.infer_rows(lr[0], 0, h // 2, hr, "serve")   # strip pieces
    ctx.infer_rows(lr[0], h // 2, h, hr, "serve")
    ctx.set_fusion(0)
    ctx.infer(lr, "serve")
    plr, phr, _ = synth_patch_pool(8, s, s * 24, seed=3, frame_hw=(s * 24 * 2, s * 24 * 4))
    ctx.pool_push(torch.from_numpy(plr).cuda(), torch.from_numpy(phr).cuda())
    for mode in (1, 3, 9):
        ctx.set_fusion(mode)
        l, hh, _ = ctx.sample_batch(0, 6, 20)
        ctx.train_step(l, hh)
    ctx.psnr_gain(torch.from_numpy(plr).cuda(), torch.from_numpy(phr).cuda())
    torch.cuda.synchronize()
    print("ok", s, B, C, h, w, flush=True)
# round 2 paths: the library-captured sampled training graph (device pool view, patch push between replays),
# publish against inference on another stream, the I420 push with out-of-frame corners, the two-set host pipeline,
# the multi-block SSE, the vectorised Adam, and a green-context SM partition
ctx = SRContext(3, 2, 48, seed=5)
plr, phr, _ = synth_patch_pool(40, 3, 3 * 30, seed=6, frame_hw=(3 * 30 * 3, 3 * 30 * 4))
ctx.pool_push(torch.from_numpy(plr[:30]).cuda(), torch.from_numpy(phr[:30]).cuda())
st = torch.cuda.Stream()
loss = torch.zeros(1, device="cuda")
with torch.cuda.stream(st):
    ctx.train_sampled(2, 8, 24, loss)
    ctx.pool_push(torch.from_numpy(plr[30:]).cuda(), torch.from_numpy(phr[30:]).cuda())
    ctx.train_sampled(2, 8, 24, loss)
lr = torch.from_numpy(synth_frames(3, 40, 272, seed=7)).cuda()
out = ctx.infer(lr, "serve")
with torch.cuda.stream(st):
    ctx.publish()
ctx.infer(lr, "serve", out=out)
lr_h = lr.cpu().pin_memory()
outs = [torch.empty((3, 120, 816, 3), dtype=torch.uint8).pin_memory() for _ in range(3)]
for k in range(3):
    ctx.infer_host_async(lr_h, outs[k], "serve")
ctx.infer_host_wait()
from oracle.color import rgb_to_i420  # test infrastructure only (the I420 planes of a synthetic frame)
y, u, v = rgb_to_i420(synth_frames(1, 64, 96, seed=8))
import numpy as np
xy = torch.from_numpy(np.array([[-3, 5], [90, 70], [8, 8]], np.int32)).cuda()
hrp = torch.from_numpy(np.zeros((3, 48, 48, 3), np.uint8)).cuda()
ctx2 = SRContext(3, 1, 16, seed=1)
ctx2.pool_push_i420(torch.from_numpy(y[0]).cuda(), torch.from_numpy(u[0]).cuda(), torch.from_numpy(v[0]).cuda(), hrp, xy)
si, stt, ni, nt = SRContext.sm_partition(40)
ctx.set_sm_split(nt)
with torch.cuda.stream(stt):
    ctx.train_sampled(2, 8, 24, loss)
with torch.cuda.stream(si):
    ctx.infer(lr, "serve", out=out)
torch.cuda.synchronize()
print("ok round-2 paths", flush=True)

"""Eagerly launched training iterations at the bench config (x3 8x48, batch 64, 48x48 LR from 60x60 pool entries)
for ncu: sample + gather, forward, loss, backward, Adam -- the kernels sr_train_sampled's graph replays."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sigcomm_kimjyyh20_b200 import SRContext  # noqa: E402
from synth import synth_patch_pool  # noqa: E402

ctx = SRContext(3, 8, 48, seed=0)
plr, phr, _ = synth_patch_pool(512, 3, 180, seed=1004, frame_hw=(1080, 1800))
ctx.pool_push(torch.from_numpy(plr).cuda(), torch.from_numpy(phr).cuda())
blr = torch.empty((64, 48, 48, 3), dtype=torch.uint8, device="cuda")
bhr = torch.empty((64, 144, 144, 3), dtype=torch.uint8, device="cuda")
loss = torch.zeros(1, device="cuda")
n = int(sys.argv[1]) if len(sys.argv) > 1 else 3
for _ in range(n):
    ctx.sample_batch(-1, 64, 48, out=(blr, bhr, None))
    ctx.train_grad(blr, bhr, loss)
    ctx.train_apply(1.0)
torch.cuda.synchronize()
print("loss", loss.item())

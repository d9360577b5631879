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

"""Gradient / loss / Adam-step errors of the GPU training paths vs the fp64 oracle on several configs."""
import os, sys
import numpy as np, torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import oracle as O
from paper_conf_sigcomm_kimjyyh20_b200 import SRContext
from synth import init_params, synth_patch_pool

def rel(a, b):
    return float(np.linalg.norm(np.asarray(a, np.float64) - b) / np.linalg.norm(b))

for (s, B, C), n, p, scale in (((2, 8, 48), 8, 48, 1.0), ((2, 8, 48), 8, 48, 2.0), ((3, 8, 48), 8, 48, 1.0),
                               ((3, 3, 48), 6, 48, 2.0), ((2, 8, 32), 8, 48, 1.0)):
    lrp, hrp, _ = synth_patch_pool(n, s, s * p, seed=41, frame_hw=(s * p * 3, s * p * 4))
    lr, hr = torch.from_numpy(lrp).cuda(), torch.from_numpy(hrp).cuda()
    out = []
    for mode, name in ((1, "virtual"), (3, "narrow")):
        ctx = SRContext(s, B, C, seed=22)
        ctx.set_params(init_params(s, B, C, seed=22) * scale)
        ctx.set_fusion(mode)
        loss = torch.zeros(1, device="cuda")
        ctx.train_grad(lr, hr, loss)
        g = ctx.grad_buffer().cpu().numpy().copy()
        pq = ctx.get_params("train")
        rl, rg = O.train_loss_and_grad(pq, lrp, hrp, s, B, C)
        out.append(f"{name}: loss rel {abs(loss.item()-rl)/rl:.2e} grad relL2 {rel(g, rg):.3e}")
    print(f"x{s} {B}x{C} n={n} p={p} w*{scale}: " + " | ".join(out), flush=True)

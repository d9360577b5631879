"""Run a few graph-replayed training iterations (for ncu launch lists)."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sigcomm_kimjyyh20_b200 import SRContext  # noqa: E402
from synth import synth_patch_pool  # noqa: E402

ctx = SRContext(3, 8, 48, seed=0)
plr, phr, _ = synth_patch_pool(256, 3, 180, seed=1, frame_hw=(540, 900))
ctx.pool_push(torch.from_numpy(plr).cuda(), torch.from_numpy(phr).cuda())
st = torch.cuda.Stream()
with torch.cuda.stream(st):
    loss = torch.zeros(1, device="cuda")
    ctx.train_sampled(int(sys.argv[1]) if len(sys.argv) > 1 else 3, 64, 48, loss)
torch.cuda.synchronize()
print("loss", loss.item())

"""Graph-replayed training iteration time (bench config) for kernel variants (sr_set_fusion bits) and SM splits."""
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sigcomm_kimjyyh20_b200 import SRContext  # noqa: E402
from synth import synth_patch_pool  # noqa: E402

plr, phr, _ = synth_patch_pool(512, 3, 180, seed=1004, frame_hw=(1080, 1800))
out = {}
for mode in [int(x) for x in os.environ.get("MODES", "1,9").split(",")]:
    ctx = SRContext(3, 8, 48, seed=0)
    ctx.set_fusion(mode)
    ctx.pool_push(torch.from_numpy(plr).cuda(), torch.from_numpy(phr).cuda())
    loss = torch.zeros(1, device="cuda")
    st = torch.cuda.Stream()
    with torch.cuda.stream(st):
        ctx.train_sampled(5, 64, 48, loss)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        ctx.train_sampled(50, 64, 48, loss)
        e1.record()
    torch.cuda.synchronize()
    out[f"fusion{mode}"] = round(e0.elapsed_time(e1) / 50, 4)
    ctx.close()
print(json.dumps(out))

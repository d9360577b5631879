"""Per-kernel-class CUDA-event breakdown of eagerly launched training iterations (bench config), on the whole GPU
and on a T-SM green-context partition (the bench's training partition)."""
import json
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


def run(st, k=10):
    with torch.cuda.stream(st):
        for _ in range(3):
            ctx.sample_batch(-1, 64, 48, out=(blr, bhr, None))
            ctx.train_grad(blr, bhr, loss)
        torch.cuda.synchronize()
        ctx.kernel_timing(True)
        for _ in range(k):
            ctx.sample_batch(-1, 64, 48, out=(blr, bhr, None))
            ctx.train_grad(blr, bhr, loss)
    stats = ctx.kernel_stats()
    ctx.kernel_timing(False)
    tot = sum(v["ms"] for v in stats.values()) / k
    out = {"ms_per_iter_eager": round(tot, 4)}
    for c, v in sorted(stats.items(), key=lambda kv: -kv[1]["ms"]):
        out[c] = {"us_per_launch": round(v["ms"] / v["launches"] * 1e3, 2), "launches_per_iter": v["launches"] // k,
                  "share": round(v["ms"] / k / tot, 4), "tflops": round(v["flops"] / (v["ms"] * 1e-3) / 1e12, 1)}
    return out


res = {"whole": run(torch.cuda.Stream())}
T = int(os.environ.get("T", "40"))
si, stt, ni, nt = SRContext.sm_partition(T)
ctx.set_sm_split(nt)
res[f"part{nt}"] = run(stt)
print(json.dumps(res, indent=1))

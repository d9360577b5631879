"""Training-iteration timing: eager (Python-driven) vs the library's CUDA-graph replay (sr_train_sampled)."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sigcomm_kimjyyh20_b200 import SRContext  # noqa: E402
from synth import synth_patch_pool  # noqa: E402

s, B, C = 3, 8, 48
ctx = SRContext(s, B, C, seed=0)
if len(sys.argv) > 1:
    ctx.set_fusion(int(sys.argv[1]))  # e.g. 9: fused data-gradient blocks
plr, phr, _ = synth_patch_pool(256, s, 180, seed=1, frame_hw=(540, 900))
ctx.pool_push(torch.from_numpy(plr).cuda(), torch.from_numpy(phr).cuda())
st = torch.cuda.Stream()
with torch.cuda.stream(st):
    loss = torch.zeros(1, device="cuda")
    blr = torch.empty((64, 48, 48, 3), dtype=torch.uint8, device="cuda")
    bhr = torch.empty((64, 144, 144, 3), dtype=torch.uint8, device="cuda")
    bidx = torch.empty(64, dtype=torch.int32, device="cuda")

    def eager(n):
        for i in range(n):
            ctx.sample_batch(i, 64, 48, out=(blr, bhr, bidx))
            ctx.train_grad(blr, bhr, loss)
            ctx.train_apply(1.0)

    for name, fn in (("eager", eager), ("graph", lambda n: ctx.train_sampled(n, 64, 48, loss))):
        fn(3)
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fn(50)
        b.record()
        torch.cuda.synchronize()
        ms = a.elapsed_time(b) / 50
        print(f"{name}: {ms:.3f} ms/iter  {64/ms*1e3:.0f} patches/s  {323.0/ms:.1f} TFLOP/s  loss {loss.item():.5f}",
              flush=True)

# per-kernel-class event timing of eager iterations
with torch.cuda.stream(st):
    ctx.kernel_timing(True)
    eager(10)
    stats = ctx.kernel_stats()
    ctx.kernel_timing(False)
tot = sum(v["ms"] for v in stats.values())
for k, v in sorted(stats.items(), key=lambda kv: -kv[1]["ms"]):
    print(f"{k:28s} n={v['launches']:4d} avg={1e3*v['ms']/v['launches']:8.1f} us  share={100*v['ms']/tot:5.1f}%  "
          f"{v['flops']/(v['ms']*1e-3)/1e12:7.1f} TF/s")
print("kernel-class total per iter (ms):", tot / 10)

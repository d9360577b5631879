"""Per-kernel-class CUDA-event timing of the bench's inference (30 x 720p -> 4K, x3 8x48)."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sigcomm_kimjyyh20_b200 import SRContext  # noqa: E402
from synth import synth_frames  # noqa: E402

ctx = SRContext(3, 8, 48, seed=0)
if os.environ.get("SR_FUSION"):  # A/B of kernel variants (sr_set_fusion bits)
    ctx.set_fusion(int(os.environ["SR_FUSION"]))
lr = torch.from_numpy(synth_frames(30, 720, 1280, seed=1003)).cuda()
hr = torch.empty((30, 2160, 3840, 3), dtype=torch.uint8, device="cuda")
for _ in range(2):
    ctx.infer(lr, "serve", out=hr)
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(5):
    ctx.infer(lr, "serve", out=hr)
e1.record()
torch.cuda.synchronize()
print(f"infer 30 frames: {e0.elapsed_time(e1) / 5:.3f} ms")
ctx.kernel_timing(True)
for _ in range(5):
    ctx.infer(lr, "serve", out=hr)
st = ctx.kernel_stats()
ctx.kernel_timing(False)
tot = sum(v["ms"] for v in st.values())
for k, v in sorted(st.items(), key=lambda kv: -kv[1]["ms"]):
    print(f"{k:28s} n={v['launches']:4d} {v['ms'] / 5:8.3f} ms/infer {100 * v['ms'] / tot:5.1f}%  "
          f"{v['flops'] / (v['ms'] * 1e-3) / 1e12:7.1f} TF/s  {v['bytes'] / (v['ms'] * 1e-3) / 1e9:7.1f} GB/s")

"""Per-kernel-class CUDA-event timing of BASELINE config 2 inference (30 x 540p -> 1080p x2, 8x32)."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sigcomm_kimjyyh20_b200 import SRContext  # noqa: E402
from synth import synth_frames  # noqa: E402

ctx = SRContext(2, 8, 32, seed=0)
if os.environ.get("SR_FUSION"):  # A/B of kernel variants (sr_set_fusion bits)
    ctx.set_fusion(int(os.environ["SR_FUSION"]))
lr = torch.from_numpy(synth_frames(30, 540, 960, seed=1002)).cuda()
hr = torch.empty((30, 1080, 1920, 3), dtype=torch.uint8, device="cuda")
for _ in range(3):
    ctx.infer(lr, out=hr)
ctx.kernel_timing(True)
for _ in range(10):
    ctx.infer(lr, out=hr)
st = ctx.kernel_stats()
for k, v in st.items():
    print(k, round(v["ms"] / v["launches"], 4), "ms", round(v["flops"] / (v["ms"] * 1e-3) / 1e12, 1), "TF/s")

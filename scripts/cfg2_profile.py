"""BASELINE config 2 inference for ncu: 30 x 540p -> 1080p x2 with the 8x32 net (k_resblock<32>, k_bodytail<32,16,2>,
u8 head), after two warm-up batches."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sigcomm_kimjyyh20_b200 import SRContext  # noqa: E402
from synth import synth_frames  # noqa: E402

ctx = SRContext(2, 8, 32, seed=0)
lr = torch.from_numpy(synth_frames(30, 540, 960, seed=1002)).cuda()
hr = torch.empty((30, 1080, 1920, 3), dtype=torch.uint8, device="cuda")
for _ in range(3):
    ctx.infer(lr, "serve", out=hr)
torch.cuda.synchronize()
print("cfg2 ok")

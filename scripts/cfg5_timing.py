"""Per-kernel-class CUDA-event timing of config 5's net on 1080p frames (x2, 8x48; 8 frames per call)."""
import os, sys
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sigcomm_kimjyyh20_b200 import SRContext  # noqa: E402
from synth import synth_frames  # noqa: E402

ctx = SRContext(2, 8, 48, seed=0)
lr = torch.from_numpy(synth_frames(8, 1080, 1920, seed=1005)).cuda()
hr = torch.empty((8, 2160, 3840, 3), dtype=torch.uint8, device="cuda")
for _ in range(3):
    ctx.infer(lr, out=hr)
ctx.kernel_timing(True)
for _ in range(10):
    ctx.infer(lr, out=hr)
torch.cuda.synchronize()
for k, v in sorted(ctx.kernel_stats().items(), key=lambda kv: -kv[1]["ms"]):
    print(f"{k} {v['ms'] / v['launches']:.4f} ms")

"""Per-class CUDA-event kernel times of eager training iterations (x3 8x48, 64 x 48x48) for set_fusion variants:
the persistent chain launches (default) vs one k_conv_roll launch per conv (bit 9)."""
import os, sys
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sigcomm_kimjyyh20_b200 import SRContext
from synth import synth_patch_pool

for fusion in [int(x) for x in sys.argv[1:]] or [1, 513]:
    ctx = SRContext(3, 8, 48, seed=0)
    ctx.set_fusion(fusion)
    dev = torch.device("cuda")
    plr, phr, _ = synth_patch_pool(256, 3, 180, seed=1004, frame_hw=(1080, 1800))
    ctx.pool_push(torch.from_numpy(plr).to(dev), torch.from_numpy(phr).to(dev))
    blr = torch.empty((64, 48, 48, 3), dtype=torch.uint8, device=dev)
    bhr = torch.empty((64, 144, 144, 3), dtype=torch.uint8, device=dev)
    bidx = torch.empty(64, dtype=torch.int32, device=dev)
    loss = torch.zeros(1, device=dev)
    for i in range(3):
        ctx.sample_batch(-1, 64, 48, out=(blr, bhr, bidx)); ctx.train_grad(blr, bhr, loss); ctx.train_apply(1.0)
    torch.cuda.synchronize()
    ctx.kernel_timing(True)
    for i in range(10):
        ctx.sample_batch(-1, 64, 48, out=(blr, bhr, bidx)); ctx.train_grad(blr, bhr, loss); ctx.train_apply(1.0)
    torch.cuda.synchronize()
    print(f"fusion={fusion}")
    print(ctx.kernel_stats())

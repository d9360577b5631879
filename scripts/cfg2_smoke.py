import os, sys, torch
sys.path.insert(0, "/root/repo")
from paper_conf_sigcomm_kimjyyh20_b200 import SRContext
from synth import synth_frames
ctx = SRContext(2, 8, 32, seed=0)
lr = torch.from_numpy(synth_frames(30, 540, 960, seed=5)).cuda()
out = ctx.infer(lr, "serve"); torch.cuda.synchronize()
print("cfg2 infer ok", out.shape, int(out.float().mean()))

import os, sys, torch
sys.path.insert(0, "/root/repo")
from paper_conf_sigcomm_kimjyyh20_b200 import SRContext
from synth import synth_frames
ctx = SRContext(3, 8, 48, seed=0)
lr = torch.from_numpy(synth_frames(30, 720, 1280, seed=1)).cuda()
hr = torch.empty((30, 2160, 3840, 3), dtype=torch.uint8, device="cuda")
si, stt, ni, nt = SRContext.sm_partition(40)
ctx.infer(lr, out=hr, stream=si)
torch.cuda.synchronize()
print("after torch.cuda.synchronize: green stream done?", si.query(), flush=True)
si.synchronize()
print("after stream sync:", si.query())

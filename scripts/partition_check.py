"""Does a green-context SM partition leave whole-GPU work unaffected?  Training iteration time on a normal stream
before any partition, on the 40-SM training partition, and on a normal stream again afterwards (set_sm_split(0))."""
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sigcomm_kimjyyh20_b200 import SRContext  # noqa: E402
from synth import synth_patch_pool, synth_frames  # noqa: E402

ctx = SRContext(3, 8, 48, seed=0)
plr, phr, _ = synth_patch_pool(512, 3, 180, seed=1004, frame_hw=(1080, 1800))
ctx.pool_push(torch.from_numpy(plr).cuda(), torch.from_numpy(phr).cuda())
lr = torch.from_numpy(synth_frames(30, 720, 1280, seed=1003)).cuda()
hr = torch.empty((30, 2160, 3840, 3), dtype=torch.uint8, device="cuda")
loss = torch.zeros(1, device="cuda")
st = torch.cuda.Stream()
out = {}


def t_train(s, k=30):
    with torch.cuda.stream(s):
        ctx.train_sampled(3, 64, 48, loss)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        ctx.train_sampled(k, 64, 48, loss)
        e1.record()
    torch.cuda.synchronize()
    return round(e0.elapsed_time(e1) / k, 4)


def t_infer(s):
    with torch.cuda.stream(s):
        ctx.infer(lr, out=hr)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        ctx.infer(lr, out=hr)
        e1.record()
    torch.cuda.synchronize()
    return round(e0.elapsed_time(e1), 3)


out["before_train"] = t_train(st)
out["before_infer"] = t_infer(st)
si, stt, ni, nt = SRContext.sm_partition(40)
ctx.set_sm_split(nt)
out["part_train40"] = t_train(stt)
out["part_infer108"] = t_infer(si)
ctx.set_sm_split(0)
out["after_train"] = t_train(st)
out["after_infer"] = t_infer(st)
st2 = torch.cuda.Stream()
out["after_train_newstream"] = t_train(st2)
print(json.dumps(out))

"""e2e serving loop A/B (bench config): sequential one-stream vs SM partition, single vs double host buffering;
per-step host timestamps to see where the end-to-end step time goes."""
import json
import os
import sys
import time

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sigcomm_kimjyyh20_b200 import SRContext  # noqa: E402
from synth import synth_frames, synth_patch_pool  # noqa: E402

ctx = SRContext(3, 8, 48, seed=0)
plr, phr, _ = synth_patch_pool(512, 3, 180, seed=1004, frame_hw=(1080, 1800))
ctx.pool_push(torch.from_numpy(plr).cuda(), torch.from_numpy(phr).cuda())
torch.cuda.synchronize()
lr_np = synth_frames(30, 720, 1280, seed=1003)
lr_host = torch.from_numpy(lr_np).pin_memory()
hr_hosts = [torch.empty((30, 2160, 3840, 3), dtype=torch.uint8).pin_memory() for _ in range(2)]
loss = torch.zeros(1, device="cuda")
stream = torch.cuda.Stream()
res = {}


def loop(si, stt, double, k=10):
    ts = []
    for i in range(k + 2):
        if i == 2:
            torch.cuda.synchronize()
            t0 = time.perf_counter()
        ctx.infer_host_async(lr_host, hr_hosts[i & 1] if double else hr_hosts[0], "serve", stream=si)
        ctx.train_sampled(10, 64, 48, loss, stream=stt)
        if not double:
            ctx.infer_host_wait()
        ts.append(time.perf_counter())
    ctx.infer_host_wait()
    torch.cuda.synchronize()
    return (time.perf_counter() - t0) / k * 1e3, [round((b - a) * 1e3, 2) for a, b in zip(ts[2:], ts[3:])]


for mode in ("seq", "p40"):
    if mode == "seq":
        si = stt = stream
    else:
        si, stt, ni, nt = SRContext.sm_partition(40)
        ctx.set_sm_split(nt)
    for double in (False, True):
        loop(si, stt, double, 2)
        ms, steps = loop(si, stt, double)
        res[f"{mode}_{'double' if double else 'single'}"] = {"ms_per_step": round(ms, 3), "host_step_ms": steps}
        print(json.dumps(res), flush=True)

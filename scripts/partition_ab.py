"""A/B: the bench step (30 x 720p -> 4K inference + 10 sampled training iterations, x3 8x48) sequential on the whole
GPU vs concurrent on disjoint SM partitions (sr_sm_partition green contexts: training on T SMs, inference on the
rest), throughput over K steps with CUDA events (both streams)."""
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sigcomm_kimjyyh20_b200 import SRContext  # noqa: E402
from synth import synth_frames, synth_patch_pool  # noqa: E402

K = int(os.environ.get("K", "10"))
ctx = SRContext(3, 8, 48, seed=0)
plr, phr, _ = synth_patch_pool(512, 3, 180, seed=1004, frame_hw=(1080, 1800))
ctx.pool_push(torch.from_numpy(plr).cuda(), torch.from_numpy(phr).cuda())
lr = torch.from_numpy(synth_frames(30, 720, 1280, seed=1003)).cuda()
hr = torch.empty((30, 2160, 3840, 3), dtype=torch.uint8, device="cuda")
loss = torch.zeros(1, device="cuda")
res = {}


def run(si, stt, k):
    e = [torch.cuda.Event(enable_timing=True) for _ in range(4)]
    torch.cuda.synchronize()
    e[0].record(si)
    stt.wait_event(e[0])
    for _ in range(k):
        with torch.cuda.stream(si):
            ctx.infer(lr, "serve", out=hr)
        with torch.cuda.stream(stt):
            ctx.train_sampled(10, 64, 48, loss)
    e[1].record(si)
    e[2].record(stt)
    torch.cuda.synchronize()
    return max(e[0].elapsed_time(e[1]), e[0].elapsed_time(e[2])) / k, e[0].elapsed_time(e[1]) / k, \
        e[0].elapsed_time(e[2]) / k


s0 = torch.cuda.Stream()
run(s0, s0, 2)
ms, a, b = run(s0, s0, K)
res["sequential"] = {"ms_per_step": round(ms, 3)}
infer_only = run(s0, s0, 1)
for T in [int(x) for x in os.environ.get("TS", "16,24,32,40,48").split(",")]:
    try:
        si, stt, ni, nt = SRContext.sm_partition(T)
    except Exception as exc:  # noqa: BLE001
        res[f"T{T}"] = {"error": str(exc)}
        continue
    ctx.set_sm_split(nt)
    run(si, stt, 2)
    ms, a, b = run(si, stt, K)
    res[f"T{T}"] = {"train_sms": nt, "infer_sms": ni, "ms_per_step": round(ms, 3), "infer_stream_ms": round(a, 3),
                    "train_stream_ms": round(b, 3)}
    ctx.set_sm_split(0)
    SRContext.sm_partition_release()
    print(json.dumps(res), flush=True)
print(json.dumps(res))

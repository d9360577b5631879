"""Repeat the NCCL-on-partition check many times to find which context diverges (diagnostics)."""
import ctypes
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sigcomm_kimjyyh20_b200 import SRContext, load  # noqa: E402
from synth import synth_patch_pool  # noqa: E402

plr, phr, _ = synth_patch_pool(64, 3, 180, seed=5, frame_hw=(1080, 1800))
si, stt, ni, nt = SRContext.sm_partition(40)
ws = torch.cuda.Stream()
bad = 0
for it in range(int(os.environ.get("REPS", "20"))):
    buf = ctypes.create_string_buffer(128)
    assert load().sr_nccl_unique_id(buf, 128) == 0
    ctxs = {"a_nccl_part": SRContext(3, 2, 32, seed=3, nccl_id=buf.raw), "b_part": SRContext(3, 2, 32, seed=3),
            "c_whole": SRContext(3, 2, 32, seed=3)}
    for c in ctxs.values():
        c.pool_push(torch.from_numpy(plr).cuda(), torch.from_numpy(phr).cuda())
    torch.cuda.synchronize()
    for k, c in ctxs.items():
        if k == "c_whole":
            c.train_sampled(4, 16, 48, stream=ws)
        else:
            c.set_sm_split(nt)
            c.train_sampled(4, 16, 48, stream=stt)
    torch.cuda.synchronize()
    ps = {k: c.get_params("train") for k, c in ctxs.items()}
    ts = {k: c.adam_state()[2] for k, c in ctxs.items()}
    ref = ps["c_whole"]
    d = {k: float(np.abs(p - ref).max()) for k, p in ps.items()}
    if any(v > 0 for v in d.values()):
        bad += 1
    print(it, ts, d, flush=True)
    for c in ctxs.values():
        c.set_sm_split(0)
        c.close()
print("bad", bad)

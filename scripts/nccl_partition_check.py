"""One-rank NCCL communicator in the library + green-context partition streams: the in-graph ncclAllReduce must
run on the training partition's stream (what bench.py does at N > 1 on every rank)."""
import ctypes
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sigcomm_kimjyyh20_b200 import SRContext, load  # noqa: E402
from synth import synth_patch_pool  # noqa: E402

buf = ctypes.create_string_buffer(128)
assert load().sr_nccl_unique_id(buf, 128) == 0
a = SRContext(3, 2, 32, seed=3, nccl_id=buf.raw)
b = SRContext(3, 2, 32, seed=3)
plr, phr, _ = synth_patch_pool(64, 3, 180, seed=5, frame_hw=(1080, 1800))
for c in (a, b):
    c.pool_push(torch.from_numpy(plr).cuda(), torch.from_numpy(phr).cuda())
torch.cuda.synchronize()
si, stt, ni, nt = SRContext.sm_partition(40)
for c in (a, b):
    c.set_sm_split(nt)
    c.train_sampled(4, 16, 48, stream=stt)
    c.train_step(*[t[:8].contiguous() for t in c.sample_batch(0, 16, 48)[:2]], stream=stt)
torch.cuda.synchronize()
pa, pb = a.get_params("train"), b.get_params("train")
print("nccl on partition stream: params equal:", np.array_equal(pa, pb), "t =", a.adam_state()[2])

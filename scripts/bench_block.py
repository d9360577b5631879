"""Fused residual-block timing + CTA-0 pipeline timeline (clock64 stamps per role and step)."""
import ctypes as C
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sigcomm_kimjyyh20_b200 import load  # noqa: E402

lib = load()
lib.sr_bench_resblock.restype = C.c_int
lib.sr_bench_resblock.argtypes = [C.c_int] * 5 + [C.c_void_p, C.c_void_p, C.c_void_p]
torch.cuda.init()
st = C.c_void_p(torch.cuda.current_stream().cuda_stream)
peak = json.load(open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                                   "MEASURED_PEAKS.json")))["bf16_tflops"]
for c, n, h, w in ((48, 8, 720, 1280), (32, 4, 540, 960)):  # (32, 30, ...) crashed the host process once: kept small
    ms = C.c_float()
    dbg = np.zeros(16 * 256, dtype=np.int64)
    rc = lib.sr_bench_resblock(c, n, h, w, 10, C.byref(ms), dbg.ctypes.data_as(C.c_void_p), st)
    fl = 2 * 2 * 9 * c * c * n * h * w
    tf = fl / (ms.value * 1e-3) / 1e12
    print(f"resblock C={c} n={n} {h}x{w} rc={rc} {ms.value*1e3:8.1f} us {tf:7.1f} TF/s {100*tf/peak:5.1f}% of burst")
    d = dbg.reshape(16, 256)
    t0 = d[0, 0]
    names = ["f_iss", "E1_iss", "E2_iss", "e1_got", "e1_trow", "e2_got", "e2_store", "mma_st", "acq1", "f_ok",
             "c2_st", "acq2", "t_ok"]
    for i in range(4, 6):
        print("  step %3d " % i + " ".join(f"{nm}={(d[e, i] - t0) if d[e, i] else -1:7d}" for e, nm in enumerate(names)))
    # block hand-off: MMA step st acquires ring-1 block of row st+2, last used by row st-3 (freed by epi1 at index
    # st-3); ring-2 likewise with conv2 rows (conv2 step st handles t row k = st-3, acquires row k+2, freed k-3)
    for st in range(8, 14):
        k = st - 3
        print(f"  step {st:3d}: acq1 wait {d[8, st] - d[7, st]:5d} (freed {d[13, st - 3] - d[7, st]:6d} rel. to step start)"
              f"  acq2 wait {d[11, st] - d[10, st]:5d} (freed {d[14, k - 3] - d[10, st]:6d} rel. to conv2 part start)"
              f"  f wait {d[9, st] - d[8, st]:5d}  t wait {d[12, st] - d[11, st]:5d}")
    for e, nm in enumerate(names[:7]):
        v = d[e, 20:200]
        v = v[v > 0]
        if len(v) > 2:
            print(f"  {nm:12s} mean step interval {np.mean(np.diff(v)):8.1f} cycles")

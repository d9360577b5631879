"""Per-CTA timeline of one wgrad launch (globaltimer stamps) at the training shape (virtual batch 48 x 3200)."""
import ctypes as C
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sigcomm_kimjyyh20_b200 import load  # noqa: E402

lib = load()
lib.sr_bench_wgrad.argtypes = [C.c_void_p] * 2 + [C.c_int] * 6 + [C.c_void_p] * 2 + [C.c_int, C.c_void_p]
st = C.c_void_p(torch.cuda.current_stream().cuda_stream)
H, W = 48, 3200
EXP = int(sys.argv[1]) if len(sys.argv) > 1 else 0
for ci, co in ((48, 48), (16, 48), (48, 32)):
    x = (torch.randn(1, H, W, ci, device="cuda") * 0.1).to(torch.bfloat16)
    dy = (torch.randn(1, H, W, co, device="cuda") * 0.1).to(torch.bfloat16)
    ms = C.c_float(0)
    dbg = np.zeros((148, 8), np.int64)
    rc = lib.sr_bench_wgrad(C.c_void_p(x.data_ptr()), C.c_void_p(dy.data_ptr()), 1, H, W, ci, co, 50,
                            C.byref(ms), dbg.ctypes.data, EXP, st)
    fl = 2 * 9 * ci * co * H * W
    print(f"wgrad {ci}x{co}: rc={rc} {ms.value * 1e3:.1f} us ({fl / ms.value / 1e9:.0f} TF/s) incl. the fused reduction")
    t0 = dbg[:, 0].min()
    d = (dbg - t0) / 1e3
    if EXP & 8:  # batched rolling kernel: slot 1 = reduction done, 2 = first MMA, 3 = MMAs issued
        names = ["entry", "reduced", "first_mma", "mma_issued", "(clock)", "first_done", "drained", "barrier"]
        skip = (4,)
    else:
        names = ["entry", "pdl", "first_full", "mma_issued", "(waited)", "done_bar", "drained", "barrier"]
        skip = (1, 4)
        clk = (dbg[:, 4] - dbg[:, 1]) / (dbg[:, 6] - dbg[:, 0])
        print(f"  SM clock during the launch: med {np.median(clk):.3f} GHz (min {clk.min():.3f}, max {clk.max():.3f})")
    for k, nm in enumerate(names):
        if k not in skip:
            print(f"  {nm:11s} min {d[:, k].min():7.2f} med {np.median(d[:, k]):7.2f} max {d[:, k].max():7.2f} us")

"""Kernel-level conv timing sweep (sr_bench_conv): TFLOP/s and % of the measured sustained bf16 peak."""
import ctypes as C
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sigcomm_kimjyyh20_b200 import load  # noqa: E402

lib = load()
lib.sr_bench_conv.restype = C.c_int
lib.sr_bench_conv.argtypes = [C.c_int] * 7 + [C.c_void_p, C.c_void_p]
torch.cuda.init()
st = C.c_void_p(torch.cuda.current_stream().cuda_stream)
peak = json.load(open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                                   "MEASURED_PEAKS.json")))["bf16_tflops"]
cases = [(48, 48, 8, 720, 1280), (32, 32, 8, 540, 960), (48, 48, 64 * 8, 48, 48), (16, 48, 8, 720, 1280),
         (48, 32, 8, 720, 1280)]
if len(sys.argv) > 1:
    cases = [tuple(int(v) for v in a.split(",")) for a in sys.argv[1:]]
for ci, co, n, h, w in cases:
    for mode, name in ((3, "no-epilogue"), (2, "store-only"), (0, "bias+relu"), (1, "bias+residual"),
                       (10, "ROLL bias+relu"), (11, "ROLL bias+res")):
        ms = C.c_float()
        rc = lib.sr_bench_conv(ci, co, n, h, w, mode, 10, C.byref(ms), st)
        fl = 2 * 9 * ci * co * n * h * w
        tf = fl / (ms.value * 1e-3) / 1e12
        print(f"{ci:3d}->{co:3d} n={n:4d} {h}x{w} {name:14s} rc={rc} {ms.value*1e3:9.1f} us  {tf:7.1f} TF/s "
              f"{100*tf/peak:5.1f}% of {peak} burst", flush=True)

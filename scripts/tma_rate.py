"""TMA load throughput: 16-B-innermost 5-D boxes (the canonical no-swizzle layouts) vs a plain 4-D box."""
import ctypes as C
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sigcomm_kimjyyh20_b200 import load  # noqa: E402

lib = load()
lib.sr_bench_tma.argtypes = [C.c_void_p, C.c_int, C.c_int, C.c_int, C.c_int, C.c_int, C.c_int, C.c_void_p, C.c_void_p]
st = C.c_void_p(torch.cuda.current_stream().cuda_stream)
H, W = 48, 3200
for Cp in (16, 48):
    act = torch.randn(1, H, W, Cp, device="cuda").to(torch.bfloat16)
    units = ((W + 63) // 64) * ((H + 3) // 4)
    for grid in (1, 148):
        for mode in (0, 1, 2):
            ms = C.c_float(0)
            passes = 20 if grid == 148 else 2
            rc = lib.sr_bench_tma(C.c_void_p(act.data_ptr()), H, W, Cp, mode, grid, passes, C.byref(ms), st)
            nbytes = 66 * 6 * Cp * 2 * units * passes * (1 if grid == 148 else 1)
            if grid == 1:
                nbytes = 66 * 6 * Cp * 2 * units * passes
            gbs = nbytes / (ms.value * 1e-3) / 1e9
            print(f"Cp={Cp} grid={grid:3d} mode={mode} rc={rc} {ms.value:8.3f} ms  {gbs:8.1f} GB/s "
                  f"({gbs / (grid if grid > 1 else 1):6.1f} GB/s per CTA)", flush=True)

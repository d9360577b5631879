"""tcgen05.mma rate for the wgrad operand pattern: MN-major SWIZZLE_32B A with a 32-B (one K row) start shift
and/or an atom stride that is not a multiple of 128 B."""
import ctypes as C
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sigcomm_kimjyyh20_b200 import load  # noqa: E402

lib = load()
st = C.c_void_p(torch.cuda.current_stream().cuda_stream)
K, reps = 64, 2000
A = torch.randn(128, K, device="cuda").to(torch.bfloat16)
cyc = torch.zeros(1, dtype=torch.int64, device="cuda")
for shift in (0, 6):
    for N in (16, 48, 144, 256):
        B = torch.randn(N, K, device="cuda").to(torch.bfloat16)
        D = torch.empty(128, N, device="cuda")
        rc = lib.sr_test_mma(C.c_void_p(A.data_ptr()), C.c_void_p(B.data_ptr()), C.c_void_p(D.data_ptr()), N, K, 2,
                             2, reps, shift, C.c_void_p(cyc.data_ptr()), st)
        torch.cuda.synchronize()
        print(f"sw32 shift={shift} N={N:3d} rc={rc} cycles/MMA={cyc.item() / (reps * K // 16 + 1):7.2f}", flush=True)

"""Which LBO/SBO assignment does tcgen05 use for MN-major SWIZZLE_32B operands?  (modes 2 / 3 of sr_test_mma)"""
import ctypes as C
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sigcomm_kimjyyh20_b200 import load  # noqa: E402

lib = load()
st = C.c_void_p(torch.cuda.current_stream().cuda_stream)
for N, K in ((48, 64), (144, 32), (16, 16)):
    A = torch.randn(128, K).to(torch.bfloat16)
    B = torch.randn(N, K).to(torch.bfloat16)
    ref = A.float() @ B.float().T
    Ad, Bd = A.cuda(), B.cuda()
    for am, bm in ((2, 0), (3, 0), (0, 2), (0, 3), (2, 2), (3, 3), (1, 1)):
        D = torch.zeros(128, N, device="cuda")
        rc = lib.sr_test_mma(C.c_void_p(Ad.data_ptr()), C.c_void_p(Bd.data_ptr()),
                             C.c_void_p(D.data_ptr()), N, K, am, bm, 0, 0, None, st)
        torch.cuda.synchronize()
        err = (D.cpu() - ref).abs().max().item()
        print(f"N={N} K={K} a={am} b={bm} rc={rc} maxerr={err:.3g}", flush=True)

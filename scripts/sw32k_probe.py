"""K-major SWIZZLE_32B A operand (the layout the rolling convs' A rows would use): plain and one-row-shifted
starts (the dx tap) against torch matmul."""
import ctypes as C
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sigcomm_kimjyyh20_b200 import load  # noqa: E402

lib = load()
st = C.c_void_p(torch.cuda.current_stream().cuda_stream)
for N, K in ((48, 64), (144, 32), (16, 16)):
    A = torch.randn(128, K).to(torch.bfloat16)
    B = torch.randn(N, K).to(torch.bfloat16)
    Ad, Bd = A.cuda(), B.cuda()
    for shift in (0, 7):
        As = A.float().clone()
        if shift == 7:
            As = torch.cat([A.float()[1:], torch.zeros(1, K)])
        ref = As @ B.float().T
        D = torch.zeros(128, N, device="cuda")
        rc = lib.sr_test_mma(C.c_void_p(Ad.data_ptr()), C.c_void_p(Bd.data_ptr()), C.c_void_p(D.data_ptr()), N, K, 4,
                             0, 0, shift, None, st)
        torch.cuda.synchronize()
        print(f"K-major SW32 N={N} K={K} shift={shift} rc={rc} maxerr={(D.cpu() - ref).abs().max().item():.3g}")

"""tcgen05.mma issue rate for K-major vs MN-major smem operands (M=128, cta_group::1, SS)."""
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
for amn, bmn in ((0, 0), (1, 1), (2, 2)):
    for N in (48, 144):
        B = torch.randn(N, K, device="cuda").to(torch.bfloat16)
        D = torch.empty(128, N, device="cuda")
        rc = lib.sr_test_mma(C.c_void_p(A.data_ptr()), C.c_void_p(B.data_ptr()), C.c_void_p(D.data_ptr()), N, K, amn,
                             bmn, reps, 0, C.c_void_p(cyc.data_ptr()), st)
        torch.cuda.synchronize()
        c = cyc.item() / (reps * K // 16 + 1)
        print(f"a_mn={amn} b_mn={bmn} N={N:3d} rc={rc} cycles/MMA={c:7.2f} floor={128 * N / 256:6.1f}", flush=True)

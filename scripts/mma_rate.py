"""tcgen05.mma (kind::f16, cta_group::1, SS) issue rate vs N at M=128, K=16 per instruction (one CTA)."""
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
for shift in (0, 1, 2):
    for N in (16, 32, 48, 64, 96, 128, 144, 192, 256):
        B = torch.randn(N, K, device="cuda").to(torch.bfloat16)
        D = torch.empty(128, N, device="cuda")
        rc = lib.sr_test_mma(C.c_void_p(A.data_ptr()), C.c_void_p(B.data_ptr()), C.c_void_p(D.data_ptr()), N, K, 0, 0,
                             reps, shift, C.c_void_p(cyc.data_ptr()), st)
        torch.cuda.synchronize()
        n_mma = reps * K // 16 + 1
        c = cyc.item() / n_mma
        floor = 128 * N / 256
        smem_b = (128 * 16 * 2 + N * 16 * 2) / c
        print(f"shift={shift} N={N:3d} rc={rc} cycles/MMA={c:7.2f} floor={floor:6.1f} eff={floor/c:5.2f} "
              f"smem read {smem_b:6.1f} B/clk", flush=True)

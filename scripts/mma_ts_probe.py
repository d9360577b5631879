"""A operand from TMEM (tcgen05.mma ... [a_tmem]): packing check against torch and MMA rate vs SS operands."""
import ctypes as C
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sigcomm_kimjyyh20_b200 import load  # noqa: E402

lib = load()
lib.sr_test_mma_ts.argtypes = [C.c_void_p] * 3 + [C.c_int] * 4 + [C.c_void_p] * 2
st = C.c_void_p(torch.cuda.current_stream().cuda_stream)
cyc = torch.zeros(1, dtype=torch.int64, device="cuda")
for N, K in ((48, 16), (144, 16), (144, 48), (96, 32), (48, 64), (96, 64), (144, 64), (256, 64)):
    A = torch.randn(128, K).to(torch.bfloat16)
    B = torch.randn(N, K).to(torch.bfloat16)
    ref = A.float() @ B.float().T
    Ad, Bd = A.cuda(), B.cuda()  # keep the device copies alive across the calls
    for pack in (0, 1):
        D = torch.zeros(128, N, device="cuda")
        rc = lib.sr_test_mma_ts(C.c_void_p(Ad.data_ptr()), C.c_void_p(Bd.data_ptr()),
                                C.c_void_p(D.data_ptr()), N, K, pack, 0, None, st)
        print(f"TS N={N} K={K} pack={pack} rc={rc} maxerr={(D.cpu() - ref).abs().max().item():.3g}", flush=True)
    reps = 200
    D = torch.zeros(128, N, device="cuda")
    lib.sr_test_mma_ts(C.c_void_p(Ad.data_ptr()), C.c_void_p(Bd.data_ptr()), C.c_void_p(D.data_ptr()),
                       N, K, 0, reps, C.c_void_p(cyc.data_ptr()), st)
    print(f"   rate: {cyc.item() / (reps * K // 16):.1f} cycles per MMA (N={N}; SS floor N/2 = {N / 2})", flush=True)
# layout probe: B = I (N = K = 16): D[m][n] = the A element the MMA reads for (row m, k = n)
N = K = 16
Ad = torch.zeros(128, K).to(torch.bfloat16).cuda()
Bd = torch.eye(16).to(torch.bfloat16).cuda()
for pack, what in ((2, "lane+1 (low +, high -)"), (3, "column+1 (low +, high -)")):
    D = torch.zeros(128, N, device="cuda")
    lib.sr_test_mma_ts(C.c_void_p(Ad.data_ptr()), C.c_void_p(Bd.data_ptr()), C.c_void_p(D.data_ptr()),
                       N, K, pack, 0, None, st)
    print("probe", what)
    Dc = D.cpu()
    for m in (0, 1, 2, 7, 8, 15, 16, 31, 32, 33, 64, 127):
        print(f"  row {m:3d}: " + " ".join(f"{v:5.0f}" for v in Dc[m].tolist()))

"""Isolated tcgen05 MMA rate (one SM, M = 128, K = 64 per iteration, bf16, SS operands) for the A layouts of the
rolling convs: K-major SWIZZLE_NONE (16-B chunk planes, a_mn = 0) vs K-major SWIZZLE_32B (a_mn = 4), B K-major
SWIZZLE_NONE; N = 48 / 96 / 144 (the dy-fold width and the two halves of a ring-wrap step)."""
import ctypes as C, os, sys
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sigcomm_kimjyyh20_b200 import load  # noqa: E402
lib = load()
st = C.c_void_p(torch.cuda.current_stream().cuda_stream)
K, reps = 64, 2000
A = torch.randn(128, K, device="cuda").to(torch.bfloat16)
cyc = torch.zeros(1, dtype=torch.int64, device="cuda")
for a_mn in (0, 4):
    for shift in (0, 3):
        for N in (48, 96, 144, 192):
            B = torch.randn(N, K, device="cuda").to(torch.bfloat16)
            D = torch.empty(128, N, device="cuda")
            rc = lib.sr_test_mma(C.c_void_p(A.data_ptr()), C.c_void_p(B.data_ptr()), C.c_void_p(D.data_ptr()), N, K,
                                 a_mn, 0, reps, shift if a_mn == 4 else (1 if shift else 0), C.c_void_p(cyc.data_ptr()), st)
            torch.cuda.synchronize()
            c = cyc.item() / (reps * K // 16 + 1)
            print(f"a_mn={a_mn} shift={shift} N={N:3d} rc={rc} cycles/MMA={c:7.2f} floor={128 * N / 256:6.1f} "
                  f"smem {(4096 + 32 * N) / c:6.1f} B/clk", flush=True)

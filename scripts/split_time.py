"""k_resblock_split timing (8 x 720p, C = 48 and 16) for build A/Bs: scripts/ab_variants.sh <reps> scripts/split_time.py <names>"""
import ctypes as C, os, sys
import numpy as np, torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sigcomm_kimjyyh20_b200 import load  # noqa: E402
os.environ["SR_BLOCK_SPLIT"] = os.environ.get("SR_BLOCK_SPLIT", "1")
lib = load()
lib.sr_bench_resblock.restype = C.c_int
lib.sr_bench_resblock.argtypes = [C.c_int] * 5 + [C.c_void_p, C.c_void_p, C.c_void_p]
st = C.c_void_p(torch.cuda.current_stream().cuda_stream)
out = []
for c in (48, 16):
    t = []
    for _ in range(5):
        ms = C.c_float()
        rc = lib.sr_bench_resblock(c, 8, 720, 1280, 10, C.byref(ms), None, st)
        t.append(ms.value * 1e3)
    out.append(f"C={c} rc={rc} {np.median(t):7.1f} us")
print(sys.argv[1] if len(sys.argv) > 1 else "", "  ".join(out), flush=True)

"""k_resblock inference timing per instantiation (GEN 0 = inference-specialised, 1/2 = runtime extras, all null):
sr_bench_resblock without stamps, median of 5 x 10 launches."""
import ctypes as C, os, sys
import numpy as np, torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sigcomm_kimjyyh20_b200 import load
lib = load()
lib.sr_bench_resblock.restype = C.c_int
lib.sr_bench_resblock.argtypes = [C.c_int] * 5 + [C.c_void_p, C.c_void_p, C.c_void_p]
st = C.c_void_p(torch.cuda.current_stream().cuda_stream)
for rep in range(2):
    for c, n, h, w in ((48, 8, 720, 1280), (16, 8, 720, 1280)):
        for g in (0, 1, 2):
            lib.sr_test_block_gen(g)
            t = []
            for _ in range(5):
                ms = C.c_float()
                rc = lib.sr_bench_resblock(c, n, h, w, 10, C.byref(ms), None, st)
                t.append(ms.value * 1e3)
            print(f"C={c} gen={g} rc={rc} median {np.median(t):8.1f} us")
lib.sr_test_block_gen(-1)

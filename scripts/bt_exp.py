"""Bodytail experiment masks (conv_bodytail.cu BtArgs::exp): event-timed 8 x 720p x3 launch per mask."""
import ctypes as C, os, sys
import numpy as np, torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sigcomm_kimjyyh20_b200 import load
lib = load()
lib.sr_bench_bodytail_dbg.restype = C.c_int
lib.sr_bench_bodytail_dbg.argtypes = [C.c_int] * 5 + [C.c_void_p, C.c_void_p, C.c_void_p]
st = C.c_void_p(torch.cuda.current_stream().cuda_stream)
for rep in range(2):
    for m in [int(x) for x in (sys.argv[1:] or ["0", "1", "2", "3", "4", "7", "8", "15"])]:
        lib.sr_test_bt_exp(m)
        dbg = np.zeros(16 * 256, np.int64); ms = C.c_float()
        t = []
        for _ in range(5):
            rc = lib.sr_bench_bodytail_dbg(48, 3, 8, 720, 1280, dbg.ctypes.data_as(C.c_void_p), C.byref(ms), st)
            t.append(ms.value * 1e3)
        d = dbg.reshape(16, 256)
        iv = np.diff(d[6, 10:100][d[6, 10:100] > 0]).mean()
        print(f"exp={m:2d} rc={rc} median {np.median(t):7.1f} us  row-step {iv:7.1f} cyc")
lib.sr_test_bt_exp(0)

"""Event-timed k_bodytail<48,32,3> launches (8 x 720p, x3) through sr_bench_bodytail_dbg: median of 15."""
import ctypes as C, os, sys
import numpy as np, torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sigcomm_kimjyyh20_b200 import load
lib = load()
lib.sr_bench_bodytail_dbg.restype = C.c_int
lib.sr_bench_bodytail_dbg.argtypes = [C.c_int] * 5 + [C.c_void_p, C.c_void_p, C.c_void_p]
st = C.c_void_p(torch.cuda.current_stream().cuda_stream)
dbg = np.zeros(16 * 256, np.int64); ms = C.c_float()
t = []
for _ in range(15):
    rc = lib.sr_bench_bodytail_dbg(48, 3, 8, 720, 1280, None if os.environ.get('NODBG') else dbg.ctypes.data_as(C.c_void_p),
                                   C.byref(ms), st)
    t.append(ms.value * 1e3)
print(f"{sys.argv[1] if len(sys.argv) > 1 else ''} rc={rc} median {np.median(t):7.1f} us  min {min(t):7.1f}")

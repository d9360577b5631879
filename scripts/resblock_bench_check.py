"""sr_bench_resblock smoke at C = 32 (the case scripts/bench_block.py crashed on), with and without the timeline."""
import ctypes as C, os, sys
import numpy as np, torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sigcomm_kimjyyh20_b200 import load
lib = load(); lib.sr_bench_resblock.restype = C.c_int
lib.sr_bench_resblock.argtypes = [C.c_int] * 5 + [C.c_void_p, C.c_void_p, C.c_void_p]
torch.cuda.init(); st = C.c_void_p(torch.cuda.current_stream().cuda_stream)
ms = C.c_float()
print("rc", lib.sr_bench_resblock(32, 4, 540, 960, 2, C.byref(ms), None, st), ms.value, flush=True)
dbg = np.zeros(16 * 256, dtype=np.int64)
print("rc", lib.sr_bench_resblock(32, 4, 540, 960, 2, C.byref(ms), dbg.ctypes.data_as(C.c_void_p), st), ms.value, flush=True)

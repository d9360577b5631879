"""CTA-0 clock64 timeline of one rolling up-conv + tail launch (8 x 720p, x3, 48 -> 27(32) channels)."""
import ctypes as C, os, sys
import numpy as np, torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sigcomm_kimjyyh20_b200 import load
lib = load()
lib.sr_bench_roll_tail_dbg.restype = C.c_int
lib.sr_bench_roll_tail_dbg.argtypes = [C.c_int] * 5 + [C.c_void_p, C.c_void_p, C.c_void_p]
st = C.c_void_p(torch.cuda.current_stream().cuda_stream)
s = int(sys.argv[1]) if len(sys.argv) > 1 else 3
dbg = np.zeros(16 * 256, np.int64); ms = C.c_float()
rc = lib.sr_bench_roll_tail_dbg(48, s, 8, 720, 1280, dbg.ctypes.data_as(C.c_void_p), C.byref(ms), st)
d = dbg.reshape(16, 256); t0 = d[8, 0]
print(f"x{s} rc={rc} {ms.value*1e3:.1f} us; setup+pdl {d[10,0]-t0}, exit {d[9,0]-t0}")
names = ["in_iss", "mma_st", "acq", "in_ok", "mma_iss", "ep_got", "ep_drained", "ep_done"]
for i in range(20, 30):
    print("  %3d " % i + " ".join(f"{nm}={(d[e, i] - t0) if d[e, i] else -1:7d}" for e, nm in enumerate(names)))
for e, nm in enumerate(names):
    v = d[e, 10:200]; v = v[v > 0]
    if len(v) > 2: print(f"  {nm:10s} interval {np.mean(np.diff(v)):7.1f}")
for lo, hi, nm in ((2, 1, "acq wait"), (3, 2, "in wait"), (4, 3, "issue"), (6, 5, "drain"), (7, 6, "epi")):
    a, b = d[lo, 10:200], d[hi, 10:200]; m = (a > 0) & (b > 0)
    print(f"  {nm:10s} mean {np.mean(a[m] - b[m]):7.1f}")

"""CTA-0 clock64 timeline of one fused body + up conv + tail launch (8 x 720p, x3, C = 48)."""
import ctypes as C, os, sys
import numpy as np, torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sigcomm_kimjyyh20_b200 import load
lib = load()
lib.sr_bench_bodytail_dbg.restype = C.c_int
lib.sr_bench_bodytail_dbg.argtypes = [C.c_int] * 5 + [C.c_void_p, C.c_void_p, C.c_void_p]
st = C.c_void_p(torch.cuda.current_stream().cuda_stream)
s = int(sys.argv[1]) if len(sys.argv) > 1 else 3
dbg = np.zeros(16 * 256, np.int64); ms = C.c_float()
rc = lib.sr_bench_bodytail_dbg(48, s, 8, 720, 1280, dbg.ctypes.data_as(C.c_void_p), C.byref(ms), st)
d = dbg.reshape(16, 256)
t0 = d[0, 0]
print(f"x{s} rc={rc} {ms.value*1e3:.1f} us")
names = {0: "f_iss", 7: "c1_st", 8: "c1_acq", 9: "c1_fok", 1: "c1_iss", 10: "c2_st", 11: "c2_acq", 12: "c2_tok",
         2: "c2_iss", 3: "e1_got", 4: "e1_done", 5: "e2_got", 13: "e2_lrw", 14: "e2_lrok", 6: "e2_done"}
for i in range(20, 28):
    print("  %3d " % i + " ".join(f"{nm}={(d[e, i] - t0) if d[e, i] else -1:7d}" for e, nm in names.items()))
for e, nm in names.items():
    v = d[e, 10:200]; v = v[v > 0]
    if len(v) > 2: print(f"  {nm:8s} interval {np.mean(np.diff(v)):7.1f}")
for hi, lo, nm in ((8, 7, "c1 acq wait"), (9, 8, "c1 f wait"), (1, 9, "c1 issue"), (11, 10, "c2 acq wait"),
                   (12, 11, "c2 t wait"), (2, 12, "c2 issue"), (4, 3, "e1 row"), (13, 5, "e2 drain"),
                   (14, 13, "e2 lr wait"), (6, 14, "e2 tail+copy")):
    a, b = d[hi, 10:200], d[lo, 10:200]; m = (a > 0) & (b > 0)
    print(f"  {nm:12s} mean {np.mean(a[m] - b[m]):7.1f}")

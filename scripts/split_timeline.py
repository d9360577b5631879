"""CTA-pair-0 clock64 timeline of k_resblock_split (8 x 720p): per-event steady-state intervals and waits.
rank 0: 0 f TMA issued, 1 conv1 step start, 2 ring blocks acquired, 3 f row landed, 4 epi1 got row, 5 t copy issued
rank 1: 1 conv2 step start, 2 blocks acquired, 3 t row landed, 4 epi2 got row, 5 store issued."""
import ctypes as C, os, sys
import numpy as np, torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sigcomm_kimjyyh20_b200 import load  # noqa: E402
os.environ["SR_BLOCK_SPLIT"] = "1"
lib = load()
lib.sr_bench_resblock.restype = C.c_int
lib.sr_bench_resblock.argtypes = [C.c_int] * 5 + [C.c_void_p, C.c_void_p, C.c_void_p]
st = C.c_void_p(torch.cuda.current_stream().cuda_stream)
for c in (48, 16):
    dbg = np.zeros(16 * 256, np.int64)
    ms = C.c_float()
    rc = lib.sr_bench_resblock(c, 8, 720, 1280, 3, C.byref(ms), dbg.ctypes.data_as(C.c_void_p), st)
    d = dbg.reshape(16, 256)
    print(f"C={c} rc={rc} {ms.value * 1e3:.1f} us")
    for rk in (0, 1):
        for e in range(6):
            v = d[rk * 8 + e, 140:250]
            v = v[v > 0]
            if len(v) > 4:
                print(f"  r{rk} ev{e} interval {np.mean(np.diff(v)):8.1f}")
        for hi, lo, nm in ((2, 1, "acq wait"), (3, 2, "input wait"), (5, 4, "epi row")):
            a, b = d[rk * 8 + hi, 140:250], d[rk * 8 + lo, 140:250]
            m = (a > 0) & (b > 0)
            if m.sum() > 4:
                print(f"  r{rk} {nm:10s} mean {np.mean(a[m] - b[m]):8.1f}")

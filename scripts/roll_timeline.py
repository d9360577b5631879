import ctypes as C, os, sys
import numpy as np, torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sigcomm_kimjyyh20_b200 import load
lib = load()
lib.sr_bench_roll_dbg.restype = C.c_int
lib.sr_bench_roll_dbg.argtypes = [C.c_int] * 6 + [C.c_void_p, C.c_void_p, C.c_void_p]
st = C.c_void_p(torch.cuda.current_stream().cuda_stream)
CI, CO = (int(sys.argv[1]), int(sys.argv[2])) if len(sys.argv) > 2 else (48, 48)
for res in (0, 1):
    dbg = np.zeros(16 * 256, np.int64); ms = C.c_float()
    rc = lib.sr_bench_roll_dbg(CI, CO, 8, 720, 1280, res, dbg.ctypes.data_as(C.c_void_p), C.byref(ms), st)
    d = dbg.reshape(16, 256); t0 = d[0, 0]
    print(f"res={res} rc={rc} {ms.value*1e3:.1f} us")
    names = ["in_iss", "mma_st", "acq", "in_ok", "mma_iss", "ep_got", "ep_drained", "ep_stored"]
    for i in range(6, 14):
        print("  %3d " % i + " ".join(f"{nm}={(d[e, i] - t0) if d[e, i] else -1:7d}" for e, nm in enumerate(names)))
    a_, b_ = d[11, 10:40], d[6, 10:40]; m_ = (a_ > 0) & (b_ > 0)
    if m_.any(): print(f"  o_free wait mean {np.mean(a_[m_] - b_[m_]):7.1f}  pack+sts {np.mean(d[12,10:40][m_] - a_[m_]):7.1f}"
                       f"  fence {np.mean(d[13,10:40][m_] - d[12,10:40][m_]):7.1f}  arrive {np.mean(d[7,10:40][m_] - d[13,10:40][m_]):7.1f}")
    for e, nm in enumerate(names):
        v = d[e, 10:40]; v = v[v > 0]
        if len(v) > 2: print(f"  {nm:10s} interval {np.mean(np.diff(v)):7.1f}")

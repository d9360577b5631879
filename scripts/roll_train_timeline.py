"""CTA-0 timeline (clock64) of one rolling conv launch at the training virtual-batch shape (1 x 48 x 3200): entry,
setup, per-input-row TMA issue / MMA / epilogue events, exit.  Where the ~20 us of a training conv go."""
import ctypes as C
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sigcomm_kimjyyh20_b200 import load  # noqa: E402

lib = load()
lib.sr_bench_roll_dbg.restype = C.c_int
lib.sr_bench_roll_dbg.argtypes = [C.c_int] * 6 + [C.c_void_p, C.c_void_p, C.c_void_p]
st = C.c_void_p(torch.cuda.current_stream().cuda_stream)
# GRID=n: n CTAs (the bench's training partition has 40 SMs); PART=n: run on an n-SM green-context partition
grid = int(os.environ.get("GRID", "0"))
if grid:
    lib.sr_test_grid_cap(grid)
if os.environ.get("PART"):
    from paper_conf_sigcomm_kimjyyh20_b200 import SRContext  # noqa: E402
    _, pst, _, _ = SRContext.sm_partition(int(os.environ["PART"]))
    st = C.c_void_p(pst.cuda_stream)
shapes = ((1, 48, 3200),) if os.environ.get("TRAIN_ONLY") else ((1, 48, 3200), (8, 720, 1280))
for shape in shapes:
    for res in (0, 1, 2):
        dbg = np.zeros(16 * 256, np.int64)
        ms = C.c_float()
        lib.sr_bench_roll_dbg(48, 48, *shape, res, dbg.ctypes.data_as(C.c_void_p), C.byref(ms), st)  # warm
        rc = lib.sr_bench_roll_dbg(48, 48, *shape, res, dbg.ctypes.data_as(C.c_void_p), C.byref(ms), st)
        d = dbg.reshape(16, 256)
        t0 = d[8, 0]
        print(f"shape={shape} res={res} rc={rc} event-timed {ms.value * 1e3:.1f} us; CTA-0 cycles from entry:")
        print(f"  setup+pdl done {d[10, 0] - t0}, exit {d[9, 0] - t0}")
        names = {0: "in_iss", 1: "mma_st", 2: "acq", 3: "in_ok", 4: "mma_iss", 5: "ep_got", 6: "ep_drained",
                 11: "ep_slot", 12: "ep_staged", 13: "ep_fenced", 7: "ep_stored"}
        for i in range(0, 12):
            print("  %3d " % i + " ".join(f"{nm}={(d[e, i] - t0) if d[e, i] else -1:7d}" for e, nm in names.items()))

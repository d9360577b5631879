"""Fused residual block (C=48, 8 x 720p) under the k_resblock benchmarking experiments: which parts bound it.
exp bits: 1 no residual load, 2 no output store, 4 no t smem write, 8 no bias re-arm, 16 no conv2 MMAs,
32 no conv1 MMAs, 64 no accumulator loads, 128 no f-row TMA after the first piece (results wrong when set)."""
import ctypes as C
import os
import subprocess
import sys

if len(sys.argv) > 1:
    import torch
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    from paper_conf_sigcomm_kimjyyh20_b200 import load  # noqa: E402
    lib = load()
    lib.sr_bench_resblock.argtypes = [C.c_int] * 5 + [C.c_void_p, C.c_void_p, C.c_void_p]
    st = C.c_void_p(torch.cuda.current_stream().cuda_stream)
    ms = C.c_float()
    lib.sr_bench_resblock(48, 8, 720, 1280, 10, C.byref(ms), None, st)
    fl = 2 * 2 * 9 * 48 * 48 * 8 * 720 * 1280
    print(f"exp={os.environ.get('SR_BLOCK_EXP', '0'):>4s} {ms.value * 1e3:8.1f} us  {fl / ms.value / 1e9:7.1f} TF/s"
          f"  ({sys.argv[1]})", flush=True)
else:
    for exp, what in ((0, "full"), (1, "no residual"), (2, "no store"), (4, "no t write"), (8, "no re-arm"),
                      (64, "no acc loads"), (16, "no conv2 MMA"), (32, "no conv1 MMA"), (48, "no MMAs"),
                      (128, "no f TMA"), (1 | 2 | 4 | 8 | 64 | 128, "MMAs only"), (7, "no res/store/t"),
                      (16 | 32 | 128, "no MMA, no f TMA")):
        subprocess.run([sys.executable, __file__, what], env=dict(os.environ, SR_BLOCK_EXP=str(exp)))

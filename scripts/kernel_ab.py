"""One-line timing of the hot kernels for build A/Bs (scripts/ab_variants.sh --cmd): k_resblock<48> (8 x 720p),
k_bodytail<48,32,3> (8 x 720p, no stamps), inference of 30 x 720p -> 4K, and the graph-replayed training
iteration (64 patches 48 -> 144, x3 8x48) on the whole GPU."""
import ctypes as C, os, sys
import numpy as np, torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sigcomm_kimjyyh20_b200 import SRContext, load  # noqa: E402
from synth import synth_frames, synth_patch_pool  # noqa: E402
lib = load()
st = C.c_void_p(torch.cuda.current_stream().cuda_stream)
lib.sr_bench_resblock.restype = C.c_int
lib.sr_bench_resblock.argtypes = [C.c_int] * 5 + [C.c_void_p, C.c_void_p, C.c_void_p]
lib.sr_bench_bodytail_dbg.restype = C.c_int
lib.sr_bench_bodytail_dbg.argtypes = [C.c_int] * 5 + [C.c_void_p, C.c_void_p, C.c_void_p]
out = {}
t = []
for _ in range(5):
    ms = C.c_float()
    lib.sr_bench_resblock(48, 8, 720, 1280, 10, C.byref(ms), None, st)
    t.append(ms.value * 1e3)
out["resblock48_us"] = np.median(t)
t = []
for _ in range(9):
    ms = C.c_float()
    lib.sr_bench_bodytail_dbg(48, 3, 8, 720, 1280, None, C.byref(ms), st)
    t.append(ms.value * 1e3)
out["bodytail_us"] = np.median(t)
ctx = SRContext(3, 8, 48, seed=0)
lr = torch.from_numpy(synth_frames(30, 720, 1280, seed=1003)).cuda()
hr = torch.empty((30, 2160, 3840, 3), dtype=torch.uint8, device="cuda")
for _ in range(2):
    ctx.infer(lr, "serve", out=hr)
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(5):
    ctx.infer(lr, "serve", out=hr)
e1.record()
torch.cuda.synchronize()
out["infer30_ms"] = e0.elapsed_time(e1) / 5
plr, phr, _ = synth_patch_pool(256, 3, 180, seed=1, frame_hw=(540, 900))
ctx.pool_push(torch.from_numpy(plr).cuda(), torch.from_numpy(phr).cuda())
loss = torch.zeros(1, device="cuda")
ctx.train_sampled(3, 64, 48, loss)
torch.cuda.synchronize()
e0.record()
ctx.train_sampled(50, 64, 48, loss)
e1.record()
torch.cuda.synchronize()
out["train_iter_ms"] = e0.elapsed_time(e1) / 50
print(sys.argv[1] if len(sys.argv) > 1 else "", " ".join(f"{k}={v:.4g}" for k, v in out.items()), flush=True)

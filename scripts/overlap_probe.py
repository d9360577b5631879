"""Do two streams of our kernels overlap under an SM split?  Big inference on stream A with (a) small inferences,
(b) the training graph on stream B; step time vs the parts alone."""
import os, sys
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench as B
from paper_conf_sigcomm_kimjyyh20_b200 import SRContext
from synth import synth_frames

dev = torch.device("cuda")
lr = torch.from_numpy(synth_frames(B.FRAMES, B.LR_H, B.LR_W, seed=1003)).to(dev)
hr = torch.empty((B.FRAMES, B.S * B.LR_H, B.S * B.LR_W, 3), dtype=torch.uint8, device=dev)
small = torch.from_numpy(synth_frames(2, 720, 1280, seed=5)).to(dev)
ctx_a = SRContext(B.S, B.BLOCKS, B.CH, seed=0)
ctx_b = SRContext(B.S, B.BLOCKS, B.CH, seed=0)
K = int(sys.argv[1]) if len(sys.argv) > 1 else 32
ctx_a.set_sm_split(K)        # ctx_a inference: 148-K SMs
ctx_b.set_sm_split(148 - K)  # ctx_b inference: K SMs
sa, sb = torch.cuda.Stream(), torch.cuda.Stream()
def ta():
    with torch.cuda.stream(sa):
        ctx_a.infer(lr, "serve", out=hr)
def tb():
    with torch.cuda.stream(sb):
        for _ in range(4):
            ctx_b.infer(small, "serve")
def timed(fns, n=4):
    for f in fns: f()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(sa); sb.wait_stream(sa)
    for _ in range(n):
        for f in fns: f()
    sa.wait_stream(sb); e1.record(sa); torch.cuda.synchronize()
    return e0.elapsed_time(e1) / n
print(f"K={K}: A alone {timed([ta]):.3f} ms, B alone {timed([tb]):.3f} ms, A+B {timed([ta, tb]):.3f} ms", flush=True)

import numpy as np, torch, sys
sys.path.insert(0, "/root/repo")
from paper_conf_sigcomm_kimjyyh20_b200 import SRContext
from synth import synth_frames
for (s,B,C,n,h,w) in ((2,1,8,2,90,600),(2,1,48,2,90,600),(2,1,32,2,90,600),(2,1,32,1,45,301),(2,1,32,1,300,130),(2,1,32,1,20,1000)):
    ctx = SRContext(s, B, C, seed=0)
    lr, _ = synth_frames(n, h, w, seed=5, scale=s)
    x = torch.from_numpy(lr).cuda()
    ctx.set_fusion(True); a = ctx.infer(x, "serve").cpu().numpy().astype(int)
    ctx.set_fusion(False); b = ctx.infer(x, "serve").cpu().numpy().astype(int)
    d = np.abs(a-b).max(axis=-1)
    print(s,B,C,n,h,w,"max", d.max(), "count>2", (d>2).sum(), flush=True)
    if d.max() > 2:
        ys, xs = np.nonzero(d[0] > 2)
        print(" rows(LR)", sorted(set((ys//s).tolist()))[:40])
        print(" cols(LR)", sorted(set((xs//s).tolist()))[:60])

import sys, os, torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sigcomm_kimjyyh20_b200 import SRContext
from synth import synth_patch_pool
s, B, C = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3])
n, p, pp = int(sys.argv[4]), int(sys.argv[5]), int(sys.argv[6])
ctx = SRContext(s, B, C, seed=0)
plr, phr, _ = synth_patch_pool(max(n, 8), s, s * pp, seed=1, frame_hw=(s * pp * 2, s * pp * 4))
ctx.pool_push(torch.from_numpy(plr).cuda(), torch.from_numpy(phr).cuda())
lr, hr, idx = ctx.sample_batch(0, n, p)
torch.cuda.synchronize(); print("sample ok", flush=True)
loss = torch.zeros(1, device="cuda")
ctx.train_grad(lr, hr, loss)
torch.cuda.synchronize(); print("train_grad ok", loss.item(), flush=True)

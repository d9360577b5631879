"""k_conv_chain timeline at the training shape (x3 8x48, 64 x 48x48 -> 1 x 48 x 3200): per (CTA, layer) globaltimer
stamps (sr_test_chain_dbg) of one eager training step; prints per-layer spans across the grid."""
import ctypes as C, os, sys
import numpy as np, torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sigcomm_kimjyyh20_b200 import SRContext, load
from synth import synth_patch_pool

lib = load()
lib.sr_test_chain_dbg.argtypes = [C.c_void_p]
ctx = SRContext(3, 8, 48, seed=0)
plr, phr, _ = synth_patch_pool(64, 3, 144, seed=3, frame_hw=(540, 900))
lr, hr = torch.from_numpy(plr).cuda(), torch.from_numpy(phr).cuda()
loss = torch.zeros(1, device="cuda")
for _ in range(3):
    ctx.train_grad(lr, hr, loss)
torch.cuda.synchronize()
G = torch.cuda.get_device_properties(0).multi_processor_count
dbg = torch.zeros(G * 20 * 8 + 20 * 64 * 4, dtype=torch.int64, device="cuda")
lib.sr_test_chain_dbg(C.c_void_p(dbg.data_ptr()))
ctx.train_grad(lr, hr, loss)   # the stamps of the last chain launch (the data-gradient chain) survive
torch.cuda.synchronize()
lib.sr_test_chain_dbg(None)
dall = dbg.cpu().numpy().astype(np.float64)
d = dall[:G * 160].reshape(G, 20, 8)
rr = dall[G * 160:].reshape(20, 64, 4)
nl = int((d[0, :, 2] > 0).sum())
t0 = d[:, 0, 5][d[:, 0, 5] > 0].min()
names = ["flags_ok", "mma_first", "mma_last", "st_issued", "published", "w_issued"]
print(f"grid {G}, layers {nl}; times in us from the first weight issue")
for l in range(nl):
    row = []
    for k in (5, 0, 1, 2, 3, 4):
        v = (d[:, l, k] - t0) / 1e3
        row.append(f"{names[k]} {v.min():7.2f}/{np.median(v):7.2f}/{v.max():7.2f}")
    print(f"L{l:2d} " + "  ".join(row))
pub = d[:, :nl, 4]
print("per-layer span (max published l - max published l-1):",
      " ".join(f"{(pub[:, l].max() - pub[:, l - 1].max()) / 1e3:.2f}" for l in range(1, nl)))
first = d[:, :nl, 0]
print("median (flags_ok l - published l-1 own):", " ".join(f"{np.median(first[:, l] - pub[:, l-1]) / 1e3:.2f}" for l in range(1, nl)))
print("median compute (published l - flags_ok l):", " ".join(f"{np.median(pub[:, l] - first[:, l]) / 1e3:.2f}" for l in range(1, nl)))
print("median mma span (mma_last - mma_first):", " ".join(f"{np.median(d[:, l, 2] - d[:, l, 1]) / 1e3:.2f}" for l in range(nl)))
print("median drain (published - mma_last):", " ".join(f"{np.median(d[:, l, 4] - d[:, l, 2]) / 1e3:.2f}" for l in range(nl)))
print("median flags->mma_first:", " ".join(f"{np.median(d[:, l, 1] - d[:, l, 0]) / 1e3:.2f}" for l in range(1, nl)))
print("median store-warp cycles in bulk_wait<3> per layer:", " ".join(f"{np.median(d[:, l, 6]):.0f}" for l in range(nl)))
print("median store-warp cycles in publish fences per layer:", " ".join(f"{np.median(d[:, l, 7]):.0f}" for l in range(nl)))

cta = int(os.environ.get("SR_CHAIN_DBG_CTA", "0"))
print(f"CTA {cta}: per-row stamps (us from the layer's first input issue): in_issue / mma / ep_drain / store")
for l in range(min(nl, 5)):
    t = rr[l]
    base_t = t[0, 0]
    rows = [i for i in range(64) if t[i, 0] > 0 or t[i, 1] > 0 or t[i, 2] > 0 or t[i, 3] > 0]
    print(f" L{l}: " + "  ".join(
        f"{i}:" + "/".join(f"{(t[i, k] - base_t) / 1e3:.1f}" if t[i, k] > 0 else "-" for k in range(4)) for i in rows))

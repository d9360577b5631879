"""Training iteration (x3 8x48, 64 x 48x48) confined to a green-context SM partition of N SMs (sr_sm_partition +
sr_set_sm_split): graph-replay ms per iteration and the eager per-kernel-class CUDA-event breakdown."""
import os, sys
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sigcomm_kimjyyh20_b200 import SRContext
from synth import synth_patch_pool

fusion = int(os.environ.get("SR_FUSION", "1"))
for n in [int(x) for x in sys.argv[1:]] or [40, 32]:
    ctx = SRContext(3, 8, 48, seed=0)
    ctx.set_fusion(fusion)
    s_inf, s_tr, n_inf, n_tr = SRContext.sm_partition(n)
    ctx.set_sm_split(n_tr)
    dev = torch.device("cuda")
    plr, phr, _ = synth_patch_pool(256, 3, 180, seed=1004, frame_hw=(1080, 1800))
    with torch.cuda.stream(s_tr):
        ctx.pool_push(torch.from_numpy(plr).to(dev), torch.from_numpy(phr).to(dev), stream=s_tr)
        loss = torch.zeros(1, device=dev)
        ctx.train_sampled(3, 64, 48, loss, stream=s_tr)
    s_tr.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with torch.cuda.stream(s_tr):
        e0.record(s_tr)
        ctx.train_sampled(20, 64, 48, loss, stream=s_tr)
        e1.record(s_tr)
    s_tr.synchronize()
    ms = e0.elapsed_time(e1) / 20
    blr = torch.empty((64, 48, 48, 3), dtype=torch.uint8, device=dev)
    bhr = torch.empty((64, 144, 144, 3), dtype=torch.uint8, device=dev)
    bidx = torch.empty(64, dtype=torch.int32, device=dev)
    ctx.kernel_timing(True)
    with torch.cuda.stream(s_tr):
        for i in range(5):
            ctx.sample_batch(-1, 64, 48, out=(blr, bhr, bidx), stream=s_tr)
            ctx.train_grad(blr, bhr, loss, stream=s_tr)
            ctx.train_apply(1.0, stream=s_tr)
    s_tr.synchronize()
    st = ctx.kernel_stats()
    tot = sum(v["ms"] for v in st.values())
    print(f"fusion={fusion} train_sms={n_tr}: graph {ms:.3f} ms/iter; eager per iter {tot / 5:.3f} ms: " +
          ", ".join(f"{k} {v['ms'] / 5 * 1e3:.0f}us" for k, v in sorted(st.items(), key=lambda kv: -kv[1]["ms"])))
    ctx.set_sm_split(0)
    del ctx
    SRContext.sm_partition_release()

"""GPU parity of exactly what bench.py times, at the bench's sizes, against the fp64 oracle (through the C ABI).

* The training iteration the bench replays (sr_train_sampled: one captured CUDA graph of sample + gather from the
  device pool view and step counter -> forward -> loss -> backward -> [allreduce] -> Adam with the device step count)
  at the bench config (x3, 8 blocks x 48 ch, batch 64, 48x48 LR patches from a pool of 60x60 LR entries), replayed
  K = 3 times with a patch push and a publish in between: every step's gradient (oracle at the GPU's own parameters,
  rel L2 <= 1e-2), loss, Adam state (oracle Adam from the GPU's state and gradient) and the whole oracle chain from
  the same start (params rel L2 <= 1e-3 after K steps; north-star bars).
* The same iteration composed from the public calls inside a caller's torch CUDA graph (sample_batch(-1) +
  train_grad + train_allreduce + train_apply_dev): sampled indices bit-exact, including patches pushed after capture.
* Whole-frame inference: one 720p frame x3 8x48 element-wise (|du8| <= 2, PSNR within 0.05 dB) and frame 29 of the
  bench's 30-frame batch bit-identical to the frame inferred alone (offsets > 2^31 bytes in the activations).
* The paper's own 120-px HR training patch (LR 60 at x2, 40 at x3).
* The other BASELINE configs at their own sizes: config 2 (x2 8x32, a whole 540p frame element-wise + frame 29 of a
  30-frame batch), config 5 (x2 8x48 1080p: a band of the whole-frame output against the oracle on the band + halo),
  config 4's second net (x2 8x32, 64 x 48x48: gradient and Adam step).
"""
import numpy as np
import pytest
import torch

import oracle as O
from synth import init_params, synth_frames, synth_patch_pool
from tests.helpers import psnr, rel_l2

pytestmark = pytest.mark.gpu

S, B, C = 3, 8, 48          # bench net (BASELINE config 3/4)
BATCH, P, PP = 64, 48, 60   # bench batch, LR patch, pool LR entry (crop offsets 0..12)


def _ctx(s, b, c, **kw):
    from paper_conf_sigcomm_kimjyyh20_b200 import SRContext
    return SRContext(s, b, c, **kw)


def _oracle_batch(seed, step, lrp, hrp, batch, p, s):
    idx, oy, ox = O.sample_indices(seed, step, lrp.shape[0], batch, lrp.shape[1], p)
    lr, hr = O.gather_patches(lrp, hrp, idx, oy, ox, p, s)
    return idx, lr, hr


def test_bench_training_graph_matches_oracle_chain():
    """sr_train_sampled at the bench config, K = 3 graph replays (Adam, batch 64, lr 1e-4)."""
    seed = 11
    ctx = _ctx(S, B, C, seed=seed)
    lrp, hrp, _ = synth_patch_pool(200, S, S * PP, seed=1004, frame_hw=(1080, 1800))
    extra_lr, extra_hr, _ = synth_patch_pool(40, S, S * PP, seed=1005, frame_hw=(1080, 1800))
    ctx.pool_push(torch.from_numpy(lrp).cuda(), torch.from_numpy(hrp).cuda())
    p0 = ctx.get_params("train").astype(np.float64)
    loss = torch.zeros(1, device="cuda")
    st = torch.cuda.Stream()
    pool_lr, pool_hr = lrp, hrp
    chain_p, chain_m, chain_v = p0.copy(), np.zeros_like(p0), np.zeros_like(p0)
    p_prev = p0
    m_prev, v_prev = np.zeros_like(p0), np.zeros_like(p0)
    launches = []
    for k in range(1, 4):
        l0 = ctx.launches
        with torch.cuda.stream(st):
            ctx.train_sampled(1, BATCH, P, loss)   # k = 1: eager + capture; k >= 2: graph replay
        st.synchronize()
        launches.append(ctx.launches - l0)
        g = ctx.grad_buffer().cpu().numpy().astype(np.float64)  # w_r g_r (w_r = 1), kept after Adam
        p_k = ctx.get_params("train").astype(np.float64)
        m_k, v_k, t_k = ctx.adam_state()
        assert t_k == k
        # the batch the device sampled at step k-1 from the pool as it stood (device pool view + step counter)
        _, blr, bhr = _oracle_batch(seed, k - 1, pool_lr, pool_hr, BATCH, P, S)
        # (a) gradient + loss at the GPU's own parameters (north-star gradient bar)
        ref_loss, ref_g = O.train_loss_and_grad(p_prev, blr, bhr, S, B, C)
        assert abs(loss.item() - ref_loss) / ref_loss < 1e-2, (k, loss.item(), ref_loss)
        assert rel_l2(g, ref_g) < 1e-2, (k, rel_l2(g, ref_g))
        # (b) the Adam update itself: oracle Adam from the GPU's state with the GPU's gradient, t = k
        # (fp32 state: beta2 = 0.999 is not representable, so 1 - beta2 carries a 1.3e-5 relative error into v)
        rp, rm, rv = O.adam_step(p_prev, m_prev, v_prev, g, k)
        assert rel_l2(m_k, rm) < 1e-5 and rel_l2(v_k, rv) < 1e-4, (k, rel_l2(m_k, rm), rel_l2(v_k, rv))
        assert rel_l2(p_k - p_prev, rp - p_prev) < 1e-3, (k, rel_l2(p_k - p_prev, rp - p_prev))
        # (c) the independent fp64 oracle chain from the same start (own gradients)
        _, cg = O.train_loss_and_grad(chain_p, blr, bhr, S, B, C)
        chain_p, chain_m, chain_v = O.adam_step(chain_p, chain_m, chain_v, cg, k)
        assert rel_l2(p_k, chain_p) < 1e-3, (k, rel_l2(p_k, chain_p))
        assert rel_l2(m_k, chain_m) < 2e-2 and rel_l2(v_k, chain_v) < 4e-2
        p_prev, m_prev, v_prev = p_k, m_k.astype(np.float64), v_k.astype(np.float64)
        if k == 1:  # new arrivals after the capture: the replayed graph's sampler must see them (device pool view)
            ctx.pool_push(torch.from_numpy(extra_lr).cuda(), torch.from_numpy(extra_hr).cuda(), stream=st)
            pool_lr = np.concatenate([lrp, extra_lr])
            pool_hr = np.concatenate([hrp, extra_hr])
        if k == 2:  # epoch end between steps: PREV <- SERVE, SERVE <- bf16(TRAIN)
            serve_before = ctx.get_params("serve")
            ctx.publish(stream=st)
            st.synchronize()
            np.testing.assert_array_equal(ctx.get_params("prev"), serve_before)
            tr = torch.from_numpy(p_k.astype(np.float32)).to(torch.bfloat16).float().numpy()
            sv = ctx.get_params("serve")
            assert np.max(np.abs(sv - tr)) <= np.max(np.abs(tr)) * 2 ** -8
    assert launches[1] == launches[2] > 10  # replays: the captured iteration's kernels, counted per replay


def test_caller_graph_iteration_indices_bitexact_and_new_arrivals():
    """The iteration composed from the public calls and captured by the caller (torch.cuda.graph): sample_batch(-1)
    draws step t's indices bit-exactly from the pool as it is at replay time (patches pushed after the capture are
    reachable: the 150 newest get weight 4)."""
    s, b, c, seed = 2, 2, 16, 5
    ctx = _ctx(s, b, c, seed=seed)
    lrp, hrp, _ = synth_patch_pool(300, s, 2 * 40, seed=61, frame_hw=(480, 960))
    new_lr, new_hr, _ = synth_patch_pool(200, s, 2 * 40, seed=62, frame_hw=(480, 960))
    ctx.pool_push(torch.from_numpy(lrp).cuda(), torch.from_numpy(hrp).cuda())
    blr = torch.empty((32, 24, 24, 3), dtype=torch.uint8, device="cuda")
    bhr = torch.empty((32, 48, 48, 3), dtype=torch.uint8, device="cuda")
    bidx = torch.empty(32, dtype=torch.int32, device="cuda")
    loss = torch.zeros(1, device="cuda")
    scale = torch.ones(1, device="cuda")

    def it():
        ctx.sample_batch(-1, 32, 24, out=(blr, bhr, bidx))
        ctx.train_grad(blr, bhr, loss)
        ctx.train_allreduce()
        ctx.train_apply_dev(scale)

    it()  # step 0 eager (sizes the workspaces)
    torch.cuda.synchronize()
    np.testing.assert_array_equal(bidx.cpu().numpy(), O.sample_indices(seed, 0, 300, 32, 40, 24)[0])
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        it()
    # the capture itself ran nothing; the device step counter is still 1
    g.replay()
    torch.cuda.synchronize()
    np.testing.assert_array_equal(bidx.cpu().numpy(), O.sample_indices(seed, 1, 300, 32, 40, 24)[0])
    ctx.pool_push(torch.from_numpy(new_lr).cuda(), torch.from_numpy(new_hr).cuda())
    g.replay()
    torch.cuda.synchronize()
    ridx, oy, ox = O.sample_indices(seed, 2, 500, 32, 40, 24)
    got = bidx.cpu().numpy()
    np.testing.assert_array_equal(got, ridx)
    assert (got >= 300).any()  # new arrivals are drawn
    rl, rh = O.gather_patches(np.concatenate([lrp, new_lr]), np.concatenate([hrp, new_hr]), ridx, oy, ox, 24, s)
    np.testing.assert_array_equal(blr.cpu().numpy(), rl)
    np.testing.assert_array_equal(bhr.cpu().numpy(), rh)
    assert ctx.pool_stats()[0] == 500


def test_train_sampled_recaptures_on_new_loss_pointer():
    """A different loss pointer after the capture is honoured (the graph is re-captured, never replayed with the
    stale pointer)."""
    ctx = _ctx(2, 1, 16, seed=3)
    lrp, hrp, _ = synth_patch_pool(50, 2, 64, seed=7, frame_hw=(256, 512))
    ctx.pool_push(torch.from_numpy(lrp).cuda(), torch.from_numpy(hrp).cuda())
    st = torch.cuda.Stream()
    l1, l2 = torch.zeros(1, device="cuda"), torch.zeros(1, device="cuda")
    with torch.cuda.stream(st):
        ctx.train_sampled(2, 8, 24, l1)
        ctx.train_sampled(1, 8, 24, l2)
    st.synchronize()
    assert l1.item() > 0 and l2.item() > 0 and l1.item() != l2.item()


@pytest.mark.parametrize("cfg,n,p", [((3, 8, 48), 64, 48), ((2, 8, 32), 30, 48), ((3, 2, 48), 5, 40),
                                     ((2, 3, 32), 3, 60)])
def test_chain_equals_per_layer_launches(cfg, n, p):
    """The persistent chain launches (k_conv_chain: the forward blocks + body conv, and the data-gradient chain, each
    one cooperative launch with cross-CTA row flags; opt-in, set_fusion bit 9) against one k_conv_roll launch per
    conv (set_fusion 0, the blocks unfused): the same MMAs in the same order and the same epilogues -> loss and
    gradient bit-identical, over several consecutive calls (the flag generation advances per launch), and within the
    north-star bars of the oracle.  Shapes: the bench's (64 x 48x48: 25 column strips, two-phase bands), the C = 32
    net, and ragged widths (a partial last strip; fewer CTAs than strips: contiguous pieces)."""
    s, Bn, Cn = cfg
    lrp, hrp, _ = synth_patch_pool(n, s, s * p, seed=51, frame_hw=(s * p * 3, s * p * 4))
    lr, hr = torch.from_numpy(lrp).cuda(), torch.from_numpy(hrp).cuda()
    out = []
    for mode in (512, 0):
        ctx = _ctx(s, Bn, Cn, seed=52)
        ctx.set_fusion(mode)
        p0 = ctx.get_params("train")
        runs = []
        for _ in range(3):
            loss = torch.zeros(1, device="cuda")
            ctx.train_grad(lr, hr, loss)
            runs.append((loss.item(), ctx.grad_buffer().clone()))
        out.append(runs)
    for (la, ga), (lb, gb) in zip(out[0], out[1]):
        assert la == lb
        assert torch.equal(ga, gb)
    if n <= 8:
        ref_loss, ref_g = O.train_loss_and_grad(p0, lrp, hrp, s, Bn, Cn)
        assert abs(out[0][0][0] - ref_loss) / ref_loss < 1e-2
        assert rel_l2(out[0][0][1].cpu().numpy(), ref_g) < 1e-2


@pytest.mark.parametrize("train_sms", [40, 24])
def test_chain_on_partition_grids(train_sms):
    """k_conv_chain at the bench's training shape (64 x 48x48 -> 25 column strips) with the grid of a training
    partition (sr_set_sm_split): 40 CTAs = two-phase bands of unequal height (15 strips x 2 bands, 10 x 1), 24 CTAs =
    fewer CTAs than strips -> contiguous pieces spanning strips; bit-identical to the per-layer launches."""
    s, Bn, Cn = 3, 8, 48
    lrp, hrp, _ = synth_patch_pool(64, s, s * 48, seed=61, frame_hw=(s * 48 * 3, s * 48 * 4))
    lr, hr = torch.from_numpy(lrp).cuda(), torch.from_numpy(hrp).cuda()
    out = []
    for mode in (512, 0):
        ctx = _ctx(s, Bn, Cn, seed=62)
        ctx.set_fusion(mode)
        ctx.set_sm_split(train_sms)
        loss = torch.zeros(1, device="cuda")
        ctx.train_grad(lr, hr, loss)
        out.append((loss.item(), ctx.grad_buffer().clone()))
        ctx.set_sm_split(0)
    assert out[0][0] == out[1][0]
    assert torch.equal(out[0][1], out[1][1])


def test_whole_720p_frame_elementwise():
    """One whole 720p frame through the x3 8x48 net (the bench's net and frame size) against the oracle, every
    output element: |du8| <= 2 and PSNR within 0.05 dB of the oracle's against the HR original."""
    ctx = _ctx(S, B, C, seed=0)
    lr, hr = synth_frames(1, 720, 1280, seed=1003, scale=S)
    got = ctx.infer(torch.from_numpy(lr).cuda(), "serve").cpu().numpy()
    ref = O.infer_u8(ctx.get_params("serve"), lr, S, B, C)
    d = np.abs(got.astype(np.int64) - ref.astype(np.int64))
    assert d.max() <= 2, d.max()
    assert abs(psnr(got, hr) - psnr(ref, hr)) < 0.05


def test_frame_29_of_bench_batch_equals_frame_alone():
    """The bench's 30-frame batch (activation tensors of 2.65 GB: byte offsets beyond 2^31) gives the last frame
    bit-identical to inferring that frame alone."""
    ctx = _ctx(S, B, C, seed=0)
    lr = torch.from_numpy(synth_frames(30, 720, 1280, seed=1003)).cuda()
    batch = ctx.infer(lr, "serve")
    alone = ctx.infer(lr[29:30].contiguous(), "serve")
    first = ctx.infer(lr[0:1].contiguous(), "serve")
    torch.cuda.synchronize()
    assert torch.equal(batch[29], alone[0])
    assert torch.equal(batch[0], first[0])


def test_cfg2_whole_540p_frame_elementwise_and_batch_tail():
    """BASELINE config 2's net and frame (x2, 8 blocks x 32 ch, 540p -> 1080p; residual blocks on CTA pairs): one
    whole frame element-wise against the oracle (|du8| <= 2, PSNR within 0.05 dB against the HR original), and
    frame 29 of the bench's 30-frame batch bit-identical to that frame inferred alone."""
    s, b, c = 2, 8, 32
    ctx = _ctx(s, b, c, seed=0)
    lr, hr = synth_frames(1, 540, 960, seed=1002, scale=s)
    got = ctx.infer(torch.from_numpy(lr).cuda(), "serve").cpu().numpy()
    ref = O.infer_u8(ctx.get_params("serve"), lr, s, b, c)
    d = np.abs(got.astype(np.int64) - ref.astype(np.int64))
    assert d.max() <= 2, d.max()
    assert abs(psnr(got, hr) - psnr(ref, hr)) < 0.05
    lr30 = torch.from_numpy(synth_frames(30, 540, 960, seed=1002)).cuda()
    batch = ctx.infer(lr30, "serve")
    alone = ctx.infer(lr30[29:30].contiguous(), "serve")
    torch.cuda.synchronize()
    assert torch.equal(batch[29], alone[0])


def test_cfg5_1080p_x2_band_elementwise():
    """BASELINE config 5's net and frame (x2, 8 x 48, 1080p -> 2160p): the HR rows of a 64-row LR band in the middle
    of a whole-frame inference against the oracle run on that band plus its receptive-field halo (2B + 4 = 20 LR
    rows each side; R12), element-wise (|du8| <= 2) -- the full 1080p frame is beyond the oracle's seconds budget."""
    s, b, c = 2, 8, 48
    ctx = _ctx(s, b, c, seed=0)
    lr, _ = synth_frames(1, 1080, 1920, seed=1005, scale=s)
    got = ctx.infer(torch.from_numpy(lr).cuda(), "serve").cpu().numpy()
    r0, r1, R = 500, 564, 2 * b + 4
    band = np.ascontiguousarray(lr[:, r0 - R:r1 + R])
    ref = O.infer_u8(ctx.get_params("serve"), band, s, b, c)[:, s * R:s * (R + r1 - r0)]
    d = np.abs(got[:, s * r0:s * r1].astype(np.int64) - ref.astype(np.int64))
    assert d.max() <= 2, d.max()


def test_cfg4_secondary_net_gradient_batch64():
    """BASELINE config 4's second net (x2, 8 x 32) at the bench's batch (64 patches of 48 x 48, virtual wide batch of
    64 x 50 columns): loss within 1e-2 and gradient rel L2 <= 1e-2 against the oracle, one Adam step rel L2 <= 1e-3."""
    s, b, c = 2, 8, 32
    ctx = _ctx(s, b, c, seed=7)
    lrp, hrp, _ = synth_patch_pool(64, s, s * 48, seed=1008, frame_hw=(960, 1600))
    p0 = ctx.get_params("train")
    lo = torch.zeros(1, device="cuda")
    ctx.train_grad(torch.from_numpy(lrp).cuda(), torch.from_numpy(hrp).cuda(), lo)
    g = ctx.grad_buffer().cpu().numpy().copy()
    ref_loss, ref_g = O.train_loss_and_grad(p0, lrp, hrp, s, b, c)
    assert abs(lo.item() - ref_loss) / ref_loss < 1e-2
    assert rel_l2(g, ref_g) < 1e-2, rel_l2(g, ref_g)
    ctx.train_apply(1.0)
    rp, _, _ = O.adam_step(p0, np.zeros_like(p0), np.zeros_like(p0), ref_g, 1)
    assert rel_l2(ctx.get_params("train"), rp) < 1e-3


@pytest.mark.parametrize("s,p", [(2, 60), (3, 40)])
def test_paper_120px_training_patch(s, p):
    """The paper's training patch: 120x120 HR output -> LR 60 at x2, 40 at x3, with the 8x48
    net; gradient and loss vs the oracle, one Adam step."""
    n = 4
    ctx = _ctx(s, B, C, seed=17)
    lrp, hrp, _ = synth_patch_pool(n, s, 120, seed=18, frame_hw=(480, 720))
    lo = torch.zeros(1, device="cuda")
    p0 = ctx.get_params("train")
    ctx.train_grad(torch.from_numpy(lrp).cuda(), torch.from_numpy(hrp).cuda(), lo)
    g = ctx.grad_buffer().cpu().numpy().copy()
    ref_loss, ref_g = O.train_loss_and_grad(p0, lrp, hrp, s, B, C)
    assert abs(lo.item() - ref_loss) / ref_loss < 1e-2
    assert rel_l2(g, ref_g) < 1e-2
    ctx.train_apply(1.0)
    rp, _, _ = O.adam_step(p0, np.zeros_like(p0), np.zeros_like(p0), ref_g, 1)
    assert rel_l2(ctx.get_params("train"), rp) < 1e-3


def test_publish_waits_for_inflight_inference():
    """sr_publish on the training stream while a long inference batch runs on another stream: the frames are
    computed entirely with the old SERVE weights (the copies wait for the in-flight inference)."""
    s, b, c = 3, 8, 48
    ctx = _ctx(s, b, c, seed=2, lr=1e-2)
    lrp, hrp, _ = synth_patch_pool(8, s, 96, seed=3, frame_hw=(480, 720))
    ctx.train_step(torch.from_numpy(lrp).cuda(), torch.from_numpy(hrp).cuda())  # TRAIN != SERVE now
    lr = torch.from_numpy(synth_frames(12, 720, 1280, seed=4)).cuda()
    ref = ctx.infer(lr, "serve").clone()
    torch.cuda.synchronize()
    a, t = torch.cuda.Stream(), torch.cuda.Stream()
    out = torch.empty_like(ref)
    with torch.cuda.stream(a):
        ctx.infer(lr, "serve", out=out)
    with torch.cuda.stream(t):
        ctx.publish()
    torch.cuda.synchronize()
    assert torch.equal(out, ref)
    after = ctx.infer(lr[:1].contiguous(), "serve")
    assert not torch.equal(after[0], ref[0])  # the publish did take effect for later calls


def test_i420_push_clamps_out_of_frame_corners():
    """External patch corners outside the frame (the client sends the location) are clamped into
    it and counted; the crops equal the oracle's crops at the clamped corners."""
    from oracle.color import crop_rgb_from_i420, rgb_to_i420
    s, pp = 2, 16
    ctx = _ctx(s, 1, 8)
    y, u, v = rgb_to_i420(synth_frames(1, 64, 96, seed=43))
    xy = np.array([[-5, 3], [90, 60], [10, 6], [200, -40]], np.int32)
    clamped = np.stack([np.clip(xy[:, 0], 0, 96 - pp), np.clip(xy[:, 1], 0, 64 - pp)], 1).astype(np.int32)
    hr = np.random.default_rng(7).integers(0, 256, (4, s * pp, s * pp, 3)).astype(np.uint8)
    ctx.pool_push_i420(*(torch.from_numpy(a[0]).cuda() for a in (y, u, v)), torch.from_numpy(hr).cuda(),
                       torch.from_numpy(xy).cuda())
    assert ctx.pool_stats() == (4, 3)
    lr_b, _, idx = ctx.sample_batch(0, 64, pp)
    crops = crop_rgb_from_i420(y, u, v, clamped, pp)
    for k, j in enumerate(idx.cpu().numpy()):
        np.testing.assert_array_equal(lr_b[k].cpu().numpy(), crops[int(j)])


def test_nccl_communicator_one_rank_path():
    """The in-library DP exchange (sr_options.nccl_id -> ncclCommInitRank in sr_create, ncclAllReduce inside
    sr_train_step and inside sr_train_sampled's captured graph) on a one-rank communicator (one GPU here): identical
    parameters to the context without a communicator; sum_r w_r is the rank's own weight."""
    from paper_conf_sigcomm_kimjyyh20_b200 import load
    import ctypes
    buf = ctypes.create_string_buffer(128)
    assert load().sr_nccl_unique_id(buf, 128) == 0
    s, b, c = 2, 2, 16
    a = _ctx(s, b, c, seed=9, nccl_id=buf.raw, dp_weight=2.0)
    r = _ctx(s, b, c, seed=9, dp_weight=2.0)
    assert a.dp_weight_sum == 2.0 and r.dp_weight_sum == 2.0
    lrp, hrp, _ = synth_patch_pool(60, s, 64, seed=10, frame_hw=(256, 512))
    lr, hr = torch.from_numpy(lrp[:6, :24, :24].copy()).cuda(), torch.from_numpy(hrp[:6, :48, :48].copy()).cuda()
    for ctx in (a, r):
        ctx.train_step(lr, hr)
        ctx.pool_push(torch.from_numpy(lrp).cuda(), torch.from_numpy(hrp).cuda())
    st = torch.cuda.Stream()
    with torch.cuda.stream(st):
        for ctx in (a, r):
            ctx.train_sampled(3, 8, 24)
    st.synchronize()
    np.testing.assert_array_equal(a.get_params("train"), r.get_params("train"))
    # and the step equals the oracle's DP aggregation of this single rank (w / sum w = 1)
    assert a.adam_state()[2] == 4


def test_binding_rejects_bad_tensors():
    from paper_conf_sigcomm_kimjyyh20_b200 import SRError
    ctx = _ctx(2, 1, 8)
    good = torch.zeros((1, 16, 16, 3), dtype=torch.uint8, device="cuda")
    for bad in (good.float(), good.cpu(), good[:, :, ::2], torch.zeros((1, 16, 16, 4), dtype=torch.uint8,
                                                                         device="cuda")):
        with pytest.raises(SRError):
            ctx.infer(bad)
    with pytest.raises(SRError):
        ctx.infer(good, out=torch.empty((1, 32, 30, 3), dtype=torch.uint8, device="cuda"))
    with pytest.raises(SRError):
        ctx.train_step(good, torch.zeros((1, 16, 16, 3), dtype=torch.uint8, device="cuda"))


@pytest.mark.parametrize("n,elems,off", [(1, 3840 * 2160 * 3, 0), (64, 180 * 180 * 3, 0), (5, 1001, 3), (3, 17, 1),
                                         (2, 70000, 7)])
def test_sse_u8_exact(n, elems, off):
    """k_sse_u8 (Q1's integer SSE; multi-block, 16-B vector body, unaligned heads/tails) == numpy's exact int64 sum,
    from a whole 4K frame pair (PSNR of a 4K frame) down to ragged items at odd byte offsets."""
    import ctypes
    from paper_conf_sigcomm_kimjyyh20_b200 import load
    r = np.random.default_rng(elems + n)
    a = r.integers(0, 256, n * elems + off, dtype=np.uint8)
    b = r.integers(0, 256, n * elems + off, dtype=np.uint8)
    b[off: off + elems // 2] = a[off: off + elems // 2]  # an identical half (a zero partial)
    da, db = torch.from_numpy(a).cuda(), torch.from_numpy(b).cuda()
    out = torch.zeros(n, dtype=torch.int64, device="cuda")
    st = load().sr_sse_u8(ctypes.c_void_p(da.data_ptr() + off), ctypes.c_void_p(db.data_ptr() + off), n, elems,
                          ctypes.c_void_p(out.data_ptr()), ctypes.c_void_p(torch.cuda.current_stream().cuda_stream))
    assert st == 0
    d = (a[off:off + n * elems].astype(np.int64) - b[off:off + n * elems].astype(np.int64)).reshape(n, elems)
    np.testing.assert_array_equal(out.cpu().numpy(), (d * d).sum(axis=1))


def test_infer_host_async_two_in_flight():
    """sr_infer_host_async with two staging sets: consecutive calls overlap (up to two in flight, a third waits for
    the first); every batch lands intact in its own host buffer, bit-identical to sr_infer on device buffers."""
    s, b, c = 3, 2, 16
    ctx = _ctx(s, b, c, seed=33)
    lrs = [synth_frames(5, 96, 160, seed=40 + k) for k in range(4)]
    ref = [ctx.infer(torch.from_numpy(x).cuda(), "serve").cpu() for x in lrs]
    lr_h = [torch.from_numpy(x).pin_memory() for x in lrs]
    outs = [torch.zeros((5, 288, 480, 3), dtype=torch.uint8).pin_memory() for _ in range(4)]
    st = torch.cuda.Stream()
    for k in range(4):
        ctx.infer_host_async(lr_h[k], outs[k], "serve", stream=st)
    ctx.infer_host_wait()
    for k in range(4):
        assert torch.equal(outs[k], ref[k]), k


def test_nccl_allreduce_on_partition_stream():
    """bench.py at N > 1 runs the DP iteration (with the library's in-graph ncclAllReduce) on the training partition's
    green-context stream: a one-rank communicator there gives the same parameters as no communicator."""
    import ctypes
    from paper_conf_sigcomm_kimjyyh20_b200 import SRContext, load
    buf = ctypes.create_string_buffer(128)
    assert load().sr_nccl_unique_id(buf, 128) == 0
    a = _ctx(3, 2, 32, seed=3, nccl_id=buf.raw)
    b = _ctx(3, 2, 32, seed=3)
    plr, phr, _ = synth_patch_pool(64, 3, 180, seed=5, frame_hw=(1080, 1800))
    for c in (a, b):
        c.pool_push(torch.from_numpy(plr).cuda(), torch.from_numpy(phr).cuda())
    torch.cuda.synchronize()
    si, stt, ni, nt = SRContext.sm_partition(40)
    assert nt == 40 and ni > 0
    for c in (a, b):
        c.set_sm_split(nt)
        c.train_sampled(4, 16, 48, stream=stt)
    stt.synchronize()  # the partition's own stream (green context)
    torch.cuda.synchronize()
    ta, tb = a.adam_state()[2], b.adam_state()[2]
    assert ta == tb == 4, (ta, tb)
    np.testing.assert_array_equal(a.get_params("train"), b.get_params("train"))
    for c in (a, b):
        c.set_sm_split(0)


def test_dp_error_paths():
    """world > 1 without a communicator: sr_train_step / sr_train_sampled / sr_train_allreduce refuse (SR_E_STATE) and
    leave TRAIN untouched, while the caller-exchange split (sr_train_grad + sr_train_apply) works; sr_dp_weight_sum is
    0 there (unknown); sr_sm_partition rejects impossible splits."""
    from paper_conf_sigcomm_kimjyyh20_b200 import SRContext, SRError
    ctx = _ctx(2, 1, 16, seed=4, world=2, rank=1)
    assert ctx.dp_weight_sum == 0.0
    lrp, hrp, _ = synth_patch_pool(8, 2, 48, seed=9, frame_hw=(192, 384))
    lr, hr = torch.from_numpy(lrp).cuda(), torch.from_numpy(hrp).cuda()
    p0 = ctx.get_params("train")
    with pytest.raises(SRError):
        ctx.train_step(lr, hr)
    ctx2 = _ctx(2, 1, 16, seed=4, world=2, rank=1)
    with pytest.raises(SRError):
        ctx2.train_allreduce()
    ctx3 = _ctx(2, 1, 16, seed=4, world=2, rank=1)
    ctx3.pool_push(lr, hr)
    with pytest.raises(SRError):
        ctx3.train_sampled(1, 4, 16)
    np.testing.assert_array_equal(_ctx(2, 1, 16, seed=4, world=2, rank=1).get_params("train"), p0)
    ok = _ctx(2, 1, 16, seed=4, world=2, rank=1)
    ok.train_grad(lr, hr)
    ok.train_apply(1.0)  # the caller's own exchange (here: none) and 1 / sum w
    assert not np.array_equal(ok.get_params("train"), p0)
    for bad in (0, 148, 1000):
        with pytest.raises(SRError):
            SRContext.sm_partition(bad)

"""Pins for the fp64 oracle against things other than itself (CPU only).

Each test names what fixes the expected value: brute force, a library routine (torch), a closed form,
a mathematical invariant (adjointness, translation equivariance), a published test vector, or a fact
printed in PAPER.md (tests/golden/paper_facts.json)."""
import json
import re
import math
import os

import numpy as np
import pytest
import torch

import oracle as O
from synth import init_params, num_params

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _rng(seed=0):
    return np.random.default_rng(seed)


# ---------------------------------------------------------------- convolution
@pytest.mark.parametrize("shape", [(2, 6, 7, 4, 5), (1, 3, 2, 3, 16), (1, 1, 1, 2, 2)])
def test_conv_matches_bruteforce(shape):
    N, H, W, Ci, Co = shape
    r = _rng(1)
    x = r.standard_normal((N, H, W, Ci))
    Wt = r.standard_normal((Co, Ci, 3, 3))
    b = r.standard_normal(Co)
    np.testing.assert_allclose(O.conv3x3(x, Wt, b), O.conv3x3_bruteforce(x, Wt, b), rtol=1e-12, atol=1e-12)


def test_conv_matches_torch_conv2d():
    r = _rng(2)
    x = r.standard_normal((2, 9, 11, 5))
    Wt = r.standard_normal((7, 5, 3, 3))
    b = r.standard_normal(7)
    ref = torch.nn.functional.conv2d(torch.from_numpy(x).permute(0, 3, 1, 2), torch.from_numpy(Wt),
                                     torch.from_numpy(b), padding=1).permute(0, 2, 3, 1).numpy()
    np.testing.assert_allclose(O.conv3x3(x, Wt, b), ref, rtol=1e-12, atol=1e-12)


def test_conv_identity_and_shift_kernels():
    r = _rng(3)
    x = r.standard_normal((1, 5, 6, 3))
    Wid = np.zeros((3, 3, 3, 3))
    for c in range(3):
        Wid[c, c, 1, 1] = 1.0
    np.testing.assert_array_equal(O.conv3x3(x, Wid), x)
    # tap (ky,kx)=(0,2): out[y,x] = in[y-1, x+1] (zero outside) -> pins the tap/offset convention
    Ws = np.zeros((3, 3, 3, 3))
    for c in range(3):
        Ws[c, c, 0, 2] = 1.0
    exp = np.zeros_like(x)
    exp[:, 1:, :-1, :] = x[:, :-1, 1:, :]
    np.testing.assert_array_equal(O.conv3x3(x, Ws), exp)


def test_dgrad_wgrad_are_adjoints():
    """<conv_W(x), dy> = <x, dgrad_W(dy)> = <W, wgrad(x, dy)> (bias-free); db = sum dy."""
    r = _rng(4)
    x = r.standard_normal((2, 7, 5, 6))
    Wt = r.standard_normal((4, 6, 3, 3))
    dy = r.standard_normal((2, 7, 5, 4))
    lhs = np.sum(O.conv3x3(x, Wt) * dy)
    assert abs(lhs - np.sum(x * O.conv3x3_dgrad(dy, Wt))) < 1e-9 * max(1, abs(lhs))
    dW, db = O.conv3x3_wgrad(x, dy)
    assert abs(lhs - np.sum(Wt * dW)) < 1e-9 * max(1, abs(lhs))
    np.testing.assert_allclose(db, dy.sum(axis=(0, 1, 2)), rtol=1e-12)


def test_dgrad_wgrad_match_torch_autograd():
    r = _rng(5)
    x = torch.from_numpy(r.standard_normal((2, 6, 8, 3))).requires_grad_(True)
    Wt = torch.from_numpy(r.standard_normal((5, 3, 3, 3))).requires_grad_(True)
    b = torch.from_numpy(r.standard_normal(5)).requires_grad_(True)
    dy = r.standard_normal((2, 6, 8, 5))
    out = torch.nn.functional.conv2d(x.permute(0, 3, 1, 2), Wt, b, padding=1).permute(0, 2, 3, 1)
    out.backward(torch.from_numpy(dy))
    np.testing.assert_allclose(O.conv3x3_dgrad(dy, Wt.detach().numpy()), x.grad.numpy(), rtol=1e-10, atol=1e-12)
    dW, db = O.conv3x3_wgrad(x.detach().numpy(), dy)
    np.testing.assert_allclose(dW, Wt.grad.numpy(), rtol=1e-10, atol=1e-12)
    np.testing.assert_allclose(db, b.grad.numpy(), rtol=1e-10, atol=1e-12)


# ---------------------------------------------------------------- pixel shuffle
@pytest.mark.parametrize("s", [2, 3, 4])
def test_pixel_shuffle_matches_torch_and_inverts(s):
    r = _rng(6)
    y = r.standard_normal((2, 4, 5, 3 * s * s))
    ref = torch.nn.functional.pixel_shuffle(torch.from_numpy(y).permute(0, 3, 1, 2), s).permute(0, 2, 3, 1).numpy()
    ps = O.pixel_shuffle(y, s)
    np.testing.assert_array_equal(ps, ref)
    np.testing.assert_array_equal(O.pixel_unshuffle(ps, s), y)


# ---------------------------------------------------------------- bilinear skip
@pytest.mark.parametrize("s", [2, 3, 4])
def test_bilinear_matches_torch_interpolate(s):
    v = _rng(7).integers(0, 256, size=(2, 7, 9, 3)).astype(np.uint8)
    ref = torch.nn.functional.interpolate(torch.from_numpy(v.astype(np.float64)).permute(0, 3, 1, 2),
                                          scale_factor=s, mode="bilinear", align_corners=False)
    ref = ref.permute(0, 2, 3, 1).numpy()
    np.testing.assert_allclose(O.bilinear_up(v, s), ref, rtol=0, atol=1e-12)


@pytest.mark.parametrize("s", [2, 3, 4])
def test_bicubic_matches_torch_interpolate(s):
    """The bicubic skip variant (R23) = PyTorch bicubic, align_corners=False, A = -0.75, clamped taps."""
    v = _rng(17).integers(0, 256, size=(2, 7, 9, 3)).astype(np.uint8)
    ref = torch.nn.functional.interpolate(torch.from_numpy(v.astype(np.float64)).permute(0, 3, 1, 2),
                                          scale_factor=s, mode="bicubic", align_corners=False)
    np.testing.assert_allclose(O.bicubic_up(v, s), ref.permute(0, 2, 3, 1).numpy(), rtol=0, atol=1e-10)


def test_bicubic_hand_computed_weights():
    """Constants are reproduced exactly (weights sum to 1), and on a ramp v[i] = 10 i the x2 outputs use the
    A = -0.75 weights worked out by hand: t = 0.75 -> (-0.03515625, 0.26171875, 0.87890625, -0.10546875) on
    taps i0-1..i0+2, t = 0.25 -> the mirror.  (A = -0.75 does not reproduce linear functions exactly.)"""
    c = np.full((1, 6, 6, 3), 77, np.uint8)
    np.testing.assert_allclose(O.bicubic_up(c, 3), 77.0, atol=1e-12)
    ramp = np.tile(np.arange(0, 120, 10, dtype=np.uint8).reshape(1, 1, 12, 1), (1, 3, 1, 3))
    up = O.bicubic_up(ramp, 2)[0, 1, :, 0]
    w75 = [-0.03515625, 0.26171875, 0.87890625, -0.10546875]
    assert abs(up[4] - 10 * sum(w * i for w, i in zip(w75, range(0, 4)))) < 1e-12        # src 1.75
    assert abs(up[5] - 10 * sum(w * i for w, i in zip(w75[::-1], range(1, 5)))) < 1e-12  # src 2.25
    assert abs(up[4] - 17.03125) < 1e-12 and abs(up[5] - 22.96875) < 1e-12


def test_bilinear_x2_values_are_sixteenths():
    """At x2 the separable weights are 1/4, 3/4: every value is an exact multiple of 1/16 (ties real)."""
    v = _rng(8).integers(0, 256, size=(1, 16, 16, 3)).astype(np.uint8)
    b = O.bilinear_up(v, 2) * 16
    np.testing.assert_array_equal(b, np.round(b))
    assert np.mean(b % 16 == 8) > 0.01  # exact .5 ties exist -> the rounding mode matters


# ---------------------------------------------------------------- whole net special cases
@pytest.mark.parametrize("s", [2, 3, 4])
def test_zero_weight_net_is_bilinear_bitexact(s):
    v = _rng(9).integers(0, 256, size=(2, 10, 12, 3)).astype(np.uint8)
    p = np.zeros(num_params(s, 2, 8), np.float32)
    out = O.infer_u8(p, v, s, 2, 8)
    ref = torch.nn.functional.interpolate(torch.from_numpy(v.astype(np.float64)).permute(0, 3, 1, 2),
                                          scale_factor=s, mode="bilinear", align_corners=False)
    ref = np.rint(ref.permute(0, 2, 3, 1).numpy()).astype(np.uint8)  # numpy rint = half-to-even
    np.testing.assert_array_equal(out, ref)


@pytest.mark.parametrize("s", [2, 3, 4])
def test_bias_only_up_conv_is_the_shuffle_permutation(s):
    """Zero input frame (skip = 0), zero weights, up-conv bias b[k] = k/255: HR pixel (s h+i, s w+j, c)
    must equal c s^2 + i s + j exactly (ESPCN/PyTorch channel order)."""
    B, C = 1, 8
    p = np.zeros(num_params(s, B, C), np.float64)
    k = 3 * s * s
    p[-k:] = np.arange(k) / 255.0
    v = np.zeros((1, 3, 4, 3), np.uint8)
    out = O.infer_u8(p, v, s, B, C)
    for c in range(3):
        for i in range(s):
            for j in range(s):
                assert np.all(out[0, i::s, j::s, c] == c * s * s + i * s + j)


def test_translation_equivariance_interior():
    s, B, C = 2, 1, 4
    p = init_params(s, B, C, seed=11)
    v = _rng(12).integers(0, 256, size=(1, 24, 24, 3)).astype(np.uint8)
    dy, dx = 2, 3
    vs = np.zeros_like(v)
    vs[:, dy:, dx:] = v[:, :-dy, :-dx]
    a = O.infer_u8(p, v, s, B, C).astype(int)
    b = O.infer_u8(p, vs, s, B, C).astype(int)
    R = 2 * B + 3 + 1
    np.testing.assert_array_equal(b[:, s * (dy + R):s * (24 - R), s * (dx + R):s * (24 - R)],
                                  a[:, s * R:s * (24 - R - dy), s * R:s * (24 - R - dx)])


# ---------------------------------------------------------------- gradients: finite differences
@pytest.mark.parametrize("s", [2, 3, 4])
def test_full_gradient_finite_difference(s):
    B, C = 2, 4
    r = _rng(13)
    p = init_params(s, B, C, seed=3).astype(np.float64) * 3.0
    lr = r.integers(0, 256, size=(2, 5, 6, 3)).astype(np.uint8)
    hr = r.integers(0, 256, size=(2, 5 * s, 6 * s, 3)).astype(np.uint8)
    loss, g = O.train_loss_and_grad(p, lr, hr, s, B, C)
    n = p.size
    idx = np.arange(n) if s == 2 else r.choice(n, size=300, replace=False)
    h = 1e-6
    fd = np.empty(idx.size)

    def L(q):
        y = O.forward(q, lr, s, B, C)
        o = O.pixel_shuffle(y, s) + O.bilinear_up(lr, s) / 255.0
        return np.mean((o - hr / 255.0) ** 2)

    for k, i in enumerate(idx):
        q = p.copy()
        q[i] += h
        lp = L(q)
        q[i] -= 2 * h
        lm = L(q)
        fd[k] = (lp - lm) / (2 * h)
    rel = np.linalg.norm(fd - g[idx]) / np.linalg.norm(fd)
    assert rel < 1e-5, rel
    assert abs(loss - L(p)) < 1e-15


@pytest.mark.parametrize("loss_kind", ["mse", "l1"])
def test_gradient_matches_torch_autograd_net(loss_kind):
    """Same net written with torch.nn.functional in float64 (library autograd); MSE (R6) and the L1 variant
    (torch's sign(0) = 0 convention)."""
    s, B, C = 3, 2, 4
    r = _rng(14)
    p = init_params(s, B, C, seed=5).astype(np.float64)
    lr = r.integers(0, 256, size=(2, 6, 5, 3)).astype(np.uint8)
    hr = r.integers(0, 256, size=(2, 18, 15, 3)).astype(np.uint8)
    loss, g = O.train_loss_and_grad(p, lr, hr, s, B, C, loss_kind=loss_kind)
    pt = torch.from_numpy(p.copy()).requires_grad_(True)
    convs, off = [], 0
    for co, ci in O.conv_shapes_oracle(s, B, C):
        W = pt[off:off + co * ci * 9].view(co, ci, 3, 3)
        off += co * ci * 9
        convs.append((W, pt[off:off + co]))
        off += co
    F = torch.nn.functional
    v = torch.from_numpy(lr.astype(np.float64)).permute(0, 3, 1, 2)
    x = v / 255.0
    f0 = F.conv2d(x, *convs[0], padding=1)
    f = f0
    for b in range(B):
        f = f + F.conv2d(F.relu(F.conv2d(f, *convs[1 + 2 * b], padding=1)), *convs[2 + 2 * b], padding=1)
    gg = f0 + F.conv2d(f, *convs[-2], padding=1)
    y = F.conv2d(gg, *convs[-1], padding=1)
    o = F.pixel_shuffle(y, s) + F.interpolate(v, scale_factor=s, mode="bilinear", align_corners=False) / 255.0
    t = torch.from_numpy(hr.astype(np.float64)).permute(0, 3, 1, 2) / 255.0
    lt = ((o - t) ** 2).mean() if loss_kind == "mse" else (o - t).abs().mean()
    lt.backward()
    assert abs(lt.item() - loss) < 1e-14
    np.testing.assert_allclose(g, pt.grad.numpy(), rtol=1e-9, atol=1e-14)


# ---------------------------------------------------------------- Adam
def test_adam_step1_closed_form():
    r = _rng(15)
    p0 = r.standard_normal(100)
    g = r.standard_normal(100)
    p1, m1, v1 = O.adam_step(p0, np.zeros(100), np.zeros(100), g, 1, lr=1e-4)
    np.testing.assert_allclose(p1, p0 - 1e-4 * g / (np.abs(g) + 1e-8), rtol=1e-14, atol=1e-16)
    np.testing.assert_allclose(m1, 0.1 * g, rtol=1e-14)
    np.testing.assert_allclose(v1, 0.001 * g * g, rtol=1e-13)


def test_adam_matches_torch_optim():
    r = _rng(16)
    p0 = r.standard_normal(50)
    pt = torch.nn.Parameter(torch.from_numpy(p0.copy()))
    opt = torch.optim.Adam([pt], lr=1e-4, betas=(0.9, 0.999), eps=1e-8)
    p, m, v = p0.copy(), np.zeros(50), np.zeros(50)
    for t in range(1, 6):
        g = r.standard_normal(50)
        pt.grad = torch.from_numpy(g.copy())
        opt.step()
        p, m, v = O.adam_step(p, m, v, g, t)
    np.testing.assert_allclose(p, pt.detach().numpy(), rtol=1e-12, atol=1e-15)


def test_dp_aggregate():
    g1, g2 = np.ones(4), 3 * np.ones(4)
    np.testing.assert_allclose(O.dp_aggregate([g1, g2]), 2 * np.ones(4))
    np.testing.assert_allclose(O.dp_aggregate([g1, g2], [1, 3]), 2.5 * np.ones(4))


# ---------------------------------------------------------------- sampler
def test_splitmix64_published_vector():
    """SplitMix64 seeded with 0: first outputs 0xE220A8397B1DCDAF, 0x6E789E6AA1B965F4 (reference
    implementation by S. Vigna)."""
    g = 0x9E3779B97F4A7C15
    assert O.srnet._mix64(g) == 0xE220A8397B1DCDAF
    assert O.srnet._mix64(2 * g % (1 << 64)) == 0x6E789E6AA1B965F4


def test_sampler_recency_weight_statistics():
    n, K, w, batch = 1000, 150, 4, 4096
    idx, oy, ox = O.sample_indices(seed=1234, step=0, n_view=n, batch=batch, p_pool=60, p=48)
    assert idx.min() >= 0 and idx.max() < n
    assert oy.min() >= 0 and oy.max() <= 12 and ox.max() <= 12
    frac_recent = np.mean(idx >= n - K)
    expect = w * K / (w * K + n - K)  # 600 / 1450
    assert abs(frac_recent - expect) < 4 * math.sqrt(expect * (1 - expect) / batch)
    # small pool: all entries are "recent"
    idx2, _, _ = O.sample_indices(seed=1, step=3, n_view=10, batch=64, p_pool=48, p=48)
    assert idx2.min() >= 0 and idx2.max() < 10


def test_sampler_is_counter_based():
    a = O.sample_indices(7, 5, 300, 16, 60, 48, rank=1, world=2)
    b = O.sample_indices(7, 5, 300, 16, 60, 48, rank=1, world=2)
    c = O.sample_indices(7, 5, 300, 16, 60, 48, rank=0, world=2)
    for x, y in zip(a, b):
        np.testing.assert_array_equal(x, y)
    assert not np.array_equal(a[0], c[0])


def test_gather_is_a_crop():
    lrp = np.arange(3 * 6 * 6 * 3, dtype=np.int64).reshape(3, 6, 6, 3).astype(np.uint8)
    hrp = np.arange(3 * 12 * 12 * 3, dtype=np.int64).reshape(3, 12, 12, 3).astype(np.uint8)
    lr, hr = O.gather_patches(lrp, hrp, [2, 0], [1, 0], [2, 1], 4, 2)
    np.testing.assert_array_equal(lr[0], lrp[2, 1:5, 2:6])
    np.testing.assert_array_equal(hr[1], hrp[0, 0:8, 2:10])


# ---------------------------------------------------------------- PSNR
def test_psnr_closed_forms():
    a = np.full((3, 8, 8, 3), 100, np.uint8)
    for d in (1, 5, 17):
        b = a + np.uint8(d)
        np.testing.assert_allclose(O.psnr_u8(a, b), 20 * math.log10(255.0 / d), rtol=1e-13)
    np.testing.assert_array_equal(O.psnr_u8(a, a), 100.0)
    pa, pb, gain = O.psnr_gain(a + np.uint8(1), a + np.uint8(2), a)
    assert abs(gain - 20 * math.log10(2.0)) < 1e-12


# ---------------------------------------------------------------- facts printed in the paper
def test_paper_facts():
    f = json.load(open(os.path.join(GOLD, "paper_facts.json")))
    g = f["grid_1080p_cells"]
    assert g["frame_hw"][0] * g["frame_hw"][1] // (g["patch"] ** 2) == g["value"]
    assert f["raw_patch_bytes"]["patch"] ** 2 * 3 == f["raw_patch_bytes"]["value"]
    for key, s in (("strip_720p", 3), ("strip_1080p", 2)):
        e = f[key]
        w, h = e["frame_hw"][1], e["frame_hw"][0] // e["pieces"]
        assert [w, h] == e["value"]
        assert [w * s, h * s * e["pieces"]] == f["strip_upscaled_4k"]["value"]
    for ingest, up, fps, delay, ngpu in f["table2_rows"]["rows"]:
        assert abs(fps - 1000.0 / delay) / fps < 0.08, (ingest, fps, delay)
    # the shapes we build: parameter counts of the configs
    assert num_params(2, 2, 8) == 4020 and num_params(2, 8, 32) == 161580
    assert num_params(2, 8, 48) == 359868 and num_params(3, 8, 48) == 366363


def test_oracle_is_independent_of_product_code():
    here = os.path.join(os.path.dirname(os.path.dirname(__file__)), "oracle")
    for fn in os.listdir(here):
        if fn.endswith(".py"):
            src = open(os.path.join(here, fn)).read()
            imports = [ln for ln in src.splitlines() if re.match(r"\s*(import|from)\s", ln)]
            for ln in imports:
                assert "paper_conf_sigcomm_kimjyyh20_b200" not in ln and "synth" not in ln, ln
                assert "ctypes" not in ln and "torch" not in ln, ln

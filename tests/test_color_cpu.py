"""The I420 boundary's colour conversion (oracle/color.py) pinned to the real-valued ITU-R BT.601 definition
(tests/golden/bt601_colors.json) and to its structural properties."""
import json
import os

import numpy as np

from oracle.color import crop_rgb_from_i420, i420_to_rgb, rgb_to_i420

G = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "bt601_colors.json")))


def _flat_blocks(rgb):
    """[k, 3] colours -> one 2x2 flat block per colour (so chroma averaging is exact)."""
    k = rgb.shape[0]
    return np.repeat(np.repeat(rgb.reshape(1, 1, k, 3), 2, axis=1), 2, axis=2).reshape(1, 2, 2 * k, 3)


def test_rgb_to_ycbcr_matches_bt601_within_one():
    rng = np.random.default_rng(0)
    cols = np.concatenate([rng.integers(0, 256, (4000, 3)), np.array([[255, 0, 0], [0, 255, 0], [0, 0, 255]])])
    y, u, v = rgb_to_i420(_flat_blocks(cols.astype(np.uint8)))
    f = G["rgb_to_ycbcr"]
    for plane, key in ((y[0, 0, ::2], "y"), (u[0, 0], "cb"), (v[0, 0], "cr")):
        c = f[key]
        exact = c[0] + (c[1] * cols[:, 0] + c[2] * cols[:, 1] + c[3] * cols[:, 2]) / 255.0
        assert np.max(np.abs(plane.astype(float) - exact)) <= f["tolerance"] + 0.5, key


def test_ycbcr_to_rgb_matches_bt601():
    rng = np.random.default_rng(1)
    yy = rng.integers(16, 236, 3000)
    cb = rng.integers(16, 241, 3000)
    cr = rng.integers(16, 241, 3000)
    y = np.repeat(yy.reshape(1, 1, -1), 2, axis=2).repeat(2, axis=1).astype(np.uint8)  # [1, 2, 2k]
    u = cb.reshape(1, 1, -1).astype(np.uint8)
    v = cr.reshape(1, 1, -1).astype(np.uint8)
    rgb = i420_to_rgb(y, u, v)[0, 0, ::2]
    f = G["ycbcr_to_rgb"]
    for k, key in enumerate("rgb"):
        c = f[key]
        exact = np.clip(c[0] * (yy - 16) + c[1] * (cb - 128.0) + c[2] * (cr - 128.0), 0, 255)
        assert np.max(np.abs(rgb[:, k] - exact)) <= f["tolerance"], key


def test_black_and_white_exact_both_ways():
    for e in G["exact"]:
        rgb = np.array(e["rgb"], np.uint8).reshape(1, 1, 1, 3).repeat(2, 1).repeat(2, 2)
        y, u, v = rgb_to_i420(rgb)
        assert (int(y[0, 0, 0]), int(u[0, 0, 0]), int(v[0, 0, 0])) == tuple(e["yuv"])
        back = i420_to_rgb(y, u, v)
        assert np.all(back == np.array(e["rgb"]))


def test_chroma_is_shared_by_its_2x2_block_and_planes_have_i420_shapes():
    rng = np.random.default_rng(2)
    rgb = rng.integers(0, 256, (2, 6, 8, 3)).astype(np.uint8)
    y, u, v = rgb_to_i420(rgb)
    assert y.shape == (2, 6, 8) and u.shape == (2, 3, 4) and v.shape == (2, 3, 4)
    back = i420_to_rgb(y, u, v)
    # pixels of one 2x2 block with equal luma decode to equal colour
    y2 = y.copy()
    y2[:, 0:2, 0:2] = y2[:, 0:1, 0:1]
    b2 = i420_to_rgb(y2, u, v)
    assert np.all(b2[:, 0, 0] == b2[:, 1, 1]) and np.all(b2[:, 0, 1] == b2[:, 1, 0])
    assert back.shape == rgb.shape


def test_round_trip_of_flat_colours_is_close():
    rng = np.random.default_rng(3)
    cols = rng.integers(16, 240, (2000, 3)).astype(np.uint8)
    rgb = _flat_blocks(cols)
    back = i420_to_rgb(*rgb_to_i420(rgb))
    assert np.max(np.abs(back.astype(int) - rgb.astype(int))) <= 3


def test_crop_is_a_window_of_the_decoded_frame():
    rng = np.random.default_rng(4)
    y = rng.integers(0, 256, (1, 10, 12)).astype(np.uint8)
    u = rng.integers(0, 256, (1, 5, 6)).astype(np.uint8)
    v = rng.integers(0, 256, (1, 5, 6)).astype(np.uint8)
    full = i420_to_rgb(y, u, v)[0]
    c = crop_rgb_from_i420(y, u, v, [(3, 1), (0, 0), (7, 5)], 4)
    assert np.array_equal(c[0], full[1:5, 3:7]) and np.array_equal(c[2], full[5:9, 7:11])

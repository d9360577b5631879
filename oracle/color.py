"""Colour-space boundary of the ingest server — TEST INFRASTRUCTURE (see oracle/__init__.py).

WebRTC hands the media server decoded I420 frames (§2: the server decodes the stream) and
the encoders downstream take I420 again (§7).  The paper does not give the conversion (DESIGN.md
reading R21), so both directions use the integer BT.601 studio-swing ("limited range") formulas of the
classic 8-bit YUV <-> RGB definition, written out here as plain integer arithmetic (floor shifts):

  I420 -> RGB (chroma sample (y//2, x//2) shared by its 2x2 block):
      C = Y - 16, D = U - 128, E = V - 128
      R = clip((298 C + 409 E + 128) >> 8),  G = clip((298 C - 100 D - 208 E + 128) >> 8),
      B = clip((298 C + 516 D + 128) >> 8)
  RGB -> I420 (U, V from the 2x2 block's rounded mean colour):
      Y = ((66 R + 129 G + 25 B + 128) >> 8) + 16
      (R', G', B') = (sum over the 2x2 block + 2) >> 2
      U = ((-38 R' - 74 G' + 112 B' + 128) >> 8) + 128,  V = ((112 R' - 94 G' - 18 B' + 128) >> 8) + 128

Frames are planar: y [n, h, w], u and v [n, h/2, w/2] (h, w even); RGB is [n, h, w, 3] u8.
"""
from __future__ import annotations

import numpy as np


def _clip8(x):
    return np.clip(x, 0, 255).astype(np.uint8)


def i420_to_rgb(y, u, v):
    y = y.astype(np.int64)
    uu = np.repeat(np.repeat(u.astype(np.int64), 2, axis=-2), 2, axis=-1)  # chroma of pixel (r, c) = (r//2, c//2)
    vv = np.repeat(np.repeat(v.astype(np.int64), 2, axis=-2), 2, axis=-1)
    c, d, e = y - 16, uu - 128, vv - 128
    r = (298 * c + 409 * e + 128) >> 8
    g = (298 * c - 100 * d - 208 * e + 128) >> 8
    b = (298 * c + 516 * d + 128) >> 8
    return np.stack([_clip8(r), _clip8(g), _clip8(b)], axis=-1)


def rgb_to_i420(rgb):
    x = rgb.astype(np.int64)
    r, g, b = x[..., 0], x[..., 1], x[..., 2]
    y = ((66 * r + 129 * g + 25 * b + 128) >> 8) + 16
    n, h, w = r.shape
    blk = x.reshape(n, h // 2, 2, w // 2, 2, 3).sum(axis=(2, 4))
    rm, gm, bm = [(blk[..., k] + 2) >> 2 for k in range(3)]
    u = ((-38 * rm - 74 * gm + 112 * bm + 128) >> 8) + 128
    v = ((112 * rm - 94 * gm - 18 * bm + 128) >> 8) + 128
    return y.astype(np.uint8), u.astype(np.uint8), v.astype(np.uint8)


def crop_rgb_from_i420(y, u, v, xy, pp):
    """LR counterparts of HR patches (§5.2: patches arrive with their location): the pp x pp RGB crop
    of the decoded frame at LR top-left (x, y) for every entry of xy [n, 2]."""
    rgb = i420_to_rgb(y, u, v)[0]
    return np.stack([rgb[yy:yy + pp, xx:xx + pp] for xx, yy in xy])

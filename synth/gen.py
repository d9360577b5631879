"""Seeded synthetic input generators (inputs only; none of the method's arithmetic lives here).

Recipe:
  * HR frames: u8 RGB = 1/f-spectrum noise (spectral slope -2 in power, 3 channels with a shared luma
    component) + random axis-aligned and oblique rectangles/edges + thin "text-like" strokes + mild
    per-frame noise.  Temporal structure: a global pan of 1-3 px/frame over a larger canvas and a scene
    cut (new sub-seed) every `cut_every` frames (the paper relies on temporal redundancy and scene
    changes).
  * LR frames: s x s area average of HR, rounded half-to-even (what a downscaling ingest client sends).
  * Patches: HR cells of the frame grid (the paper's 120x120 cells) with
    their area-averaged LR counterparts, pushed in arrival order.
  * Weights: SplitMix64 stream (seed), uniform +-1/sqrt(9*Cin) for every W and b, drawn in the canonical
    parameter order (per conv: W in OIHW order, then b).  This is the input the method starts from; the
    C++ library's sr_create() carries an independent transcription, checked bit-exact by a test.
"""
from __future__ import annotations

import numpy as np

MASK64 = (1 << 64) - 1
GAMMA = 0x9E3779B97F4A7C15


def mix64(z: int) -> int:
    """SplitMix64 finaliser on a Python int (mod 2^64)."""
    z &= MASK64
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & MASK64
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & MASK64
    return z ^ (z >> 31)


def splitmix64_stream(seed: int, n: int) -> np.ndarray:
    """n successive SplitMix64 outputs: state += GAMMA; out = mix64(state).  Vectorised in uint64."""
    k = np.arange(1, n + 1, dtype=np.uint64)
    with np.errstate(over="ignore"):
        z = np.uint64(seed & MASK64) + k * np.uint64(GAMMA)
        z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
        z = z ^ (z >> np.uint64(31))
    return z


def conv_shapes(scale: int, blocks: int, channels: int):
    """(Cout, Cin) of every 3x3 conv in canonical order: head, (b.conv1, b.conv2) x B, body, up."""
    C = channels
    shapes = [(C, 3)]
    for _ in range(blocks):
        shapes += [(C, C), (C, C)]
    shapes += [(C, C), (3 * scale * scale, C)]
    return shapes


def num_params(scale: int, blocks: int, channels: int) -> int:
    return sum(co * ci * 9 + co for co, ci in conv_shapes(scale, blocks, channels))


def init_params(scale: int, blocks: int, channels: int, seed: int = 0) -> np.ndarray:
    """Flat fp32 canonical parameter vector: per conv W[Cout][Cin][3][3] then b[Cout].

    u = (z >> 40) * 2^-24 in [0,1); value = fp32((2u - 1) * (1/sqrt(9*Cin))), computed in fp64 then
    rounded once to fp32 (the C++ transcription does the same in double)."""
    n = num_params(scale, blocks, channels)
    z = splitmix64_stream(seed, n)
    u = (z >> np.uint64(40)).astype(np.float64) * (2.0 ** -24)
    bound = np.empty(n, dtype=np.float64)
    off = 0
    for co, ci in conv_shapes(scale, blocks, channels):
        cnt = co * ci * 9 + co
        bound[off:off + cnt] = 1.0 / np.sqrt(9.0 * ci)
        off += cnt
    return ((2.0 * u - 1.0) * bound).astype(np.float32)


# ----------------------------------------------------------------------------------------------------
# frames
# ----------------------------------------------------------------------------------------------------

def _pink_noise(rng: np.random.Generator, h: int, w: int) -> np.ndarray:
    """Zero-mean 1/f noise (amplitude ~ 1/f), unit std, float32 [h, w]."""
    white = rng.standard_normal((h, w)).astype(np.float32)
    spec = np.fft.rfft2(white)
    fy = np.fft.fftfreq(h)[:, None]
    fx = np.fft.rfftfreq(w)[None, :]
    f = np.sqrt(fy * fy + fx * fx)
    f[0, 0] = 1.0
    spec *= (1.0 / np.maximum(f, 1.0 / max(h, w))).astype(np.float32)
    spec[0, 0] = 0
    out = np.fft.irfft2(spec, s=(h, w)).astype(np.float32)
    out /= out.std() + 1e-6
    return out


def _canvas(seed: int, h: int, w: int) -> np.ndarray:
    """One scene: float32 [h, w, 3] in 0..255."""
    rng = np.random.default_rng(seed)
    luma = _pink_noise(rng, h, w)
    img = np.empty((h, w, 3), dtype=np.float32)
    base = rng.uniform(60, 190, size=3).astype(np.float32)
    chroma = _pink_noise(rng, h, w)
    mix = rng.uniform(-1.0, 1.0, size=3).astype(np.float32)
    for c in range(3):
        img[..., c] = base[c] + 38.0 * luma + 12.0 * mix[c] * chroma
    yy, xx = np.mgrid[0:h, 0:w].astype(np.float32)
    # rectangles / edges (axis-aligned and oblique half-planes)
    for _ in range(12):
        y0, x0 = rng.integers(0, h), rng.integers(0, w)
        hh, ww = rng.integers(h // 20 + 1, h // 3 + 2), rng.integers(w // 20 + 1, w // 3 + 2)
        col = rng.uniform(0, 255, size=3).astype(np.float32)
        img[y0:y0 + hh, x0:x0 + ww, :] = 0.3 * img[y0:y0 + hh, x0:x0 + ww, :] + 0.7 * col
    for _ in range(4):
        ang = rng.uniform(0, np.pi)
        d = rng.uniform(-0.3, 0.3) * (h + w)
        m = (np.cos(ang) * (xx - w / 2) + np.sin(ang) * (yy - h / 2)) > d
        img[m] += rng.uniform(-50, 50, size=3).astype(np.float32)
    # text-like strokes: short thin dark/bright bars in rows
    for _ in range(max(1, (h * w) // 40000)):
        y0, x0 = rng.integers(0, max(1, h - 8)), rng.integers(0, max(1, w - 40))
        length = rng.integers(4, 40)
        val = 20.0 if rng.random() < 0.5 else 235.0
        if rng.random() < 0.5:
            img[y0:y0 + 2, x0:x0 + length, :] = val
        else:
            img[y0:y0 + min(length, 12), x0:x0 + 2, :] = val
    return img


def area_downsample(hr: np.ndarray, s: int) -> np.ndarray:
    """s x s area average of u8 HR [..., H, W, 3] -> u8 LR, round half to even (np.rint)."""
    *lead, H, W, C = hr.shape
    assert H % s == 0 and W % s == 0
    v = hr.reshape(*lead, H // s, s, W // s, s, C).astype(np.float64).mean(axis=(-4, -2))
    return np.rint(v).astype(np.uint8)


def synth_frames(n: int, h: int, w: int, seed: int, scale: int | None = None, cut_every: int = 300,
                 pan_max: int = 3):
    """n u8 frames [n, h, w, 3] with a global pan and scene cuts.

    If `scale` is given, frames are produced at HR (h*scale, w*scale) and the function returns
    (lr [n,h,w,3], hr [n,h*s,w*s,3]); otherwise it returns LR-resolution frames only (bench inputs)."""
    s = scale or 1
    H, W = h * s, w * s
    rng = np.random.default_rng(seed)
    margin = pan_max * max(n, 1) * s + 1
    frames = np.empty((n, H, W, 3), dtype=np.uint8)
    canvas = None
    py = px = 0
    for i in range(n):
        if i % cut_every == 0:
            canvas = _canvas(int(rng.integers(0, 2 ** 31)), H + margin, W + margin)
            py = px = 0
            dy, dx = int(rng.integers(-pan_max, pan_max + 1)), int(rng.integers(1, pan_max + 1))
        oy = int(np.clip(margin // 2 + py, 0, margin - 1))
        ox = int(np.clip(px, 0, margin - 1))
        fr = canvas[oy:oy + H, ox:ox + W, :] + rng.normal(0, 1.5, size=(H, W, 3)).astype(np.float32)
        frames[i] = np.clip(np.rint(fr), 0, 255).astype(np.uint8)
        py += dy * s
        px += dx * s
    if scale is None:
        return frames
    return area_downsample(frames, s), frames


def synth_patch_pool(n: int, scale: int, hr_patch: int, seed: int, frame_hw=(1080, 1920)):
    """n (LR, HR) patch pairs in arrival order: HR cells hr_patch x hr_patch of synthetic HR frames
    (the 16x9 grid of 120x120 cells at 1080p), LR = area average / scale.

    Returns (lr u8 [n, P, P, 3], hr u8 [n, sP, sP, 3], arrival int64 [n])."""
    assert hr_patch % scale == 0
    H, W = frame_hw
    rng = np.random.default_rng(seed)
    gy, gx = H // hr_patch, W // hr_patch
    per_frame = gy * gx
    hr = np.empty((n, hr_patch, hr_patch, 3), dtype=np.uint8)
    i = 0
    fidx = 0
    while i < n:
        canvas = _canvas(int(rng.integers(0, 2 ** 31)) + fidx, gy * hr_patch, gx * hr_patch)
        canvas = np.clip(np.rint(canvas), 0, 255).astype(np.uint8)
        cells = rng.permutation(gy * gx)[:per_frame]
        for c in cells:
            if i >= n:
                break
            cy, cx = divmod(int(c), gx)
            hr[i] = canvas[cy * hr_patch:(cy + 1) * hr_patch, cx * hr_patch:(cx + 1) * hr_patch]
            i += 1
        fidx += 1
    lr = area_downsample(hr, scale)
    return lr, hr, np.arange(n, dtype=np.int64)

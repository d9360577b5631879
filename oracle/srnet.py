"""fp64 numpy oracle of the LiveNAS SR hot path (TEST INFRASTRUCTURE; see oracle/__init__.py).

Citations are PAPER.md line numbers (+ section).  Where the paper is silent the DESIGN.md reading
("Readings" table, R1..R18, which restates SURVEY.md §8(c)) is named.

Network (§7 L1241-1242 names the NAS "ultra-high" model without giving its topology; the
north star fixes the family: 3x3 conv, ReLU, residual add, pixel-shuffle upsampling with a bilinear
skip; reading R1):
    x  = v / 255                                    (R3: RGB u8 in, /255, no mean shift)
    f0 = conv_head(x)                               (3 -> C)
    f  = f0;  for b in 1..B:  f = f + conv_b2(relu(conv_b1(f)))     (EDSR-style block, no BN, scale 1)
    g  = f0 + conv_body(f)                          (global skip)
    y  = conv_up(g)                                 (C -> 3 s^2, ESPCN sub-pixel conv)
    out255 = 255 * PS_s(y) + bilinear_s(v)          (bilinear = the WebRTC baseline)
    inference: u8 = rint(clip(out255, 0, 255))      (R5: clamp then round-half-to-even)
    training:  o = PS_s(y) + bilinear_s(v)/255, loss = mean((o - hr/255)^2)     (R6: MSE, no clamp)
Every conv is 3x3, stride 1, with bias and zero "same" padding at the image border (R4).
"""
from __future__ import annotations

import math

import numpy as np

MASK64 = (1 << 64) - 1
GAMMA = 0x9E3779B97F4A7C15


# ----------------------------------------------------------------------------------------------------
# topology and parameter layout (R1; canonical order = head, (b.conv1, b.conv2) x B, body, up)
# ----------------------------------------------------------------------------------------------------

def conv_shapes_oracle(scale, blocks, channels):
    C = channels
    return [(C, 3)] + [(C, C)] * (2 * blocks) + [(C, C), (3 * scale * scale, C)]


def unpack_params(flat, scale, blocks, channels):
    """Flat canonical vector -> list of (W[Cout,Cin,3,3] fp64, b[Cout] fp64)."""
    flat = np.asarray(flat, dtype=np.float64)
    out, off = [], 0
    for co, ci in conv_shapes_oracle(scale, blocks, channels):
        W = flat[off:off + co * ci * 9].reshape(co, ci, 3, 3)
        off += co * ci * 9
        b = flat[off:off + co]
        off += co
        out.append((W, b))
    assert off == flat.size, (off, flat.size)
    return out


def pack_params(convs):
    return np.concatenate([np.concatenate([W.ravel(), b.ravel()]) for W, b in convs])


# ----------------------------------------------------------------------------------------------------
# 3x3 convolution: the plain definition (R4)
#   out[n,y,x,co] = b[co] + sum_{ky,kx in 0..2} sum_ci W[co,ci,ky,kx] * in[n, y+ky-1, x+kx-1, ci]
# ----------------------------------------------------------------------------------------------------

def conv3x3(x, W, b=None):
    """x [N,H,W,Cin] -> [N,H,W,Cout]; the sum over taps written as 9 matrix products."""
    x = np.asarray(x, dtype=np.float64)
    N, H, Wd, Ci = x.shape
    Co = W.shape[0]
    xp = np.pad(x, ((0, 0), (1, 1), (1, 1), (0, 0)))
    out = np.zeros((N, H, Wd, Co))
    for ky in range(3):
        for kx in range(3):
            out += xp[:, ky:ky + H, kx:kx + Wd, :] @ W[:, :, ky, kx].T
    if b is not None:
        out += b
    return out


def conv3x3_bruteforce(x, W, b):
    """7-nested-loop direct convolution (pin for conv3x3 on tiny tensors)."""
    N, H, Wd, Ci = x.shape
    Co = W.shape[0]
    out = np.zeros((N, H, Wd, Co))
    for n in range(N):
        for y in range(H):
            for xx in range(Wd):
                for co in range(Co):
                    acc = float(b[co])
                    for ky in range(3):
                        for kx in range(3):
                            yy, xs = y + ky - 1, xx + kx - 1
                            if 0 <= yy < H and 0 <= xs < Wd:
                                for ci in range(Ci):
                                    acc += W[co, ci, ky, kx] * x[n, yy, xs, ci]
                    out[n, y, xx, co] = acc
    return out


def conv3x3_dgrad(dy, W):
    """dL/dx of out = conv3x3(x, W): dx[y,x,ci] = sum_{ky,kx,co} W[co,ci,ky,kx] dy[y+1-ky, x+1-kx, co]
    (full correlation with the 180-degree-rotated kernel, Cin/Cout swapped; zero outside)."""
    dy = np.asarray(dy, dtype=np.float64)
    N, H, Wd, Co = dy.shape
    Ci = W.shape[1]
    dyp = np.pad(dy, ((0, 0), (1, 1), (1, 1), (0, 0)))
    dx = np.zeros((N, H, Wd, Ci))
    for ky in range(3):
        for kx in range(3):
            dx += dyp[:, 2 - ky:2 - ky + H, 2 - kx:2 - kx + Wd, :] @ W[:, :, ky, kx]
    return dx


def conv3x3_wgrad(x, dy):
    """dW[co,ci,ky,kx] = sum_{n,y,x} dy[n,y,x,co] * x[n, y+ky-1, x+kx-1, ci];  db[co] = sum dy."""
    x = np.asarray(x, dtype=np.float64)
    dy = np.asarray(dy, dtype=np.float64)
    N, H, Wd, Ci = x.shape
    Co = dy.shape[-1]
    xp = np.pad(x, ((0, 0), (1, 1), (1, 1), (0, 0)))
    dW = np.zeros((Co, Ci, 3, 3))
    d2 = dy.reshape(-1, Co)
    for ky in range(3):
        for kx in range(3):
            dW[:, :, ky, kx] = d2.T @ xp[:, ky:ky + H, kx:kx + Wd, :].reshape(-1, Ci)
    return dW, d2.sum(axis=0)


# ----------------------------------------------------------------------------------------------------
# pixel shuffle (ESPCN sub-pixel layout; PyTorch channel order, R1):
#   PS(y)[n, s*h+i, s*w+j, c] = y[n, h, w, c*s^2 + i*s + j]
# ----------------------------------------------------------------------------------------------------

def pixel_shuffle(y, s):
    N, H, W, K = y.shape
    c_out = K // (s * s)
    out = np.empty((N, H * s, W * s, c_out), dtype=y.dtype)
    for c in range(c_out):
        for i in range(s):
            for j in range(s):
                out[:, i::s, j::s, c] = y[..., c * s * s + i * s + j]
    return out


def pixel_unshuffle(o, s):
    N, Hs, Ws, c_out = o.shape
    y = np.empty((N, Hs // s, Ws // s, c_out * s * s), dtype=o.dtype)
    for c in range(c_out):
        for i in range(s):
            for j in range(s):
                y[..., c * s * s + i * s + j] = o[:, i::s, j::s, c]
    return y


# ----------------------------------------------------------------------------------------------------
# bilinear up-scaling (the WebRTC baseline; Fig. 7).  R2: half-pixel centres
# (align_corners=False): src = (dst + 0.5)/s - 0.5, clamped below at 0; i0 = floor(src),
# i1 = min(i0 + 1, n - 1), out = (1 - l) v[i0] + l v[i1], l = src - i0; horizontal pass, then vertical.
# ----------------------------------------------------------------------------------------------------

def _bilinear_axis(v, s, axis):
    n = v.shape[axis]
    dst = np.arange(n * s, dtype=np.float64)
    src = np.maximum((dst + 0.5) / s - 0.5, 0.0)
    i0 = np.floor(src).astype(np.int64)
    i1 = np.minimum(i0 + 1, n - 1)
    lam = src - i0
    a = np.take(v, i0, axis=axis)
    b = np.take(v, i1, axis=axis)
    shape = [1] * v.ndim
    shape[axis] = n * s
    lam = lam.reshape(shape)
    return (1.0 - lam) * a + lam * b


def bilinear_up(v_u8, s):
    """u8 [N,H,W,3] -> fp64 [N,sH,sW,3] on the 0..255 scale."""
    v = np.asarray(v_u8, dtype=np.float64)
    return _bilinear_axis(_bilinear_axis(v, s, 2), s, 1)


# ----------------------------------------------------------------------------------------------------
# bicubic up-scaling (the skip variant of SURVEY §8(f) NEXT 3; north star "bilinear/bicubic"; reading R23):
# Keys cubic convolution with A = -0.75 (PyTorch bicubic, align_corners=False): src = (dst + 0.5)/s - 0.5 (no
# clamp), i0 = floor(src), t = src - i0, out = sum_{k=-1..2} w(k - t) v[clamp(i0 + k, 0, n-1)],
# w(x) = (A+2)|x|^3 - (A+3)|x|^2 + 1 for |x| <= 1, A|x|^3 - 5A|x|^2 + 8A|x| - 4A for 1 < |x| < 2.
# ----------------------------------------------------------------------------------------------------

def _cubic_w(x, A=-0.75):
    x = abs(x)
    if x <= 1.0:
        return (A + 2.0) * x ** 3 - (A + 3.0) * x ** 2 + 1.0
    if x < 2.0:
        return A * x ** 3 - 5.0 * A * x ** 2 + 8.0 * A * x - 4.0 * A
    return 0.0


def _bicubic_axis(v, s, axis):
    n = v.shape[axis]
    out_shape = list(v.shape)
    out_shape[axis] = n * s
    out = np.zeros(out_shape, dtype=np.float64)
    for dst in range(n * s):
        src = (dst + 0.5) / s - 0.5
        i0 = int(np.floor(src))
        t = src - i0
        acc = 0.0
        for k in range(-1, 3):
            idx = min(max(i0 + k, 0), n - 1)
            acc = acc + _cubic_w(k - t) * np.take(v, idx, axis=axis)
        sl = [slice(None)] * v.ndim
        sl[axis] = dst
        out[tuple(sl)] = acc
    return out


def bicubic_up(v_u8, s):
    """u8 [N,H,W,3] -> fp64 [N,sH,sW,3] on the 0..255 scale (horizontal pass, then vertical)."""
    v = np.asarray(v_u8, dtype=np.float64)
    return _bicubic_axis(_bicubic_axis(v, s, 2), s, 1)


def skip_up(v_u8, s, skip="bilinear"):
    return bilinear_up(v_u8, s) if skip == "bilinear" else bicubic_up(v_u8, s)


# ----------------------------------------------------------------------------------------------------
# network forward (see module docstring)
# ----------------------------------------------------------------------------------------------------

def forward(flat_params, lr_u8, scale, blocks, channels, keep=False):
    """Returns y (the up-conv output, [N,H,W,3s^2]) and, if keep, the saved activations."""
    convs = unpack_params(flat_params, scale, blocks, channels)
    x = np.asarray(lr_u8, dtype=np.float64) / 255.0
    Wh, bh = convs[0]
    f0 = conv3x3(x, Wh, bh)
    f = f0
    fs, ts = [f0], []
    for blk in range(blocks):
        W1, b1 = convs[1 + 2 * blk]
        W2, b2 = convs[2 + 2 * blk]
        t = np.maximum(conv3x3(f, W1, b1), 0.0)
        f = f + conv3x3(t, W2, b2)
        ts.append(t)
        fs.append(f)
    Wb, bb = convs[1 + 2 * blocks]
    g = f0 + conv3x3(f, Wb, bb)
    Wu, bu = convs[2 + 2 * blocks]
    y = conv3x3(g, Wu, bu)
    if keep:
        return y, dict(x=x, fs=fs, ts=ts, g=g, convs=convs)
    return y


def infer_u8(flat_params, lr_u8, scale, blocks, channels, return_float=False, skip="bilinear"):
    """Inference output: u8 = rint(clip(255 PS(y) + bilinear(v), 0, 255)) (R5); skip="bicubic" for R23."""
    y = forward(flat_params, lr_u8, scale, blocks, channels)
    o255 = 255.0 * pixel_shuffle(y, scale) + skip_up(lr_u8, scale, skip)
    u8 = np.rint(np.clip(o255, 0.0, 255.0)).astype(np.uint8)
    if return_float:
        return u8, o255
    return u8


# ----------------------------------------------------------------------------------------------------
# training: MSE loss (R6) and the analytic backward pass (chain rule written out by hand)
# ----------------------------------------------------------------------------------------------------

def train_loss_and_grad(flat_params, lr_u8, hr_u8, scale, blocks, channels, loss_kind="mse", skip="bilinear"):
    """Returns (loss, flat gradient) of L = mean over all HR elements of (o - hr/255)^2,
    o = PS(y) + bilinear(v)/255 (no clamp).  Gradient w.r.t. the parameters only (no input grad)."""
    y, a = forward(flat_params, lr_u8, scale, blocks, channels, keep=True)
    convs = a["convs"]
    o = pixel_shuffle(y, scale) + skip_up(lr_u8, scale, skip) / 255.0
    t = np.asarray(hr_u8, dtype=np.float64) / 255.0
    n_el = o.size
    if loss_kind == "mse":
        loss = float(np.sum((o - t) ** 2) / n_el)
        do = 2.0 * (o - t) / n_el
    elif loss_kind == "l1":
        loss = float(np.sum(np.abs(o - t)) / n_el)
        do = np.sign(o - t) / n_el
    else:
        raise ValueError(loss_kind)
    dy = pixel_unshuffle(do, scale)
    grads = [None] * len(convs)
    fs, ts, g, x = a["fs"], a["ts"], a["g"], a["x"]
    # up conv
    Wu, _ = convs[-1]
    grads[-1] = conv3x3_wgrad(g, dy)
    dg = conv3x3_dgrad(dy, Wu)
    # body conv (g = f0 + conv_body(f_B))
    Wb, _ = convs[-2]
    grads[-2] = conv3x3_wgrad(fs[-1], dg)
    df = conv3x3_dgrad(dg, Wb)
    # residual blocks in reverse: f_b = f_{b-1} + conv2(relu(conv1(f_{b-1})))
    for blk in reversed(range(blocks)):
        W1, _ = convs[1 + 2 * blk]
        W2, _ = convs[2 + 2 * blk]
        tb = ts[blk]
        grads[2 + 2 * blk] = conv3x3_wgrad(tb, df)
        dt = conv3x3_dgrad(df, W2) * (tb > 0.0)        # ReLU' = 1[pre-activation > 0] = 1[t > 0]
        grads[1 + 2 * blk] = conv3x3_wgrad(fs[blk], dt)
        df = df + conv3x3_dgrad(dt, W1)                # residual path adds
    df0 = df + dg                                      # global skip adds
    grads[0] = conv3x3_wgrad(x, df0)
    return loss, pack_params(grads)


def dp_aggregate(grads, weights=None):
    """Weighted gradient aggregation across ranks (§6.2; weights unspecified in
    the paper, R11): g = sum_r w_r g_r / sum_r w_r."""
    grads = [np.asarray(g, dtype=np.float64) for g in grads]
    w = np.ones(len(grads)) if weights is None else np.asarray(weights, dtype=np.float64)
    return sum(wi * gi for wi, gi in zip(w, grads)) / w.sum()


def adam_step(p, m, v, g, t, lr=1e-4, beta1=0.9, beta2=0.999, eps=1e-8):
    """Adam (Kingma & Ba, PAPER.md L1247-1248 [53]; lr 1e-4 L1250; R7: PyTorch defaults, bias-corrected,
    no weight decay).  t counts from 1.  Returns (p, m, v) in fp64."""
    p = np.asarray(p, dtype=np.float64)
    g = np.asarray(g, dtype=np.float64)
    m = beta1 * np.asarray(m, dtype=np.float64) + (1.0 - beta1) * g
    v = beta2 * np.asarray(v, dtype=np.float64) + (1.0 - beta2) * g * g
    mhat = m / (1.0 - beta1 ** t)
    vhat = v / (1.0 - beta2 ** t)
    p = p - lr * mhat / (np.sqrt(vhat) + eps)
    return p, m, v


# ----------------------------------------------------------------------------------------------------
# recency-weighted mini-batch sampler (§6.2: the K = 150 most recent patches get
# four times the weight; R10: integer weights, with replacement) and LR/HR crop gather
# (patches carry timestamp + location).  Counter-based RNG (R10):
#   u_k = mix64(seed + GAMMA * ((((t*G + r) * 2^20 + j) * 4) + k + 1))   (mod 2^64), k = 0,1,2
# ----------------------------------------------------------------------------------------------------

def _mix64(z):
    z &= MASK64
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & MASK64
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & MASK64
    return z ^ (z >> 31)


def _u(seed, t, G, r, j, k):
    ctr = ((((t * G + r) << 20) + j) * 4 + k + 1) & MASK64
    return _mix64((seed + GAMMA * ctr) & MASK64)


def sample_indices(seed, step, n_view, batch, p_pool, p, rank=0, world=1, recent_k=150, recent_w=4):
    """Returns (idx[batch] in 0..n_view-1 of the rank's pool view, oy[batch], ox[batch]).
    Index rule: K' = min(K, n), W = w K' + (n - K'), q = floor(u0 W / 2^64);
    q < w K' -> n-1-floor(q/w) (newest first) else q - w K' (oldest first).
    Crop offsets o = floor(u (Pp - P + 1) / 2^64)."""
    n = n_view
    kp = min(recent_k, n)
    Wt = recent_w * kp + (n - kp)
    idx = np.empty(batch, np.int64)
    oy = np.empty(batch, np.int64)
    ox = np.empty(batch, np.int64)
    span = p_pool - p + 1
    for j in range(batch):
        q = (_u(seed, step, world, rank, j, 0) * Wt) >> 64
        idx[j] = (n - 1 - q // recent_w) if q < recent_w * kp else (q - recent_w * kp)
        oy[j] = (_u(seed, step, world, rank, j, 1) * span) >> 64
        ox[j] = (_u(seed, step, world, rank, j, 2) * span) >> 64
    return idx, oy, ox


def gather_patches(lr_pool, hr_pool, idx, oy, ox, p, scale):
    """Byte copy: LR crop [oy:oy+P, ox:ox+P], HR crop at (s*oy, s*ox) of size sP."""
    lr = np.stack([lr_pool[i, y:y + p, x:x + p] for i, y, x in zip(idx, oy, ox)])
    sp = scale * p
    hr = np.stack([hr_pool[i, scale * y:scale * y + sp, scale * x:scale * x + sp]
                   for i, y, x in zip(idx, oy, ox)])
    return lr, hr


# ----------------------------------------------------------------------------------------------------
# quality (§6.1: HQ patches as reference, PSNR of the SR'd patch; L1659-1661 PSNR;
# Q_DNN = improvement due to SR, L896-917; R13/R14: RGB u8, per-patch PSNR averaged, cap 100 dB)
# ----------------------------------------------------------------------------------------------------

def psnr_u8(a_u8, b_u8):
    """Per-patch PSNR over the leading axis: SSE exact integer; 10 log10(255^2 count / SSE)."""
    a = np.asarray(a_u8).astype(np.int64)
    b = np.asarray(b_u8).astype(np.int64)
    n = a.shape[0]
    out = np.empty(n)
    for i in range(n):
        sse = int(np.sum((a[i] - b[i]) ** 2))
        cnt = a[i].size
        out[i] = 100.0 if sse == 0 else 10.0 * math.log10(255.0 * 255.0 * cnt / sse)
    return out


def psnr_gain(sr_a_u8, sr_b_u8, hr_u8):
    """(mean PSNR of A, mean PSNR of B, gain = A - B), each against the HR reference patches."""
    pa = float(np.mean(psnr_u8(sr_a_u8, hr_u8)))
    pb = float(np.mean(psnr_u8(sr_b_u8, hr_u8)))
    return pa, pb, pa - pb

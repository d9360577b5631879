"""Shared test utilities (no method arithmetic: rounding/layout helpers and comparison metrics)."""
import numpy as np
import torch


def bf16_round(a):
    """Round to bf16 (RNE) and return float64."""
    return torch.from_numpy(np.ascontiguousarray(a, dtype=np.float32)).to(torch.bfloat16).to(torch.float64).numpy()


def to_dev_bf16(a_nhwc, cpad):
    """float NHWC -> device bf16 NHWC with channels zero-padded to cpad."""
    a = np.asarray(a_nhwc, dtype=np.float32)
    n, h, w, c = a.shape
    out = np.zeros((n, h, w, cpad), np.float32)
    out[..., :c] = a
    return torch.from_numpy(out).to(torch.bfloat16).cuda().contiguous()


def from_dev_bf16(t, c=None):
    a = t.float().cpu().numpy().astype(np.float64)
    return a if c is None else a[..., :c]


def rel_l2(a, b):
    a = np.asarray(a, np.float64).ravel()
    b = np.asarray(b, np.float64).ravel()
    return float(np.linalg.norm(a - b) / max(np.linalg.norm(b), 1e-300))


def psnr(a_u8, b_u8):
    d = np.asarray(a_u8, np.float64) - np.asarray(b_u8, np.float64)
    mse = np.mean(d * d)
    return 100.0 if mse == 0 else 10 * np.log10(255.0 ** 2 / mse)


def rup16(c):
    return (c + 15) // 16 * 16

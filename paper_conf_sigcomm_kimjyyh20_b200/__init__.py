"""B200-native LiveNAS super-resolution hot path (SIGCOMM '20, Kim et al.).

`SRContext` is a thin Python face of the C ABI in include/sr.h (libsr.so): torch is used for device memory
and streams only; all compute runs in the library's sm_100a kernels.  See DESIGN.md.
"""
from __future__ import annotations

import ctypes as C

from . import _lib
from ._lib import MODELS, SRError, check, load, sr_options, sr_quality  # noqa: F401
from ._lib import SR_EV_NONE, SR_EV_RESUME, SR_EV_SUSPEND, SR_SUSPENDED, SR_TRAINING  # noqa: F401

__all__ = ["SRContext", "Controller", "load", "SRError", "MODELS"]


def _ptr(t):
    return C.c_void_p(t.data_ptr()) if t is not None else None


def _chk(t, shape=None, dtype="uint8", cuda=True, name="tensor", min_numel=None):
    """Argument check before a raw pointer crosses the C ABI (the library cannot see dtype, device, strides or
    extent): the dtype, device kind, contiguity and exact shape (or a minimum element count) must match."""
    import torch
    want = getattr(torch, dtype)
    if not isinstance(t, torch.Tensor):
        raise SRError(f"{name}: expected a torch.Tensor, got {type(t).__name__}")
    if t.dtype != want:
        raise SRError(f"{name}: dtype {t.dtype}, expected {want}")
    if t.is_cuda != cuda:
        raise SRError(f"{name}: must be a {'CUDA' if cuda else 'host (CPU)'} tensor")
    if not t.is_contiguous():
        raise SRError(f"{name}: must be contiguous")
    if shape is not None and tuple(t.shape) != tuple(shape):
        raise SRError(f"{name}: shape {tuple(t.shape)}, expected {tuple(shape)}")
    if min_numel is not None and t.numel() < min_numel:
        raise SRError(f"{name}: needs >= {min_numel} elements, has {t.numel()}")
    return t


def _nhwc3(t, name, cuda=True):
    """u8 [n, h, w, 3] (an image batch)."""
    if t.dim() != 4 or t.shape[-1] != 3:
        raise SRError(f"{name}: expected [n, h, w, 3], got {tuple(t.shape)}")
    return _chk(t, None, "uint8", cuda, name)


def _loss(loss):
    return None if loss is None else _chk(loss, None, "float32", True, "loss", min_numel=1)


def _stream(stream):
    import torch
    s = stream if stream is not None else torch.cuda.current_stream()
    return C.c_void_p(s.cuda_stream)


def _model(m):
    return MODELS[m] if isinstance(m, str) else int(m)


class Controller:
    """Algorithm 1's Training/Suspended state machine (App. A), held in the library's sr_controller
    struct.  `update(diff)` is one training epoch (Training) or one validation period (Suspended); it is host
    logic and needs no GPU.  `SRContext.controller_step` measures the diff on the GPU and calls it."""

    STATES = {SR_TRAINING: "training", SR_SUSPENDED: "suspended"}
    EVENTS = {SR_EV_NONE: None, SR_EV_SUSPEND: "suspend", SR_EV_RESUME: "resume"}

    def __init__(self, thresh_sat: float, count_sat: int, thresh_online: float, count_online: int):
        self.lib = load()
        self.c = _lib.sr_controller()
        check(self.lib.sr_controller_init(C.byref(self.c), thresh_sat, count_sat, thresh_online, count_online),
              None, "sr_controller_init")

    @property
    def state(self) -> str:
        return self.STATES[self.c.state]

    @property
    def patience(self) -> int:
        return self.c.patience

    def update(self, diff: float):
        ev = C.c_int(0)
        check(self.lib.sr_controller_update(C.byref(self.c), float(diff), C.byref(ev)), None,
              "sr_controller_update")
        return self.EVENTS[ev.value]


class SRContext:
    """One per-stream SR network (sr_create).  Tensors passed in must be CUDA uint8 NHWC, contiguous."""

    def __init__(self, scale: int, blocks: int, channels: int, seed: int = 0, lr: float = 0.0,
                 world: int = 1, rank: int = 0, dp_weight: float = 0.0, recent_k: int = 0, recent_w: int = 0,
                 pool_capacity: int = 0, loss: str = "mse", skip: str = "bilinear", nccl_id: bytes | None = None,
                 device: int | None = None):
        """nccl_id: the 128-byte id of the DP group (parallel.nccl_id_broadcast), given to every rank -> the ctx owns
        an NCCL communicator and train_step / train_sampled exchange the gradient themselves (sr_options.nccl_id).
        device: CUDA ordinal (default: torch's current device)."""
        import torch
        if not torch.cuda.is_available():
            raise SRError("SRContext needs a CUDA device (no CPU fallback)")
        self.lib = load()
        self.scale, self.blocks, self.channels = scale, blocks, channels
        if nccl_id is not None and len(nccl_id) != 128:
            raise SRError("nccl_id must be the 128 bytes of an ncclUniqueId")
        self._id_buf = C.create_string_buffer(bytes(nccl_id), 128) if nccl_id is not None else None
        opt = sr_options(seed=seed, lr=lr, world=world, rank=rank, dp_weight=dp_weight, recent_k=recent_k,
                         recent_w=recent_w, pool_capacity=pool_capacity, loss={"mse": 0, "l1": 1}[loss],
                         skip={"bilinear": 0, "bicubic": 1}[skip],
                         device=torch.cuda.current_device() if device is None else int(device),
                         nccl_id=C.cast(self._id_buf, C.c_void_p) if self._id_buf is not None else None)
        h = C.c_void_p()
        st = self.lib.sr_create(scale, blocks, channels, C.byref(opt), C.byref(h))
        if st != 0:
            raise SRError(f"sr_create({scale},{blocks},{channels}) failed with status {st}")
        self.h = h

    def close(self):
        if getattr(self, "h", None):
            self.lib.sr_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    # ---------------------------------------------------------------- parameters
    @property
    def num_params(self) -> int:
        return int(self.lib.sr_num_params(self.h))

    def get_params(self, which="train"):
        import numpy as np
        out = np.empty(self.num_params, dtype=np.float32)
        check(self.lib.sr_get_params(self.h, _model(which), out.ctypes.data_as(C.c_void_p), out.size), self.h,
              "sr_get_params")
        return out

    def set_params(self, flat):
        import numpy as np
        a = np.ascontiguousarray(flat, dtype=np.float32)
        check(self.lib.sr_set_params(self.h, a.ctypes.data_as(C.c_void_p), a.size), self.h, "sr_set_params")

    # ---------------------------------------------------------------- inference
    def infer(self, lr, which="serve", out=None, stream=None):
        import torch
        n, h, w, _ = _nhwc3(lr, "lr").shape
        s = self.scale
        if out is None:
            out = torch.empty((n, s * h, s * w, 3), dtype=torch.uint8, device=lr.device)
        _chk(out, (n, s * h, s * w, 3), name="out")
        check(self.lib.sr_infer(self.h, _model(which), _ptr(lr), n, h, w, _ptr(out), _stream(stream)), self.h,
              "sr_infer")
        return out

    def infer_host(self, lr_host, out_host, which="serve", stream=None):
        """lr_host / out_host: CPU uint8 tensors (pinned for speed)."""
        n, h, w, _ = _nhwc3(lr_host, "lr_host", cuda=False).shape
        _chk(out_host, (n, self.scale * h, self.scale * w, 3), cuda=False, name="out_host")
        check(self.lib.sr_infer_host(self.h, _model(which), _ptr(lr_host), n, h, w, _ptr(out_host),
                                     _stream(stream)), self.h, "sr_infer_host")
        return out_host

    def infer_host_async(self, lr_host, out_host, which="serve", stream=None):
        """sr_infer_host_async: enqueue H2D / compute / D2H and return; out_host is valid after infer_host_wait()."""
        n, h, w, _ = _nhwc3(lr_host, "lr_host", cuda=False).shape
        _chk(out_host, (n, self.scale * h, self.scale * w, 3), cuda=False, name="out_host")
        check(self.lib.sr_infer_host_async(self.h, _model(which), _ptr(lr_host), n, h, w, _ptr(out_host),
                                           _stream(stream)), self.h, "sr_infer_host_async")
        return out_host

    def infer_host_wait(self):
        check(self.lib.sr_infer_host_wait(self.h), self.h, "sr_infer_host_wait")

    def infer_rows(self, lr_frame, row0, row1, hr_frame, which="serve", stream=None):
        if lr_frame.dim() != 3 or lr_frame.shape[-1] != 3:
            raise SRError(f"lr_frame: expected [h, w, 3], got {tuple(lr_frame.shape)}")
        h, w, _ = _chk(lr_frame, None, name="lr_frame").shape
        _chk(hr_frame, (self.scale * h, self.scale * w, 3), name="hr_frame")
        check(self.lib.sr_infer_rows(self.h, _model(which), _ptr(lr_frame), h, w, row0, row1, _ptr(hr_frame),
                                     _stream(stream)), self.h, "sr_infer_rows")
        return hr_frame

    def infer_i420(self, y, u, v, which="serve", out=None, stream=None):
        """I420 in (y [n,h,w], u/v [n,h/2,w/2] uint8 CUDA), I420 out at s x (sr_infer_i420)."""
        import torch
        if y.dim() != 3:
            raise SRError(f"y: expected [n, h, w], got {tuple(y.shape)}")
        n, h, w = _chk(y, None, name="y").shape
        _chk(u, (n, h // 2, w // 2), name="u")
        _chk(v, (n, h // 2, w // 2), name="v")
        s = self.scale
        if out is None:
            out = (torch.empty((n, s * h, s * w), dtype=torch.uint8, device=y.device),
                   torch.empty((n, s * h // 2, s * w // 2), dtype=torch.uint8, device=y.device),
                   torch.empty((n, s * h // 2, s * w // 2), dtype=torch.uint8, device=y.device))
        _chk(out[0], (n, s * h, s * w), name="out[0]")
        _chk(out[1], (n, s * h // 2, s * w // 2), name="out[1]")
        _chk(out[2], (n, s * h // 2, s * w // 2), name="out[2]")
        check(self.lib.sr_infer_i420(self.h, _model(which), _ptr(y), _ptr(u), _ptr(v), n, h, w, _ptr(out[0]),
                                     _ptr(out[1]), _ptr(out[2]), _stream(stream)), self.h, "sr_infer_i420")
        return out

    # ---------------------------------------------------------------- training
    def _patches(self, lr, hr, name="patches"):
        n, p, p2, _ = _nhwc3(lr, name + " lr").shape
        if p != p2:
            raise SRError(f"{name} lr: patches must be square, got {tuple(lr.shape)}")
        _chk(hr, (n, self.scale * p, self.scale * p, 3), name=name + " hr")
        return n, p

    def train_step(self, lr, hr, loss=None, stream=None):
        """Forward, loss, backward, [NCCL gradient exchange when the ctx has a communicator], Adam (sr_train_step)."""
        n, p = self._patches(lr, hr)
        _loss(loss)
        check(self.lib.sr_train_step(self.h, _ptr(lr), _ptr(hr), n, p, _ptr(loss), _stream(stream)), self.h,
              "sr_train_step")

    def train_grad(self, lr, hr, loss=None, stream=None):
        n, p = self._patches(lr, hr)
        _loss(loss)
        check(self.lib.sr_train_grad(self.h, _ptr(lr), _ptr(hr), n, p, _ptr(loss), _stream(stream)), self.h,
              "sr_train_grad")

    def grad_buffer(self):
        """torch view of the flat fp32 gradient (for an NCCL allreduce via torch.distributed)."""
        import torch
        ptr = self.lib.sr_grad_buffer(self.h)
        n = self.num_params
        return _wrap_device_f32(ptr, n, torch.cuda.current_device())

    def train_apply(self, grad_scale=1.0, stream=None):
        check(self.lib.sr_train_apply(self.h, C.c_float(grad_scale), _stream(stream)), self.h, "sr_train_apply")

    def train_apply_dev(self, scale_dev, stream=None):
        """Adam with the gradient scale read from a device float tensor (graph-capturable)."""
        _chk(scale_dev, None, "float32", True, "scale_dev", min_numel=1)
        check(self.lib.sr_train_apply_dev(self.h, _ptr(scale_dev), _stream(stream)), self.h, "sr_train_apply_dev")

    def train_allreduce(self, stream=None):
        """The DP exchange alone (sr_train_allreduce): NCCL sum-allreduce of the gradient buffer."""
        check(self.lib.sr_train_allreduce(self.h, _stream(stream)), self.h, "sr_train_allreduce")

    @property
    def dp_weight_sum(self) -> float:
        """sum_r w_r over the DP group (sr_dp_weight_sum)."""
        return float(self.lib.sr_dp_weight_sum(self.h))

    def adam_state(self):
        """(m, v, t): TRAIN's Adam moments (fp32, canonical layout) and step count (sr_get_adam_state)."""
        import numpy as np
        m = np.empty(self.num_params, np.float32)
        v = np.empty(self.num_params, np.float32)
        t = C.c_int64(0)
        check(self.lib.sr_get_adam_state(self.h, m.ctypes.data_as(C.c_void_p), v.ctypes.data_as(C.c_void_p), m.size,
                                         C.byref(t)), self.h, "sr_get_adam_state")
        return m, v, int(t.value)

    def pool_stats(self):
        """(arrivals, clamped_crops) from the device counters (sr_pool_stats)."""
        a, c = C.c_int64(0), C.c_int64(0)
        check(self.lib.sr_pool_stats(self.h, C.byref(a), C.byref(c)), self.h, "sr_pool_stats")
        return int(a.value), int(c.value)

    def pool_push(self, lr, hr, stream=None):
        n, pp = self._patches(lr, hr, "pool")
        check(self.lib.sr_pool_push(self.h, _ptr(lr), _ptr(hr), n, pp, None, _stream(stream)), self.h,
              "sr_pool_push")

    def pool_push_i420(self, y, u, v, hr, xy, stream=None):
        """HR patches hr [n,s*pp,s*pp,3] with LR counterparts cropped from one decoded I420 frame (y [h,w], u/v
        [h/2,w/2]) at LR corners xy [n,2] int32 (x, y)."""
        h, w = _chk(y, None, name="y").shape[-2:]
        if y.dim() != 2:
            raise SRError(f"y: expected one frame [h, w], got {tuple(y.shape)}")
        _chk(u, (h // 2, w // 2), name="u")
        _chk(v, (h // 2, w // 2), name="v")
        n, pp = _nhwc3(hr, "hr").shape[0], hr.shape[1] // self.scale
        _chk(hr, (n, self.scale * pp, self.scale * pp, 3), name="hr")
        _chk(xy, (n, 2), "int32", name="xy")
        check(self.lib.sr_pool_push_i420(self.h, _ptr(y), _ptr(u), _ptr(v), h, w, _ptr(hr), _ptr(xy), n, pp, None,
                                         _stream(stream)), self.h, "sr_pool_push_i420")

    @property
    def pool_size(self) -> int:
        return int(self.lib.sr_pool_size(self.h))

    def sample_batch(self, step, batch, p, out=None, stream=None):
        import torch
        s = self.scale
        if out is None:
            lr = torch.empty((batch, p, p, 3), dtype=torch.uint8, device="cuda")
            hr = torch.empty((batch, s * p, s * p, 3), dtype=torch.uint8, device="cuda")
            idx = torch.empty(batch, dtype=torch.int32, device="cuda")
        else:
            lr, hr, idx = out
        _chk(lr, (batch, p, p, 3), name="out lr")
        _chk(hr, (batch, s * p, s * p, 3), name="out hr")
        if idx is not None:
            _chk(idx, (batch,), "int32", name="out idx")
        check(self.lib.sr_sample_batch(self.h, step, batch, p, _ptr(lr), _ptr(hr), _ptr(idx), _stream(stream)),
              self.h, "sr_sample_batch")
        return lr, hr, idx

    def train_sampled(self, iters, batch, p, loss=None, stream=None):
        """`iters` sampled training iterations from one captured CUDA graph (sr_train_sampled; with a communicator
        each iteration includes the NCCL gradient exchange)."""
        _loss(loss)
        check(self.lib.sr_train_sampled(self.h, iters, batch, p, _ptr(loss), _stream(stream)), self.h,
              "sr_train_sampled")

    def publish(self, stream=None):
        check(self.lib.sr_publish(self.h, _stream(stream)), self.h, "sr_publish")

    def psnr_gain(self, lr, hr, a="serve", b="bilinear", stream=None):
        q = sr_quality()
        n, p = self._patches(lr, hr, "validation")
        check(self.lib.sr_psnr_gain(self.h, _model(a), _model(b), _ptr(lr), _ptr(hr), n, p, C.byref(q),
                                    _stream(stream)), self.h, "sr_psnr_gain")
        return q.psnr_a, q.psnr_b, q.gain

    def controller_step(self, ctrl: Controller, lr, hr, stream=None) -> dict:
        """Epoch-end / validation hook (sr_controller_step): PSNR of SERVE/PREV/INIT/bilinear on the recent
        patches, Algorithm 1's diff and transition, and the Q_DNN feedback."""
        r = _lib.sr_epoch_report()
        n, p = self._patches(lr, hr, "validation")
        check(self.lib.sr_controller_step(self.h, C.byref(ctrl.c), _ptr(lr), _ptr(hr), n, p, C.byref(r),
                                          _stream(stream)), self.h, "sr_controller_step")
        out = {f: getattr(r, f) for f, _ in r._fields_}
        out["state_before"] = Controller.STATES[r.state_before]
        out["state_after"] = Controller.STATES[r.state_after]
        out["event"] = Controller.EVENTS[r.event]
        return out

    def patch_select(self, raw, dec, cell=120, max_sel=10, seed=0, step=0, stream=None):
        """The ingest client's patch selection (sr_patch_select): [(x, y), ...] of the kept cells in order."""
        import numpy as np
        if raw.dim() != 3 or raw.shape[-1] != 3:
            raise SRError(f"raw: expected [h, w, 3], got {tuple(raw.shape)}")
        h, w = _chk(raw, None, name="raw").shape[:2]
        _chk(dec, (h, w, 3), name="dec")
        xy = np.zeros(2 * max(max_sel, 1), np.int32)
        n = C.c_int(0)
        check(self.lib.sr_patch_select(self.h, _ptr(raw), _ptr(dec), h, w, cell, max_sel, seed, step,
                                       xy.ctypes.data_as(C.c_void_p), C.byref(n), _stream(stream)), self.h,
              "sr_patch_select")
        return [(int(xy[2 * i]), int(xy[2 * i + 1])) for i in range(n.value)]

    def set_fusion(self, fuse_blocks=True):
        check(self.lib.sr_set_fusion(self.h, int(fuse_blocks)), self.h, "sr_set_fusion")

    @staticmethod
    def sm_partition(train_sms):
        """sr_sm_partition: (infer_stream, train_stream, infer_sms, train_sms) -- torch ExternalStreams whose kernels
        run on disjoint SM partitions (green contexts); release with SRContext.sm_partition_release()."""
        import torch
        lib = load()
        si, stt = C.c_void_p(), C.c_void_p()
        ni, nt = C.c_int(0), C.c_int(0)
        check(lib.sr_sm_partition(int(train_sms), C.byref(si), C.byref(stt), C.byref(ni), C.byref(nt)), None,
              "sr_sm_partition")
        return (torch.cuda.ExternalStream(si.value), torch.cuda.ExternalStream(stt.value), int(ni.value),
                int(nt.value))

    @staticmethod
    def sm_partition_release():
        check(load().sr_sm_partition_release(), None, "sr_sm_partition_release")

    def set_sm_split(self, train_sms):
        """sr_set_sm_split: training-side calls use train_sms SMs, inference-side calls the rest (0 = all)."""
        check(self.lib.sr_set_sm_split(self.h, int(train_sms)), self.h, "sr_set_sm_split")

    def kernel_timing(self, enable=True):
        check(self.lib.sr_kernel_timing(self.h, int(enable)), self.h, "sr_kernel_timing")

    def kernel_stats(self):
        import json
        buf = C.create_string_buffer(1 << 16)
        n = self.lib.sr_kernel_stats(self.h, buf, len(buf))
        if n < 0:
            raise SRError(f"sr_kernel_stats failed: {n}")
        return json.loads(buf.value.decode())

    @property
    def launches(self) -> int:
        return int(self.lib.sr_launch_count(self.h))


def _wrap_device_f32(ptr, n, device):
    """Zero-copy torch tensor over a device pointer owned by the ctx (via __cuda_array_interface__)."""
    import torch

    class _Arr:
        __cuda_array_interface__ = {"shape": (n,), "typestr": "<f4", "data": (ptr, False), "version": 3,
                                    "strides": None}
    return torch.as_tensor(_Arr(), device=f"cuda:{device}")

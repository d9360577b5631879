#!/usr/bin/env python
"""Achieved HBM bandwidth of the memory-bound kernels of the hot path (SURVEY.md §8(d) memory-bound list), live with
CUDA events on the launching stream, against MEASURED_PEAKS.json hbm_gbs; run it under
`ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum -k regex:'k_adam|k_sample_gather|
k_sse_u8|k_conv_roll|k_pack_weights'` for the DRAM traffic per launch.

Algorithmic bytes per launch:
  * k_adam (T6): read p, m, v, g + write p, m, v = 28 B per parameter; at the bench net (366,363 params) and on a
    64 Mi-parameter flat buffer (bandwidth-bound size);
  * k_sample_gather (T1): the crops read + written, 2 x 64 x (48^2 + 144^2) x 3 B at the bench batch;
  * k_sse_u8 (Q1): 2 B per sample pair; one 4K frame pair (49.8 MB) and the 64 validation patches of the bench;
  * k_conv_roll<16,48,0,u8> (A1 head, inference): 3 B in + 96 B out per LR pixel (30 720p frames).
"""
from __future__ import annotations

import ctypes
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import argparse
    ap = argparse.ArgumentParser()
    ap.add_argument("--only", default="", help="comma list of: adam_small,adam64m,gather,sse4k,sseval,infer")
    args = ap.parse_args()
    only = set(x for x in args.only.split(",") if x)

    def want(k):
        return not only or k in only
    import numpy as np
    import torch
    from paper_conf_sigcomm_kimjyyh20_b200 import SRContext, load
    from synth import synth_frames, synth_patch_pool
    lib = load()
    peak = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json"))).get("hbm_gbs", 6538.0) \
        if os.path.exists(os.path.join(ROOT, "MEASURED_PEAKS.json")) else 6538.0
    st = torch.cuda.current_stream()
    sp = ctypes.c_void_p(st.cuda_stream)
    rows = []

    def timeit(fn, reps=20, warm=3):
        for _ in range(warm):
            fn()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(reps):
            fn()
        e1.record()
        torch.cuda.synchronize()
        return e0.elapsed_time(e1) / reps

    # ---- Adam
    for n in [n for n, k in ((366363, "adam_small"), (64 << 20, "adam64m")) if want(k)]:
        p = torch.randn(n, device="cuda") * 0.05
        m = torch.zeros(n, device="cuda")
        v = torch.zeros(n, device="cuda")
        g = torch.randn(n, device="cuda") * 1e-3
        f10 = lambda: lib.sr_test_adam(ctypes.c_void_p(p.data_ptr()), ctypes.c_void_p(m.data_ptr()),  # noqa: E731
                                       ctypes.c_void_p(v.data_ptr()), ctypes.c_void_p(g.data_ptr()), n, 10,
                                       ctypes.c_float(1e-4), sp)
        ms = timeit(f10, reps=5) / 10  # (includes the 1-thread step-counter kernel between Adam launches)
        rows.append(("k_adam", f"{n} params", 28 * n, ms))
        del p, m, v, g
    # ---- sample + gather at the bench batch (x3, pool of 60x60 LR entries)
    ctx = SRContext(3, 8, 48, seed=0)
    plr, phr, _ = synth_patch_pool(512, 3, 180, seed=1004, frame_hw=(1080, 1800))
    ctx.pool_push(torch.from_numpy(plr).cuda(), torch.from_numpy(phr).cuda())
    blr = torch.empty((64, 48, 48, 3), dtype=torch.uint8, device="cuda")
    bhr = torch.empty((64, 144, 144, 3), dtype=torch.uint8, device="cuda")
    if want("gather"):
        ms = timeit(lambda: ctx.sample_batch(-1, 64, 48, out=(blr, bhr, None)))
        rows.append(("k_sample_gather", "64 x (48^2 + 144^2) x 3 B", 2 * 64 * (48 * 48 + 144 * 144) * 3, ms))
    # ---- SSE: one 4K frame pair; the bench's 64 validation patches (180x180 HR)
    a = torch.from_numpy(synth_frames(1, 2160, 3840, seed=1)).cuda()
    b = torch.from_numpy(synth_frames(1, 2160, 3840, seed=2)).cuda()
    out = torch.zeros(64, dtype=torch.int64, device="cuda")
    el = 2160 * 3840 * 3
    if want("sse4k"):
        ms = timeit(lambda: lib.sr_sse_u8(ctypes.c_void_p(a.data_ptr()), ctypes.c_void_p(b.data_ptr()), 1, el,
                                          ctypes.c_void_p(out.data_ptr()), sp))
        rows.append(("k_sse_u8", "one 4K frame pair", 2 * el, ms))
    va = torch.from_numpy(phr[:64].copy()).cuda()
    vb = torch.from_numpy(phr[64:128].copy()).cuda()
    el = 180 * 180 * 3
    if want("sseval"):
        ms = timeit(lambda: lib.sr_sse_u8(ctypes.c_void_p(va.data_ptr()), ctypes.c_void_p(vb.data_ptr()), 64, el,
                                          ctypes.c_void_p(out.data_ptr()), sp))
        rows.append(("k_sse_u8", "64 validation patches 180x180", 2 * 64 * el, ms))
    # ---- head conv from u8 (inference of 30 720p frames, timed per kernel class by the library)
    if not want("infer"):
        out_rows = []
        for name, shape, by, ms in rows:
            gbs = by / (ms * 1e-3) / 1e9
            out_rows.append({"kernel": name, "shape": shape, "algorithmic_bytes": int(by), "ms": round(ms, 5),
                             "GB/s": round(gbs, 1), "frac_of_hbm": round(gbs / peak, 4)})
        print(json.dumps({"hbm_peak_gbs": peak, "rows": out_rows}, indent=1))
        return
    lr = torch.from_numpy(synth_frames(30, 720, 1280, seed=1003)).cuda()
    hr = torch.empty((30, 2160, 3840, 3), dtype=torch.uint8, device="cuda")
    for _ in range(3):
        ctx.infer(lr, "serve", out=hr)
    ctx.kernel_timing(True)
    for _ in range(10):
        ctx.infer(lr, "serve", out=hr)
    stats = ctx.kernel_stats()
    ctx.kernel_timing(False)
    h = stats["conv_roll_16x48"]
    rows.append(("k_conv_roll<16,48,u8> (head)", "30 x 720p", h["bytes"] / h["launches"], h["ms"] / h["launches"]))
    bt = stats["bodytail_48x32"]
    rows.append(("k_bodytail<48,32,3> (body+up+tail)", "30 x 720p, bytes only", bt["bytes"] / bt["launches"],
                 bt["ms"] / bt["launches"]))
    out_rows = []
    for name, shape, by, ms in rows:
        gbs = by / (ms * 1e-3) / 1e9
        out_rows.append({"kernel": name, "shape": shape, "algorithmic_bytes": int(by), "ms": round(ms, 5),
                         "GB/s": round(gbs, 1), "frac_of_hbm": round(gbs / peak, 4)})
    print(json.dumps({"hbm_peak_gbs": peak, "rows": out_rows}, indent=1))


if __name__ == "__main__":
    main()

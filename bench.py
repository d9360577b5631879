#!/usr/bin/env python
"""Benchmark of the LiveNAS SR hot path on B200 (one process per GPU).

Workload (BASELINE.json config 3 + config 4): per rank and per step
  * A1-A4  super-resolve a batch of 30 synthetic 720p LR frames to 4K (x3, 8 res blocks x 48 ch)  [sr_infer]
  * T1-T6  10 online-training iterations (the paper's cadence: 50 iterations per 5-s epoch = one per 3 frames
           at 30 fps, PAPER.md L916-917 / L1247-1250): recency-weighted sample + gather of 64 patches
           (48x48 LR -> 144x144 HR), forward, MSE, backward, [NCCL allreduce of the gradient over NVLink
           when N > 1], Adam                                                                         [sr_sample_batch,
                                                                                                       sr_train_grad, sr_train_apply]
  * T7     at each epoch end (every 50 iterations = every 5th step, L1247-1253): publish (TRAIN -> SERVE)
                                                                                                     [sr_publish]
  * Q1     and Algorithm 1's epoch-end evaluation on 64 recent patches: PSNR of SERVE, PREV, INIT and bilinear,
           the saturation diff and Q_DNN (reported; the bench stays in the Training state, whose work is
           the expensive one, so every epoch does the same work)                                     [sr_controller_step]
The headline metric is 4K frames/s summed over ranks (weak scaling: frames are sharded, 30 per rank per step);
training patches/s is reported beside it.  `--impl reference` times the fp64 CPU oracle (the paper has no code).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

S, BLOCKS, CH = 3, 8, 48
LR_H, LR_W = 720, 1280
FRAMES = 30
ITERS = 10
EPOCH_ITERS = 50  # training iterations per epoch; publish + Algorithm 1 at its end
BATCH, PATCH = 64, 48
POOL_N, POOL_LR = 512, 60           # pool entries: 60x60 LR / 180x180 HR (crop offsets span 0..12)
VAL_N = 64
FLOP_PER_LR_PX = 2 * 9 * (3 * CH + 2 * BLOCKS * CH * CH + CH * CH + CH * 3 * S * S)
# one training iteration: forward + data-grad (no input grad for the head) + weight-grad
TRAIN_FLOP = BATCH * PATCH * PATCH * (3 * FLOP_PER_LR_PX - 2 * 9 * 3 * CH)


def peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        return {}


def dist_env():
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return world, rank, local


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled every 200 ms during the timed region."""

    FIELDS = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
              "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
              "clocks_event_reasons.sw_power_cap")

    def __init__(self, index):
        self.index = index
        self.p = None

    def start(self):
        try:
            self.p = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.FIELDS}",
                                       "--format=csv,noheader,nounits", "-lms", "200"],
                                      stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except Exception:
            self.p = None

    def stop(self):
        if self.p is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.p.terminate()
        out, _ = self.p.communicate(timeout=10)
        rows = []
        for ln in out.strip().splitlines():
            parts = [x.strip() for x in ln.split(",")]
            if len(parts) == 7:
                try:
                    rows.append((float(parts[0]), float(parts[1]), float(parts[2]), parts[3:]))
                except ValueError:
                    pass
        if not rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["no samples"]}
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in rows for i, v in enumerate(r[3]) if v.lower().startswith("active")})
        loaded = [r for r in rows if r[2] > 300.0] or rows
        return {"sm_mhz": statistics.median(r[0] for r in loaded), "sm_max_mhz": max(r[1] for r in rows),
                "reasons": reasons, "samples": len(rows), "samples_under_load": len(loaded)}


def run_ours(args):
    import numpy as np
    import torch
    import torch.distributed as dist
    from paper_conf_sigcomm_kimjyyh20_b200 import Controller, SRContext
    from paper_conf_sigcomm_kimjyyh20_b200.parallel import dp_allreduce_grad_dev, max_over_ranks
    from synth import synth_frames, synth_patch_pool

    world, rank, local = dist_env()
    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    dev = torch.device("cuda", local)
    frames = args.frames
    ctx = SRContext(S, BLOCKS, CH, seed=0, world=world, rank=rank)
    # ---- synthetic inputs (seeded; per-rank frame shard)
    lr_np = synth_frames(frames, LR_H, LR_W, seed=1003 + rank)
    lr = torch.from_numpy(lr_np).to(dev)
    hr = torch.empty((frames, S * LR_H, S * LR_W, 3), dtype=torch.uint8, device=dev)
    plr, phr, _ = synth_patch_pool(POOL_N, S, S * POOL_LR, seed=1004, frame_hw=(1080, 1800))
    ctx.pool_push(torch.from_numpy(plr).to(dev), torch.from_numpy(phr).to(dev))
    val_lr = torch.from_numpy(plr[-VAL_N:]).to(dev)
    val_hr = torch.from_numpy(phr[-VAL_N:]).to(dev)
    blr = torch.empty((BATCH, PATCH, PATCH, 3), dtype=torch.uint8, device=dev)
    bhr = torch.empty((BATCH, S * PATCH, S * PATCH, 3), dtype=torch.uint8, device=dev)
    bidx = torch.empty(BATCH, dtype=torch.int32, device=dev)
    loss = torch.zeros(1, dtype=torch.float32, device=dev)
    grad = ctx.grad_buffer()
    state = {"q": None}

    wdev = torch.ones(1, dtype=torch.float32, device=dev)  # this rank's gradient weight w_r
    inv_w = wdev.reciprocal()  # single GPU: the Adam scale 1 / w_0 (no exchange step)

    def train_iter():
        ctx.sample_batch(-1, BATCH, PATCH, out=(blr, bhr, bidx))   # device-side step counter
        ctx.train_grad(blr, bhr, loss)                            # grad <- w_r g_r
        # NCCL sum-allreduce over NVLink (N > 1) -> Adam scale 1 / sum_r w_r
        scale = dp_allreduce_grad_dev(grad, wdev) if world > 1 else inv_w
        ctx.train_apply_dev(scale)

    # one training iteration captured as a CUDA graph (after an eager warm-up that sizes the workspaces)
    train_iter()
    torch.cuda.synchronize()
    graph = None
    launches_per_iter = 0
    if not args.no_graph:
        graph = torch.cuda.CUDAGraph()
        lc = ctx.launches
        try:
            with torch.cuda.graph(graph):
                train_iter()
            launches_per_iter = ctx.launches - lc   # our kernels inside one captured iteration
        except Exception as exc:  # e.g. a collective that cannot be captured: launch the iterations eagerly
            print(f"[bench] rank {rank}: training-iteration graph capture failed ({exc}); eager iterations",
                  file=sys.stderr, flush=True)
            graph = None
            torch.cuda.synchronize()

    ctrl = Controller(thresh_sat=0.05, count_sat=2, thresh_online=0.5, count_online=2)
    state["iters"] = 0  # training iterations since the last epoch end

    def epoch_eval():
        r = ctx.controller_step(ctrl, val_lr, val_hr)
        if ctrl.state != "training":  # keep the measured work constant (see the docstring)
            ctrl.c.state, ctrl.c.patience = 0, 0
        state["q"] = r
        state["epochs"] = state.get("epochs", 0) + 1

    def train_iters():
        for _ in range(args.iters):
            if graph is not None:
                graph.replay()
            else:
                train_iter()
        state["iters"] += args.iters
        if state["iters"] >= EPOCH_ITERS:  # epoch end (50 iterations, L1247-1250): publish + Algorithm 1
            state["iters"] = 0
            ctx.publish()
            epoch_eval()

    def step():
        ctx.infer(lr, "serve", out=hr)
        train_iters()

    def barrier():
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()

    for _ in range(args.warmup):
        step()
    barrier()
    state["iters"], state["epochs"] = 0, 0  # the timed region starts at an epoch boundary
    clk = ClockSampler(local)
    clk.start()
    l0 = ctx.launches
    ctx.kernel_timing(True)
    barrier()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(args.steps):
        step()
    e1.record()
    barrier()
    ms = e0.elapsed_time(e1)
    epochs_timed = state["epochs"]
    launches = ctx.launches - l0 + (launches_per_iter * args.iters * args.steps if graph is not None else 0)
    stats = ctx.kernel_stats()
    ctx.kernel_timing(False)
    clocks = clk.stop()
    ms = max_over_ranks(ms, device=dev)

    # ---- training iteration alone (informational; the step above already contains it)
    t0, t1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    t0.record()
    for _ in range(20):
        if graph is not None:
            graph.replay()
        else:
            train_iter()
    t1.record()
    torch.cuda.synchronize()
    train_iter_ms = t0.elapsed_time(t1) / 20

    # ---- end-to-end: host (pinned) frames in, host frames out, through the C ABI (sr_infer_host)
    lr_host = torch.from_numpy(lr_np).pin_memory()
    hr_host = torch.empty((frames, S * LR_H, S * LR_W, 3), dtype=torch.uint8).pin_memory()
    loss_host = torch.zeros(1, dtype=torch.float32).pin_memory()

    def step_e2e():
        # a serving loop: frames in and out through the host API; the training iterations are enqueued behind the
        # inference and run while the last HR chunks drain over PCIe; the step ends when its HR frames are in host
        # memory (sr_infer_host_wait) and its loss has been read back
        ctx.infer_host_async(lr_host, hr_host, "serve")
        train_iters()
        loss_host.copy_(loss, non_blocking=True)
        ctx.infer_host_wait()

    step_e2e()
    barrier()
    state["iters"] = 0
    e2, e3 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e2.record()
    for _ in range(args.steps):
        step_e2e()
    e3.record()
    barrier()
    ms_e2e = max_over_ranks(e2.elapsed_time(e3), device=dev)

    if rank == 0:
        pk = peaks()
        sustained = pk.get("bf16_tflops_sustained") or 1393.0
        # dominant kernel = class with the largest share of kernel time
        dom, dv = max(stats.items(), key=lambda kv: kv[1]["ms"])
        achieved = dv["flops"] / (dv["ms"] * 1e-3) / 1e12
        ktot = sum(v["ms"] for v in stats.values())
        total_frames = frames * args.steps * world
        fps = total_frames / (ms * 1e-3)
        fps_e2e = total_frames / (ms_e2e * 1e-3)
        conv_flops = sum(v["flops"] for v in stats.values())
        line = {
            "metric": "4K SR frames/s (720p->2160p x3, 8x48) with online training at the paper's cadence",
            "value": round(fps, 3),
            "unit": "frames/s",
            "n_gpus": world,
            "steps": args.steps,
            "warmup": args.warmup,
            "ms_per_step": round(ms / args.steps, 3),
            "higher_is_better": True,
            "scaling": "weak",
            "vs_baseline": None,
            "dtype": "bf16",
            "data": "synthetic (seeded 1/f frames + edges + strokes, pan; random-init weights)",
            "config": {
                "workload": f"cfg3+cfg4: {frames}x 720p->4K x3 frames + {args.iters} train iters (64x 48->144) "
                            "+ publish + Algorithm-1 evaluation at each epoch end (every 50 iterations) per rank",
                "net": f"x{S}, {BLOCKS} blocks x {CH} ch", "frames_per_rank": frames,
                "train_iters_per_step": args.iters, "batch": BATCH, "patch_lr": PATCH,
                "epoch_ends_timed": epochs_timed,
                "parallelism": f"frames sharded x{world}, DP training (NCCL allreduce)" if world > 1 else "1 GPU",
                "l2": "working set > L2 (one 720p activation tensor at 48 ch = 88 MB; 30 frames per step)",
            },
            "train_patches_per_s": round(BATCH * args.iters * args.steps * world / (ms * 1e-3), 1),
            "train_iter": {"ms": round(train_iter_ms, 4), "tflops": round(TRAIN_FLOP / (train_iter_ms * 1e-3) / 1e12, 1),
                           "graph": graph is not None, "note": "one sampled training iteration alone (rank 0)"},
            "quality_gain_db": round(state["q"]["q_dnn"], 4) if state["q"] else None,
            "alg1_last": {k: (round(v, 4) if isinstance(v, float) else v) for k, v in state["q"].items()}
            if state["q"] else None,
            "tensor_tflops_all_convs": round(conv_flops / (sum(v["ms"] for v in stats.values()) * 1e-3) / 1e12, 1),
            "kernel_share": {k: round(v["ms"] / ktot, 4) for k, v in sorted(stats.items(), key=lambda kv: -kv[1]["ms"])},
            "kernel_share_note": "CUDA-event time per kernel class of the eagerly launched kernels (inference, "
                                 "Algorithm-1 evaluation); the graph-replayed training kernels are in train_iter",
            "roofline": {"bound": "tensor", "kernel": dom, "achieved": round(achieved, 1),
                         "peak": sustained, "unit": "TFLOP/s", "frac": round(achieved / sustained, 4),
                         "peak_kind": "measured bf16_tflops_sustained (MEASURED_PEAKS.json)",
                         "traffic": traffic_of(dom, frames), "traffic_unit": "bytes per launch (ncu dram read+write)",
                         "algorithmic_bytes": round(dv["bytes"] / dv["launches"]),
                         "launches": dv["launches"], "avg_ms": round(dv["ms"] / dv["launches"], 4)},
            "e2e": {"value": round(fps_e2e, 3), "unit": "frames/s",
                    "h2d_bytes_per_step": int(lr_host.numel()), "d2h_bytes_per_step": int(hr_host.numel() + 4)},
            "gpu_launches": int(launches),
            "clocks": clocks,
        }
        if not args.no_cpu_baseline:
            line["cpu_baseline"] = cpu_baseline(frames, args.iters)
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


def cpu_baseline(frames, iters, band_rows=None, train_patches=None):
    """The fp64 numpy oracle, as it stands, on a bounded sample of the same workload: one 120-row band of a
    720p frame through the x3 8x48 net and one training step on 16 patches; scaled to the step's units."""
    import numpy as np
    import oracle as O
    from synth import init_params, synth_frames, synth_patch_pool
    band_rows = band_rows or int(os.environ.get("SR_CPU_BAND_ROWS", "120"))
    train_patches = train_patches or int(os.environ.get("SR_CPU_TRAIN_PATCHES", "16"))
    p = init_params(S, BLOCKS, CH, seed=0)
    lr = synth_frames(1, band_rows, LR_W, seed=1003)
    t0 = time.perf_counter()
    O.infer_u8(p, lr, S, BLOCKS, CH)
    t_band = time.perf_counter() - t0
    plr, phr, _ = synth_patch_pool(train_patches, S, S * PATCH, seed=1004, frame_hw=(432, 576))
    t0 = time.perf_counter()
    _, g = O.train_loss_and_grad(p, plr, phr, S, BLOCKS, CH)
    O.adam_step(p, np.zeros_like(g), np.zeros_like(g), g, 1)
    t_train = time.perf_counter() - t0
    t_frame = t_band * LR_H / band_rows
    t_step = frames * t_frame + iters * t_train * BATCH / train_patches
    cores = len(os.sched_getaffinity(0))
    return {"value": round(frames / t_step, 6), "unit": "frames/s", "cores": cores, "kind": "oracle",
            "sample": f"{band_rows}x{LR_W} LR band ({t_band:.2f}s) + 1 train step on {train_patches} patches "
                      f"({t_train:.2f}s), scaled to {frames} frames + {iters} x {BATCH}-patch iterations",
            "train_patches_per_s": round(train_patches / t_train, 3)}


def run_reference(args):
    world, rank, _ = dist_env()
    if rank != 0:
        return
    frames, iters = args.frames, args.iters
    vals = []
    for _ in range(args.warmup):
        cpu_baseline(frames, iters, band_rows=24, train_patches=4)
    for _ in range(args.steps):
        vals.append(cpu_baseline(frames, iters, band_rows=24, train_patches=4))
    v = statistics.median(x["value"] for x in vals)
    cb = dict(vals[-1])
    cb["value"] = v
    print(json.dumps({
        "impl": "reference", "metric": "4K SR frames/s (720p->2160p x3, 8x48) with online training at the paper's cadence",
        "value": v, "unit": "frames/s", "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64",
        "data": "synthetic", "config": {"workload": f"cfg3+cfg4 per step (oracle on a bounded sample)"},
        "cpu_baseline": cb, "e2e": {"value": v, "unit": "frames/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }), flush=True)


def traffic_of(kernel_class, frames):
    """DRAM bytes per launch of the dominant kernel from the committed ncu capture (profiles/r01_traffic.json),
    when it was taken on the same launch shape; else None."""
    try:
        with open(os.path.join(ROOT, "profiles", "r01_traffic.json")) as f:
            t = json.load(f).get(kernel_class)
    except (OSError, ValueError):
        return None
    if not t or t.get("frames") != frames or (t.get("h"), t.get("w")) != (LR_H, LR_W):
        return None
    return int(t["dram_read"] + t["dram_write"])


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--frames", type=int, default=FRAMES)
    ap.add_argument("--iters", type=int, default=ITERS)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-graph", action="store_true", help="launch the training iterations eagerly")
    args = ap.parse_args()
    if args.impl == "reference":
        run_reference(args)
    else:
        run_ours(args)


if __name__ == "__main__":
    main()

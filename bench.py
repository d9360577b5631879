#!/usr/bin/env python
"""Benchmark of the LiveNAS SR hot path on B200 (one process per GPU).

Workload of one step (BASELINE.json configs 3 + 4), per rank:
  * A1-A4  super-resolve a batch of 30 synthetic 720p LR frames to 4K (x3, 8 res blocks x 48 ch)  [sr_infer]
  * ingest 3 arriving (LR, HR) patch pairs into the device pool (one second of video at 30 fps; the paper's client
           sends ~6 patches per 2 s)                                           [sr_pool_push]
  * T1-T6  10 online-training iterations (the paper's cadence: 50 iterations per 5-s epoch = one per 3 frames at
           30 fps, L916-917 / L1247-1250): recency-weighted sample + gather of 64 patches (48x48 LR -> 144x144 HR),
           forward, MSE, backward, [N > 1: NCCL sum-allreduce of w_r g_r inside the library], Adam -- one CUDA graph
           per iteration, captured and replayed by the library                                      [sr_train_sampled]
  * T7     at each epoch end (every 50 iterations = every 5th step, L1247-1253): publish (TRAIN -> SERVE) [sr_publish]
  * Q1     and Algorithm 1's epoch-end evaluation on 64 recent patches: PSNR of SERVE, PREV, INIT and bilinear, the
           saturation diff and Q_DNN [sr_controller_step].  Constant-work mode: the controller's decisions are
           reported (alg1) but the bench keeps training, so every epoch does the same work.
The headline metric is 4K frames/s summed over ranks (weak scaling: 30 frames per rank per step); training
patches/s beside it.  Beside the headline, the same JSON line carries:
  * cfg2: 540p -> 1080p x2 with the 8x32 net, batch of 30 frames (BASELINE config 2), frames/s + its roofline;
  * cfg4: training alone at the maximum rate (patches/s, ms per iteration, TFLOP/s, the dominant training kernel's
    roofline, the allreduce time at N > 1);
  * cpu_baseline: the fp64 oracle on ONE whole 720p frame and ONE whole 64-patch training step (all host cores,
    BLAS threads stated) plus the step at one thread.
`--gpus N` without a torchrun environment re-launches itself under torch.distributed.run with N ranks.
`--impl reference` times the fp64 CPU oracle (the paper has no code to install).  `--workload live` runs the
config-5 live-ingest harness instead (scripts/live_ingest.py).
"""
from __future__ import annotations

import argparse
import json
import os
import socket
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
ARRIVALS_PER_STEP = 3               # patches arriving per second of video (L3279-3281)
VAL_N = 64
FLOP_PER_LR_PX = 2 * 9 * (3 * CH + 2 * BLOCKS * CH * CH + CH * CH + CH * 3 * S * S)
# one training iteration: forward + data-grad (no input grad for the head) + weight-grad
TRAIN_FLOP = BATCH * PATCH * PATCH * (3 * FLOP_PER_LR_PX - 2 * 9 * 3 * CH)
# config 2 (BASELINE.json): 540p -> 1080p x2, 8 x 32, batch of 30 frames
C2_S, C2_B, C2_C, C2_H, C2_W = 2, 8, 32, 540, 960
C2_FLOP_PER_LR_PX = 2 * 9 * (3 * C2_C + 2 * C2_B * C2_C * C2_C + C2_C * C2_C + C2_C * 3 * C2_S * C2_S)
METRIC = "4K SR frames/s (720p->2160p x3, 8x48) with online training at the paper's cadence"


def workload_config(frames, iters, world):
    """The `config` object of the JSON line -- identical in both arms (the driver compares them)."""
    return {
        "workload": f"cfg3+cfg4: {frames}x 720p->4K x3 frames + {ARRIVALS_PER_STEP} patch arrivals + {iters} train "
                    f"iters (64x 48->144) + publish + Algorithm-1 evaluation at each epoch end (every 50 "
                    f"iterations) per rank",
        "net": f"x{S}, {BLOCKS} blocks x {CH} ch", "frames_per_rank": frames, "train_iters_per_step": iters,
        "batch": BATCH, "patch_lr": PATCH, "pool_lr_entry": POOL_LR,
        "parallelism": f"frames sharded x{world}, DP training (NCCL allreduce in libsr)" if world > 1 else "1 GPU",
        "l2": "working set > L2 (one 720p activation tensor at 48 ch = 88 MB; 30 frames per step)",
    }


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


def _roofline(stats, cls, peak, peak_kind, traffic=None):
    v = stats[cls]
    achieved = v["flops"] / (v["ms"] * 1e-3) / 1e12
    return {"bound": "tensor", "kernel": cls, "achieved": round(achieved, 1), "peak": round(peak, 1), "unit": "TFLOP/s",
            "frac": round(achieved / peak, 4), "peak_kind": peak_kind, "traffic": traffic,
            "traffic_unit": "bytes per launch (ncu dram read+write)",
            "algorithmic_bytes": round(v["bytes"] / v["launches"]), "launches": v["launches"],
            "avg_ms": round(v["ms"] / v["launches"], 4)}


def run_ours(args):
    import numpy as np
    import torch
    import torch.distributed as dist
    from paper_conf_sigcomm_kimjyyh20_b200 import Controller, SRContext
    from paper_conf_sigcomm_kimjyyh20_b200.parallel import max_over_ranks, nccl_id_broadcast
    from synth import synth_frames, synth_patch_pool

    world, rank, local = dist_env()
    if args.gpus and world != args.gpus:
        raise SystemExit(f"bench: --gpus {args.gpus} but WORLD_SIZE={world}")
    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    dev = torch.device("cuda", local)
    frames = args.frames
    # the DP group's NCCL communicator lives in the library (sr_options.nccl_id): rank 0 draws the id
    nccl_id = nccl_id_broadcast() if world > 1 else None
    ctx = SRContext(S, BLOCKS, CH, seed=0, world=world, rank=rank, nccl_id=nccl_id)
    stream = torch.cuda.Stream(device=dev)  # whole-GPU stream (setup, cfg4, cfg2)
    # The step's inference and training run concurrently on disjoint SM partitions (sr_sm_partition, green contexts:
    # the paper's server runs inference and online training side by side, §7): inference on `s_inf`,
    # patch arrivals + training + publish + Algorithm 1 on `s_tr`; --partition 0 issues both on one stream instead.
    part = None
    if args.partition > 0:
        try:
            s_inf, s_tr, n_inf, n_tr = SRContext.sm_partition(args.partition)
            ctx.set_sm_split(n_tr)
            part = {"train_sms": n_tr, "infer_sms": n_inf}
        except Exception as exc:  # noqa: BLE001 -- e.g. a driver without green contexts
            print(f"[bench] SM partition unavailable ({exc}); sequential step", file=sys.stderr, flush=True)
            part = {"error": str(exc)}
    if part is None or "error" in part:
        s_inf = s_tr = stream
    # ---- synthetic inputs (seeded; per-rank frame shard; every rank holds the same pool and samples its chunk)
    lr_np = synth_frames(frames, LR_H, LR_W, seed=1003 + rank)
    lr = torch.from_numpy(lr_np).to(dev)
    hr = torch.empty((frames, S * LR_H, S * LR_W, 3), dtype=torch.uint8, device=dev)
    plr, phr, _ = synth_patch_pool(POOL_N, S, S * POOL_LR, seed=1004, frame_hw=(1080, 1800))
    n_arr = ARRIVALS_PER_STEP * (2 * args.warmup + 2 * args.steps + 4)
    alr, ahr, _ = synth_patch_pool(n_arr, S, S * POOL_LR, seed=1006, frame_hw=(1080, 1800))
    arr_lr, arr_hr = torch.from_numpy(alr).to(dev), torch.from_numpy(ahr).to(dev)
    val_lr = torch.from_numpy(plr[-VAL_N:]).to(dev)
    val_hr = torch.from_numpy(phr[-VAL_N:]).to(dev)
    loss = torch.zeros(1, dtype=torch.float32, device=dev)
    state = {"q": None, "iters": 0, "epochs": 0, "arr": 0, "events": []}
    with torch.cuda.stream(stream):
        ctx.pool_push(torch.from_numpy(plr).to(dev), torch.from_numpy(phr).to(dev))
    torch.cuda.synchronize()  # the pool is filled before the training stream samples it
    ctrl = Controller(thresh_sat=0.05, count_sat=2, thresh_online=0.5, count_online=2)

    def arrive():
        a = state["arr"] % (n_arr // ARRIVALS_PER_STEP)
        sl = slice(a * ARRIVALS_PER_STEP, (a + 1) * ARRIVALS_PER_STEP)
        ctx.pool_push(arr_lr[sl], arr_hr[sl], stream=s_tr)
        state["arr"] += 1

    def epoch_eval():
        r = ctx.controller_step(ctrl, val_lr, val_hr, stream=s_tr)
        if r["event"]:
            state["events"].append(r["event"])
        if ctrl.state != "training":  # constant-work mode (see the docstring): keep training every epoch
            ctrl.c.state, ctrl.c.patience = 0, 0
        state["q"] = r
        state["epochs"] += 1

    def train_iters():
        ctx.train_sampled(args.iters, BATCH, PATCH, loss, stream=s_tr)  # library-captured graph, replayed
        state["iters"] += args.iters
        if state["iters"] >= EPOCH_ITERS:  # epoch end (50 iterations, L1247-1250): publish + Algorithm 1
            state["iters"] = 0
            ctx.publish(stream=s_tr)  # waits for the inference in flight on s_inf (sr_publish)
            epoch_eval()

    def step():
        ctx.infer(lr, "serve", out=hr, stream=s_inf)
        arrive()
        train_iters()

    def barrier():
        if world > 1:
            dist.barrier()
        for s_ in (s_inf, s_tr):  # the partitions' streams (green contexts) explicitly
            s_.synchronize()
        torch.cuda.synchronize()

    def t_start():
        e = torch.cuda.Event(enable_timing=True)
        e.record(s_inf)
        s_tr.wait_event(e)
        return e

    def t_stop(e0):
        evs = []
        for s_ in (s_inf, s_tr, stream):
            ev = torch.cuda.Event(enable_timing=True)
            ev.record(s_)
            evs.append(ev)
        for ev in evs:
            ev.synchronize()
        torch.cuda.synchronize()
        return max(e0.elapsed_time(ev) for ev in evs)

    for _ in range(args.warmup):
        step()
    barrier()
    state["iters"], state["epochs"], state["events"] = 0, 0, []  # the timed region starts at an epoch boundary
    clk = ClockSampler(local)
    clk.start()
    l0 = ctx.launches
    ctx.kernel_timing(True)
    barrier()
    e0 = t_start()
    for _ in range(args.steps):
        step()
    ms = t_stop(e0)
    barrier()
    epochs_timed = state["epochs"]
    launches = ctx.launches - l0
    stats = ctx.kernel_stats()
    ctx.kernel_timing(False)
    clocks = clk.stop()
    ms = max_over_ranks(ms, device=dev)
    alg1 = {"mode": "constant-work: decisions are computed and reported but the bench keeps training",
            "epochs_timed": epochs_timed, "events_timed": list(state["events"]),
            "last": {k: (round(v, 4) if isinstance(v, float) else v) for k, v in state["q"].items()}
            if state["q"] else None}

    # ---- end-to-end: host (pinned) frames in, host frames out, through the C ABI (sr_infer_host_async)
    lr_host = torch.from_numpy(lr_np).pin_memory()
    hr_hosts = [torch.empty((frames, S * LR_H, S * LR_W, 3), dtype=torch.uint8).pin_memory() for _ in range(2)]
    hr_host = hr_hosts[0]
    loss_host = torch.zeros(1, dtype=torch.float32).pin_memory()
    nstep = [0]

    def step_e2e():
        # a serving loop: frames in and out through the host API (sr_infer_host_async: H2D / SR / D2H pipelined by
        # the library, two batches in flight into two host output buffers); patch arrivals and the training
        # iterations run beside it on the training stream and the step's loss is read back to the host
        ctx.infer_host_async(lr_host, hr_hosts[nstep[0] & 1], "serve", stream=s_inf)
        nstep[0] += 1
        arrive()
        train_iters()
        ev = torch.cuda.Event()
        ev.record(s_tr)
        stream.wait_event(ev)
        with torch.cuda.stream(stream):
            loss_host.copy_(loss, non_blocking=True)

    step_e2e()
    ctx.infer_host_wait()
    barrier()
    state["iters"] = 0
    e2 = t_start()
    for _ in range(args.steps):
        step_e2e()
    ctx.infer_host_wait()  # every step's HR frames are in host memory before the region closes
    ms_e2e = max_over_ranks(t_stop(e2), device=dev)
    barrier()
    if part is not None and "error" not in part:
        ctx.set_sm_split(0)  # the rest runs on the whole GPU

    # ---- config 4: training alone at the maximum rate (sampled iterations from the captured graph)
    n_tr = 100
    t0, t1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with torch.cuda.stream(stream):  # re-capture for the whole-GPU grids (and any workspace growth) before timing
        ctx.train_sampled(3, BATCH, PATCH, loss)
    barrier()
    with torch.cuda.stream(stream):
        t0.record()
        ctx.train_sampled(n_tr, BATCH, PATCH, loss)
        t1.record()
    barrier()
    tr_ms = max_over_ranks(t0.elapsed_time(t1), device=dev) / n_tr
    allreduce_us = None
    if world > 1:
        a0, a1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        with torch.cuda.stream(stream):
            for _ in range(5):
                ctx.train_allreduce()
            a0.record()
            for _ in range(50):
                ctx.train_allreduce()
            a1.record()
        barrier()
        allreduce_us = max_over_ranks(a0.elapsed_time(a1), device=dev) / 50 * 1e3
    # per-kernel shares of one training iteration: the same kernels launched eagerly with event timing
    ctx.kernel_timing(True)
    with torch.cuda.stream(stream):
        blr = torch.empty((BATCH, PATCH, PATCH, 3), dtype=torch.uint8, device=dev)
        bhr = torch.empty((BATCH, S * PATCH, S * PATCH, 3), dtype=torch.uint8, device=dev)
        for _ in range(10):
            ctx.sample_batch(-1, BATCH, PATCH, out=(blr, bhr, None))
            ctx.train_grad(blr, bhr, loss)
    tstats = ctx.kernel_stats()
    ctx.kernel_timing(False)
    barrier()

    # ---- config 2 (BASELINE.json): 540p -> 1080p x2, 8x32, batch of 30 frames, inference alone
    c2 = None
    if not args.no_cfg2:
        ctx2 = SRContext(C2_S, C2_B, C2_C, seed=0)
        lr2 = torch.from_numpy(synth_frames(frames, C2_H, C2_W, seed=1002 + rank)).to(dev)
        hr2 = torch.empty((frames, C2_S * C2_H, C2_S * C2_W, 3), dtype=torch.uint8, device=dev)
        with torch.cuda.stream(stream):
            for _ in range(3):
                ctx2.infer(lr2, "serve", out=hr2)
        barrier()
        ctx2.kernel_timing(True)
        c0, c1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        with torch.cuda.stream(stream):
            c0.record()
            for _ in range(args.steps):
                ctx2.infer(lr2, "serve", out=hr2)
            c1.record()
        barrier()
        c2_ms = max_over_ranks(c0.elapsed_time(c1), device=dev)
        c2_stats = ctx2.kernel_stats()
        c2 = {"c2_ms": c2_ms, "stats": c2_stats}
        ctx2.close()

    if rank == 0:
        pk = peaks()
        sustained = pk.get("bf16_tflops_sustained") or 1393.0
        pk_kind = "measured bf16_tflops_sustained (MEASURED_PEAKS.json)"
        dom = max(stats.items(), key=lambda kv: kv[1]["ms"])[0]
        # with the SM partition the inference kernels run on infer_sms of the SMs: their roofline peak is that share
        # of the measured whole-GPU peak
        inf_share, inf_note = 1.0, ""
        if part is not None and "error" not in part:
            nsm = torch.cuda.get_device_properties(dev).multi_processor_count
            inf_share = part["infer_sms"] / nsm
            inf_note = f" x {part['infer_sms']}/{nsm} SMs (the inference partition the kernel ran on)"
        ktot = sum(v["ms"] for v in stats.values())
        total_frames = frames * args.steps * world
        fps = total_frames / (ms * 1e-3)
        fps_e2e = total_frames / (ms_e2e * 1e-3)
        conv_flops = sum(v["flops"] for v in stats.values())
        tdom = max(tstats.items(), key=lambda kv: kv[1]["ms"])[0]
        tktot = sum(v["ms"] for v in tstats.values())
        line = {
            "metric": METRIC,
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
            "config": workload_config(frames, args.iters, world),
            "concurrency": ({"mode": "inference and training on disjoint SM partitions (green contexts)", **part}
                            if part is not None and "error" not in part else
                            {"mode": "sequential on one stream", **(part or {})}),
            "train_patches_per_s": round(BATCH * args.iters * args.steps * world / (ms * 1e-3), 1),
            "quality_gain_db": round(state["q"]["q_dnn"], 4) if state["q"] else None,
            "alg1": alg1,
            "tensor_tflops_all_convs": round(conv_flops / (ktot * 1e-3) / 1e12, 1),
            "kernel_share": {k: round(v["ms"] / ktot, 4) for k, v in sorted(stats.items(), key=lambda kv: -kv[1]["ms"])},
            "kernel_share_note": "CUDA-event time per kernel class of the eagerly launched kernels (inference, "
                                 "Algorithm-1 evaluation); the graph-replayed training kernels are in cfg4",
            "roofline": _roofline(stats, dom, sustained * inf_share, pk_kind + inf_note, traffic_of(dom, frames)),
            "e2e": {"value": round(fps_e2e, 3), "unit": "frames/s",
                    "h2d_bytes_per_step": int(lr_host.numel()),
                    "d2h_bytes_per_step": int(hr_host.numel() + loss_host.numel() * 4)},
            "gpu_launches": int(launches),
            "clocks": clocks,
            "cfg4_train": {
                "workload": "BASELINE config 4: sampled training iterations alone at the maximum rate, 64 x 48x48 LR "
                            "patches (x3, 8x48), Adam; DP over ranks with the NCCL allreduce inside the graph",
                "patches_per_s": round(BATCH * world / (tr_ms * 1e-3), 1), "ms_per_iter": round(tr_ms, 4),
                "tflops": round(TRAIN_FLOP / (tr_ms * 1e-3) / 1e12, 1),
                "frac_of_sustained": round(TRAIN_FLOP / (tr_ms * 1e-3) / 1e12 / sustained, 4),
                "allreduce_us": round(allreduce_us, 2) if allreduce_us is not None else None,
                "allreduce_bytes": ctx.num_params * 4,
                "roofline": _roofline(tstats, tdom, sustained, pk_kind, traffic_of(tdom, 1, PATCH, BATCH * (PATCH + 2))),
                "kernel_share": {k: round(v["ms"] / tktot, 4)
                                 for k, v in sorted(tstats.items(), key=lambda kv: -kv[1]["ms"])},
                "kernel_share_note": "eager event-timed launches of the same kernels (sample, forward, backward; "
                                     "per-class shares); ms_per_iter is the graph replay",
            },
        }
        if c2 is not None:
            cst = c2["stats"]
            cdom = max(cst.items(), key=lambda kv: kv[1]["ms"])[0]
            c2fps = frames * args.steps * world / (c2["c2_ms"] * 1e-3)
            line["cfg2"] = {
                "workload": f"BASELINE config 2: {frames} x 540p -> 1080p x2, 8 blocks x 32 ch, inference only",
                "frames_per_s": round(c2fps, 2), "ms_per_batch": round(c2["c2_ms"] / args.steps, 3),
                "tflops": round(c2fps * C2_H * C2_W * C2_FLOP_PER_LR_PX / 1e12, 1),
                "roofline": _roofline(cst, cdom, sustained, pk_kind, traffic_of(cdom, frames, C2_H, C2_W)),
                "kernel_share": {k: round(v["ms"] / sum(x["ms"] for x in cst.values()), 4)
                                 for k, v in sorted(cst.items(), key=lambda kv: -kv[1]["ms"])},
            }
        if not args.no_cpu_baseline:
            line["cpu_baseline"] = cpu_baseline()
        print(json.dumps(line), flush=True)
    # (the SM partitions stay until process exit: torch may still record events on their streams at teardown)
    if world > 1:
        dist.destroy_process_group()


def _cpu_model():
    try:
        for ln in open("/proc/cpuinfo"):
            if ln.startswith("model name"):
                return ln.split(":", 1)[1].strip()
    except OSError:
        pass
    return None


def cpu_baseline():
    """The fp64 numpy oracle, as it stands, on whole units of the workload (no extrapolation): ONE whole 720p frame
    through the x3 8x48 net (frames/s) and ONE whole 64-patch training step (forward + backward + Adam; patches/s),
    with BLAS threads = all host cores available to the process, then the training step again at one thread."""
    import numpy as np
    from threadpoolctl import threadpool_info, threadpool_limits

    import oracle as O
    from synth import init_params, synth_frames, synth_patch_pool
    cores = len(os.sched_getaffinity(0))
    p = init_params(S, BLOCKS, CH, seed=0)
    lr = synth_frames(1, LR_H, LR_W, seed=1003)
    plr, phr, _ = synth_patch_pool(BATCH, S, S * PATCH, seed=1004, frame_hw=(432, 576))

    def train_step():
        _, g = O.train_loss_and_grad(p, plr, phr, S, BLOCKS, CH)
        O.adam_step(p, np.zeros_like(g), np.zeros_like(g), g, 1)

    with threadpool_limits(limits=cores):
        blas = [d.get("num_threads") for d in threadpool_info() if d.get("user_api") == "blas"]
        t0 = time.perf_counter()
        O.infer_u8(p, lr, S, BLOCKS, CH)
        t_frame = time.perf_counter() - t0
        t0 = time.perf_counter()
        train_step()
        t_step = time.perf_counter() - t0
    with threadpool_limits(limits=1):
        t0 = time.perf_counter()
        train_step()
        t_step1 = time.perf_counter() - t0
    return {"value": round(1.0 / t_frame, 6), "unit": "frames/s", "cores": cores, "kind": "oracle",
            "sample": f"one whole 720x1280 LR frame -> 4K through the x3 8x48 net ({t_frame:.2f} s; frames/s = 1/t) "
                      f"and one whole training step on 64 48x48 patches, forward + backward + Adam ({t_step:.2f} s); "
                      f"BLAS threads {blas}; training step at 1 thread {t_step1:.2f} s",
            "train_patches_per_s": round(BATCH / t_step, 4), "blas_threads": blas[0] if blas else None,
            "one_thread": {"train_patches_per_s": round(BATCH / t_step1, 4), "blas_threads": 1},
            "cpu_model": _cpu_model()}


REF_BAND = 180  # rows of the 720p frame per reference-arm step (a quarter frame)


def run_reference(args):
    """The oracle (the paper has no code) on the box's host cores: each step super-resolves one
    quarter of a 720p frame (a 180-row band, zero padded at its edges like a frame) through the x3 8x48 net;
    value = 0.25 frame per step / the measured time.  Only rank 0 runs (N > 1: the others exit)."""
    world, rank, _ = dist_env()
    if rank != 0:
        return
    from threadpoolctl import threadpool_limits

    import oracle as O
    from synth import init_params, synth_frames
    cores = len(os.sched_getaffinity(0))
    p = init_params(S, BLOCKS, CH, seed=0)
    lr = synth_frames(1, LR_H, LR_W, seed=1003)
    band = args.ref_band
    bands = [lr[:, i * band:(i + 1) * band] for i in range(LR_H // band)]
    with threadpool_limits(limits=cores):
        for i in range(args.warmup):
            O.infer_u8(p, bands[i % len(bands)][:, :16], S, BLOCKS, CH)  # untimed warm-up on a sliver
        t = 0.0
        for i in range(args.steps):
            t0 = time.perf_counter()
            O.infer_u8(p, bands[i % len(bands)], S, BLOCKS, CH)
            t += time.perf_counter() - t0
    frac = band / LR_H
    v = frac * args.steps / t
    print(json.dumps({
        "impl": "reference", "metric": METRIC, "value": round(v, 6), "unit": "frames/s", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(t / args.steps * 1e3, 3),
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": workload_config(args.frames, args.iters, world),
        "cpu_baseline": {"value": round(v, 6), "unit": "frames/s", "cores": cores, "kind": "oracle",
                         "sample": f"per step one {band}x{LR_W} band ({band}/{LR_H} frame) of a 720p frame through "
                                   f"the x3 8x48 net; inference only (the oracle's training is reported by cpu_baseline of "
                                   f"the product arm)"},
        "e2e": {"value": round(v, 6), "unit": "frames/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }), flush=True)


def traffic_of(kernel_class, frames, h=None, w=None):
    """DRAM bytes per launch of a dominant kernel from the committed ncu captures (profiles/r01_traffic.json: the
    headline's inference kernels; profiles/r02_traffic.json: the cfg4 / cfg2 side lines), when taken on the same
    launch shape; else None."""
    h = LR_H if h is None else h
    w = LR_W if w is None else w
    for name in ("r02_traffic.json", "r01_traffic.json"):
        try:
            with open(os.path.join(ROOT, "profiles", name)) as f:
                t = json.load(f).get(kernel_class)
        except (OSError, ValueError):
            continue
        if t and t.get("frames") == frames and (t.get("h"), t.get("w")) == (h, w):
            return int(t["dram_read"] + t["dram_write"])
    return None


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def relaunch(n):
    """`--gpus N` outside torchrun: run this script under torch.distributed.run with N ranks (127.0.0.1
    rendezvous); NCCL_DEBUG=INFO so the communicator's rank lines are in the log."""
    env = dict(os.environ)
    env.setdefault("NCCL_DEBUG", "INFO")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={n}",
           "--master-addr", "127.0.0.1", "--master-port", str(_free_port()), os.path.abspath(__file__)] + sys.argv[1:]
    return subprocess.call(cmd, env=env)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--frames", type=int, default=FRAMES)
    ap.add_argument("--iters", type=int, default=ITERS)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-cfg2", action="store_true")
    ap.add_argument("--workload", choices=["cfg3", "live"], default="cfg3")
    ap.add_argument("--partition", type=int, default=40,
                    help="SMs of the training partition (green contexts); 0 = inference and training sequential")
    ap.add_argument("--ref-band", type=int, default=REF_BAND, help=argparse.SUPPRESS)
    args, extra = ap.parse_known_args()
    if extra and args.workload != "live":  # the live harness takes its own options (--streams, --seconds, --i420, ...)
        ap.error(f"unrecognized arguments: {' '.join(extra)}")
    if args.warmup < 3:
        raise SystemExit("bench: --warmup must be >= 3")
    if "WORLD_SIZE" not in os.environ and args.gpus > 1:
        raise SystemExit(relaunch(args.gpus))
    if dist_env()[0] > 1:
        os.environ.setdefault("NCCL_DEBUG", "INFO")
    if args.workload == "live":
        from scripts.live_ingest import main as live_main
        raise SystemExit(live_main(sys.argv[1:]))
    if args.impl == "reference":
        run_reference(args)
    else:
        run_ours(args)


if __name__ == "__main__":
    main()

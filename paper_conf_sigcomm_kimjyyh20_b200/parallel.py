"""Host-side multi-GPU plumbing of the hot path (one process per GPU, torch.distributed over NCCL/NVLink).

Only sharding arithmetic and the gradient exchange live here; every FLOP runs in libsr.so.

* Inference shards naturally (§6.2):
    - throughput mode: frames round-robin / contiguous per rank, no collective (`frame_shard`);
    - latency mode: one frame split into equal horizontal pieces, one per GPU (`strip_rows`, 720p -> 3 x 240
      rows, L1192-1194); the library adds an exact halo (reading R12) so stitching is bit-exact.
* Training is data-parallel over patches (L1210-1220): the pool is partitioned by arrival sequence
  (`pool_view`, mirrored in sr_sample_batch), each rank computes w_r * g_r, one sum-allreduce of the flat
  fp32 gradient (NCCL; gloo on CPU for tests), then Adam with g = sum_r w_r g_r / sum_r w_r (`dp_allreduce_grad`).
"""
from __future__ import annotations


def frame_shard(n_frames: int, world: int, rank: int) -> range:
    """Contiguous frame range of `rank` (weak scaling: every rank gets n_frames // world (+1))."""
    lo = n_frames * rank // world
    hi = n_frames * (rank + 1) // world
    return range(lo, hi)


def strip_rows(h: int, world: int, rank: int) -> tuple[int, int]:
    """Equal horizontal pieces of an LR frame (the paper's intra-frame split): rows [r0, r1)."""
    return h * rank // world, h * (rank + 1) // world


def pool_view(n_avail: int, world: int, rank: int) -> tuple[int, int]:
    """Arrival-order chunk [lo, hi) of the n_avail pooled patches that rank samples from (oldest first)."""
    return n_avail * rank // world, n_avail * (rank + 1) // world


def dp_allreduce_grad(grad, weight: float = 1.0, group=None) -> float:
    """In-place sum-allreduce of `grad` (already scaled by this rank's weight w_r inside sr_train_grad) and of
    the weights; returns the Adam grad_scale = 1 / sum_r w_r, so the update uses sum_r w_r g_r / sum_r w_r."""
    import torch
    import torch.distributed as dist
    if not dist.is_initialized() or dist.get_world_size(group) == 1:
        return 1.0 / weight
    dist.all_reduce(grad, op=dist.ReduceOp.SUM, group=group)
    w = torch.tensor([float(weight)], dtype=torch.float64, device=grad.device)
    dist.all_reduce(w, op=dist.ReduceOp.SUM, group=group)
    return 1.0 / float(w.item())


def dp_allreduce_grad_dev(grad, weight_dev, group=None):
    """Graph-capturable variant: sum-allreduce `grad` and the 1-element weight tensor `weight_dev` on the device and
    return a device tensor holding 1 / sum_r w_r (feed it to SRContext.train_apply_dev)."""
    import torch.distributed as dist
    w = weight_dev.clone()
    if dist.is_initialized() and dist.get_world_size(group) > 1:
        dist.all_reduce(grad, op=dist.ReduceOp.SUM, group=group)
        dist.all_reduce(w, op=dist.ReduceOp.SUM, group=group)
    return w.reciprocal()


def max_over_ranks(value: float, device=None, group=None) -> float:
    """Max of a scalar over ranks (timings are reported as the slowest rank)."""
    import torch
    import torch.distributed as dist
    if not dist.is_initialized() or dist.get_world_size(group) == 1:
        return value
    t = torch.tensor([float(value)], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX, group=group)
    return float(t.item())

"""Host-side multi-GPU plumbing of the hot path (one process per GPU, torch.distributed for rendezvous and timing).

No arithmetic of the method lives here: sharding index ranges, the NCCL id hand-out and a max-over-ranks of a
timing.  Every FLOP, including the data-parallel gradient exchange, runs in libsr.so.

* Inference shards naturally (§6.2):
    - throughput mode: frames round-robin / contiguous per rank, no collective (`frame_shard`);
    - latency mode: one frame split into equal horizontal pieces, one per GPU (`strip_rows`, 720p -> 3 x 240
      rows, L1192-1194); the library adds an exact halo (reading R12) so stitching is bit-exact.
* Training is data-parallel over patches (L1210-1220): the pool is partitioned by arrival sequence (`pool_view`,
  mirrored on the device by sr_sample_batch), each rank computes w_r * g_r, and the ctx's own NCCL communicator sums
  them (sr_train_step / sr_train_sampled / sr_train_allreduce); Adam applies 1 / sum_r w_r.  The communicator is
  created inside sr_create from an ncclUniqueId that rank 0 draws and `nccl_id_broadcast` hands to every rank.
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


def nccl_id_broadcast(group=None) -> bytes:
    """The 128-byte ncclUniqueId of the DP group: drawn by rank 0 through the library (sr_nccl_unique_id) and
    broadcast over the process group (gloo or NCCL), so every rank passes the same bytes to SRContext(nccl_id=...)."""
    import ctypes as C

    import torch
    import torch.distributed as dist

    from ._lib import SRError, load
    backend = dist.get_backend(group)
    dev = torch.device("cuda", torch.cuda.current_device()) if backend == "nccl" else torch.device("cpu")
    buf = torch.zeros(128, dtype=torch.uint8)
    if dist.get_rank(group) == 0:
        raw = C.create_string_buffer(128)
        st = load().sr_nccl_unique_id(raw, 128)
        if st != 0:
            raise SRError(f"sr_nccl_unique_id failed with status {st}")
        buf = torch.frombuffer(bytearray(raw.raw), dtype=torch.uint8).clone()
    t = buf.to(dev)
    dist.broadcast(t, src=0, group=group)
    return bytes(t.cpu().numpy().tobytes())


def max_over_ranks(value: float, device=None, group=None) -> float:
    """Max of a scalar over ranks (timings are reported as the slowest rank)."""
    import torch
    import torch.distributed as dist
    if not dist.is_initialized() or dist.get_world_size(group) == 1:
        return value
    t = torch.tensor([float(value)], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX, group=group)
    return float(t.item())

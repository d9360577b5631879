"""Multi-rank host logic on CPU (gloo, world size 2): sharding arithmetic, the NCCL id hand-out, max-over-ranks
timing, and the DP exchange protocol the library runs (sum-allreduce of w_r g_r, then Adam with 1 / sum_r w_r)."""
import os
import socket
import tempfile

import numpy as np
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle as O
from paper_conf_sigcomm_kimjyyh20_b200.parallel import (frame_shard, max_over_ranks, nccl_id_broadcast, pool_view,
                                                         strip_rows)
from synth import init_params


def test_sharding_arithmetic():
    for n, g in ((30, 1), (30, 4), (7, 8), (240, 3)):
        got = [list(frame_shard(n, g, r)) for r in range(g)]
        assert sum(got, []) == list(range(n))
        assert max(map(len, got)) - min(map(len, got)) <= 1
    # the paper's pieces: 720p -> 3 x 240 rows, 1080p -> 3 x 360 rows
    assert [strip_rows(720, 3, r) for r in range(3)] == [(0, 240), (240, 480), (480, 720)]
    assert [strip_rows(1080, 3, r)[1] - strip_rows(1080, 3, r)[0] for r in range(3)] == [360] * 3
    views = [pool_view(1001, 4, r) for r in range(4)]
    assert views[0][0] == 0 and views[-1][1] == 1001
    assert all(views[i][1] == views[i + 1][0] for i in range(3))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, out_dir, weights):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    s, B, C = 2, 1, 4
    p = init_params(s, B, C, seed=4).astype(np.float64)
    r = np.random.default_rng(100 + rank)  # each rank: its own arrival chunk of patches
    lr = r.integers(0, 256, size=(2, 6, 6, 3)).astype(np.uint8)
    hr = r.integers(0, 256, size=(2, 12, 12, 3)).astype(np.uint8)
    _, g = O.train_loss_and_grad(p, lr, hr, s, B, C)
    w = weights[rank]
    # the protocol libsr runs on the device (sr_train_grad pre-scales by w_r; sr_create allreduces the weights once;
    # sr_train_allreduce sums the gradients; k_adam applies 1 / sum_r w_r), here over gloo on the oracle's gradients
    gt = torch.from_numpy(g * w)
    dist.all_reduce(gt, op=dist.ReduceOp.SUM)
    wt = torch.tensor([w], dtype=torch.float64)
    dist.all_reduce(wt, op=dist.ReduceOp.SUM)
    agg = gt.numpy() / float(wt.item())
    t = max_over_ranks(float(rank + 1))
    nid = nccl_id_broadcast()
    np.save(os.path.join(out_dir, f"id{rank}.npy"), np.frombuffer(nid, np.uint8))
    np.save(os.path.join(out_dir, f"agg{rank}.npy"), agg)
    np.save(os.path.join(out_dir, f"g{rank}.npy"), g)
    np.save(os.path.join(out_dir, f"max{rank}.npy"), np.array([t]))
    dist.destroy_process_group()


def _run(weights):
    with tempfile.TemporaryDirectory() as d:
        mp.spawn(_worker, args=(2, _free_port(), d, weights), nprocs=2, join=True)
        aggs = [np.load(os.path.join(d, f"agg{r}.npy")) for r in range(2)]
        gs = [np.load(os.path.join(d, f"g{r}.npy")) for r in range(2)]
        mx = [float(np.load(os.path.join(d, f"max{r}.npy"))[0]) for r in range(2)]
        ids = [np.load(os.path.join(d, f"id{r}.npy")) for r in range(2)]
    return aggs, gs, mx, ids


def test_dp_allreduce_gloo_uniform_equals_union_batch():
    aggs, gs, mx, ids = _run([1.0, 1.0])
    np.testing.assert_array_equal(aggs[0], aggs[1])          # every rank applies identical bits
    np.testing.assert_allclose(aggs[0], O.dp_aggregate(gs), rtol=1e-12)
    assert mx == [2.0, 2.0]
    # rank 0's ncclUniqueId (drawn by libsr's sr_nccl_unique_id) reaches every rank byte for byte
    assert ids[0].size == 128 and ids[0].any()
    np.testing.assert_array_equal(ids[0], ids[1])


def test_dp_allreduce_gloo_recency_weights():
    """Larger weight for the rank holding the newer patches (reading R11)."""
    aggs, gs, _, _ = _run([1.0, 4.0])
    np.testing.assert_allclose(aggs[1], O.dp_aggregate(gs, [1.0, 4.0]), rtol=1e-12)

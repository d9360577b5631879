"""Intra-frame pieces across processes (§6.2): each process super-resolves its
strip of one frame with sr_infer_rows and writes its HR rows straight into a frame buffer owned by another process
(CUDA IPC: the same mapping a peer GPU's buffer gets over NVLink), and the stitched frame is bit-identical to
whole-frame inference (reading R12: exact halo).  One GPU here, so both processes share it."""
import os

import pytest
import torch
import torch.multiprocessing as mp

pytestmark = pytest.mark.gpu

S, B, C = 3, 2, 16
H, W = 96, 272


def _piece(rank, world, q_in, q_out):
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import torch as T
    from paper_conf_sigcomm_kimjyyh20_b200 import SRContext
    from paper_conf_sigcomm_kimjyyh20_b200.parallel import strip_rows
    T.cuda.set_device(0)
    lr, hr = q_in.get()             # CUDA tensors shared by the owner process (IPC handles)
    ctx = SRContext(S, B, C, seed=7)
    r0, r1 = strip_rows(H, world, rank)
    ctx.infer_rows(lr, r0, r1, hr, "serve")
    T.cuda.synchronize()
    q_out.put(rank)
    q_in.get()                      # keep the mapping alive until the owner has read the frame


def test_strip_pieces_written_across_processes_bitexact():
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    from paper_conf_sigcomm_kimjyyh20_b200 import SRContext
    from synth import synth_frames
    ctx = mp.get_context("spawn")
    world = 3  # the paper's three pieces (L1192-1194)
    lr = torch.from_numpy(synth_frames(1, H, W, seed=8)[0]).cuda()
    hr = torch.full((S * H, S * W, 3), 9, dtype=torch.uint8, device="cuda")
    qs_in = [ctx.Queue() for _ in range(world)]
    q_out = ctx.Queue()
    procs = [ctx.Process(target=_piece, args=(r, world, qs_in[r], q_out)) for r in range(world)]
    for p in procs:
        p.start()
    for q in qs_in:
        q.put((lr, hr))
    done = sorted(q_out.get(timeout=300) for _ in range(world))
    assert done == list(range(world))
    torch.cuda.synchronize()
    ref = SRContext(S, B, C, seed=7).infer(lr[None].contiguous(), "serve")[0]
    torch.cuda.synchronize()
    stitched = hr.clone()
    for q in qs_in:
        q.put(None)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    assert torch.equal(stitched, ref)

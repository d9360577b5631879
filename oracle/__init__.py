"""fp64 CPU ORACLE for the LiveNAS SR hot path — TEST INFRASTRUCTURE, NOT PRODUCT CODE.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / `--impl reference` leg may import
this package.  It shares no code with paper_conf_sigcomm_kimjyyh20_b200/ (the CUDA path) and imports
nothing from it.  Every function cites the PAPER.md passage it follows (PAPER.md = the extracted text
of Kim et al., "Neural-Enhanced Live Streaming", SIGCOMM '20) or the DESIGN.md reading it takes where
the paper is silent.

Parity pins (tests/test_oracle_pins.py, `-m "not gpu"`): brute-force 7-loop conv, identity/delta
kernels, pixel shuffle as a permutation, zero-weight net == bilinear skip (bit-exact u8, checked
against torch.nn.functional.interpolate), finite-difference gradients of the whole net, PSNR closed
form, Adam step-1 closed form (and torch.optim.Adam), sampler statistics, paper arithmetic facts,
Algorithm 1 (oracle/controller.py) against traces worked out by hand from App. A (tests/golden/alg1_traces.json),
the I420 conversion (oracle/color.py) against the real-valued BT.601 matrices, and the client's patch selection
(oracle/patch_select.py) against frames whose degraded cells are known by construction.
"parity unpinned": none of the functions below; the learning-direction check (loss falls) is a
sanity check only.
"""
from .srnet import (  # noqa: F401
    conv3x3, conv3x3_bruteforce, conv3x3_dgrad, conv3x3_wgrad, pixel_shuffle, pixel_unshuffle,
    bilinear_up, bicubic_up, unpack_params, pack_params, forward, infer_u8, train_loss_and_grad, adam_step,
    dp_aggregate, sample_indices, gather_patches, psnr_u8, psnr_gain, conv_shapes_oracle,
)
from .controller import Algorithm1, epoch_report  # noqa: F401
from .patch_select import select_patches  # noqa: F401

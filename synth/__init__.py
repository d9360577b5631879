"""Seeded synthetic inputs shared by the oracle tests, the GPU parity tests and bench.py.

This package holds NO arithmetic of the method (no conv, no pixel shuffle, no bilinear skip, no loss,
no Adam, no sampler, no PSNR). It only draws inputs: frames, patches, and the random-init weights the
method starts from (the paper starts from a DIV2K/NTIRE-trained DNN, PAPER.md:L1142-1146 / L1670-1671,
which does not exist here, so weights are a seeded draw passed in as an input).
"""
from .gen import (  # noqa: F401
    GAMMA, mix64, splitmix64_stream, init_params, conv_shapes, num_params,
    synth_frames, synth_patch_pool, area_downsample,
)

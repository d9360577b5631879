"""Client-side patch selection (§5.2), oracle pins: frames whose degraded cells are known by
construction, the strict comparison, the 1080p grid, and the permutation."""
import numpy as np

from oracle.patch_select import cell_sse, permutation, select_patches


def _frame(h, w, seed):
    return np.random.default_rng(seed).integers(0, 256, (h, w, 3)).astype(np.uint8)


def test_exactly_the_degraded_cells_are_selected():
    raw = _frame(240, 360, 0)            # 2 x 3 cells of 120
    dec = raw.copy()
    dec[0:120, 120:240] ^= 7             # cells (x=120, y=0) and (x=0, y=120) get errors, the rest are perfect
    dec[120:240, 0:120] ^= 3
    sel = select_patches(raw, dec, cell=120, max_sel=10, seed=5)
    assert sorted(sel) == [(0, 120), (120, 0)]


def test_max_sel_caps_and_order_follows_the_permutation():
    raw = _frame(360, 480, 1)            # 3 x 4 = 12 cells
    dec = raw.copy()
    bad = [(0, 0), (1, 2), (2, 3), (0, 3), (2, 1)]
    for cy, cx in bad:
        dec[cy * 120:(cy + 1) * 120, cx * 120:(cx + 1) * 120] ^= 1
    sel = select_patches(raw, dec, cell=120, max_sel=3, seed=9, step=2)
    assert len(sel) == 3
    perm = permutation(12, 9, 2)
    expect = [(c % 4 * 120, c // 4 * 120) for c in perm if (c // 4, c % 4) in bad][:3]
    assert sel == expect


def test_uniform_error_selects_nothing_strict_comparison():
    raw = _frame(240, 240, 2)
    dec = raw ^ 1                        # every sample off by exactly 1 -> every cell's PSNR equals the frame's
    assert select_patches(raw, dec, cell=120) == []


def test_1080p_grid_is_16x9_cells_of_120():
    raw = np.zeros((1080, 1920, 3), np.uint8)
    sse, cnt = cell_sse(raw, raw, 120)
    assert sse.shape == (9, 16) and np.all(cnt == 120 * 120 * 3)


def test_partial_cells_count_for_the_frame_but_are_never_candidates():
    raw = _frame(130, 250, 3)            # whole cells: 1 x 2; partial border row/column
    dec = raw.copy()
    dec[120:, :] ^= 255                  # only the partial row is bad -> raises the frame error, selects nothing
    assert select_patches(raw, dec, cell=120) == []
    sse, cnt = cell_sse(raw, dec, 120)
    assert sse.shape == (2, 3) and cnt.sum() == 130 * 250 * 3


def test_permutation_is_a_permutation():
    for n in (1, 2, 7, 144):
        p = permutation(n, 123, 4)
        assert sorted(p) == list(range(n))
    assert permutation(144, 1, 0) != permutation(144, 1, 1)

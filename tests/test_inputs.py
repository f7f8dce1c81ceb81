"""Seeded input generators (inputs.py): the block-defined matrices of config 5 give the
same columns whatever slab is drawn (SURVEY 8(e) "Inputs"), so a rank's slab at any
world size is a slice of the one global matrix."""
import numpy as np

from paper_conf_ipps_00020c20_b200 import inputs
from paper_conf_ipps_00020c20_b200.sharded import slab_bounds


def test_blocked_slabs_are_slices_of_the_global_matrix():
    rows, cols = 96, 10000
    full = inputs.uniform_f16_blocked(rows, cols, 7, block=1024)
    assert full.shape == (rows, cols) and full.flags["F_CONTIGUOUS"]
    assert -1.0 <= float(full.min()) and float(full.max()) <= 1.0
    for world in (1, 2, 3, 8):
        for r in range(world):
            n0, n1 = slab_bounds(cols, world, r)
            sl = inputs.uniform_f16_blocked(rows, cols, 7, block=1024, col0=n0, ncols=n1 - n0)
            assert np.array_equal(sl.view(np.uint16), full[:, n0:n1].view(np.uint16))


def test_blocked_integer_range_and_slices():
    full = inputs.integer_f16_blocked(64, 5000, 3, -1, 1, block=512)
    assert set(np.unique(full).tolist()) == {-1.0, 0.0, 1.0}
    sl = inputs.integer_f16_blocked(64, 5000, 3, -1, 1, block=512, col0=1500, ncols=2000)
    assert np.array_equal(sl, full[:, 1500:3500])


def test_blocked_seeds_differ_per_block():
    x = inputs.uniform_f16_blocked(128, 2048, 1, block=1024)
    assert not np.array_equal(x[:, :1024], x[:, 1024:])

"""The seeded input generator: C, numpy and pure-Python
implementations agree bit for bit, and the value ranges are as stated."""
import numpy as np
import pytest

import nugen


@pytest.mark.parametrize("kind", ["uniform", "int", "eye", "ones", "rank1", "zeros", "temp", "power"])
def test_three_implementations_agree(kind):
    rows, cols, ncols, i0, j0 = 13, 37, 101, 5, 17
    c = nugen.fill(rows, cols, seed=3, mat=1, kind=kind, i0=i0, j0=j0, ncols=ncols)
    n = nugen.fill_numpy(rows, cols, seed=3, mat=1, kind=kind, i0=i0, j0=j0, ncols=ncols)
    assert np.array_equal(c.view(np.uint32), n.view(np.uint32))
    for (r, k) in [(0, 0), (3, 7), (12, 36)]:
        assert c[r, k] == nugen.entry_py(3, 1, kind, ncols, i0 + r, j0 + k)
        assert c[r, k] == nugen.entry(3, 1, kind, ncols, i0 + r, j0 + k)


def test_uniform_range_and_granularity():
    x = nugen.fill(256, 512, seed=1, mat=1).astype(np.float64)
    assert x.min() >= -1.0 and x.max() < 1.0
    q = x * 2.0 ** 23
    assert np.array_equal(q, np.round(q))          # 2^-23 granularity, exact fp32
    assert abs(x.mean()) < 0.01 and abs(x.var() - 1 / 3) < 0.01


def test_int_range():
    x = nugen.fill(64, 64, seed=2, mat=2, kind="int")
    assert x.min() >= -8 and x.max() <= 8 and set(np.unique(x)) <= set(range(-8, 9))


def test_block_regeneration_matches_full_matrix():
    full = nugen.fill(40, 50, seed=5, mat=2)
    blk = nugen.fill(7, 9, seed=5, mat=2, i0=11, j0=23, ncols=50)
    assert np.array_equal(full[11:18, 23:32], blk)


def test_a_and_b_differ_and_seeds_differ():
    a = nugen.fill(16, 16, seed=1, mat=nugen.MAT_A)
    b = nugen.fill(16, 16, seed=1, mat=nugen.MAT_B)
    a2 = nugen.fill(16, 16, seed=2, mat=nugen.MAT_A)
    assert not np.array_equal(a, b) and not np.array_equal(a, a2)


def test_hotspot_grid_ranges():
    t = nugen.fill(128, 256, seed=6, mat=nugen.MAT_T, kind="temp").astype(np.float64)
    p = nugen.fill(128, 256, seed=6, mat=nugen.MAT_P, kind="power").astype(np.float64)
    assert t.min() >= 320.0 and t.max() < 340.0 and abs(t.mean() - 330.0) < 0.2
    assert p.min() >= 0.0 and p.max() < 0.5
    q = p * 2.0 ** 25
    assert np.array_equal(q, np.round(q))           # exact fp32, 2^-25 granularity

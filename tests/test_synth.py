"""The shared seeded input recipes (synth/): determinism and structure."""
import numpy as np

import synth


def test_locations_deterministic_and_in_unit_square():
    x1, y1 = synth.locations(1600, seed=0)
    x2, y2 = synth.locations(1600, seed=0)
    assert np.array_equal(x1, x2) and np.array_equal(y1, y2)
    assert x1.min() > 0 and x1.max() < 1 and y1.min() > 0 and y1.max() < 1


def test_morton_order_is_a_permutation_of_the_grid():
    xg, yg = synth.jittered_grid(400, seed=3)
    xs, ys = synth.morton_sort(xg, yg)
    a = np.sort(xg * 7 + yg)
    b = np.sort(xs * 7 + ys)
    assert np.array_equal(a, b)
    k = synth.morton_keys(xs, ys)
    assert np.all(np.diff(k.astype(np.int64)) >= 0)


def test_jitter_stays_in_cell():
    side = 20
    x, y = synth.jittered_grid(side * side, seed=1)
    i = np.repeat(np.arange(side), side)
    assert np.all(np.abs(x * side - (i + 0.5)) <= 0.4 + 1e-12)


def test_normal_vector_seeded():
    assert np.array_equal(synth.normal_vector(10, 1), synth.normal_vector(10, 1))

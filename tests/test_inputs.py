"""The seeded R-MAT generator: exact n, m, simple graph,
sorted rows, and independence from the thread count."""
import numpy as np

import inputs


def test_rmat_shape_and_hygiene():
    off, nbr = inputs.rmat(3000, 40000, seed=2)
    assert off.size == 3001 and nbr.size == 40000 and off[-1] == 40000
    assert np.all(np.diff(off.astype(np.int64)) >= 0)
    assert nbr.max() < 3000
    for v in range(3000):
        row = nbr[off[v]:off[v + 1]]
        assert np.all(np.diff(row.astype(np.int64)) > 0)   # ascending, no duplicates
        assert v not in row                                 # no self loops


def test_rmat_thread_count_independent_and_seeded():
    a = inputs.rmat(5000, 60000, seed=7, nthreads=1)
    b = inputs.rmat(5000, 60000, seed=7, nthreads=5)
    c = inputs.rmat(5000, 60000, seed=8, nthreads=5)
    assert np.array_equal(a[0], b[0]) and np.array_equal(a[1], b[1])
    assert not np.array_equal(a[1], c[1])


def test_rmat_is_skewed():
    off, nbr = inputs.config_graph("C1")
    d = np.diff(off.astype(np.int64))
    assert d.max() > 20 * d.mean()


def test_small_graph_helpers():
    off, nbr = inputs.from_edges(4, [(0, 1), (2, 1), (1, 3)])
    assert off.tolist() == [0, 0, 2, 2, 3] and nbr.tolist() == [0, 2, 1]

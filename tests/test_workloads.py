"""The config-5 generator in C (workloads/banded_markov.c) emits exactly the
arrays of the numpy definition workloads.banded_markov."""
import numpy as np
import pytest

import workloads as W


@pytest.mark.parametrize("n,mu,width,irr,seed", [
    (2, 3, 2, False, 1), (33, 6, 8, True, 3), (777, 5, 2, False, 3), (1000, 10, 64, True, 3),
    (5000, 15, 5000, True, 3), (20000, 10, 1024, False, 1), (20000, 7, 32768, True, 2), (4096, 10, 3, True, 9)])
def test_c_generator_matches_numpy(n, mu, width, irr, seed):
    a = W.banded_markov(n, mu, width, irr, seed)
    b = W.banded_markov_fast(n, mu, width, irr, seed)
    for x, y in zip(a, b):
        assert x.dtype == y.dtype and np.array_equal(x, y)


def test_c_generator_structure():
    r, c, v = W.banded_markov_fast(100000, 10, 1024, False, 1)
    assert np.all(np.diff(c) >= 0) and np.all(r != c)
    assert np.all((v >= 1.0) & (v < 2.0))
    assert np.all(np.abs(r.astype(np.int64) - c) <= 1024)
    assert len(r) == 100000 * 9 - 2     # mu-1 off-diagonals per column, minus the two edge backbones

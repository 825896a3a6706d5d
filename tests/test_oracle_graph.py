"""Pins of the oracle's graph construction (reading Q14) and hub selection (reading Q7)."""
import numpy as np
import pytest

import gen
import oracle
from helpers import np_canonical, random_multigraph


@pytest.mark.parametrize("seed", range(10))
def test_canonical_csr_matches_numpy(seed):
    rng = np.random.default_rng(seed)
    n = int(rng.integers(1, 300))
    m = int(rng.integers(0, 3000))
    src, dst, w = random_multigraph(rng, n, m, wset=tuple(range(1, 9)))
    g = oracle.canonical_csr(n, src, dst, w)
    ptr, col, wt = np_canonical(n, src, dst, w)
    assert np.array_equal(g.ptr, ptr)
    assert np.array_equal(g.col, col)
    assert np.array_equal(g.wt, wt)


def test_canonical_rmat():
    n = 1 << 12
    src, dst, w = gen.rmat(n, 16 * n, seed=11)
    g = oracle.canonical_csr(n, src, dst, w)
    ptr, col, wt = np_canonical(n, src, dst, w)
    assert np.array_equal(g.ptr, ptr) and np.array_equal(g.col, col) and np.array_equal(g.wt, wt)
    assert g.m < src.size  # R-MAT produces duplicates and self-loops


@pytest.mark.parametrize("seed", range(5))
def test_transpose_matches_numpy(seed):
    rng = np.random.default_rng(100 + seed)
    n = int(rng.integers(1, 200))
    src, dst, w = random_multigraph(rng, n, int(rng.integers(0, 2000)))
    g = oracle.canonical_csr(n, src, dst, w)
    gr = oracle.transpose(g)
    u = np.repeat(np.arange(n), np.diff(g.ptr))
    # reverse edges (v -> u, w) canonical order = sorted by (v, u)
    ptr, col, wt = np_canonical(n, g.col, u.astype(np.uint32), g.wt)
    assert np.array_equal(gr.ptr, ptr) and np.array_equal(gr.col, col) and np.array_equal(gr.wt, wt)


def test_hubs_topdeg():
    n = 1 << 11
    src, dst, w = gen.rmat(n, 8 * n, seed=12)
    g = oracle.canonical_csr(n, src, dst, w)
    gr = oracle.transpose(g)
    deg = np.diff(g.ptr) + np.diff(gr.ptr)
    order = np.lexsort((np.arange(n), -deg))     # degree desc, id asc
    for K in (1, 5, 20):
        assert np.array_equal(oracle.hubs_topdeg(g, gr, K), order[:K].astype(np.uint32))
    # ties: all-equal degrees pick ids 0..K-1
    ring = np.arange(10, dtype=np.uint32)
    g2 = oracle.canonical_csr(10, ring, (ring + 1) % 10, np.ones(10, np.uint32))
    assert list(oracle.hubs_topdeg(g2, oracle.transpose(g2), 3)) == [0, 1, 2]

"""Input generator properties (gen/): determinism, chunking, ranges, permutation, skew."""
import numpy as np

import gen


def test_deterministic_and_chunkable():
    n = 1000
    a = gen.rmat(n, 5000, seed=3)
    b = gen.rmat(n, 5000, seed=3)
    for x, y in zip(a, b):
        assert np.array_equal(x, y)
    c1 = gen.rmat(n, 2000, seed=3)
    c2 = gen.rmat(n, 3000, seed=3, e0=2000)
    for x, y, z in zip(a, c1, c2):
        assert np.array_equal(x, np.concatenate([y, z]))
    d = gen.rmat(n, 5000, seed=4)
    assert not np.array_equal(a[0], d[0])


def test_ranges():
    for n in (1, 2, 3, 1000, 1 << 12):
        s, d, w = gen.rmat(n, 4000, w_max=23, seed=7)
        assert s.max() < n and d.max() < n
        assert w.min() >= 1 and w.max() <= 23
    s, d, w = gen.rmat(1 << 10, 100000, w_max=64, seed=1)
    assert set(np.unique(w)) == set(range(1, 65))


def test_permutation_is_bijection():
    lib = gen._load()
    for n in (2, 5, 1000, 4097):
        img = np.array([lib.gen_permute(x, n, 9) for x in range(n)])
        assert np.array_equal(np.sort(img), np.arange(n))


def test_rmat_skew_and_thresholds():
    tA, tAB, tABC = gen.thresholds(*gen.RMAT1[:3])
    assert tA == int(0.57 * 2 ** 32) and tABC == int(0.95 * 2 ** 32)
    n = 1 << 14
    s, d, w = gen.rmat(n, 16 * n, seed=1, permute=False)
    deg = np.bincount(s, minlength=n)
    assert deg.max() > 50 * deg.mean()          # power-law hubs
    # without permutation vertex 0 (all-'a' quadrant path) is the largest hub
    assert deg.argmax() == 0


def test_sample_sources():
    n = 1000
    s, d, w = gen.rmat(n, 3000, seed=5)
    src = gen.sample_sources(n, s, d, 10, seed=42)
    assert src.size == 10 and np.all(np.isin(src, s[s != d]))
    assert np.array_equal(src, gen.sample_sources(n, s, d, 10, seed=42))


def test_generator_vertex_zero_is_the_top_hub():
    """Reading N10: configs[0]'s "vertex 0" is the R-MAT generator's vertex 0, which the Feistel
    permutation moves; it is the highest-degree vertex of the C1 graph, while id 0 is isolated."""
    c = gen.CONFIGS["c1"]
    s, d, _ = c.edges()
    v0 = gen.generator_vertex(c, 0)
    keep = s != d
    deg = np.bincount(s[keep], minlength=c.n) + np.bincount(d[keep], minlength=c.n)
    assert deg.argmax() == v0 and deg[0] == 0
    u, v, _ = gen.rmat(c.n, 1000, c.abcd, c.w_max, c.seed, permute=False)
    up, vp, _ = gen.rmat(c.n, 1000, c.abcd, c.w_max, c.seed, permute=True)
    assert all(gen.generator_vertex(c, int(a)) == int(b) for a, b in zip(u[:50], up[:50]))

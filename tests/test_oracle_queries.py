"""Pins of the oracle's query definition (Table 6).

Each check compares oracle.query / oracle.bellman_ford with something fixed
independently of the oracle's C code:
  * brute-force enumeration of all simple paths (n <= 8),
  * scipy.sparse.csgraph shortest paths (SSSP, BFS),
  * threshold reachability (SSWP = max t reachable over edges w >= t; SSNP = min t over w <= t),
  * Viterbi with power-of-two weights = 2^-(SSSP over log2 w) exactly,
  * REACH = (BFS < inf); Viterbi with all weights 1 = REACH.
"""
import numpy as np
import pytest
import scipy.sparse as sp
from scipy.sparse.csgraph import breadth_first_order, dijkstra

import gen
import oracle
from helpers import INF32, KINDS, brute_force, np_canonical, random_multigraph, rmat_small


def _csr(n, src, dst, w):
    g = oracle.canonical_csr(n, src, dst, w)
    return g


@pytest.mark.parametrize("seed", range(40))
def test_query_equals_brute_force(seed):
    rng = np.random.default_rng(seed)
    n = int(rng.integers(1, 9))
    m = int(rng.integers(0, 3 * n + 1))
    src, dst, w = random_multigraph(rng, n, m)
    g = _csr(n, src, dst, w)
    for kind in KINDS:
        for s in range(n):
            bf = brute_force(kind, n, g.ptr, g.col, g.wt, s)
            q = oracle.query(kind, g, s)
            assert np.array_equal(q, bf), (kind, s)
            b = oracle.bellman_ford(kind, g, s)
            assert np.array_equal(b, bf), (kind, s)


def test_kind_operators_table6():
    """(+) and the selection of Table 6 on scalar cases fixed by arithmetic."""
    assert oracle._load().or_extend(0, 5, 7) == 12          # SSSP: Val(u)+w
    assert oracle._load().or_extend(1, 5, 7) == 5           # SSWP: min(Val(u), w)
    assert oracle._load().or_extend(2, 5, 7) == 7           # SSNP: max(Val(u), w)
    v = np.array([oracle._load().or_extend(3, int(np.float32(1.0).view(np.uint32)), 3)],
                 dtype=np.uint32).view(np.float32)[0]
    assert v == np.float32(1.0) / np.float32(3.0)           # Viterbi: Val(u)/w in binary32
    assert oracle._load().or_extend(4, 5, 99) == 6          # BFS: +1 regardless of w
    assert oracle._load().or_extend(5, 1, 99) == 1          # REACH: Val(u)
    # selection: MIN for SSSP/SSNP/BFS, MAX for SSWP/Viterbi/REACH
    assert oracle._load().or_better(0, 3, 4) and not oracle._load().or_better(0, 4, 3)
    assert oracle._load().or_better(1, 4, 3) and oracle._load().or_better(5, 1, 0)


def _scipy_graph(g, weights):
    return sp.csr_matrix((weights.astype(np.float64), g.col.astype(np.int64), g.ptr), shape=(g.n, g.n))


@pytest.mark.parametrize("scale,seed", [(8, 1), (10, 2), (12, 3)])
def test_sssp_and_bfs_match_scipy(scale, seed):
    n, src, dst, w = rmat_small(scale, 8, seed)
    g = _csr(n, src, dst, w)
    A = _scipy_graph(g, g.wt)
    U = _scipy_graph(g, np.ones(g.m))
    rng = np.random.default_rng(seed)
    for s in rng.integers(0, n, size=6):
        d = dijkstra(A, indices=int(s))
        q = oracle.query("sssp", g, int(s))
        exp = np.where(np.isinf(d), INF32, d).astype(np.uint64)
        assert np.array_equal(q.astype(np.uint64), exp)
        h = dijkstra(U, indices=int(s), unweighted=True)
        qb = oracle.query("bfs", g, int(s))
        assert np.array_equal(qb.astype(np.uint64), np.where(np.isinf(h), INF32, h).astype(np.uint64))
        reach = oracle.query("reach", g, int(s))
        assert np.array_equal(reach, (~np.isinf(h)).astype(np.uint32))


def _reach_mask(g, s, keep):
    """Vertices reachable from s using only edges with keep[i] (scipy BFS)."""
    A = sp.csr_matrix((np.ones(int(keep.sum())), g.col[keep].astype(np.int64),
                       np.concatenate([[0], np.cumsum([keep[g.ptr[u]:g.ptr[u + 1]].sum()
                                                       for u in range(g.n)])]).astype(np.int64)),
                      shape=(g.n, g.n))
    order = breadth_first_order(A, s, directed=True, return_predecessors=False)
    mask = np.zeros(g.n, dtype=bool)
    mask[order] = True
    return mask


@pytest.mark.parametrize("scale,seed", [(7, 4), (9, 5)])
def test_sswp_ssnp_threshold_reachability(scale, seed):
    """SSWP(s,v) = max t: v reachable over edges w >= t; SSNP(s,v) = min t over edges w <= t."""
    n, src, dst, w = rmat_small(scale, 8, seed, w_max=16)
    g = _csr(n, src, dst, w)
    rng = np.random.default_rng(seed)
    ts = np.unique(g.wt)
    for s in rng.integers(0, n, size=3):
        s = int(s)
        wide = np.zeros(n, dtype=np.int64)
        narrow = np.full(n, INF32, dtype=np.int64)
        for t in ts:                       # increasing t
            wide[_reach_mask(g, s, g.wt >= t)] = t
        for t in ts[::-1]:                 # decreasing t
            narrow[_reach_mask(g, s, g.wt <= t)] = t
        wide[s] = INF32
        narrow[s] = 0
        assert np.array_equal(oracle.query("sswp", g, s).astype(np.int64), wide)
        assert np.array_equal(oracle.query("ssnp", g, s).astype(np.int64), narrow)


@pytest.mark.parametrize("scale,seed", [(8, 6), (10, 7)])
def test_viterbi_powers_of_two_exact(scale, seed):
    """Division by 2^k is exact in binary32, so Viterbi = ldexp(1, -SSSP(log2 w)) exactly
    while the exponent stays above the subnormal floor (2^-149)."""
    n, src, dst, _ = rmat_small(scale, 8, seed)
    rng = np.random.default_rng(seed)
    k = rng.integers(1, 7, size=src.size)            # w in {2,4,...,64}
    g = _csr(n, src, dst, (1 << k).astype(np.uint32))
    L = _scipy_graph(g, np.log2(g.wt).astype(np.float64))
    for s in rng.integers(0, n, size=5):
        d = dijkstra(L, indices=int(s))
        q = oracle.as_float(oracle.query("viterbi", g, int(s)))
        exp = np.where(np.isinf(d) | (d > 149), 0.0, np.ldexp(1.0, -np.where(np.isinf(d), 0, d).astype(np.int64)))
        assert np.array_equal(q, exp.astype(np.float32))


def test_viterbi_unit_weights_is_reach():
    n, src, dst, _ = rmat_small(9, 8, 8)
    g = _csr(n, src, dst, np.ones(src.size, dtype=np.uint32))
    for s in (0, 3, 17):
        v = oracle.as_float(oracle.query("viterbi", g, s))
        r = oracle.query("reach", g, s)
        assert np.array_equal(v, r.astype(np.float32))


def test_viterbi_close_to_f64_definition():
    """Binary32 chained division stays within path_len * 2^-24 relative of the exact product
    (north_star's 1e-6 relative bound for diameter-scale paths)."""
    rng = np.random.default_rng(9)
    n = 7
    for _ in range(20):
        src, dst, w = random_multigraph(rng, n, 18, wset=(1, 2, 3, 5, 7, 11, 13, 23))
        g = _csr(n, src, dst, w)
        for s in range(n):
            q = oracle.as_float(oracle.query("viterbi", g, s)).astype(np.float64)
            # exact f64 max-product by brute force over simple paths
            best = np.zeros(n)
            best[s] = 1.0

            def visit(u, on, p):
                for i in range(int(g.ptr[u]), int(g.ptr[u + 1])):
                    v = int(g.col[i])
                    if v in on:
                        continue
                    pv = p / float(g.wt[i])
                    best[v] = max(best[v], pv)
                    on.add(v)
                    visit(v, on, pv)
                    on.discard(v)
            visit(s, {s}, 1.0)
            assert np.allclose(q, best, rtol=1e-6, atol=0)


def test_empty_and_isolated():
    g = _csr(1, np.zeros(0, np.uint32), np.zeros(0, np.uint32), np.zeros(0, np.uint32))
    for kind in KINDS:
        q = oracle.query(kind, g, 0)
        assert q[0] == oracle.source_val(kind)
    g = _csr(4, np.array([1, 2], np.uint32), np.array([2, 3], np.uint32), np.array([5, 6], np.uint32))
    q = oracle.query("sssp", g, 0)
    assert list(q) == [0, INF32, INF32, INF32]
    q = oracle.query("sssp", g, 1)
    assert list(q) == [INF32, 0, 5, 11]


def test_init_values_reading_q1():
    f = lambda x: int(np.array([x], dtype=np.float32).view(np.uint32)[0])
    assert [oracle.init_val(k) for k in KINDS] == [INF32, 0, INF32, f(0.0), INF32, 0]
    assert [oracle.source_val(k) for k in KINDS] == [0, INF32, 0, f(1.0), 0, 1]


@pytest.mark.parametrize("seed", range(4))
def test_wcc_oracle_pins(seed):
    """NEXT-3 WCC (Table 6 WCC row): the label fixpoint is the minimum vertex id of
    the weak component.  Pinned against scipy's weak connected components (an independent
    algorithm) plus the invariants label(v) <= v, label(label(v)) == label(v), and equal labels
    at both ends of every edge."""
    import scipy.sparse as sp
    import scipy.sparse.csgraph as csg
    rng = np.random.default_rng(seed)
    n = int(rng.integers(1, 3000))
    src, dst, w = gen.rmat(max(n, 2), int(rng.integers(0, 3 * n + 1)), seed=seed + 11) if n > 1 else (
        np.zeros(0, np.uint32), np.zeros(0, np.uint32), np.zeros(0, np.uint32))
    n = max(n, 2)
    g = oracle.canonical_csr(n, src, dst, w)
    lab = oracle.wcc(g)
    a = sp.csr_matrix((np.ones(g.m), g.col, g.ptr), shape=(n, n))
    nc, comp = csg.connected_components(a, directed=True, connection="weak")
    mins = np.full(nc, n)
    np.minimum.at(mins, comp, np.arange(n))
    assert np.array_equal(lab, mins[comp].astype(np.uint32))
    assert np.all(lab <= np.arange(n)) and np.array_equal(lab[lab], lab)
    rows = np.repeat(np.arange(n), np.diff(g.ptr))
    assert np.array_equal(lab[rows], lab[g.col])
    assert np.array_equal(oracle.query("wcc", g, 0), lab)


@pytest.mark.parametrize("kind", KINDS)
def test_query_batch_equals_single_queries(kind):
    """or_query_batch (the OpenMP driver the full-size parity tests and the CPU baseline use)
    returns, row by row, exactly or_query of each source — any thread count, repeated and
    out-of-order sources included; or_query itself is pinned above (brute force, scipy,
    threshold reachability, closed forms)."""
    n, src, dst, w = rmat_small(10, 8, 91)
    g = oracle.canonical_csr(n, src, dst, w)
    rng = np.random.default_rng(5)
    sources = np.concatenate([rng.integers(0, n, 13), [7, 7, 0, n - 1]]).astype(np.uint32)
    for threads in (1, 3, 8):
        out = oracle.query_batch(kind, g, sources, nthreads=threads)
        assert out.shape == (sources.size, n)
        for i, s in enumerate(sources):
            assert np.array_equal(out[i], oracle.query(kind, g, int(s))), (kind, threads, i)
    assert oracle.query_batch(kind, g, np.zeros(0, np.uint32)).shape == (0, n)

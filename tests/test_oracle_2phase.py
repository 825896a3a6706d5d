"""Pins of the oracle's Algorithm 3 (2Phase) and FULL-mode evaluation.

Invariants fixed by the paper and the mathematics:
  * 2Phase result == definition (oracle.query) on 100% of vertices,
    with the real CG AND with arbitrary sub-graph proxies (random edge subsets, empty, G itself);
  * phase-1 values are never better than final ones (sub-graph monotonicity);
  * the Complete Core Graph (all non-zero-centrality edges) makes phase 1 exact;
  * every vertex reached from s pushes its full G out-list in phase 2 (FirstPhase2Visit).
"""
import numpy as np
import pytest

import oracle
from helpers import KINDS, random_multigraph, rmat_small


def _worse_or_equal(kind, a, b):
    """a is not better than b under the kind's selection."""
    if kind in ("sssp", "ssnp", "bfs"):
        return np.all(a >= b)
    if kind == "viterbi":
        return np.all(oracle.as_float(a) <= oracle.as_float(b))
    return np.all(a <= b)


@pytest.mark.parametrize("kind", KINDS)
@pytest.mark.parametrize("seed", [1, 2, 3])
def test_2phase_equals_definition_real_cg(kind, seed):
    n, src, dst, w = rmat_small(10, 8, seed, w_max=11)
    g = oracle.canonical_csr(n, src, dst, w)
    gr = oracle.transpose(g)
    hubs = oracle.hubs_topdeg(g, gr, 8)
    cg = oracle.subgraph(g, oracle.cg_for_kind(kind, g, gr, hubs))
    rng = np.random.default_rng(seed)
    for s in rng.integers(0, n, size=8):
        s = int(s)
        ref = oracle.query(kind, g, s)
        val, p1, st = oracle.two_phase(kind, g, cg, s)
        assert np.array_equal(val, ref)
        assert _worse_or_equal(kind, p1, val)
        assert st["unvisited_p2"] == 0
        assert val[s] == oracle.source_val(kind)
        full, fst = oracle.full_bsp(kind, g, s)
        assert np.array_equal(full, ref)
        assert st["reached"] == fst["reached"]


@pytest.mark.parametrize("seed", range(12))
def test_2phase_any_proxy(seed):
    rng = np.random.default_rng(seed)
    n = int(rng.integers(1, 30))
    src, dst, w = random_multigraph(rng, n, int(rng.integers(0, 5 * n)))
    g = oracle.canonical_csr(n, src, dst, w)
    for frac in (0.0, 0.1, 0.5, 1.0):
        flags = (rng.random(g.m) < frac).astype(np.uint8)
        proxy = oracle.subgraph(g, flags)
        for kind in KINDS:
            for s in range(n):
                val, p1, st = oracle.two_phase(kind, g, proxy, s)
                assert np.array_equal(val, oracle.query(kind, g, s)), (kind, s, frac)
                assert _worse_or_equal(kind, p1, val)
                if frac == 1.0:
                    assert np.array_equal(p1, val)       # proxy == G: phase 1 is exact


@pytest.mark.parametrize("kind", KINDS)
def test_complete_core_graph_is_exact(kind):
    """cCG = all edges tight for some source (non-zero centrality): phase 1 exact."""
    rng = np.random.default_rng(5)
    n = 24
    src, dst, w = random_multigraph(rng, n, 80, wset=(1, 2, 3, 4, 5, 6))
    g = oracle.canonical_csr(n, src, dst, w)
    u_of = np.repeat(np.arange(n), np.diff(g.ptr))
    ccg = np.zeros(g.m, dtype=np.uint8)
    for s in range(n):
        val = oracle.query(kind, g, s)
        for i in range(g.m):
            u, v = int(u_of[i]), int(g.col[i])
            if val[u] != oracle.init_val(kind):
                cand = oracle._load().or_extend(oracle.KINDS[kind], int(val[u]),
                                                1 if kind == "bfs" else int(g.wt[i]))
                if cand == val[v]:
                    ccg[i] = 1
    cg = oracle.subgraph(g, ccg)
    for s in range(n):
        val, p1, st = oracle.two_phase(kind, g, cg, s)
        assert np.array_equal(p1, val)
        assert st["precise_p1"] == st["reached"]


def test_2phase_precision_sanity_rmat():
    """Loose distributional sanity (parity UNPINNED): CG % and p1 precision."""
    n, src, dst, w = rmat_small(12, 16, 1, w_max=13)
    g = oracle.canonical_csr(n, src, dst, w)
    gr = oracle.transpose(g)
    hubs = oracle.hubs_topdeg(g, gr, 20)
    flags = oracle.cg_alg1("sssp", g, gr, hubs)
    frac = flags.sum() / g.m
    assert 0.02 < frac < 0.40
    cg = oracle.subgraph(g, flags)
    _, _, st = oracle.two_phase("sssp", g, cg, int(hubs[0]))
    assert st["precise_p1"] >= 0.8 * st["reached"]
    full, fst = oracle.full_bsp("sssp", g, int(hubs[0]))
    assert st["edges_p1"] + st["edges_p2"] < fst["edges_p2"]

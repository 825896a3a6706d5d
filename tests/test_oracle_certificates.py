"""Pins of oracle O7: the precision certificates of the Reduced(E)
optimization — Theorem 1 for SSSP / BFS, its bottleneck analogs for SSWP / SSNP,
REACH's lattice top.  A certificate claims a phase-1 value is already final, so:

* P5 itself: every certified vertex is precise (p1(v) == the query's final value), on every
  vertex of random multigraphs and small RMAT graphs, all sources;
* closed forms: a hub reached in phase 1 is certified through Theorem 1 (a) with v = h (the
  Algorithm 1 CG holds the backward shortest-path tree of h, so p1(h) is exact and the bound
  d(s,h) - d(h,h) = d(s,h) meets it); on a weighted path whose last vertex is the hub, every
  vertex after the source is certified;
* coverage: the bottleneck certificates cover most reached vertices of RMAT graphs (SURVEY
  appendix: 67-70 %), Theorem 1 only a few — a checker that certified nothing would fail here.
"""
import numpy as np
import pytest

import oracle
from helpers import random_multigraph, rmat_small

CERT_KINDS = ("sssp", "bfs", "sswp", "ssnp", "reach")


def _setup(n, src, dst, w, kind, K):
    g = oracle.canonical_csr(n, src, dst, w)
    gr = oracle.transpose(g)
    hubs = oracle.hubs_topdeg(g, gr, min(K, n))
    cg = oracle.subgraph(g, oracle.cg_for_kind(kind, g, gr, hubs))
    hf, hb = oracle.hub_values(kind, g, gr, hubs)
    return g, gr, hubs, cg, hf, hb


@pytest.mark.parametrize("kind", CERT_KINDS)
@pytest.mark.parametrize("seed", range(5))
def test_certified_implies_precise(kind, seed):
    rng = np.random.default_rng(500 + seed)
    if seed < 3:
        n = int(rng.integers(2, 60))
        src, dst, w = random_multigraph(rng, n, 5 * n)
    else:
        n, src, dst, w = rmat_small(9, 8, 40 + seed, w_max=23)
    g, gr, hubs, cg, hf, hb = _setup(n, src, dst, w, kind, 6)
    for s in range(n):
        final = oracle.query(kind, g, s)
        _, p1, _ = oracle.two_phase(kind, g, cg, s)
        cert = oracle.certified(kind, s, p1, hf, hb).astype(bool)
        bad = np.nonzero(cert & (p1 != final))[0]
        assert bad.size == 0, f"{kind} s={s}: certified but imprecise at {bad[:5]}"
        assert not (cert & (p1 == oracle.init_val(kind))).any()  # only reached vertices


@pytest.mark.parametrize("kind", ("sssp", "sswp", "ssnp"))
def test_hubs_reached_in_phase1_are_certified(kind):
    n, src, dst, w = rmat_small(10, 8, 77, w_max=23)
    g, gr, hubs, cg, hf, hb = _setup(n, src, dst, w, kind, 8)
    checked = 0
    for s in np.random.default_rng(1).choice(n, 40, replace=False):
        s = int(s)
        final = oracle.query(kind, g, s)
        _, p1, _ = oracle.two_phase(kind, g, cg, s)
        cert = oracle.certified(kind, s, p1, hf, hb)
        for h in hubs:
            h = int(h)
            if h != s and final[h] != oracle.init_val(kind):
                assert p1[h] == final[h] and cert[h] == 1, (kind, s, h)
                checked += 1
    assert checked > 20


def test_path_to_hub_is_fully_certified():
    n = 10
    src = np.arange(n - 1, dtype=np.uint32)
    w = np.array([3, 1, 4, 1, 5, 9, 2, 6, 5], np.uint32)
    g = oracle.canonical_csr(n, src, src + 1, w)
    gr = oracle.transpose(g)
    hubs = np.array([n - 1], np.uint32)  # the path's end
    for kind in ("sssp", "bfs"):
        cg = oracle.subgraph(g, oracle.cg_alg1(kind, g, gr, hubs))
        hf, hb = oracle.hub_values(kind, g, gr, hubs)
        for s in range(n - 1):
            _, p1, _ = oracle.two_phase(kind, g, cg, s)
            cert = oracle.certified(kind, s, p1, hf, hb)
            assert cert[s:].all() and not cert[:s].any(), (kind, s)
            if kind == "sssp":
                assert list(p1[s:]) == list(np.concatenate([[0], np.cumsum(w[s:])]))


def test_coverage_bottleneck_vs_theorem1():
    n, src, dst, w = rmat_small(11, 8, 78, w_max=23)
    cover = {}
    for kind in ("sssp", "sswp", "ssnp", "reach"):
        g, gr, hubs, cg, hf, hb = _setup(n, src, dst, w, kind, 20)
        tot = c = 0
        for s in np.random.default_rng(2).choice(np.nonzero(np.diff(g.ptr))[0], 10, replace=False):
            _, p1, _ = oracle.two_phase(kind, g, cg, int(s))
            reached = p1 != oracle.init_val(kind)
            reached[int(s)] = False
            cert = oracle.certified(kind, int(s), p1, hf, hb).astype(bool)
            tot += int(reached.sum())
            c += int((cert & reached).sum())
        cover[kind] = c / max(tot, 1)
    assert cover["reach"] == 1.0
    assert cover["sswp"] > 0.4 and cover["ssnp"] > 0.4, cover
    assert 0.0 < cover["sssp"] < cover["sswp"], cover

"""Pins of the oracle's Core Graph builders.

Algorithm 1: the worked example of Table 2 / Figure 4 (P:848-984,
tests/golden/table2_fig4.txt) — the CG edge set, both all-pairs tables, the
Fig 4 row/column, the connectivity edge and its effect — plus the property
that Alg 1's forward (backward) tight edges preserve Q(h) on G (on G^R).

Algorithm 2: a hand-worked trace (tests/golden/alg2_worked.txt),
reachability preservation for the first hub, and an independent
level-synchronous formulation (the one the GPU emulates: winner of each newly
labeled vertex = minimum (FIFO rank of parent, edge position)).
"""
from collections import deque

import numpy as np
import pytest

import oracle
from conftest import read_golden
from helpers import INF32, random_multigraph, rmat_small


def _table2():
    gd = read_golden("table2_fig4.txt")
    e = np.array([[int(r[0]) - 1, int(r[1]) - 1, int(r[2])] for r in gd["edges"]], dtype=np.uint32)
    g = oracle.canonical_csr(9, e[:, 0], e[:, 1], e[:, 2])
    return gd, g


def _mat(rows):
    return np.array([[INF32 if x == "inf" else int(x) for x in r] for r in rows], dtype=np.uint64)


def _edge_set(g, flags):
    u = np.repeat(np.arange(g.n), np.diff(g.ptr))
    return {(int(u[i]), int(g.col[i])) for i in np.nonzero(flags)[0]}


def _apsp(g):
    return np.stack([oracle.query("sssp", g, s) for s in range(g.n)]).astype(np.uint64)


def test_table2_g_apsp():
    gd, g = _table2()
    assert g.m == 17                       # "G with 17 Edges" (Table 2 caption)
    assert np.array_equal(_apsp(g), _mat(gd["apsp_g"]))


def test_fig4_row_and_column():
    gd, g = _table2()
    assert np.array_equal(oracle.query("sssp", g, 6).astype(np.uint64), _mat(gd["fig4b"])[0])
    gr = oracle.transpose(g)               # SSSP(* -> 7) = SSSP(7) on G^R
    assert np.array_equal(oracle.query("sssp", gr, 6).astype(np.uint64), _mat(gd["fig4c"])[0])


def test_table2_alg1_core_graph():
    gd, g = _table2()
    gr = oracle.transpose(g)
    hubs = np.array([int(gd["hubs"][0][0]) - 1], dtype=np.uint32)
    flags = oracle.cg_alg1("sssp", g, gr, hubs, connectivity=False)
    expect = {(int(a) - 1, int(b) - 1) for a, b in gd["cg"]}
    assert _edge_set(g, flags) == expect and len(expect) == 8
    cg = oracle.subgraph(g, flags)
    assert np.array_equal(_apsp(cg), _mat(gd["apsp_cg"]))        # Table 2 bottom
    # connectivity step (Alg 1 l.8-12): 6 -> 4 (lowest weight out-edge of 6)
    flags_c = oracle.cg_alg1("sssp", g, gr, hubs, connectivity=True)
    added = _edge_set(g, flags_c) - expect
    assert added == {(int(a) - 1, int(b) - 1) for a, b in gd["connectivity"]}
    cgc = oracle.subgraph(g, flags_c)
    assert np.array_equal(oracle.query("sssp", cgc, 5).astype(np.uint64), _mat(gd["sssp6_cg_conn"])[0])
    # 2Phase on the CG reproduces G exactly for every source
    for s in range(9):
        val, p1, st = oracle.two_phase("sssp", g, cgc, s)
        assert np.array_equal(val, oracle.query("sssp", g, s))


@pytest.mark.parametrize("kind", ["sssp", "sswp", "ssnp", "viterbi"])
@pytest.mark.parametrize("seed", [1, 2])
def test_alg1_preserves_hub_queries(kind, seed):
    """Forward tight edges keep Q(h) exact on the CG; backward ones keep Q(h) on CG^R exact."""
    n, src, dst, w = rmat_small(10, 8, seed, w_max=11)
    g = oracle.canonical_csr(n, src, dst, w)
    gr = oracle.transpose(g)
    hubs = oracle.hubs_topdeg(g, gr, 5)
    cg = oracle.subgraph(g, oracle.cg_alg1(kind, g, gr, hubs, connectivity=True))
    cgr = oracle.transpose(cg)
    for h in hubs:
        assert np.array_equal(oracle.query(kind, cg, int(h)), oracle.query(kind, g, int(h)))
        assert np.array_equal(oracle.query(kind, cgr, int(h)), oracle.query(kind, gr, int(h)))
    # CG is a sub-graph of G on all vertices; every outdeg>0 vertex keeps an out-edge
    assert cg.m <= g.m
    od = np.diff(g.ptr)
    assert np.all(np.diff(cg.ptr)[od > 0] > 0)


def test_alg1_connectivity_choice():
    # vertex 0 has three out-edges and is on no solution path of hub 4 (separate component)
    src = np.array([0, 0, 0, 4], np.uint32)
    dst = np.array([1, 2, 3, 5], np.uint32)
    w = np.array([5, 2, 9, 1], np.uint32)
    g = oracle.canonical_csr(6, src, dst, w)
    gr = oracle.transpose(g)
    hubs = np.array([4], np.uint32)
    for kind, exp in (("sssp", (0, 2)), ("ssnp", (0, 2)), ("viterbi", (0, 2)), ("sswp", (0, 3))):
        es = _edge_set(g, oracle.cg_alg1(kind, g, gr, hubs, connectivity=True))
        assert exp in es, kind
        assert sum(1 for e in es if e[0] == 0) == 1


def test_alg2_worked_example():
    gd = read_golden("alg2_worked.txt")
    n = int(gd["n"][0][0])
    e = np.array([[int(a), int(b)] for a, b in gd["edges"]], dtype=np.uint32)
    g = oracle.canonical_csr(n, e[:, 0], e[:, 1], np.ones(len(e), np.uint32))
    gr = oracle.transpose(g)
    hubs = np.array([int(x) for x in gd["hubs"][0]], dtype=np.uint32)
    flags = oracle.cg_alg2(g, gr, hubs)
    assert list(flags) == [int(x) for x in gd["flags"][0]]


def _alg2_levelsync(g, gr, hubs, per_direction=False):
    """Independent formulation of Alg 2: level-synchronous traversal where each newly
    labeled vertex's discovering edge is the one with minimum (rank of parent in FIFO
    order, position in the parent's adjacency), and the next level is ordered by that key.
    per_direction: one label array for the forward traversals and one for the backward ones
    (reading Q9')."""
    n = g.n
    qids = {False: np.zeros(n, dtype=np.int64)}
    qids[True] = np.zeros(n, dtype=np.int64) if per_direction else qids[False]
    flags = np.zeros(g.m, dtype=np.uint8)

    def g_edge(u, v):  # position of G edge u->v
        lo, hi = int(g.ptr[u]), int(g.ptr[u + 1])
        i = lo + int(np.searchsorted(g.col[lo:hi], v))
        assert i < hi and g.col[i] == v
        return i

    for k, h in enumerate(hubs):
        lab = k + 1
        for graph, rev in ((g, False), (gr, True)):
            qid = qids[rev]
            level = [int(h)]
            while level:
                win = {}
                for r, u in enumerate(level):
                    for j, i in enumerate(range(int(graph.ptr[u]), int(graph.ptr[u + 1]))):
                        v = int(graph.col[i])
                        if qid[v] == lab:
                            continue
                        if qid[v] == 0:
                            key = (r, j)
                            if v not in win or key < win[v][0]:
                                win[v] = (key, u)
                        else:
                            flags[g_edge(v, u) if rev else g_edge(u, v)] = 1
                nxt = sorted(win.items(), key=lambda kv: kv[1][0])
                for v, (_, u) in nxt:
                    qid[v] = lab
                    flags[g_edge(v, u) if rev else g_edge(u, v)] = 1
                level = [v for v, _ in nxt]
    return flags


@pytest.mark.parametrize("seed", range(6))
def test_alg2_equals_levelsync_formulation(seed):
    rng = np.random.default_rng(seed)
    if seed < 3:
        n = int(rng.integers(2, 40))
        src, dst, w = random_multigraph(rng, n, 4 * n)
    else:
        n, src, dst, w = rmat_small(9, 6, seed)
    g = oracle.canonical_csr(n, src, dst, w)
    gr = oracle.transpose(g)
    hubs = oracle.hubs_topdeg(g, gr, min(5, n))
    assert np.array_equal(oracle.cg_alg2(g, gr, hubs), _alg2_levelsync(g, gr, hubs))
    # the per-direction variant (reading Q9', the default general CG of BFS / REACH / WCC)
    assert np.array_equal(oracle.cg_alg2(g, gr, hubs, per_direction=True),
                          _alg2_levelsync(g, gr, hubs, per_direction=True))


@pytest.mark.parametrize("seed", range(4))
def test_alg2_per_direction_is_union_of_directions(seed):
    """With one Qid per direction, the forward traversals never see the backward labels and vice
    versa, so the CG is the union of Alg 2 run forward-only on G and forward-only on G^R (its
    edges reversed back into G, Alg 2 l.9): a mistake such as the backward traversal reusing
    the forward labels, or not reversing its edges, breaks this identity."""
    if seed < 2:
        rng = np.random.default_rng(100 + seed)
        n = int(rng.integers(3, 60))
        src, dst, w = random_multigraph(rng, n, 5 * n)
    else:
        n, src, dst, w = rmat_small(9, 8, 30 + seed)
    g = oracle.canonical_csr(n, src, dst, w)
    gr = oracle.transpose(g)
    hubs = oracle.hubs_topdeg(g, gr, min(6, n))
    empty = oracle.CSR(n, np.zeros(n + 1, np.int64), np.zeros(0, np.uint32), np.zeros(0, np.uint32))
    fwd = oracle.cg_alg2(g, empty, hubs)                 # forward traversals only, on G
    bwd_r = oracle.cg_alg2(gr, empty, hubs)              # forward-only on G^R: flags in G^R's order
    bwd = np.zeros(g.m, np.uint8)                        # G^R edge (v -> u) is G edge (u -> v)
    for v in range(n):
        for i in range(int(gr.ptr[v]), int(gr.ptr[v + 1])):
            if bwd_r[i]:
                u = int(gr.col[i])
                lo, hi = int(g.ptr[u]), int(g.ptr[u + 1])
                bwd[lo + int(np.searchsorted(g.col[lo:hi], v))] = 1
    union = np.maximum(fwd, bwd)
    per_dir = oracle.cg_alg2(g, gr, hubs, per_direction=True)
    assert np.array_equal(per_dir, union)


@pytest.mark.parametrize("seed", [3, 4])
def test_alg2_first_hub_reachability(seed):
    n, src, dst, w = rmat_small(10, 8, seed)
    g = oracle.canonical_csr(n, src, dst, w)
    gr = oracle.transpose(g)
    hubs = oracle.hubs_topdeg(g, gr, 8)
    cg = oracle.subgraph(g, oracle.cg_alg2(g, gr, hubs))
    h = int(hubs[0])
    assert np.array_equal(oracle.query("reach", cg, h), oracle.query("reach", g, h))
    assert cg.m < g.m


def test_alg2_single_hub_is_bfs_tree():
    """With one hub and a fresh Qid, Traverse(h, G) adds exactly one discovering edge per
    vertex reached from h (plus the first edge back into h when h lies on a cycle)."""
    n, src, dst, w = rmat_small(9, 8, 21)
    g = oracle.canonical_csr(n, src, dst, w)
    gr = oracle.transpose(g)
    h = int(oracle.hubs_topdeg(g, gr, 1)[0])
    # forward-only count: run Alg 2 on a graph whose reverse has no edges into/out of anything
    empty = oracle.CSR(n, np.zeros(n + 1, np.int64), np.zeros(0, np.uint32), np.zeros(0, np.uint32))
    flags = oracle.cg_alg2(g, empty, np.array([h], np.uint32))
    reach = oracle.query("reach", g, h)
    on_cycle = bool(reach[np.asarray(gr.col[gr.ptr[h]:gr.ptr[h + 1]], dtype=np.int64)].any())
    assert int(flags.sum()) == int(reach.sum()) - 1 + int(on_cycle)

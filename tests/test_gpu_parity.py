"""GPU parity: the CUDA path through the C ABI vs the CPU oracle, element by element.

Bars: CSR/CSC, CG edge sets, hub ids and all integer-kind values are
bit-exact; Viterbi values are bit-exact too (fallback bound 1e-6 relative, north_star).
"""
import numpy as np
import pytest
import torch

import gen
import oracle
from gpu_util import assert_values_equal, both, gpu_graph, to_dev, to_np
from helpers import KINDS, random_multigraph

pytestmark = pytest.mark.gpu


# ------------------------------------------------------------------ inputs
def test_device_generator_matches_host():
    from paper_conf_eurosys_0002a0a024_b200 import rmat_device
    for n, m, seed, permute, wm in ((1 << 12, 50_000, 1, True, 64), (4_847_571, 200_000, 2, True, 23),
                                   (1000, 30_000, 3, False, 7), (3, 100, 4, True, 1)):
        hs, hd, hw = gen.rmat(n, m, w_max=wm, seed=seed, permute=permute)
        ds, dd, dw = rmat_device(n, m, w_max=wm, seed=seed, permute=permute, device="cuda:0")
        assert np.array_equal(to_np(ds), hs) and np.array_equal(to_np(dd), hd) and np.array_equal(to_np(dw), hw)


# ------------------------------------------------------------------ a1, a2: CSR / CSC
@pytest.mark.parametrize("seed", range(6))
def test_csr_csc_bit_equal(seed):
    rng = np.random.default_rng(seed)
    n = int(rng.integers(1, 3000))
    src, dst, w = random_multigraph(rng, n, int(rng.integers(0, 20000)), wset=tuple(range(1, 70)))
    g, og = both(n, src, dst, w)
    assert g.m == og.m
    ptr, idx, ww = g.export()
    assert np.array_equal(ptr.cpu().numpy(), og.ptr)
    assert np.array_equal(to_np(idx), og.col) and np.array_equal(to_np(ww), og.wt)
    ogr = oracle.transpose(og)
    ptr, idx, ww = g.export(transpose=True)
    assert np.array_equal(ptr.cpu().numpy(), ogr.ptr)
    assert np.array_equal(to_np(idx), ogr.col) and np.array_equal(to_np(ww), ogr.wt)


def test_csr_rmat16_and_wide_weights():
    n, m = 1 << 16, 16 << 16
    for wm in (64, 1 << 20):   # packed edge words, then the (dst, w) pair layout
        src, dst, w = gen.rmat(n, m, w_max=wm, seed=1)
        g, og = both(n, src, dst, w)
        ptr, idx, ww = g.export()
        assert np.array_equal(ptr.cpu().numpy(), og.ptr)
        assert np.array_equal(to_np(idx), og.col) and np.array_equal(to_np(ww), og.wt)


def test_graph_input_errors():
    from paper_conf_eurosys_0002a0a024_b200 import CGInvalid
    with pytest.raises(CGInvalid):
        gpu_graph(4, np.array([0, 9]), np.array([1, 2]), np.array([1, 1]))
    with pytest.raises(CGInvalid):
        gpu_graph(4, np.array([0, 1]), np.array([1, 2]), np.array([1, 0]))


# ------------------------------------------------------------------ a8-a13: queries
def _check_queries(n, src, dst, w, sources, kinds=KINDS, modes=("full", "2phase"), K=8):
    g, og = both(n, src, dst, w)
    ogr = oracle.transpose(og)
    for kind in kinds:
        if "2phase" in modes:
            g.build(kind, K=min(K, n))
        for mode in modes:
            out = to_np(g.query(kind, to_dev(sources), mode=mode))
            for i, s in enumerate(sources):
                assert_values_equal(out[i], oracle.query(kind, og, int(s)), kind, f"{kind}/{mode}/s={s}")
    g.close()
    return og, ogr


@pytest.mark.parametrize("seed", range(8))
def test_queries_small_random(seed):
    rng = np.random.default_rng(seed)
    n = int(rng.integers(1, 200))
    src, dst, w = random_multigraph(rng, n, int(rng.integers(0, 6 * n + 1)))
    _check_queries(n, src, dst, w, np.arange(n, dtype=np.uint32))


def test_queries_rmat16_config1():
    """configs[0]: RMAT scale-16 ef16, w 1..64 — vertex 0 (isolated in the permuted ids), the
    generator's vertex 0 (the config's query, reading N10) + 64 sampled sources."""
    c = gen.CONFIGS["c1"]
    src, dst, w = c.edges()
    sources = np.concatenate([[0, gen.generator_vertex(c, 0)], gen.sample_sources(c.n, src, dst, 64, seed=42)])
    sources = sources.astype(np.uint32)
    _check_queries(c.n, src, dst, w, sources, K=20)


def test_edge_cases():
    # n = 1, no edges
    _check_queries(1, np.zeros(0, np.uint32), np.zeros(0, np.uint32), np.zeros(0, np.uint32), np.array([0], np.uint32),
                   K=1)
    # isolated source and a source with outdeg 0 in a two-component graph with self-loops, duplicates
    src = np.array([0, 0, 1, 2, 2, 4, 5, 5, 6], np.uint32)
    dst = np.array([1, 1, 2, 0, 2, 5, 6, 6, 4], np.uint32)
    w = np.array([3, 2, 64, 1, 5, 1, 7, 3, 2], np.uint32)
    _check_queries(8, src, dst, w, np.arange(8, dtype=np.uint32), K=2)


def test_long_chain_loop_control():
    n = 100_000
    src = np.arange(n - 1, dtype=np.uint32)
    dst = src + 1
    w = (src % 7 + 1).astype(np.uint32)
    _check_queries(n, src, dst, w, np.array([0, n // 2], np.uint32), kinds=("sssp", "bfs", "viterbi", "reach"),
                   modes=("full",))


def test_f16_lane_overflow_falls_back():
    """SSSP and BFS run in binary16 lanes, exact for integers below 2048; a candidate of 2048 or
    more sets the lane-overflow flag and the call re-runs in u32 lanes: a 2500-vertex chain
    (levels / distances up to 2499) plus shortcuts, 2Phase and FULL, several sources."""
    n = 2500
    src = np.concatenate([np.arange(n - 1), [0, 1, 2]]).astype(np.uint32)
    dst = np.concatenate([np.arange(1, n), [1300, 1450, 2499]]).astype(np.uint32)
    w = np.ones(src.size, np.uint32)
    _check_queries(n, src, dst, w, np.array([0, 5, 100, 400, 2490], np.uint32), kinds=("sssp", "bfs", "reach", "sswp"),
                   K=4)


def test_wide_weights_use_u32_lanes():
    """SSWP / SSNP values are edge weights: binary16 lanes (32 queries per pass) only while
    w_max <= 2048; wider weights run in u32 lanes (16 per pass, cg_stats.batch_queries tells
    which), with the same results."""
    rng = np.random.default_rng(12)
    n, m = 3000, 24000
    src, dst = rng.integers(0, n, m).astype(np.uint32), rng.integers(0, n, m).astype(np.uint32)
    for w_hi, qb in ((2000, 32), (5000, 16)):
        w = rng.integers(1, w_hi + 1, m).astype(np.uint32)
        g, og = both(n, src, dst, w)
        sources = np.arange(0, 40, dtype=np.uint32)
        for kind in ("sswp", "ssnp"):
            g.build(kind, K=8)
            out, st = g.query(kind, to_dev(sources), mode="2phase", stats=True)
            out = to_np(out)
            assert all(x["batch_queries"] == qb for x in st), (kind, w_hi)
            for i, s in enumerate(sources):
                assert_values_equal(out[i], oracle.query(kind, og, int(s)), kind, f"w<={w_hi} {kind} s={s}")
        g.close()


def test_star_hub_chunks():
    """A hub with 10^6 out-edges: its row is split over many warps and CTAs by the edge-balanced
    S2 (a window row longer than any warp's share, dynamic tail tiles)."""
    leaves = 1_000_000
    n = leaves + 2
    src = np.concatenate([np.zeros(leaves, np.uint32), np.arange(1, 2001, dtype=np.uint32)])
    dst = np.concatenate([np.arange(1, leaves + 1, dtype=np.uint32), np.full(2000, n - 1, np.uint32)])
    rng = np.random.default_rng(3)
    w = rng.integers(1, 65, size=src.size).astype(np.uint32)
    _check_queries(n, src, dst, w, np.array([0, 5], np.uint32), kinds=("sssp", "sswp", "reach"), K=2)


def test_viterbi_powers_of_two_exact():
    n, m = 1 << 12, 16 << 12
    src, dst, _ = gen.rmat(n, m, seed=6)
    rng = np.random.default_rng(6)
    w = (1 << rng.integers(1, 7, size=m)).astype(np.uint32)
    _check_queries(n, src, dst, w, np.arange(0, n, 97, dtype=np.uint32), kinds=("viterbi",))


# ------------------------------------------------------------------ a3-a7: Core Graph
@pytest.mark.parametrize("kind", KINDS)
def test_core_graph_edge_set_and_hubs(kind):
    n, m = 1 << 14, 16 << 14
    src, dst, w = gen.rmat(n, m, w_max=15, seed=11)
    g, og = both(n, src, dst, w)
    ogr = oracle.transpose(og)
    info = g.build(kind, K=20)
    hubs = oracle.hubs_topdeg(og, ogr, 20)
    assert info["hubs"] == [int(h) for h in hubs]
    exp = oracle.cg_for_kind(kind, og, ogr, hubs)
    got = g.core_flags(kind).cpu().numpy()
    assert got.size == exp.size
    bad = np.nonzero(got != exp)[0]
    assert bad.size == 0, f"{kind}: {bad.size} CG edges differ"
    assert info["m_cg"] == int(exp.sum())


@pytest.mark.parametrize("kind", KINDS)
def test_phase1_values_and_precision(kind):
    """p1 (the phase-1 fixpoint on CG) and impacted / reached / precise counts are unique: equal
    to the oracle's Alg 3."""
    n, m = 1 << 13, 16 << 13
    src, dst, w = gen.rmat(n, m, w_max=31, seed=5)
    g, og = both(n, src, dst, w)
    ogr = oracle.transpose(og)
    g.build(kind, K=20)
    cg = oracle.subgraph(og, oracle.cg_for_kind(kind, og, ogr, oracle.hubs_topdeg(og, ogr, 20)))
    sources = gen.sample_sources(n, src, dst, 16, seed=9)
    out, p1, stats = g.query(kind, to_dev(sources), mode="2phase", p1=True, stats=True)
    out, p1 = to_np(out), to_np(p1)
    for i, s in enumerate(sources):
        val, op1, st = oracle.two_phase(kind, og, cg, int(s))
        assert_values_equal(out[i], val, kind, f"final s={s}")
        assert_values_equal(p1[i], op1, kind, f"p1 s={s}")
        assert stats[i]["reached"] == st["reached"]
        assert stats[i]["precise_p1"] == st["precise_p1"]
        assert stats[i]["impacted"] == st["impacted"]


def test_hub_policies_and_errors():
    from paper_conf_eurosys_0002a0a024_b200 import CGInvalid, CGNoCoreGraph
    n, m = 1 << 12, 8 << 12
    src, dst, w = gen.rmat(n, m, seed=2)
    g, og = both(n, src, dst, w)
    with pytest.raises(CGNoCoreGraph):
        g.query("sssp", to_dev(np.array([1], np.uint32)), mode="2phase")
    with pytest.raises(CGInvalid):
        g.build("sssp", K=0)
    with pytest.raises(CGInvalid):
        g.build("sssp", hubs=[n + 5])
    with pytest.raises(CGInvalid):
        g.query("sssp", to_dev(np.array([n], np.uint32)), mode="full", stats=True)
    info = g.build("sssp", hubs=[3, 17, 99])
    assert info["hubs"] == [3, 17, 99]
    ogr = oracle.transpose(og)
    exp = oracle.cg_alg1("sssp", og, ogr, np.array([3, 17, 99], np.uint32))
    got = g.core_flags("sssp").cpu().numpy()
    assert np.array_equal(got, exp)
    info = g.build("sswp", K=10, policy="sampled", seed=123)
    assert len(set(info["hubs"])) == 10
    s = gen.sample_sources(n, src, dst, 8, seed=1)
    out = to_np(g.query("sswp", to_dev(s), mode="2phase"))
    for i, x in enumerate(s):
        assert_values_equal(out[i], oracle.query("sswp", og, int(x)), "sswp")


def test_query_host_end_to_end():
    n, m = 1 << 14, 16 << 14
    src, dst, w = gen.rmat(n, m, seed=4)
    g, og = both(n, src, dst, w)
    g.build("ssnp", K=20)
    s = gen.sample_sources(n, src, dst, 7, seed=3)
    out = g.query_host("ssnp", torch.from_numpy(s.astype(np.int64)), mode="2phase", batch=3)
    got = out.view(torch.int32).numpy().view(np.uint32)
    for i, x in enumerate(s):
        assert_values_equal(got[i], oracle.query("ssnp", og, int(x)), "ssnp")


def test_alg_options_match_oracle():
    """Alg 1 for REACH/BFS and Alg 2 with connectivity (the options of readings Q11/Q12)."""
    n, m = 1 << 12, 12 << 12
    src, dst, w = gen.rmat(n, m, seed=8)
    g, og = both(n, src, dst, w)
    ogr = oracle.transpose(og)
    hubs = oracle.hubs_topdeg(og, ogr, 10)
    g.build("bfs", K=10, alg="specialized")
    assert np.array_equal(g.core_flags("bfs").cpu().numpy(), oracle.cg_alg1("bfs", og, ogr, hubs))
    g.build("reach", K=10, alg="general", connectivity=True)
    assert np.array_equal(g.core_flags("reach").cpu().numpy(), oracle.cg_alg2(og, ogr, hubs, connectivity=True))


def test_rmat18_all_kinds_many_tiles():
    """A mid-size graph (2^18 vertices, 4 M edges): many S1 rounds per CTA, multi-window hub
    rows shared by several warps and CTAs, dense and sparse frontiers in both phases — every kind
    in both modes against the oracle."""
    n, m = 1 << 18, 16 << 18
    src, dst, w = gen.rmat(n, m, w_max=19, seed=13)
    g, og = both(n, src, dst, w)
    sources = np.concatenate([[0], gen.sample_sources(n, src, dst, 5, seed=2)]).astype(np.uint32)
    for kind in KINDS:
        g.build(kind, K=20)
        for mode in ("full", "2phase"):
            out = to_np(g.query(kind, to_dev(sources), mode=mode))
            for i, s in enumerate(sources):
                assert_values_equal(out[i], oracle.query(kind, og, int(s)), kind, f"{kind}/{mode}/s={s}")


@pytest.mark.parametrize("engine", ["single", "u32", "packed"])
def test_single_and_batched_engines(engine, monkeypatch):
    """CG_BATCH=0 runs every source through the single-query engine; otherwise sources run in
    batches (NEXT-2): "u32" forces u32 value lanes (16 queries per pass, CG_LANES=32), "packed"
    is the default (binary16 lanes for SSSP / SSWP / SSNP / BFS, bit lanes for REACH, 32 per pass).  Ragged
    tails (45 sources: 2 full u32 passes + 13; 1 packed pass + 13), all kinds, both modes,
    phase-1 values and the unique per-query counts must match the oracle."""
    if engine == "single":
        monkeypatch.setenv("CG_BATCH", "0")
    elif engine == "u32":
        monkeypatch.setenv("CG_LANES", "32")
    batch = engine
    n, m = 1 << 14, 16 << 14
    src, dst, w = gen.rmat(n, m, w_max=27, seed=21)
    g, og = both(n, src, dst, w)
    ogr = oracle.transpose(og)
    hubs = oracle.hubs_topdeg(og, ogr, 20)
    sources = np.concatenate([[0, 0], gen.sample_sources(n, src, dst, 43, seed=4)]).astype(np.uint32)
    for kind in KINDS:
        g.build(kind, K=20)
        cg = oracle.subgraph(og, oracle.cg_for_kind(kind, og, ogr, hubs))
        out, p1, st = g.query(kind, to_dev(sources), mode="2phase", p1=True, stats=True)
        out, p1 = to_np(out), to_np(p1)
        full = to_np(g.query(kind, to_dev(sources), mode="full"))
        for i, s in enumerate(sources):
            val, op1, ost = oracle.two_phase(kind, og, cg, int(s))
            assert_values_equal(out[i], val, kind, f"B={batch} {kind} 2phase s={s}")
            assert_values_equal(full[i], val, kind, f"B={batch} {kind} full s={s}")
            assert_values_equal(p1[i], op1, kind, f"B={batch} {kind} p1 s={s}")
            assert (st[i]["reached"], st[i]["precise_p1"], st[i]["impacted"]) == \
                (ost["reached"], ost["precise_p1"], ost["impacted"]), (batch, kind, int(s))


@pytest.mark.parametrize("rest", ["0", "1"])
def test_first_sweep_over_g_minus_cg(rest, monkeypatch):
    """Reading N7: after phase 1 every CG edge is at its fixpoint, so phase 2's first sweep may
    relax only G minus the CG (CG_REST=1, the default) — values, phase-1 values and the
    reached / precise / impacted counts are those of the full first sweep (CG_REST=0) and the
    oracle's, for every kind, with an Alg 1 CG (connectivity edges included) and Alg 2's."""
    monkeypatch.setenv("CG_REST", rest)
    n, m = 1 << 15, 16 << 15
    src, dst, w = gen.rmat(n, m, w_max=17, seed=41)
    g, og = both(n, src, dst, w)
    ogr = oracle.transpose(og)
    hubs = oracle.hubs_topdeg(og, ogr, 20)
    sources = np.concatenate([[0], gen.sample_sources(n, src, dst, 36, seed=5)]).astype(np.uint32)
    for kind in KINDS:
        g.build(kind, K=20)
        cg = oracle.subgraph(og, oracle.cg_for_kind(kind, og, ogr, hubs))
        out, p1, st = g.query(kind, to_dev(sources), mode="2phase", p1=True, stats=True)
        out, p1 = to_np(out), to_np(p1)
        for i, s in enumerate(sources):
            val, op1, ost = oracle.two_phase(kind, og, cg, int(s))
            assert_values_equal(out[i], val, kind, f"rest={rest} {kind} s={s}")
            assert_values_equal(p1[i], op1, kind, f"rest={rest} {kind} p1 s={s}")
            assert (st[i]["reached"], st[i]["precise_p1"], st[i]["impacted"]) == \
                (ost["reached"], ost["precise_p1"], ost["impacted"]), (rest, kind, int(s))


@pytest.mark.parametrize("dyn", ["0", "1"])
def test_static_and_dynamic_s2_split(dyn, monkeypatch):
    """S2's edge split: fully static (CG_DYN=0) or half static + tiles taken from a per-iteration
    counter (the default for iterations with >= 1,024 list edges per warp, i.e. >= 2.4 M edges:
    the dense iterations of RMAT-18 with 32 sources)."""
    monkeypatch.setenv("CG_DYN", dyn)
    n, m = 1 << 18, 16 << 18
    src, dst, w = gen.rmat(n, m, w_max=19, seed=17)
    g, og = both(n, src, dst, w)
    sources = gen.sample_sources(n, src, dst, 32, seed=12)
    for kind in ("sssp", "viterbi", "bfs"):
        g.build(kind, K=20)
        for mode in ("2phase", "full"):
            out = to_np(g.query(kind, to_dev(sources), mode=mode))
            for i, s in enumerate(sources[:8]):
                assert_values_equal(out[i], oracle.query(kind, og, int(s)), kind, f"dyn={dyn} {kind} {mode}")


@pytest.mark.parametrize("bits_below", ["0", "4294967295"])
def test_batched_frontier_modes(bits_below, monkeypatch):
    """The batched engine keeps the union frontier either as bitmap bits set by S2 or as the
    per-vertex query masks scanned by S1 (chosen per iteration); force each everywhere."""
    monkeypatch.setenv("CG_BITS_BELOW", bits_below)
    n, m = 1 << 15, 16 << 15
    src, dst, w = gen.rmat(n, m, w_max=15, seed=33)
    g, og = both(n, src, dst, w)
    sources = gen.sample_sources(n, src, dst, 20, seed=8)
    for kind in ("sssp", "viterbi", "reach"):
        g.build(kind, K=20)
        for mode in ("2phase", "full"):
            out = to_np(g.query(kind, to_dev(sources), mode=mode))
            for i, s in enumerate(sources):
                assert_values_equal(out[i], oracle.query(kind, og, int(s)), kind, f"bits<{bits_below} {kind} {mode}")


@pytest.mark.parametrize("reduced,lanes", [("0", ""), ("0x3f", ""), ("0x3f", "32")])
def test_reduced_pull_completion(reduced, lanes, monkeypatch):
    """NEXT-1: phase 2 = one pull sweep over the in-edges of vertices whose phase-1 value is not
    certified (Theorem 1 P:1321-1371 and its bottleneck analogs; REACH: the lattice top), then
    push.  Off (0) and on for every kind that has a certificate (0x3f; the hub certificates need
    u32 lanes, forced by CG_LANES=32): identical to the oracle."""
    monkeypatch.setenv("CG_REDUCED", reduced)
    if lanes:
        monkeypatch.setenv("CG_LANES", lanes)
    n, m = 1 << 15, 16 << 15
    src, dst, w = gen.rmat(n, m, w_max=9, seed=44)
    g, og = both(n, src, dst, w)
    sources = np.concatenate([[0], gen.sample_sources(n, src, dst, 21, seed=6)]).astype(np.uint32)
    for kind in KINDS:
        g.build(kind, K=20)
        out = to_np(g.query(kind, to_dev(sources), mode="2phase"))
        for i, s in enumerate(sources):
            assert_values_equal(out[i], oracle.query(kind, og, int(s)), kind, f"reduced={reduced} {kind} s={s}")


def test_general_cg_per_direction():
    """Reading Q9 option: Alg 2 with one Qid[] per traversal direction == the oracle's option."""
    n, m = 1 << 13, 12 << 13
    src, dst, w = gen.rmat(n, m, seed=17)
    g, og = both(n, src, dst, w)
    ogr = oracle.transpose(og)
    hubs = oracle.hubs_topdeg(og, ogr, 12)
    g.build("reach", K=12, alg="general_perdir")
    assert np.array_equal(g.core_flags("reach").cpu().numpy(), oracle.cg_alg2(og, ogr, hubs, per_direction=True))
    s = gen.sample_sources(n, src, dst, 9, seed=3)
    for kind in ("reach", "bfs"):
        out = to_np(g.query(kind, to_dev(s), mode="2phase"))
        for i, x in enumerate(s):
            assert_values_equal(out[i], oracle.query(kind, og, int(x)), kind, "perdir")


@pytest.mark.parametrize("kind", ["sssp", "sswp", "ssnp", "viterbi"])
def test_partial_builds_merge_to_full_core_graph(kind):
    """NEXT-4: the flags of hub shards (cg_build_partial), OR-ed and installed with
    cg_build_from_flags, give exactly the single-call Core Graph (Algorithm 1 is a union over
    hubs), and 2Phase queries on it match the oracle."""
    n, m = 1 << 13, 16 << 13
    src, dst, w = gen.rmat(n, m, w_max=29, seed=61)
    g, og = both(n, src, dst, w)
    ref = g.build(kind, K=20)
    ref_flags = g.core_flags(kind).cpu().numpy()
    merged = None
    for b, e in ((0, 7), (7, 13), (13, 20)):
        f = g.build_partial(kind, K=20, hub_range=(b, e))
        merged = f.clone() if merged is None else torch.maximum(merged, f)
    info = g.build_from_flags(kind, merged, K=20)
    ogr = oracle.transpose(og)
    exp = oracle.cg_alg1(kind, og, ogr, np.array(ref["hubs"], np.uint32), connectivity=True)
    assert np.array_equal(ref_flags, exp)  # the single-call build is the oracle's Algorithm 1 CG
    assert np.array_equal(g.core_flags(kind).cpu().numpy(), exp)  # ... and so is the merged one
    assert info["m_cg"] == ref["m_cg"] == int(exp.sum()) and info["hubs"] == ref["hubs"]
    # the shards' raw flags are the oracle's Alg 1 marks of their hubs (no connectivity edges)
    f0 = g.build_partial(kind, K=20, hub_range=(0, 7)).cpu().numpy()
    assert np.array_equal(f0, oracle.cg_alg1(kind, og, ogr, np.array(ref["hubs"][:7], np.uint32),
                                             connectivity=False))
    sources = gen.sample_sources(n, src, dst, 9, seed=2)
    out = to_np(g.query(kind, to_dev(sources), mode="2phase"))
    for i, s in enumerate(sources):
        assert_values_equal(out[i], oracle.query(kind, og, int(s)), kind, f"merged {kind} s={s}")
    from paper_conf_eurosys_0002a0a024_b200 import CGUnsupported
    with pytest.raises(CGUnsupported):
        g.build_partial("reach", K=4, hub_range=(0, 2))


def test_core_graph_save_load(tmp_path):
    """NEXT-4 persistence: a saved Core Graph loads into a fresh Graph of the same edges (same
    flags, hubs, results) and is refused by a different graph."""
    from paper_conf_eurosys_0002a0a024_b200 import CGInvalid, Graph
    n, m = 1 << 13, 16 << 13
    src, dst, w = gen.rmat(n, m, w_max=29, seed=62)
    g, og = both(n, src, dst, w)
    sources = gen.sample_sources(n, src, dst, 7, seed=3)
    for kind in ("sssp", "reach"):
        info = g.build(kind, K=16)
        path = str(tmp_path / f"{kind}.cg")
        g.save_core(kind, path)
        g2 = Graph(n, to_dev(src), to_dev(dst), to_dev(w))
        info2 = g2.load_core(kind, path)
        assert info2["m_cg"] == info["m_cg"] and info2["hubs"] == info["hubs"]
        ogr = oracle.transpose(og)
        hubs = np.array(info["hubs"], np.uint32)
        exp = (oracle.cg_alg1(kind, og, ogr, hubs) if kind == "sssp"
               else oracle.cg_alg2(og, ogr, hubs, per_direction=True))  # the kind's CG (reading Q9')
        assert np.array_equal(g2.core_flags(kind).cpu().numpy(), exp)  # loaded == oracle CG
        assert np.array_equal(g.core_flags(kind).cpu().numpy(), exp)
        out = to_np(g2.query(kind, to_dev(sources), mode="2phase"))
        for i, s in enumerate(sources):
            assert_values_equal(out[i], oracle.query(kind, og, int(s)), kind, f"loaded {kind} s={s}")
        g2.close()
    src3, dst3, w3 = gen.rmat(n, m, w_max=29, seed=63)
    g3 = Graph(n, to_dev(src3), to_dev(dst3), to_dev(w3))
    with pytest.raises(CGInvalid):
        g3.load_core("sssp", str(tmp_path / "sssp.cg"))
    with pytest.raises(CGInvalid):
        g3.load_core("sssp", str(tmp_path / "missing.cg"))


@pytest.mark.parametrize("seed", range(3))
def test_wcc_small_random(seed):
    """NEXT-3 WCC: labels (minimum id of the weak component) from FULL and 2PHASE equal the
    oracle on random multigraphs (isolated vertices, duplicates, self-loops); phase-1 labels
    equal the oracle's WCC of the Core Graph alone (label propagation on CG ∪ CG^R from the
    vertex ids converges to the CG's weak components: reading W2)."""
    rng = np.random.default_rng(100 + seed)
    n = int(rng.integers(2, 400))
    src, dst, w = random_multigraph(rng, n, int(rng.integers(0, 3 * n + 1)))
    g, og = both(n, src, dst, w)
    ogr = oracle.transpose(og)
    exp = oracle.wcc(og)
    g.build("wcc", K=min(8, n))
    flags = oracle.cg_alg2(og, ogr, oracle.hubs_topdeg(og, ogr, min(8, n)), per_direction=True)
    assert np.array_equal(g.core_flags("wcc").cpu().numpy(), flags)
    for mode in ("full", "2phase"):
        out = to_np(g.query("wcc", None, mode=mode))
        assert out.shape == (1, n)
        assert np.array_equal(out[0], exp), mode
    _, p1 = g.query("wcc", None, mode="2phase", p1=True)
    assert np.array_equal(to_np(p1)[0], oracle.wcc(oracle.subgraph(og, flags)))


def test_wcc_rmat_and_errors():
    from paper_conf_eurosys_0002a0a024_b200 import CGInvalid
    n, m = 1 << 15, 8 << 15
    src, dst, w = gen.rmat(n, m, seed=71)
    g, og = both(n, src, dst, w)
    exp = oracle.wcc(og)
    g.build("reach", K=20)  # WCC shares REACH's general CG
    for mode in ("full", "2phase"):
        out, st = g.query("wcc", None, mode=mode, stats=True)
        assert np.array_equal(to_np(out)[0], exp), mode
        assert st[0]["batch_queries"] == 1
    with pytest.raises(CGInvalid):
        g.query("wcc", to_dev(np.array([0, 1], np.uint32)), mode="full")
    host = g.query_host("wcc", np.array([0], np.uint32), mode="2phase")
    assert np.array_equal(host.numpy()[0], exp)

"""The §8(b) boundary contract on the GPU: sticky device errors, asynchrony, output formats,
per-phase times, stream ordering, and the binary16 value-lane limits (reading N3).

The problem statement's query is Q(s) over all vertices; Algorithm 3's two phases
 are what ms_p1 / ms_p2 time.
"""
import numpy as np
import pytest
import torch

import gen
import oracle
from gpu_util import assert_values_equal, both, to_dev, to_np
from helpers import KINDS

pytestmark = pytest.mark.gpu


def _rmat(scale, ef, seed, w_max=23):
    n, m = 1 << scale, ef << scale
    src, dst, w = gen.rmat(n, m, w_max=w_max, seed=seed)
    return n, src, dst, w


def test_device_source_out_of_range_is_sticky_einval():
    """A source id >= n in a DEVICE array, no stats: cg_query stays asynchronous (CG_OK), the
    bad query's row holds InitVal, the other rows are right; cg_graph_status then returns
    CG_EINVAL, and so would the next query call; the error is cleared once returned."""
    from paper_conf_eurosys_0002a0a024_b200 import CGInvalid
    n, src, dst, w = _rmat(12, 8, 71)
    g, og = both(n, src, dst, w)
    for kind in ("sssp", "reach", "viterbi"):
        g.build(kind, K=8)
        good = gen.sample_sources(n, src, dst, 3, seed=5)
        s = np.array([good[0], n + 7, good[1], good[2]], np.uint32)
        for mode in ("2phase", "full"):
            out = g.query(kind, to_dev(s), mode=mode)  # asynchronous: no error yet
            with pytest.raises(CGInvalid):
                g.status()
            g.status()  # cleared
            o = to_np(out)
            assert (o[1] == oracle.init_val(kind)).all()
            for i in (0, 2, 3):
                assert_values_equal(o[i], oracle.query(kind, og, int(s[i])), kind, f"{kind}/{mode}")
        # the pending error is also returned by the next query call (which does no work)
        g.query(kind, to_dev(s), mode="2phase")
        torch.cuda.synchronize()
        with pytest.raises(CGInvalid):
            g.query(kind, to_dev(good), mode="2phase")
        g.status()
    # the single-query engine (one source) reports the same way
    g.query("sssp", to_dev(np.array([n], np.uint32)), mode="full")
    with pytest.raises(CGInvalid):
        g.status()
    # with stats the call synchronises and fails itself
    with pytest.raises(CGInvalid):
        g.query("sssp", to_dev(np.array([0, n], np.uint32)), mode="2phase", stats=True)
    g.status()
    g.close()


def test_sssp_query_returns_before_the_kernel_finishes():
    """cg_query without stats does no host synchronisation, also for SSSP / BFS whose binary16
    lanes need an overflow check (done on the device by a guarded u32 re-run)."""
    n, src, dst, w = _rmat(21, 16, 72)
    g, og = both(n, src, dst, w)
    sources = to_dev(gen.sample_sources(n, src, dst, 64, seed=9))
    stream = torch.cuda.current_stream()
    for kind in ("sssp", "bfs"):
        g.build(kind, K=20)
        out = g.query(kind, sources, mode="2phase")  # warm
        torch.cuda.synchronize()
        pending = 0
        for _ in range(3):
            g.query(kind, sources, mode="2phase", out=out)
            pending += not stream.query()  # still running when the call returned
            torch.cuda.synchronize()
        assert pending == 3, kind
    g.close()


@pytest.mark.parametrize("kind", ["sswp", "ssnp", "sssp"])
def test_weight_2048_in_binary16_lanes(kind):
    """w_max == 2048 is the largest weight binary16 lanes hold exactly: SSWP / SSNP values equal
    to 2048 and SSSP distances reaching 2048 (overflow flag -> u32 re-run) match the oracle."""
    rng = np.random.default_rng(73)
    n, m = 3000, 20000
    src, dst = rng.integers(0, n, m).astype(np.uint32), rng.integers(0, n, m).astype(np.uint32)
    w = rng.choice(np.array([1, 2, 7, 1000, 2047, 2048], np.uint32), m)
    g, og = both(n, src, dst, w)
    assert g.w_max == 2048
    g.build(kind, K=8)
    sources = np.arange(0, 40, dtype=np.uint32)
    for mode in ("2phase", "full"):
        out, st = g.query(kind, to_dev(sources), mode=mode, stats=True)
        out = to_np(out)
        for i, s in enumerate(sources):
            exp = oracle.query(kind, og, int(s))
            assert_values_equal(out[i], exp, kind, f"{kind}/{mode}/s={s}")
        if kind != "sssp":
            assert all(x["batch_queries"] == 32 for x in st)  # binary16 lanes
            assert (np.stack([oracle.query(kind, og, int(s)) for s in sources]) == 2048).any()
    # the asynchronous path (device-guarded re-run) gives the same values
    out = to_np(g.query(kind, to_dev(sources), mode="2phase"))
    for i, s in enumerate(sources):
        assert_values_equal(out[i], oracle.query(kind, og, int(s)), kind, f"{kind}/async/s={s}")
    g.close()


def u16np(t):
    torch.cuda.synchronize()
    return t.view(torch.int16).cpu().numpy().view(np.uint16)


def _u16_of(exp):
    e = exp.astype(np.int64)
    return np.where(e == 0xFFFFFFFF, 0xFFFF, e).astype(np.uint16)


def _bits_of(exp):
    n = exp.size
    b = np.zeros(((n + 31) // 32) * 32, np.uint64)
    b[:n] = exp != 0
    words = (b.reshape(-1, 32) << np.arange(32, dtype=np.uint64)).sum(axis=1)
    return words.astype(np.uint32)


def test_narrow_output_formats():
    """CG_OUT_U16 (SSSP, SSWP, SSNP, BFS, REACH) and CG_OUT_BITS (REACH) carry exactly the
    oracle's values, device and host (cg_query_host_fmt) paths; VITERBI / WCC refuse U16, only
    REACH takes BITS; a value >= 0xFFFF in U16 is a sticky CG_EOVERFLOW."""
    from paper_conf_eurosys_0002a0a024_b200 import CGInvalid, CGOverflow
    n, src, dst, w = _rmat(13, 8, 74)
    g, og = both(n, src, dst, w)
    sources = np.concatenate([[0], gen.sample_sources(n, src, dst, 37, seed=3)]).astype(np.uint32)
    for kind in ("sssp", "sswp", "ssnp", "bfs", "reach"):
        g.build(kind, K=8)
        exp = [oracle.query(kind, og, int(s)) for s in sources]
        for mode in ("2phase", "full"):
            o16 = u16np(g.query(kind, to_dev(sources), mode=mode, fmt="u16"))
            h16 = u16np(g.query_host(kind, sources, mode=mode, fmt="u16", batch=16))
            for i in range(len(sources)):
                assert np.array_equal(o16[i], _u16_of(exp[i])), (kind, mode, i)
                assert np.array_equal(h16[i], _u16_of(exp[i])), (kind, mode, i)
            if kind == "reach":
                ob = g.query(kind, to_dev(sources), mode=mode, fmt="bits").view(torch.int32).cpu().numpy()
                hb = g.query_host(kind, sources, mode=mode, fmt="bits", batch=7).view(torch.int32).numpy()
                for i in range(len(sources)):
                    assert np.array_equal(ob[i].view(np.uint32), _bits_of(exp[i])), (mode, i)
                    assert np.array_equal(hb[i].view(np.uint32), _bits_of(exp[i])), (mode, i)
    g.build("viterbi", K=4)
    for kind, fmt in (("viterbi", "u16"), ("sssp", "bits"), ("wcc", "u16")):
        with pytest.raises(CGInvalid):
            g.query(kind, to_dev(sources[:2]) if kind != "wcc" else None, mode="full", fmt=fmt)
    g.close()
    # a chain of weight-40 edges: SSSP distances pass 0xFFFF -> sticky CG_EOVERFLOW
    n = 2000
    src = np.arange(n - 1, dtype=np.uint32)
    g, og = both(n, src, src + 1, np.full(n - 1, 40, np.uint32))
    g.query("sssp", to_dev(np.array([0, 5], np.uint32)), mode="full", fmt="u16")
    with pytest.raises(CGOverflow):
        g.status()
    out = u16np(g.query("sssp", to_dev(np.array([1900, 1950], np.uint32)), mode="full", fmt="u16"))
    g.status()  # short distances fit
    assert np.array_equal(out[0], _u16_of(oracle.query("sssp", og, 1900)))
    g.close()


def test_phase_times_in_stats():
    """cg_stats.ms_p1 / ms_p2: device time of init + phase 1 and of phase 2 + output of the
    pass that ran the query (> 0; FULL has no phase 1)."""
    n, src, dst, w = _rmat(16, 16, 75)
    g, og = both(n, src, dst, w)
    sources = to_dev(gen.sample_sources(n, src, dst, 40, seed=4))
    for kind in ("sssp", "reach", "viterbi"):
        g.build(kind, K=20)
        _, st2 = g.query(kind, sources, mode="2phase", stats=True)
        _, stf = g.query(kind, sources, mode="full", stats=True)
        assert all(x["ms_p1"] > 0 and x["ms_p2"] > 0 for x in st2), kind
        assert all(x["ms_p2"] > 0 and x["ms_p1"] >= 0 for x in stf), kind
        assert all(x["ms_p1"] + x["ms_p2"] < 1000 for x in st2)
    _, st1 = g.query("sssp", sources[:1], mode="2phase", stats=True)  # single-query engine
    assert st1[0]["batch_queries"] == 1 and st1[0]["ms_p1"] > 0 and st1[0]["ms_p2"] > 0
    g.close()


def test_calls_on_two_streams_are_ordered():
    """Calls on one graph issued on different streams run in issue order (they share the
    workspace): results equal the single-stream ones."""
    n, src, dst, w = _rmat(16, 16, 76)
    g, og = both(n, src, dst, w)
    srcs = [gen.sample_sources(n, src, dst, 33, seed=s) for s in (1, 2, 3, 4)]
    kinds = ("sssp", "reach", "sswp", "bfs")
    for k in kinds:
        g.build(k, K=16)
    ref = [to_np(g.query(k, to_dev(s))) for k, s in zip(kinds, srcs)]
    streams = [torch.cuda.Stream() for _ in range(2)]
    sds = [to_dev(s) for s in srcs]  # kept alive until every stream is done (caching allocator)
    torch.cuda.synchronize()
    outs = []
    for i, (k, sd) in enumerate(zip(kinds, sds)):
        with torch.cuda.stream(streams[i % 2]):
            outs.append(g.query(k, sd))
    torch.cuda.synchronize()
    for r, o in zip(ref, outs):
        assert np.array_equal(r, to_np(o))
    g.close()


def test_split_core_graph_layout():
    """NEXT-3 split CSR: the Core Graph is one reordered copy of G's edges per kind
    with the CG edges first; the exported membership flags equal the oracle's CG and every kind
    still matches the oracle through it (2Phase; the first sweep reads G minus the CG)."""
    n, src, dst, w = _rmat(14, 12, 77, w_max=29)
    g, og = both(n, src, dst, w)
    ogr = oracle.transpose(og)
    sources = gen.sample_sources(n, src, dst, 21, seed=6)
    for kind in KINDS:
        info = g.build(kind, K=12)
        hubs = np.array(info["hubs"], np.uint32)
        exp = oracle.cg_for_kind(kind, og, ogr, hubs)
        assert np.array_equal(g.core_flags(kind).cpu().numpy(), exp), kind
        assert info["m_cg"] == int(exp.sum())
        out = to_np(g.query(kind, to_dev(sources), mode="2phase"))
        for i, s in enumerate(sources):
            assert_values_equal(out[i], oracle.query(kind, og, int(s)), kind, f"split {kind} s={s}")
    g.close()


def test_query_host_async_calls_overlap_and_complete():
    """cg_query_host_async: six calls of different kinds (and formats) back to back on one graph,
    each in several device batches so the two result slots are reused within and across calls,
    one cg_graph_status at the end — every row equals the oracle; a synchronous call follows on the
    same graph."""
    n, src, dst, w = _rmat(14, 16, 91)
    g, og = both(n, src, dst, w)
    sources = gen.sample_sources(n, src, dst, 9, seed=13)
    fmts = {"sssp": "u16", "sswp": "u32", "ssnp": "u16", "viterbi": "u32", "bfs": "u16", "reach": "bits"}
    for kind in KINDS:
        g.build(kind, K=12)
    outs = {}
    for i, kind in enumerate(KINDS):
        cols, dt = g.row_shape(fmts[kind])
        outs[kind] = torch.empty((len(sources), cols), dtype=dt, pin_memory=True)
        g.query_host(kind, torch.from_numpy(sources.astype(np.int64)), mode="2phase" if i % 2 == 0 else "full",
                     out=outs[kind], batch=2 + i % 3, fmt=fmts[kind], sync=False)
    g.status()  # waits for the stream and the graph's copy stream
    for kind in KINDS:
        got = outs[kind]
        for i, s in enumerate(sources):
            exp = oracle.query(kind, og, int(s))
            if fmts[kind] == "u16":
                assert np.array_equal(got[i].view(torch.int16).numpy().view(np.uint16), _u16_of(exp)), (kind, s)
            elif fmts[kind] == "bits":
                assert np.array_equal(got[i].view(torch.int32).numpy().view(np.uint32), _bits_of(exp)), (kind, s)
            else:
                assert_values_equal(got[i].view(torch.int32).numpy().view(np.uint32), exp, kind, f"{kind}/async")
    sync = g.query_host("sssp", torch.from_numpy(sources.astype(np.int64)), mode="2phase", batch=4)
    for i, s in enumerate(sources):
        assert_values_equal(sync[i].view(torch.int32).numpy().view(np.uint32), oracle.query("sssp", og, int(s)),
                            "sssp", "sync after async")
    g.close()


@pytest.mark.parametrize("n", [4099, 4160, 4161, 63, 1])
def test_u16_rows_any_alignment(n):
    """CG_OUT_U16 rows start at u16 index q * n: for odd n every other row starts at an odd index, and
    the transpose writes vertex pairs with 4 B stores, so rows of both parities, tiles ending exactly
    at n (n = 64 k, 64 k + 1), tiny graphs and ragged batches (33, 45 sources: two passes, the last
    partial) must all hold the oracle's values."""
    rng = np.random.default_rng(n)
    m = 8 * n
    src = rng.integers(0, n, m).astype(np.uint32)
    dst = rng.integers(0, n, m).astype(np.uint32)
    w = rng.integers(1, 24, m).astype(np.uint32)
    g, og = both(n, src, dst, w)
    for ns in (33, 45):
        sources = rng.integers(0, n, ns).astype(np.uint32)
        for kind in ("sssp", "bfs", "reach"):
            g.build(kind, K=min(8, n))
            for mode in ("2phase", "full"):
                got = u16np(g.query(kind, to_dev(sources), mode=mode, fmt="u16"))
                for i, s in enumerate(sources):
                    assert np.array_equal(got[i], _u16_of(oracle.query(kind, og, int(s)))), (n, ns, kind, mode, i)
    g.close()

"""CPU ORACLE — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import this package.  The
product path (``paper_conf_eurosys_0002a0a024_b200``) never imports it and shares no code with it.

Thin ctypes marshalling over ``oracle/oracle.c`` (plain C, see its header
for the PAPER.md passage each function follows).  Every function here only
converts numpy arrays to pointers and back.

Parity status:
  canonical_csr / transpose   pinned (numpy lexsort canonicalisation, tests/test_oracle_graph.py)
  query (all six kinds)       pinned (brute force n<=8, scipy dijkstra, threshold BFS,
                              powers-of-two Viterbi, Table 2 / Fig 4 golden)
  bellman_ford                pinned (== brute force / query)
  hubs_topdeg                 pinned (argsort of total degree)
  cg_alg1                     pinned (Table 2 / Fig 4 golden; hub-query preservation property)
  cg_alg2                     pinned (hand-worked golden; reachability preservation property)
  two_phase / full_bsp        pinned (== query on every vertex; complete-CG exactness; p1 <= final)
  certified (O7)              pinned (certified => precise on every vertex; hubs reached in phase 1
                              are certified by Theorem 1 (a); closed forms on a path graph)
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None

KINDS = {"sssp": 0, "sswp": 1, "ssnp": 2, "viterbi": 3, "bfs": 4, "reach": 5, "wcc": 6}
KIND_NAMES = {v: k for k, v in KINDS.items()}


def build(force: bool = False) -> str:
    """Compile oracle/oracle.c -> oracle/liboracle.so (gcc, -O2, OpenMP, strict IEEE)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-fPIC", "-shared", "-std=c11",
                               "-fno-fast-math", "-ffp-contract=off", "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


class _Stats(ctypes.Structure):
    _fields_ = [(k, ctypes.c_int64) for k in (
        "iters_p1", "iters_p2", "edges_p1", "edges_p2", "updates_p1", "updates_p2",
        "impacted", "reached", "precise_p1", "unvisited_p2")]


def _load():
    global _lib
    if _lib is not None:
        return _lib
    build()
    lib = ctypes.CDLL(_LIB)
    i64, u32, i32, c_int = ctypes.c_int64, ctypes.c_uint32, ctypes.c_int32, ctypes.c_int
    P = ctypes.c_void_p
    sig = {
        "or_init_val": (u32, [c_int]),
        "or_source_val": (u32, [c_int]),
        "or_extend": (u32, [c_int, u32, u32]),
        "or_better": (c_int, [c_int, u32, u32]),
        "or_canonical_csr": (i64, [i64, i64, P, P, P, P, P, P]),
        "or_transpose": (None, [i64, P, P, P, P, P, P]),
        "or_query": (i64, [c_int, i64, P, P, P, u32, P]),
        "or_query_batch": (i64, [c_int, i64, P, P, P, i64, P, P, c_int]),
        "or_bellman_ford": (i64, [c_int, i64, P, P, P, u32, P]),
        "or_hubs_topdeg": (None, [i64, P, P, i32, P]),
        "or_cg_alg1": (i64, [c_int, i64, P, P, P, P, P, P, i32, P, c_int, P]),
        "or_cg_alg2": (i64, [i64, P, P, P, P, i32, P, c_int, c_int, P]),
        "or_subgraph": (i64, [i64, P, P, P, P, P, P, P]),
        "or_2phase": (None, [c_int, i64, P, P, P, P, P, P, u32, P, P, ctypes.POINTER(_Stats)]),
        "or_full_bsp": (None, [c_int, i64, P, P, P, u32, P, ctypes.POINTER(_Stats)]),
        "or_wcc": (None, [i64, P, P, P]),
        "or_certified": (None, [c_int, i64, u32, P, i32, P, P, P]),
    }
    for name, (res, args) in sig.items():
        f = getattr(lib, name)
        f.restype = res
        f.argtypes = args
    _lib = lib
    return lib


def _p(a: np.ndarray):
    assert a.flags["C_CONTIGUOUS"]
    return ctypes.c_void_p(a.ctypes.data)


def _kind(kind) -> int:
    return KINDS[kind] if isinstance(kind, str) else int(kind)


def init_val(kind) -> int:
    return int(_load().or_init_val(_kind(kind)))


def source_val(kind) -> int:
    return int(_load().or_source_val(_kind(kind)))


@dataclass
class CSR:
    """Canonical CSR of G (or of a sub-graph / G^R): ptr int64[n+1], col u32[m], wt u32[m]."""
    n: int
    ptr: np.ndarray
    col: np.ndarray
    wt: np.ndarray

    @property
    def m(self) -> int:
        return int(self.ptr[-1])

    def outdeg(self) -> np.ndarray:
        return np.diff(self.ptr)


def canonical_csr(n: int, src, dst, w) -> CSR:
    src = np.ascontiguousarray(src, dtype=np.uint32)
    dst = np.ascontiguousarray(dst, dtype=np.uint32)
    w = np.ascontiguousarray(w, dtype=np.uint32)
    m = src.size
    ptr = np.zeros(n + 1, dtype=np.int64)
    col = np.empty(max(m, 1), dtype=np.uint32)
    wt = np.empty(max(m, 1), dtype=np.uint32)
    mc = _load().or_canonical_csr(n, m, _p(src), _p(dst), _p(w), _p(ptr), _p(col), _p(wt))
    return CSR(n, ptr, col[:mc].copy(), wt[:mc].copy())


def transpose(g: CSR) -> CSR:
    cptr = np.zeros(g.n + 1, dtype=np.int64)
    row = np.empty(max(g.m, 1), dtype=np.uint32)
    wt = np.empty(max(g.m, 1), dtype=np.uint32)
    _load().or_transpose(g.n, _p(g.ptr), _p(_nz(g.col)), _p(_nz(g.wt)), _p(cptr), _p(row), _p(wt))
    return CSR(g.n, cptr, row[:g.m].copy(), wt[:g.m].copy())


def _nz(a: np.ndarray) -> np.ndarray:
    """ctypes needs a valid pointer even for empty arrays."""
    return a if a.size else np.zeros(1, dtype=a.dtype)


def query(kind, g: CSR, s: int) -> np.ndarray:
    if kind == "wcc" or kind == 6:
        return wcc(g)  # a whole-graph query: the source is ignored
    out = np.empty(g.n, dtype=np.uint32)
    _load().or_query(_kind(kind), g.n, _p(g.ptr), _p(_nz(g.col)), _p(_nz(g.wt)), int(s), _p(out))
    return out


def wcc(g: CSR) -> np.ndarray:
    """WCC labels (NEXT-3): the minimum vertex id of each vertex's weakly connected component
    (the fixpoint of Table 6's WCC row), by union-find over the undirected edges."""
    out = np.empty(g.n, dtype=np.uint32)
    _load().or_wcc(g.n, _p(g.ptr), _p(_nz(g.col)), _p(out))
    return out


def query_batch(kind, g: CSR, sources, nthreads: int = 0) -> np.ndarray:
    srcs = np.ascontiguousarray(sources, dtype=np.uint32)
    out = np.empty((srcs.size, g.n), dtype=np.uint32)
    nthreads = nthreads or os.cpu_count() or 1
    _load().or_query_batch(_kind(kind), g.n, _p(g.ptr), _p(_nz(g.col)), _p(_nz(g.wt)), srcs.size,
                           _p(_nz(srcs)), _p(out), nthreads)
    return out


def bellman_ford(kind, g: CSR, s: int) -> np.ndarray:
    out = np.empty(g.n, dtype=np.uint32)
    _load().or_bellman_ford(_kind(kind), g.n, _p(g.ptr), _p(_nz(g.col)), _p(_nz(g.wt)), int(s), _p(out))
    return out


def hubs_topdeg(g: CSR, gr: CSR, K: int) -> np.ndarray:
    hubs = np.empty(K, dtype=np.uint32)
    _load().or_hubs_topdeg(g.n, _p(g.ptr), _p(gr.ptr), K, _p(hubs))
    return hubs


def cg_alg1(kind, g: CSR, gr: CSR, hubs, connectivity: bool = True) -> np.ndarray:
    """Edge flags (u8[m], G's CSR order) of Algorithm 1's Core Graph."""
    hubs = np.ascontiguousarray(hubs, dtype=np.uint32)
    flags = np.zeros(max(g.m, 1), dtype=np.uint8)
    _load().or_cg_alg1(_kind(kind), g.n, _p(g.ptr), _p(_nz(g.col)), _p(_nz(g.wt)), _p(gr.ptr),
                       _p(_nz(gr.col)), _p(_nz(gr.wt)), hubs.size, _p(_nz(hubs)),
                       1 if connectivity else 0, _p(flags))
    return flags[:g.m].copy()


def cg_alg2(g: CSR, gr: CSR, hubs, per_direction: bool = False, connectivity: bool = False) -> np.ndarray:
    """Edge flags (u8[m], G's CSR order) of Algorithm 2's general Core Graph."""
    hubs = np.ascontiguousarray(hubs, dtype=np.uint32)
    flags = np.zeros(max(g.m, 1), dtype=np.uint8)
    _load().or_cg_alg2(g.n, _p(g.ptr), _p(_nz(g.col)), _p(gr.ptr), _p(_nz(gr.col)), hubs.size,
                       _p(_nz(hubs)), 1 if per_direction else 0, 1 if connectivity else 0, _p(flags))
    return flags[:g.m].copy()


def subgraph(g: CSR, flags: np.ndarray) -> CSR:
    flags = np.ascontiguousarray(flags, dtype=np.uint8)
    k = int(flags.sum())
    sptr = np.zeros(g.n + 1, dtype=np.int64)
    scol = np.empty(max(k, 1), dtype=np.uint32)
    swt = np.empty(max(k, 1), dtype=np.uint32)
    _load().or_subgraph(g.n, _p(g.ptr), _p(_nz(g.col)), _p(_nz(g.wt)), _p(_nz(flags)), _p(sptr),
                        _p(scol), _p(swt))
    return CSR(g.n, sptr, scol[:k].copy(), swt[:k].copy())


def _stats_dict(st: _Stats) -> dict:
    return {k: int(getattr(st, k)) for k, _ in _Stats._fields_}


def two_phase(kind, g: CSR, cg: CSR, s: int):
    """Algorithm 3 in sequential BSP order: (final values, phase-1 values, stats dict)."""
    val = np.empty(g.n, dtype=np.uint32)
    p1 = np.empty(g.n, dtype=np.uint32)
    st = _Stats()
    _load().or_2phase(_kind(kind), g.n, _p(g.ptr), _p(_nz(g.col)), _p(_nz(g.wt)), _p(cg.ptr),
                      _p(_nz(cg.col)), _p(_nz(cg.wt)), int(s), _p(val), _p(p1), ctypes.byref(st))
    return val, p1, _stats_dict(st)


def full_bsp(kind, g: CSR, s: int):
    """FULL mode (baseline): Alg 3 init then Process on G until empty: (values, stats)."""
    val = np.empty(g.n, dtype=np.uint32)
    st = _Stats()
    _load().or_full_bsp(_kind(kind), g.n, _p(g.ptr), _p(_nz(g.col)), _p(_nz(g.wt)), int(s), _p(val),
                        ctypes.byref(st))
    return val, _stats_dict(st)


def cg_for_kind(kind, g: CSR, gr: CSR, hubs) -> np.ndarray:
    """The CG each kind uses by default (readings Q12, Q9'): Alg 1 for SSSP/SSWP/SSNP/Viterbi,
    Alg 2 with one Qid[] per traversal direction for BFS/REACH (reading Q9')."""
    k = _kind(kind)
    if k in (KINDS["bfs"], KINDS["reach"]):
        return cg_alg2(g, gr, hubs, per_direction=True)
    return cg_alg1(k, g, gr, hubs)


def as_float(vals: np.ndarray) -> np.ndarray:
    """Viterbi value words -> float32 view."""
    return np.ascontiguousarray(vals, dtype=np.uint32).view(np.float32)


def hub_values(kind, g: CSR, gr: CSR, hubs):
    """The Identify queries' values (Alg 1 l.4-5): (hf, hb) with hf[k] = Q(h_k) on G ("d(h, .)")
    and hb[k] = Q(h_k) on G^R ("d(., h)"), each [K, n] uint32."""
    hf = np.stack([query(kind, g, int(h)) for h in hubs]) if len(hubs) else np.zeros((0, g.n), np.uint32)
    hb = np.stack([query(kind, gr, int(h)) for h in hubs]) if len(hubs) else np.zeros((0, g.n), np.uint32)
    return np.ascontiguousarray(hf, dtype=np.uint32), np.ascontiguousarray(hb, dtype=np.uint32)


def certified(kind, s: int, p1: np.ndarray, hf: np.ndarray, hb: np.ndarray) -> np.ndarray:
    """O7 (NEXT-1): u8[n], 1 where Theorem 1 or its SSWP / SSNP bottleneck analog
    (or REACH's lattice top) proves the phase-1 value p1(v) precise (see oracle.c)."""
    p1 = np.ascontiguousarray(p1, dtype=np.uint32)
    n = p1.size
    out = np.zeros(max(n, 1), dtype=np.uint8)
    _load().or_certified(_kind(kind), n, int(s), _p(_nz(p1)), int(hf.shape[0]), _p(_nz(hf.reshape(-1))),
                         _p(_nz(hb.reshape(-1))), _p(out))
    return out[:n].copy()

"""Independent test helpers: small-graph generators, a numpy canonicaliser and a
pure-Python brute-force path enumerator.  None of this is shared with the
oracle's C code or with the CUDA path; it exists to PIN them.
"""
from __future__ import annotations

import numpy as np

KINDS = ("sssp", "sswp", "ssnp", "viterbi", "bfs", "reach")
INF32 = 0xFFFFFFFF


def np_canonical(n, src, dst, w):
    """Canonical edge set by numpy: drop self-loops, min weight per (u, v), sorted by (u, v).

    Returns (ptr int64[n+1], col u32, wt u32)."""
    src = np.asarray(src, dtype=np.int64)
    dst = np.asarray(dst, dtype=np.int64)
    w = np.asarray(w, dtype=np.int64)
    keep = src != dst
    src, dst, w = src[keep], dst[keep], w[keep]
    order = np.lexsort((w, dst, src))
    src, dst, w = src[order], dst[order], w[order]
    if src.size:
        first = np.ones(src.size, dtype=bool)
        first[1:] = (src[1:] != src[:-1]) | (dst[1:] != dst[:-1])
        src, dst, w = src[first], dst[first], w[first]
    ptr = np.zeros(n + 1, dtype=np.int64)
    np.add.at(ptr, src + 1, 1)
    ptr = np.cumsum(ptr)
    return ptr, dst.astype(np.uint32), w.astype(np.uint32)


def random_multigraph(rng, n, m, wset=(1, 2, 3, 5, 7, 11, 13, 64), self_loops=True):
    src = rng.integers(0, n, size=m).astype(np.uint32)
    dst = rng.integers(0, n, size=m).astype(np.uint32)
    if not self_loops:
        dst = np.where(src == dst, (dst + 1) % n, dst).astype(np.uint32)
    w = rng.choice(np.asarray(wset, dtype=np.uint32), size=m).astype(np.uint32)
    return src, dst, w


def _fold(kind, path_weights):
    """Value at the end of a path: left fold of the kind's (+) from SourceInitVal."""
    if kind == "sssp":
        return sum(int(x) for x in path_weights)
    if kind == "bfs":
        return len(path_weights)
    if kind == "sswp":
        return min([INF32] + [int(x) for x in path_weights])
    if kind == "ssnp":
        return max([0] + [int(x) for x in path_weights])
    if kind == "reach":
        return 1
    if kind == "viterbi":
        v = np.float32(1.0)
        for x in path_weights:
            v = np.float32(v / np.float32(x))
        return v
    raise ValueError(kind)


def brute_force(kind, n, ptr, col, wt, s):
    """Select over ALL simple s->v paths (cycles never improve a monotone (+)) of the fold.

    Returns u32 value words (Viterbi as f32 bit patterns) with the kind's InitVal for
    unreachable vertices and SourceInitVal at s (reading Q1)."""
    is_min = kind in ("sssp", "ssnp", "bfs")
    best = [None] * n
    best[s] = _fold(kind, [])

    def visit(u, on_path, weights):
        for i in range(int(ptr[u]), int(ptr[u + 1])):
            v = int(col[i])
            if v in on_path:
                continue
            ws = weights + [int(wt[i])]
            val = _fold(kind, ws)
            if v != s:
                if best[v] is None or (val < best[v] if is_min else val > best[v]):
                    best[v] = val
            on_path.add(v)
            visit(v, on_path, ws)
            on_path.discard(v)

    visit(s, {s}, [])
    out = np.empty(n, dtype=np.uint32)
    for v in range(n):
        b = best[v]
        if kind == "viterbi":
            f = np.float32(0.0) if b is None else np.float32(b)
            out[v] = np.array([f], dtype=np.float32).view(np.uint32)[0]
        elif b is None:
            out[v] = INF32 if is_min else 0
        else:
            out[v] = int(b)
    # the source: SourceInitVal (Q1)
    out[s] = {"sssp": 0, "ssnp": 0, "bfs": 0, "sswp": INF32, "reach": 1,
              "viterbi": int(np.array([1.0], dtype=np.float32).view(np.uint32)[0])}[kind]
    return out


def rmat_small(scale, ef, seed, w_max=64):
    import gen
    n = 1 << scale
    return (n,) + gen.rmat(n, ef * n, w_max=w_max, seed=seed)

"""Helpers shared by the -m gpu parity tests: build the CUDA-path graph from numpy edges, and
the oracle side from the SAME edges (inputs come only from gen/ or the test itself)."""
import numpy as np
import pytest
import torch

import oracle

requires_cuda = pytest.mark.skipif(not torch.cuda.is_available(), reason="needs a CUDA device")


def dev():
    return torch.device("cuda:0")


def to_dev(a: np.ndarray) -> torch.Tensor:
    return torch.from_numpy(np.ascontiguousarray(a, dtype=np.uint32).view(np.int32)).to(dev())


def to_np(t: torch.Tensor) -> np.ndarray:
    torch.cuda.synchronize()
    if t.dtype == torch.float32:
        t = t.view(torch.int32)
    elif t.dtype == torch.uint32:
        t = t.view(torch.int32)
    return t.cpu().numpy().view(np.uint32)


def gpu_graph(n, src, dst, w):
    from paper_conf_eurosys_0002a0a024_b200 import Graph
    return Graph(n, to_dev(src), to_dev(dst), to_dev(w), device=dev())


def both(n, src, dst, w):
    """(CUDA-path Graph, oracle CSR) for the same raw edge list."""
    return gpu_graph(n, src, dst, w), oracle.canonical_csr(n, src, dst, w)


def assert_values_equal(got: np.ndarray, exp: np.ndarray, kind: str, ctx=""):
    """Bit-exact for the integer kinds; Viterbi: north_star allows 1e-6 relative, the f32
    relaxation is in fact order-independent, so equality is asserted first and the
    tolerance is the documented fallback bound."""
    if kind == "viterbi":
        g = got.view(np.float32)
        e = exp.view(np.float32)
        if not np.array_equal(got, exp):
            assert np.allclose(g, e, rtol=1e-6, atol=0), f"{ctx}: viterbi beyond 1e-6 rel"
            raise AssertionError(f"{ctx}: viterbi within 1e-6 but not bit-exact "
                                 f"({int((got != exp).sum())} vertices)")
    else:
        bad = np.nonzero(got != exp)[0]
        assert bad.size == 0, f"{ctx}: {bad.size} mismatches, first v={bad[:5]} got={got[bad[:5]]} exp={exp[bad[:5]]}"

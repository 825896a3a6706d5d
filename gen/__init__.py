"""Seeded synthetic-input generator (input recipe only; no method arithmetic).

Serves both the CPU oracle (via this host C implementation) and the CUDA
path (which carries an independent device twin of the same counter-based
definition, see ``gen/rmat.c`` for the definition and DESIGN.md "Input
recipe").  Config shapes follow BASELINE.json ``configs`` and SURVEY.md §8(d).
"""
from __future__ import annotations

import ctypes
import math
import os
import subprocess
from dataclasses import dataclass, field

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "rmat.c")
_LIB = os.path.join(_HERE, "libgen.so")
_lib = None


def build(force: bool = False) -> str:
    """Compile gen/rmat.c into gen/libgen.so with gcc (OpenMP)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-fPIC", "-shared", "-std=c11",
                               "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        u32p = ctypes.POINTER(ctypes.c_uint32)
        lib.gen_rmat.argtypes = [ctypes.c_uint64, ctypes.c_uint32, ctypes.c_uint32, ctypes.c_uint32,
                                 ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int, ctypes.c_uint64,
                                 ctypes.c_uint64, u32p, u32p, u32p]
        lib.gen_rmat.restype = None
        lib.gen_scale.argtypes = [ctypes.c_uint64]
        lib.gen_scale.restype = ctypes.c_uint32
        lib.gen_splitmix64.argtypes = [ctypes.c_uint64]
        lib.gen_splitmix64.restype = ctypes.c_uint64
        lib.gen_permute.argtypes = [ctypes.c_uint64, ctypes.c_uint64, ctypes.c_uint64]
        lib.gen_permute.restype = ctypes.c_uint64
        _lib = lib
    return _lib


def thresholds(a: float, b: float, c: float) -> tuple[int, int, int]:
    """Integer quadrant thresholds floor(p * 2^32), clamped to u32."""
    def t(p: float) -> int:
        return max(0, min(0xFFFFFFFF, int(math.floor(p * 4294967296.0))))
    return t(a), t(a + b), t(a + b + c)


def splitmix64(x: int) -> int:
    return int(_load().gen_splitmix64(x & 0xFFFFFFFFFFFFFFFF))


def scale_of(n: int) -> int:
    return int(_load().gen_scale(n))


def rmat(n: int, m: int, abcd=(0.57, 0.19, 0.19, 0.05), w_max: int = 64, seed: int = 1,
         permute: bool = True, e0: int = 0):
    """Edges [e0, e0+m) of the R-MAT stream: (src, dst, w) as uint32 numpy arrays."""
    lib = _load()
    tA, tAB, tABC = thresholds(abcd[0], abcd[1], abcd[2])
    src = np.empty(m, dtype=np.uint32)
    dst = np.empty(m, dtype=np.uint32)
    w = np.empty(m, dtype=np.uint32)
    p = ctypes.POINTER(ctypes.c_uint32)
    if m:
        lib.gen_rmat(n, tA, tAB, tABC, w_max, seed, 1 if permute else 0, e0, m,
                     src.ctypes.data_as(p), dst.ctypes.data_as(p), w.ctypes.data_as(p))
    return src, dst, w


def generator_vertex(cfg, x: int = 0) -> int:
    """Vertex x of the R-MAT generator (before the vertex-id permutation) in the permuted ids of
    `cfg`'s graph.  BASELINE configs[0] queries "vertex 0": in an unpermuted Graph500 R-MAT that is
    the a-quadrant corner, the highest-degree vertex; after the permutation it is
    gen_permute(0) (reading N10).  Id 0 of the permuted graph is an isolated vertex."""
    return int(_load().gen_permute(x, cfg.n, cfg.seed))


def log_weight_max(n: int) -> int:
    """Paper's weight range upper end log(n)+1, read as floor(log2 n)+1."""
    return int(math.floor(math.log2(max(n, 2)))) + 1


@dataclass(frozen=True)
class Config:
    """One synthetic workload of BASELINE.json ``configs``."""
    name: str
    n: int
    m: int
    abcd: tuple = (0.57, 0.19, 0.19, 0.05)
    w_max: int = 64
    seed: int = 1
    note: str = ""
    kinds: tuple = field(default=("sssp",))

    def edges(self):
        return rmat(self.n, self.m, self.abcd, self.w_max, self.seed)


RMAT1 = (0.57, 0.19, 0.19, 0.05)
RMAT2 = (0.67, 0.14, 0.14, 0.05)
ALL_KINDS = ("sssp", "sswp", "ssnp", "viterbi", "bfs", "reach")

CONFIGS = {
    # configs[0]: RMAT scale-16, edgefactor 16, w 1..64, one SSSP query from vertex 0
    "c1": Config("c1-rmat16", 1 << 16, 16 << 16, RMAT1, 64, 1,
                 "RMAT scale-16 ef16, w U{1..64}, seed 1", ("sssp",)),
    # configs[1]: LiveJournal-shaped RMAT, all six kinds (the bench workload)
    "c2": Config("c2-livejournal-rmat", 4_847_571, 68_993_773, RMAT1, log_weight_max(4_847_571), 2,
                 "LiveJournal-shaped RMAT1, w U{1..23}, seed 2", ALL_KINDS),
    # configs[2]: Twitter-shaped (TTW size, Table 3)
    "c3": Config("c3-twitter-rmat", 41_652_231, 1_468_365_182, RMAT1, log_weight_max(41_652_231), 3,
                 "Twitter(TTW)-shaped RMAT1, w U{1..26}, seed 3", ("sssp", "sswp")),
    # configs[3]: Friendster-shaped
    "c4": Config("c4-friendster-rmat", 65_608_366, 1_806_067_135, RMAT1, log_weight_max(65_608_366), 4,
                 "Friendster-shaped RMAT1, w U{1..26}, seed 4", ("bfs", "reach", "viterbi")),
    # configs[4]: UK-domain-shaped, RMAT2 params for web-like skew
    "c5": Config("c5-uk-rmat2", 39_459_925, 936_364_282, RMAT2, log_weight_max(39_459_925), 5,
                 "UK-domain-shaped RMAT2, w U{1..26}, seed 5", ("sssp", "sswp", "reach")),
}


def source_candidates(n: int, src: np.ndarray, dst: np.ndarray) -> np.ndarray:
    """Sorted ids of the vertices with a non-self-loop out-edge in the RAW edge list: exactly the
    vertices with outdeg > 0 after canonicalization, so neither side's CSR is needed."""
    has_out = np.zeros(n, dtype=bool)
    keep = src != dst
    has_out[src[keep]] = True
    return np.nonzero(has_out)[0].astype(np.uint32)


def sample_from(cand: np.ndarray, count: int, seed: int) -> np.ndarray:
    """`count` sources drawn uniformly from `cand`, seeded, distinct when possible."""
    if cand.size == 0:
        return np.zeros(0, dtype=np.uint32)
    rng = np.random.default_rng(seed)
    replace = count > cand.size
    return np.sort(rng.choice(cand, size=count, replace=replace)).astype(np.uint32)


def sample_sources(n: int, src: np.ndarray, dst: np.ndarray, count: int, seed: int) -> np.ndarray:
    """Uniform sources over vertices with outdeg > 0, seeded, distinct when possible."""
    return sample_from(source_candidates(n, src, dst), count, seed)

"""B200-native Core Graph hot path (Jiang et al., EuroSys '24): CSR/CSC builder, on-GPU Core
Graph construction (Alg 1 / Alg 2) and 2Phase push relaxation (Alg 3) for SSSP, SSWP, SSNP,
Viterbi, BFS and REACH, behind the C ABI in include/cg.h.

The CUDA library (csrc/ -> libcoregraph_b200.so) is the only compute path; there is no CPU
fallback.  ``Graph`` marshals tensors to the ABI.
"""
from . import multi  # noqa: F401
from .graph import CG_ALGS, FORMATS, HUB_POLICIES, KINDS, MODES, Graph, kernel_launches, kind_id, rmat_device  # noqa: F401
from ._lib import CGError, CGInvalid, CGNoCoreGraph, CGOverflow, CGUnsupported  # noqa: F401

__all__ = ["Graph", "rmat_device", "KINDS", "MODES", "FORMATS", "HUB_POLICIES", "CG_ALGS", "kernel_launches", "kind_id",
           "CGError", "CGInvalid", "CGNoCoreGraph", "CGOverflow", "CGUnsupported"]

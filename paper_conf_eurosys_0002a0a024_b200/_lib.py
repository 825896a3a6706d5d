"""ctypes binding of include/cg.h (argument marshalling only).

Every function of the C ABI is declared here with the same name; PyTorch is used only to
own device memory (its caching allocator is installed as the library's allocator) and to
provide the CUDA stream handle.  There is no CPU fallback: if the shared library is
missing and cannot be built, importing this module raises.
"""
from __future__ import annotations

import ctypes
import os
import re

from . import _build

HERE = os.path.dirname(os.path.abspath(__file__))
HEADER = os.path.join(os.path.dirname(HERE), "include", "cg.h")

STATUS = {0: "CG_OK", -1: "CG_EINVAL", -2: "CG_ENOMEM", -3: "CG_ECUDA", -4: "CG_ENOCG",
          -5: "CG_EOVERFLOW", -7: "CG_EUNSUPPORTED", -8: "CG_EINTERNAL"}


class CGError(RuntimeError):
    def __init__(self, code: int, func: str, detail: str):
        self.code = code
        self.status = STATUS.get(code, str(code))
        super().__init__(f"{func}: {self.status}: {detail}")


class CGInvalid(CGError, ValueError):
    pass


class CGNoCoreGraph(CGError):
    pass


class CGOverflow(CGError, OverflowError):
    pass


class CGUnsupported(CGError):
    pass


_EXC = {-1: CGInvalid, -4: CGNoCoreGraph, -5: CGOverflow, -7: CGUnsupported}


class Stats(ctypes.Structure):
    _fields_ = [("iters_p1", ctypes.c_int64), ("iters_p2", ctypes.c_int64),
                ("edges_p1", ctypes.c_int64), ("edges_p2", ctypes.c_int64),
                ("updates_p1", ctypes.c_int64), ("updates_p2", ctypes.c_int64),
                ("frontier_p1", ctypes.c_int64), ("frontier_p2", ctypes.c_int64),
                ("impacted", ctypes.c_int64), ("reached", ctypes.c_int64),
                ("precise_p1", ctypes.c_int64),
                ("scanned_p1", ctypes.c_int64), ("scanned_p2", ctypes.c_int64),
                ("batch_queries", ctypes.c_int32), ("row_bytes", ctypes.c_int32),
                ("ms_p1", ctypes.c_float), ("ms_p2", ctypes.c_float)]

    def as_dict(self) -> dict:
        return {k: (float(getattr(self, k)) if k.startswith("ms_") else int(getattr(self, k)))
                for k, _ in self._fields_}


ALLOC_FN = ctypes.CFUNCTYPE(ctypes.c_void_p, ctypes.c_size_t, ctypes.c_void_p, ctypes.c_void_p)
FREE_FN = ctypes.CFUNCTYPE(None, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p)

_P = ctypes.c_void_p
_SIGS = {
    "cg_set_allocator": (ctypes.c_int, [ALLOC_FN, FREE_FN, _P]),
    "cg_graph_create": (ctypes.c_int, [ctypes.c_int, ctypes.c_int64, ctypes.c_int64, _P, _P, _P, _P,
                                       ctypes.POINTER(_P)]),
    "cg_graph_destroy": (ctypes.c_int, [_P]),
    "cg_graph_info": (ctypes.c_int, [_P, ctypes.POINTER(ctypes.c_int64), ctypes.POINTER(ctypes.c_int64),
                                     ctypes.POINTER(ctypes.c_uint32)]),
    "cg_graph_export": (ctypes.c_int, [_P, ctypes.c_int, _P, _P, _P, _P]),
    "cg_build": (ctypes.c_int, [_P, ctypes.c_int, ctypes.c_int32, ctypes.c_int, _P, ctypes.c_uint64, _P]),
    "cg_build_ex": (ctypes.c_int, [_P, ctypes.c_int, ctypes.c_int32, ctypes.c_int, _P, ctypes.c_uint64,
                                   ctypes.c_int, ctypes.c_int32, _P]),
    "cg_core_info": (ctypes.c_int, [_P, ctypes.c_int, ctypes.POINTER(ctypes.c_int64),
                                    ctypes.POINTER(ctypes.c_int32), _P, ctypes.POINTER(ctypes.c_float)]),
    "cg_core_export": (ctypes.c_int, [_P, ctypes.c_int, _P, _P]),
    "cg_build_partial": (ctypes.c_int, [_P, ctypes.c_int, ctypes.c_int32, ctypes.c_int, _P, ctypes.c_uint64,
                                        ctypes.c_int32, ctypes.c_int32, _P, _P]),
    "cg_build_from_flags": (ctypes.c_int, [_P, ctypes.c_int, ctypes.c_int32, ctypes.c_int, _P, ctypes.c_uint64,
                                           _P, ctypes.c_int32, _P]),
    "cg_core_save": (ctypes.c_int, [_P, ctypes.c_int, ctypes.c_char_p, _P]),
    "cg_core_load": (ctypes.c_int, [_P, ctypes.c_int, ctypes.c_char_p, _P]),
    "cg_query": (ctypes.c_int, [_P, ctypes.c_int, _P, ctypes.c_int32, ctypes.c_int, _P, _P, _P]),
    "cg_query_ex": (ctypes.c_int, [_P, ctypes.c_int, _P, ctypes.c_int32, ctypes.c_int, _P, _P, _P, _P]),
    "cg_query_fmt": (ctypes.c_int, [_P, ctypes.c_int, _P, ctypes.c_int32, ctypes.c_int, ctypes.c_int, _P, _P, _P,
                                    _P]),
    "cg_graph_status": (ctypes.c_int, [_P, _P]),
    "cg_query_host": (ctypes.c_int, [_P, ctypes.c_int, _P, ctypes.c_int32, ctypes.c_int, _P, ctypes.c_int32, _P]),
    "cg_query_host_fmt": (ctypes.c_int, [_P, ctypes.c_int, _P, ctypes.c_int32, ctypes.c_int, ctypes.c_int, _P,
                                         ctypes.c_int32, _P]),
    "cg_query_host_async": (ctypes.c_int, [_P, ctypes.c_int, _P, ctypes.c_int32, ctypes.c_int, ctypes.c_int, _P,
                                         ctypes.c_int32, _P]),
    "cg_rmat_generate": (ctypes.c_int, [ctypes.c_uint64, ctypes.c_uint32, ctypes.c_uint32, ctypes.c_uint32,
                                        ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int32, ctypes.c_uint64,
                                        ctypes.c_uint64, _P, _P, _P, _P]),
    "cg_kernel_launches": (ctypes.c_int64, []),
    "cg_status_string": (ctypes.c_char_p, [ctypes.c_int]),
    "cg_last_error": (ctypes.c_char_p, []),
}


def header_functions() -> list[str]:
    """Function names declared in include/cg.h (the ABI surface)."""
    with open(HEADER) as f:
        text = re.sub(r"/\*.*?\*/", "", f.read(), flags=re.S)
    return sorted(set(re.findall(r"\b(cg_[a-z_0-9]+)\s*\(", text)) - {"cg_alloc_fn", "cg_free_fn"})


_lib = None


def lib(build: bool = True) -> ctypes.CDLL:
    """Load (building first if stale) the CUDA library.  Raises if it cannot be produced."""
    global _lib
    if _lib is None:
        path = os.environ.get("CGB_LIB")  # an experiment variant built by _build.build(out=...)
        if not path:
            if build:
                _build.build()
            path = _build.LIB
        if not os.path.exists(path):
            raise ImportError(f"CUDA library {path} is missing (no CPU fallback exists)")
        L = ctypes.CDLL(path)
        for name, (res, args) in _SIGS.items():
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        _lib = L
    return _lib


def check(code: int, func: str) -> None:
    if code != 0:
        detail = (lib().cg_last_error() or b"").decode(errors="replace")
        raise _EXC.get(code, CGError)(code, func, detail)


def call(name: str, *args) -> None:
    check(getattr(lib(), name)(*args), name)


# ------------------------------------------------------------------ torch allocator plumbing
_alloc_keep = []


def install_torch_allocator() -> None:
    """Route the library's device allocations through PyTorch's caching allocator."""
    if _alloc_keep:
        return
    import torch

    def _alloc(nbytes, stream, ctx):
        try:
            dev = torch.cuda.current_device()
            return torch.cuda.caching_allocator_alloc(int(nbytes), dev, int(stream or 0))
        except Exception:  # noqa: BLE001 - the C side turns NULL into CG_ENOMEM
            return None

    def _free(ptr, stream, ctx):
        try:
            torch.cuda.caching_allocator_delete(int(ptr))
        except Exception:  # noqa: BLE001
            pass

    a, f = ALLOC_FN(_alloc), FREE_FN(_free)
    _alloc_keep.extend([a, f])
    call("cg_set_allocator", a, f, None)

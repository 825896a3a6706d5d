"""Python face of the C ABI (include/cg.h): ``Graph`` built on a CUDA device, Core Graph
construction and 2Phase / full-graph queries.  Marshalling only — every step runs in the
library's CUDA kernels; tensors are PyTorch-owned device (or pinned host) memory.
"""
from __future__ import annotations

import ctypes
import math

import torch

from . import _lib

KINDS = {"sssp": 0, "sswp": 1, "ssnp": 2, "viterbi": 3, "bfs": 4, "reach": 5, "wcc": 6}
MODES = {"2phase": 0, "full": 1}
HUB_POLICIES = {"topdeg": 0, "sampled": 1, "given": 2}
CG_ALGS = {"auto": 0, "specialized": 1, "general": 2, "general_perdir": 3}
FORMATS = {"u32": 0, "u16": 1, "bits": 2}  # cg_out_format


def kind_id(kind) -> int:
    if isinstance(kind, str):
        if kind not in KINDS:
            raise ValueError(f"unknown kind {kind!r}; one of {sorted(KINDS)}")
        return KINDS[kind]
    return int(kind)


def _ptr(t) -> ctypes.c_void_p:
    return ctypes.c_void_p(t.data_ptr() if t is not None and t.numel() else 0)


def _stream(device) -> ctypes.c_void_p:
    return ctypes.c_void_p(torch.cuda.current_stream(device).cuda_stream)


def _u32(t: torch.Tensor, device) -> torch.Tensor:
    """Reinterpret/convert an integer tensor to a contiguous uint32 tensor on `device`."""
    if not isinstance(t, torch.Tensor):
        t = torch.as_tensor(t)
    if t.dtype in (torch.int32, torch.uint32):
        t = t.view(torch.uint32) if t.dtype == torch.int32 else t
    else:
        t = t.to(torch.int64).to(torch.uint32) if t.dtype != torch.uint32 else t
    return t.to(device).contiguous()


def rmat_device(n: int, m: int, abcd=(0.57, 0.19, 0.19, 0.05), w_max: int = 64, seed: int = 1,
                permute: bool = True, device=None, e0: int = 0):
    """Draw the seeded R-MAT edge list (gen/rmat.c recipe) directly in HBM via the device twin."""
    device = torch.device(device or "cuda")
    _lib.install_torch_allocator()

    def t(p):
        return max(0, min(0xFFFFFFFF, int(math.floor(p * 4294967296.0))))
    tA, tAB, tABC = t(abcd[0]), t(abcd[0] + abcd[1]), t(abcd[0] + abcd[1] + abcd[2])
    src = torch.empty(m, dtype=torch.uint32, device=device)
    dst = torch.empty(m, dtype=torch.uint32, device=device)
    w = torch.empty(m, dtype=torch.uint32, device=device)
    with torch.cuda.device(device):
        _lib.call("cg_rmat_generate", n, tA, tAB, tABC, w_max, seed, 1 if permute else 0, e0, m,
                  _ptr(src), _ptr(dst), _ptr(w), _stream(device))
    return src, dst, w


class Graph:
    """G(V,E) on one CUDA device with its Core Graphs (cg_graph_create / cg_build / cg_query)."""

    def __init__(self, n: int, src, dst, w, device=None):
        self.device = torch.device(device or (src.device if isinstance(src, torch.Tensor) and src.is_cuda
                                              else "cuda"))
        if self.device.index is None:
            self.device = torch.device("cuda", torch.cuda.current_device())
        _lib.install_torch_allocator()
        src, dst, w = (_u32(x, self.device) for x in (src, dst, w))
        if not (src.numel() == dst.numel() == w.numel()):
            raise ValueError("src, dst, w must have the same length")
        h = ctypes.c_void_p()
        with torch.cuda.device(self.device):
            _lib.call("cg_graph_create", self.device.index, int(n), src.numel(), _ptr(src), _ptr(dst), _ptr(w),
                      _stream(self.device), ctypes.byref(h))
        self._h = h
        nn, mm, wm = ctypes.c_int64(), ctypes.c_int64(), ctypes.c_uint32()
        _lib.call("cg_graph_info", self._h, ctypes.byref(nn), ctypes.byref(mm), ctypes.byref(wm))
        self.n, self.m, self.w_max = nn.value, mm.value, wm.value

    @classmethod
    def rmat(cls, n: int, m: int, abcd=(0.57, 0.19, 0.19, 0.05), w_max: int = 64, seed: int = 1,
             device=None) -> "Graph":
        src, dst, w = rmat_device(n, m, abcd, w_max, seed, True, device)
        g = cls(n, src, dst, w, device=src.device)
        del src, dst, w
        return g

    # -------------------------------------------------------------- lifetime
    def close(self) -> None:
        h, self._h = getattr(self, "_h", None), None
        if h:
            with torch.cuda.device(self.device):
                _lib.call("cg_graph_destroy", h)

    def __del__(self):
        try:
            self.close()
        except Exception:  # noqa: BLE001 - interpreter shutdown
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    # -------------------------------------------------------------- graph
    def export(self, transpose: bool = False, ptr_only: bool = False):
        """(ptr int64[n+1], idx uint32[m], w uint32[m]) of the canonical CSR (or CSC); with
        ptr_only the edge arrays are not copied (returned as None)."""
        ptr = torch.empty(self.n + 1, dtype=torch.int64, device=self.device)
        idx = None if ptr_only else torch.empty(self.m, dtype=torch.uint32, device=self.device)
        w = None if ptr_only else torch.empty(self.m, dtype=torch.uint32, device=self.device)
        with torch.cuda.device(self.device):
            _lib.call("cg_graph_export", self._h, 1 if transpose else 0, _ptr(ptr), _ptr(idx), _ptr(w),
                      _stream(self.device))
        return ptr, idx, w

    # -------------------------------------------------------------- core graph
    def build(self, kind, K: int = 20, policy: str = "topdeg", hubs=None, seed: int = 0, alg: str = "auto",
              connectivity: bool | None = None) -> dict:
        """cg_build_ex: Core Graph for `kind`; returns core_info(kind)."""
        pol = HUB_POLICIES[policy]
        harr = None
        if hubs is not None:
            pol = HUB_POLICIES["given"]
            hl = [int(x) for x in hubs]
            K = len(hl)
            harr = (ctypes.c_uint32 * K)(*hl)
        conn = -1 if connectivity is None else (1 if connectivity else 0)
        with torch.cuda.device(self.device):
            _lib.call("cg_build_ex", self._h, kind_id(kind), int(K), pol,
                      ctypes.cast(harr, ctypes.c_void_p) if harr is not None else None,
                      int(seed), CG_ALGS[alg], conn, _stream(self.device))
        return self.core_info(kind)

    @staticmethod
    def _hubs_arg(K, policy, hubs):
        pol = HUB_POLICIES[policy]
        harr = None
        if hubs is not None:
            pol = HUB_POLICIES["given"]
            hl = [int(x) for x in hubs]
            K = len(hl)
            harr = (ctypes.c_uint32 * K)(*hl)
        return K, pol, (ctypes.cast(harr, ctypes.c_void_p) if harr is not None else None), harr

    def build_partial(self, kind, K: int = 20, hub_range=(0, None), policy: str = "topdeg", hubs=None,
                      seed: int = 0) -> torch.Tensor:
        """cg_build_partial (NEXT-4): Algorithm 1 edge flags (uint8[m], G's CSR order) of the hubs
        hub_range = [begin, end) of the K hubs the policy selects."""
        K, pol, hp, _keep = self._hubs_arg(K, policy, hubs)
        b, e = hub_range
        e = K if e is None else e
        flags = torch.empty(max(self.m, 1), dtype=torch.uint8, device=self.device)
        with torch.cuda.device(self.device):
            _lib.call("cg_build_partial", self._h, kind_id(kind), int(K), pol, hp, int(seed), int(b), int(e),
                      _ptr(flags), _stream(self.device))
        return flags[:self.m]

    def build_from_flags(self, kind, flags: torch.Tensor, K: int = 20, policy: str = "topdeg", hubs=None,
                         seed: int = 0, connectivity: bool | None = None) -> dict:
        """cg_build_from_flags (NEXT-4): install merged Algorithm 1 flags as the kind's CG."""
        K, pol, hp, _keep = self._hubs_arg(K, policy, hubs)
        flags = flags.to(self.device, torch.uint8).contiguous()
        conn = -1 if connectivity is None else (1 if connectivity else 0)
        with torch.cuda.device(self.device):
            _lib.call("cg_build_from_flags", self._h, kind_id(kind), int(K), pol, hp, int(seed), _ptr(flags), conn,
                      _stream(self.device))
        return self.core_info(kind)

    def save_core(self, kind, path: str) -> None:
        """cg_core_save (NEXT-4): write the kind's Core Graph to a host file."""
        with torch.cuda.device(self.device):
            _lib.call("cg_core_save", self._h, kind_id(kind), str(path).encode(), _stream(self.device))

    def load_core(self, kind, path: str) -> dict:
        """cg_core_load (NEXT-4): install a saved Core Graph (same graph required)."""
        with torch.cuda.device(self.device):
            _lib.call("cg_core_load", self._h, kind_id(kind), str(path).encode(), _stream(self.device))
        return self.core_info(kind)

    def core_info(self, kind) -> dict:
        m_cg, K, ms = ctypes.c_int64(), ctypes.c_int32(), ctypes.c_float()
        _lib.call("cg_core_info", self._h, kind_id(kind), ctypes.byref(m_cg), ctypes.byref(K), None,
                  ctypes.byref(ms))
        hubs = (ctypes.c_uint32 * max(K.value, 1))()
        _lib.call("cg_core_info", self._h, kind_id(kind), None, None, ctypes.cast(hubs, ctypes.c_void_p), None)
        return {"m_cg": m_cg.value, "K": K.value, "hubs": list(hubs)[:K.value], "build_ms": ms.value,
                "edge_fraction": m_cg.value / self.m if self.m else 0.0}

    def core_flags(self, kind) -> torch.Tensor:
        flags = torch.empty(self.m, dtype=torch.uint8, device=self.device)
        with torch.cuda.device(self.device):
            _lib.call("cg_core_export", self._h, kind_id(kind), _ptr(flags), _stream(self.device))
        return flags

    # -------------------------------------------------------------- queries
    def row_shape(self, fmt: str = "u32") -> tuple:
        """(elements, dtype) of one output row in cg_out_format `fmt`."""
        if fmt == "u16":
            return self.n, torch.uint16
        if fmt == "bits":
            return (self.n + 31) // 32, torch.uint32
        return self.n, torch.uint32

    def query(self, kind, sources, mode: str = "2phase", out: torch.Tensor | None = None,
              p1: torch.Tensor | bool | None = None, stats: bool = False, fmt: str = "u32"):
        """Evaluate Q(s) for every s in `sources`; returns uint32 [n_src, n] (float32 view for Viterbi).

        fmt: "u32" (default), "u16" (uint16 rows, 0xFFFFFFFF as 0xFFFF) or "bits" (REACH: bit-packed
        uint32 rows) — cg_out_format.  p1=True (or a uint32 [n_src, n] tensor) also returns the
        phase-1 values (2phase only).  stats=True returns per-query counters (synchronises)."""
        k = kind_id(kind)
        if k == KINDS["wcc"] and sources is None:  # whole-graph query: one row of labels
            sources = [0]
        src = _u32(sources, self.device).reshape(-1)
        ns = src.numel()
        if out is None:
            cols, dt = self.row_shape(fmt)
            out = torch.empty((ns, cols), dtype=dt, device=self.device)
        if p1 is True:
            p1 = torch.empty((ns, self.n), dtype=torch.uint32, device=self.device)
        st = (_lib.Stats * max(ns, 1))() if stats else None
        with torch.cuda.device(self.device):
            _lib.call("cg_query_fmt", self._h, k, _ptr(src), ns, MODES[mode], FORMATS[fmt], _ptr(out),
                      _ptr(p1) if isinstance(p1, torch.Tensor) else None,
                      ctypes.cast(st, ctypes.c_void_p) if st is not None else None, _stream(self.device))
        res = out.view(torch.float32) if (k == KINDS["viterbi"] and fmt == "u32") else out
        extra = []
        if isinstance(p1, torch.Tensor):
            extra.append(p1.view(torch.float32) if k == KINDS["viterbi"] else p1)
        if stats:
            extra.append([st[i].as_dict() for i in range(ns)])
        return (res, *extra) if extra else res

    def query_host(self, kind, sources, mode: str = "2phase", out: torch.Tensor | None = None,
                   batch: int = 0, fmt: str = "u32", sync: bool = True) -> torch.Tensor:
        """cg_query_host_fmt: host sources in, host (pinned) values out in `fmt`, copies overlapped
        with compute.  sync=False: cg_query_host_async — out (pinned) is complete after
        `self.status()` (cg_graph_status); keep it alive until then (the sources are staged)."""
        k = kind_id(kind)
        src = sources if isinstance(sources, torch.Tensor) else torch.as_tensor(sources)
        src = src.to(torch.int64).to(torch.uint32).contiguous().cpu()
        ns = src.numel()
        if out is None:
            cols, dt = self.row_shape(fmt)
            out = torch.empty((ns, cols), dtype=dt, pin_memory=True)
        with torch.cuda.device(self.device):
            _lib.call("cg_query_host_fmt" if sync else "cg_query_host_async", self._h, k, _ptr(src), ns, MODES[mode],
                      FORMATS[fmt], _ptr(out), int(batch), _stream(self.device))

        return out.view(torch.float32) if (k == KINDS["viterbi"] and fmt == "u32") else out

    def status(self) -> None:
        """cg_graph_status: synchronise and raise the graph's pending sticky device error, if any."""
        with torch.cuda.device(self.device):
            _lib.call("cg_graph_status", self._h, _stream(self.device))


def kernel_launches() -> int:
    return int(_lib.lib().cg_kernel_launches())

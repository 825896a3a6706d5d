#!/usr/bin/env python
"""Workload for compute-sanitizer (memcheck / racecheck / synccheck / initcheck): every kernel of
the library on a C1-sized RMAT graph (2^16 vertices, 2^20 edges) — graph build, all Core Graph
constructions (Alg 1, Alg 2, partial + merge), every kind in FULL and 2PHASE through both engines
(batched: binary16 / u32 / bit / label lanes; single-query), narrow outputs, the host path, and
the certificate pull (NEXT-1).  Results are checked against the oracle so a silent corruption
under the sanitizer also fails.

    compute-sanitizer --tool memcheck --kernel-name regex:'^(?!.*(at::|cub|elementwise|vectorized))' \
        python tools/sanitize_run.py
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import numpy as np
    import torch

    import gen
    import oracle
    from paper_conf_eurosys_0002a0a024_b200 import Graph

    scale = int(os.environ.get("SAN_SCALE", "16"))
    n, m = 1 << scale, 16 << scale
    src, dst, w = gen.rmat(n, m, w_max=64, seed=1)
    dev = torch.device("cuda:0")
    t = lambda a: torch.from_numpy(np.ascontiguousarray(a, np.uint32).view(np.int32)).to(dev)  # noqa: E731
    g = Graph(n, t(src), t(dst), t(w), device=dev)
    og = oracle.canonical_csr(n, src, dst, w)
    sources = gen.sample_sources(n, src, dst, 40, seed=7)
    bad = 0
    for kind in ("sssp", "sswp", "ssnp", "viterbi", "bfs", "reach"):
        g.build(kind, K=20)
        exp = oracle.query_batch(kind, og, sources[:3])
        for mode in ("full", "2phase"):
            out = g.query(kind, t(sources), mode=mode)
            one = g.query(kind, t(sources[:1]), mode=mode)  # single-query engine
            torch.cuda.synchronize()
            o = out.view(torch.int32).cpu().numpy().view(np.uint32)
            bad += int((o[:3] != exp).sum()) + int((one.view(torch.int32).cpu().numpy().view(np.uint32)[0] != exp[0]).sum())
        _, p1, st = g.query(kind, t(sources), mode="2phase", p1=True, stats=True)
        if kind != "viterbi":
            g.query(kind, t(sources), mode="2phase", fmt="u16" if kind != "reach" else "bits")
        g.query_host(kind, sources[:5], mode="2phase")
    os.environ["CG_REDUCED"] = "7"   # certificate pull for SSSP / SSWP / SSNP in u32 lanes too
    os.environ["CG_LANES"] = "32"
    for kind in ("sssp", "sswp", "ssnp", "reach"):
        g.build(kind, K=20)
        out = g.query(kind, t(sources), mode="2phase")
        torch.cuda.synchronize()
        bad += int((out.view(torch.int32).cpu().numpy().view(np.uint32)[:3] != oracle.query_batch(kind, og, sources[:3])).sum())
    del os.environ["CG_REDUCED"], os.environ["CG_LANES"]
    wcc = g.query("wcc", None, mode="2phase")
    g.query("wcc", None, mode="full")
    f = g.build_partial("sswp", K=20, hub_range=(0, 10))
    f2 = g.build_partial("sswp", K=20, hub_range=(10, 20))
    g.build_from_flags("sswp", torch.maximum(f, f2), K=20)
    g.status()
    torch.cuda.synchronize()
    bad += int((wcc.view(torch.int32).cpu().numpy().view(np.uint32)[0] != oracle.wcc(og)).sum())
    g.close()
    print("sanitize workload done, mismatches:", bad)
    sys.exit(1 if bad else 0)


if __name__ == "__main__":
    main()

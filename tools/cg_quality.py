#!/usr/bin/env python
"""CG quality on a config: edge fraction, phase-1 precision, 2Phase vs FULL edges and time, for
chosen CG algorithms / hub policies / hub counts — the Table 4 (CG %E), Table 5 (precision) and
Fig 3 / Table 13 (K) analogs; BASELINE.json configs[4] is the K sweep on C5:

    python tools/cg_quality.py --config c5 --kinds sssp,sswp,reach --K 5,10,20,40,60,80,100 \
        --policy topdeg,sampled --sources 10 > profiles/r1_ksweep_c5.jsonl

End-to-end speedup = FULL ms / 2Phase ms for the same batch of sources (one cg_query call each,
CUDA events, median of --reps after one warm-up); build_ms is the Core Graph build (a3-a7)."""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    p = argparse.ArgumentParser()
    p.add_argument("--config", default="c2")
    p.add_argument("--kinds", default="sssp,sswp,ssnp,viterbi,bfs,reach")
    p.add_argument("--algs", default="auto")
    p.add_argument("--K", default="20")
    p.add_argument("--policy", default="topdeg")
    p.add_argument("--sources", type=int, default=16)
    p.add_argument("--reps", type=int, default=3)
    a = p.parse_args()
    import numpy as np
    import torch

    import gen
    from paper_conf_eurosys_0002a0a024_b200 import Graph
    cfg = gen.CONFIGS[a.config]
    from paper_conf_eurosys_0002a0a024_b200 import rmat_device
    src_d, dst_d, w_d = rmat_device(cfg.n, cfg.m, cfg.abcd, cfg.w_max, cfg.seed, True, "cuda:0")
    has = torch.zeros(cfg.n, dtype=torch.bool, device="cuda:0")
    keep = src_d.view(torch.int32) != dst_d.view(torch.int32)
    has[src_d.view(torch.int32)[keep].to(torch.int64)] = True
    cand = torch.nonzero(has).flatten().cpu().numpy().astype(np.uint32)
    g = Graph(cfg.n, src_d, dst_d, w_d, device="cuda:0")
    del src_d, dst_d, w_d
    for K in [int(x) for x in a.K.split(",")]:
        for policy in a.policy.split(","):
            for alg in a.algs.split(","):
                for kind in a.kinds.split(","):
                    info = g.build(kind, K=K, policy=policy, alg=alg, seed=7)
                    srcs = torch.from_numpy(gen.sample_from(cand, a.sources, seed=99).astype(np.int64)).to(torch.uint32)
                    out, p1, st = g.query(kind, srcs, mode="2phase", p1=True, stats=True)
                    _, stf = g.query(kind, srcs, mode="full", stats=True)
                    reached = sum(x["reached"] for x in st)
                    prec = sum(x["precise_p1"] for x in st)
                    e2 = sum(x["edges_p1"] + x["edges_p2"] for x in st)
                    ef = sum(x["edges_p2"] for x in stf)

                    def timed(mode):
                        g.query(kind, srcs, mode=mode)
                        ts = []
                        for _ in range(a.reps):
                            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                            torch.cuda.synchronize()
                            e0.record()
                            g.query(kind, srcs, mode=mode)
                            e1.record()
                            torch.cuda.synchronize()
                            ts.append(e0.elapsed_time(e1))
                        return sorted(ts)[len(ts) // 2]
                    ms2, msf = timed("2phase"), timed("full")
                    per_q = [round(100 * x["precise_p1"] / x["reached"], 2) if x["reached"] else 100.0 for x in st]
                    print(json.dumps({"config": cfg.name, "kind": kind, "alg": alg, "K": K, "policy": policy,
                                      "cg_edge_pct": round(100 * info["edge_fraction"], 3),
                                      "p1_precision_pct": round(100 * prec / max(reached, 1), 3),
                                      "min_query_precision_pct": min(per_q), "edges_2phase_over_full": round(e2 / max(ef, 1), 3),
                                      "build_ms": round(info["build_ms"], 1), "n_sources": len(srcs),
                                      "ms_2phase": round(ms2, 3), "ms_full": round(msf, 3),
                                      "speedup_2phase_vs_full": round(msf / ms2, 3)}), flush=True)


if __name__ == "__main__":
    main()

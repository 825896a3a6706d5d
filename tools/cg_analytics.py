#!/usr/bin/env python
"""Core Graph analytics (analogs of the paper's Fig 3, Table 1, Fig 9 and
Table 17 on a synthetic config), from the library's own exports — no new kernels:

* growth   (Fig 3): CG edges (before connectivity edges) after the Identify queries
             of the first k hubs, k = 1..K (Algorithm 1 kinds, cg_build_partial per hub);
* sharing  (Table 1): average number of hubs (of K; forward + backward Identify
             queries) whose tight-edge sets contain a CG edge;
* degrees  (Fig 9): log2-binned out-degree histograms of G and of the CG;
* overlap  (Table 17): |top-t by degree in G ∩ top-t by degree in CG| for
             t = 1,000 / 10,000 / 100,000.

    python tools/cg_analytics.py --config c2 --kinds sssp,reach > profiles/r1_cg_analytics_c2.json
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    p = argparse.ArgumentParser()
    p.add_argument("--config", default="c2")
    p.add_argument("--kinds", default="sssp,sswp,reach")
    p.add_argument("--K", type=int, default=20)
    a = p.parse_args()
    import torch

    import gen
    from paper_conf_eurosys_0002a0a024_b200 import Graph

    cfg = gen.CONFIGS[a.config]
    dev = torch.device("cuda:0")
    g = Graph.rmat(cfg.n, cfg.m, cfg.abcd, cfg.w_max, cfg.seed, device=dev)
    ptr = g.export(ptr_only=True)[0]
    rptr = g.export(transpose=True, ptr_only=True)[0]
    deg_g = (ptr[1:] - ptr[:-1]) + (rptr[1:] - rptr[:-1])  # total degree (reading Q7)
    outdeg_g = ptr[1:] - ptr[:-1]
    row_of_edge = torch.repeat_interleave(torch.arange(g.n, device=dev), outdeg_g)
    _, col, _ = g.export()
    col = col.to(torch.int64)

    def hist(d):
        d = d.to(torch.int64)
        b = torch.where(d > 0, torch.floor(torch.log2(d.clamp(min=1).double())).to(torch.int64) + 1, 0)
        h = torch.bincount(b)
        return {("0" if i == 0 else f"[{2 ** (i - 1)},{2 ** i})"): int(c) for i, c in enumerate(h.tolist()) if c}

    res = {"config": cfg.name, "n": g.n, "m": g.m, "K": a.K, "kinds": {}}
    for kind in a.kinds.split(","):
        info = g.build(kind, K=a.K)
        flags = g.core_flags(kind).to(torch.bool)
        out = {"m_cg": info["m_cg"], "edge_pct": 100.0 * info["m_cg"] / g.m, "build_ms": info["build_ms"]}
        if kind in ("sssp", "sswp", "ssnp", "viterbi"):
            cum = torch.zeros(g.m, dtype=torch.bool, device=dev)
            count = torch.zeros(g.m, dtype=torch.int32, device=dev)
            growth = []
            for k in range(a.K):
                f = g.build_partial(kind, K=a.K, hub_range=(k, k + 1)).to(torch.bool)
                cum |= f
                count += f.to(torch.int32)
                growth.append(int(cum.sum().item()))
            g.build(kind, K=a.K)  # reinstall the full CG (partial builds do not replace it)
            out["growth_edges_after_k_hubs"] = growth
            tight = flags & (count > 0)  # CG edges chosen by some hub (not only a connectivity edge)
            out["avg_hubs_selecting_a_cg_edge"] = float(count[tight].double().mean().item()) if tight.any() else 0.0
            out["connectivity_edges"] = int((flags & (count == 0)).sum().item())
        cg_out = torch.bincount(row_of_edge[flags], minlength=g.n)
        cg_in = torch.bincount(col[flags], minlength=g.n)
        deg_cg = cg_out + cg_in
        out["outdeg_hist_G"] = hist(outdeg_g)
        out["outdeg_hist_CG"] = hist(cg_out)
        overlap = {}
        for t in (1000, 10000, 100000):
            t = min(t, g.n)
            # ties to the smaller id (reading Q7): sort by (-degree, id)
            key_g = deg_g.to(torch.int64) * (g.n + 1) + (g.n - torch.arange(g.n, device=dev))
            key_c = deg_cg.to(torch.int64) * (g.n + 1) + (g.n - torch.arange(g.n, device=dev))
            tg = torch.topk(key_g, t).indices
            tc = torch.topk(key_c, t).indices
            overlap[str(t)] = int(torch.isin(tg, tc).sum().item())
        out["top_degree_overlap"] = overlap
        res["kinds"][kind] = out
    print(json.dumps(res))


if __name__ == "__main__":
    main()

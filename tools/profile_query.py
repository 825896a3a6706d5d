#!/usr/bin/env python
"""One query-kernel launch inside an NVTX range "prof", for ncu:

    ncu --set full --nvtx --nvtx-include "prof/" --clock-control none --import-source on \
        -o gpurun_out/prof python tools/profile_query.py --config c2 --kind sssp --mode 2phase
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    p = argparse.ArgumentParser()
    p.add_argument("--config", default="c2")
    p.add_argument("--kind", default="sssp")
    p.add_argument("--mode", default="2phase")
    p.add_argument("--batch", type=int, default=32)
    p.add_argument("--repeat", type=int, default=1)
    p.add_argument("--fmt", default="u32", help="output rows: u32 / u16 / bits (cg_out_format)")
    a = p.parse_args()
    import numpy as np
    import torch

    import gen
    from paper_conf_eurosys_0002a0a024_b200 import Graph

    cfg = gen.CONFIGS[a.config]
    g = Graph.rmat(cfg.n, cfg.m, cfg.abcd, cfg.w_max, cfg.seed, device="cuda:0")
    if a.mode == "2phase":
        g.build(a.kind, K=20)
    ptr, _, _ = g.export()
    deg = (ptr[1:] - ptr[:-1]).cpu().numpy()
    rng = np.random.default_rng(1000)
    srcs = torch.from_numpy(rng.choice(np.nonzero(deg > 0)[0], size=a.batch).astype(np.int64)).to(torch.uint32).cuda()
    cols, dt = g.row_shape(a.fmt)
    out = torch.empty((a.batch, cols), dtype=dt, device="cuda:0")
    g.query(a.kind, srcs, mode=a.mode, out=out, fmt=a.fmt)  # warm
    torch.cuda.synchronize()
    for _ in range(a.repeat):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.nvtx.range_push("prof")
        e0.record()
        g.query(a.kind, srcs, mode=a.mode, out=out, fmt=a.fmt)
        e1.record()
        torch.cuda.nvtx.range_pop()
        torch.cuda.synchronize()
        print(f"query {a.kind} {a.mode} batch={a.batch}: {e0.elapsed_time(e1):.3f} ms (events)", flush=True)
    print("done")


if __name__ == "__main__":
    main()

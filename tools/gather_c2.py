#!/usr/bin/env python
"""Write C2's canonical CSR destinations (edge order: the FULL sweep's row-gather stream) as uint32 to a
file for tools/gather_peak.cu:  python tools/gather_c2.py /tmp/c2_dst.bin"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main(path):
    import numpy as np

    import gen
    from paper_conf_eurosys_0002a0a024_b200 import Graph

    cfg = gen.CONFIGS["c2"]
    g = Graph.rmat(cfg.n, cfg.m, cfg.abcd, cfg.w_max, cfg.seed, device="cuda:0")
    _, idx, _ = g.export()
    idx.cpu().numpy().view(np.uint32).tofile(path)
    print(cfg.n, g.m)


if __name__ == "__main__":
    main(sys.argv[1])

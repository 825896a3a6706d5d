#!/usr/bin/env python
"""Device -> pinned-host copy bandwidth of this box (the ceiling of bench.py's e2e leg)."""
import time

import torch

for mb in (64, 256, 1024):
    d = torch.empty(mb << 20, dtype=torch.uint8, device="cuda")
    h = torch.empty(mb << 20, dtype=torch.uint8, pin_memory=True)
    for _ in range(3):
        h.copy_(d, non_blocking=True)
    torch.cuda.synchronize()
    t = time.perf_counter()
    for _ in range(10):
        h.copy_(d, non_blocking=True)
    torch.cuda.synchronize()
    el = time.perf_counter() - t
    print(f"D2H pinned {mb} MiB: {10 * (mb << 20) / el / 1e9:.1f} GB/s")

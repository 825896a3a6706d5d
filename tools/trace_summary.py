#!/usr/bin/env python
"""Summarise a CG_TRACE log (stderr of tools/profile_query.py under CG_TRACE=1): the last kernel
launch that ran iterations, one line per iteration (list size, edges, S1 / S2 microseconds, edge rate)."""
import re
import sys


def main(path):
    lines = open(path).read().splitlines()
    blocks, cur = [], None
    for ln in lines:
        if ln.startswith("CG_TRACE_KERNEL"):
            cur = [ln]
            blocks.append(cur)
        elif ln.startswith("CG_TRACE ") and cur is not None:
            cur.append(ln)
    blk = [b for b in blocks if len(b) > 1][-1]
    print(blk[0])
    tot = {1: 0.0, 2: 0.0}
    for ln in blk[1:]:
        m = dict(re.findall(r"(\w+)=([\d.]+)", ln))
        s1, s2, e = float(m["s1"]), float(m["s2"]), int(m["edges"])
        tot[int(m["phase"])] += s1 + s2
        print(f"it={m['it']:>3} ph={m['phase']} q0={m['q0']:>2} list={int(m['list']):>8} act={int(m['active']):>8} "
              f"E={e:>9} s1={s1:7.1f} s2={s2:7.1f} rate={e / max(s2, 0.1) / 1e3:6.1f}G/s")
    print("phase totals (us):", {k: round(v, 1) for k, v in tot.items()})


if __name__ == "__main__":
    main(sys.argv[1])

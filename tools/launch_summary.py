#!/usr/bin/env python
"""Per-kernel launch count / total time / share from an ncu --metrics gpu__time_duration.sum csv."""
import collections
import csv
import sys


def main(path):
    rows = [r for r in csv.reader(open(path)) if len(r) > 14 and r[12] == "gpu__time_duration.sum"]
    tot = collections.Counter()
    cnt = collections.Counter()
    for r in rows:
        tot[r[4]] += float(r[14].replace(",", "")) / 1e6
        cnt[r[4]] += 1
    s = sum(tot.values()) or 1
    print(f"{'launches':>8} {'total_ms':>10} {'ms/launch':>10} {'share':>6}  kernel")
    for k, v in tot.most_common():
        print(f"{cnt[k]:8d} {v:10.3f} {v / cnt[k]:10.3f} {100 * v / s:5.1f}%  {k[:110]}")


if __name__ == "__main__":
    main(sys.argv[1])

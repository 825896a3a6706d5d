#!/usr/bin/env python
"""Summarise an ncu report: headline metrics + top SASS stall lines (with CUDA source lines)."""
import csv
import io
import subprocess
import sys


def run(rep, *args):
    return subprocess.run(["ncu", "-i", rep, *args], capture_output=True, text=True).stdout


def raw(rep):
    r = list(csv.reader(io.StringIO(run(rep, "--page", "raw", "--csv"))))
    out = []
    for row in r[2:]:
        out.append({h: (v, u) for h, u, v in zip(r[0], r[1], row)})
    return out


KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum", "dram__throughput.avg.pct_of_peak_sustained_elapsed",
        "lts__t_sectors.sum", "lts__t_sector_hit_rate.pct", "l1tex__t_sector_hit_rate.pct", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "smsp__issue_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread", "launch__grid_size",
        "lts__throughput.avg.pct_of_peak_sustained_elapsed", "l1tex__throughput.avg.pct_of_peak_sustained_active"]


def main(rep, top=25):
    for k in raw(rep):
        print({key: k.get(key, ("?", ""))[0] + " " + k.get(key, ("", ""))[1] for key in KEYS})
        stalls = {h: float(v[0].replace(",", "") or 0) for h, v in k.items()
                  if h.startswith("smsp__pcsamp_warps_issue_stalled_") and not h.endswith("not_issued")}
        tot = sum(stalls.values()) or 1
        print("stalls:", {h.replace("smsp__pcsamp_warps_issue_stalled_", ""): round(100 * v / tot, 1)
                          for h, v in sorted(stalls.items(), key=lambda x: -x[1])[:8]})
    txt = run(rep, "--page", "source", "--csv", "--print-source=sass")
    rows = list(csv.reader(io.StringIO(txt)))
    hdr = None
    data = []
    for r in rows:
        if r and r[0] == "Address":
            hdr = r
            continue
        if hdr and len(r) == len(hdr):
            data.append(dict(zip(hdr, r)))
    if not data:
        return
    key = "Warp Stall Sampling (All Samples)"
    tot = sum(float(d[key] or 0) for d in data) or 1
    print("top SASS by stall samples:")
    for d in sorted(data, key=lambda d: -float(d[key] or 0))[:top]:
        print(f"  {100 * float(d[key]) / tot:5.1f}%  {d['Source'][:70]:70s} exec={d['Instructions Executed']}")


if __name__ == "__main__":
    main(sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else 25)

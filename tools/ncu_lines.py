#!/usr/bin/env python
"""Stall samples aggregated per CUDA source line of an ncu report (needs -lineinfo):
    python tools/ncu_lines.py report.ncu-rep [top]"""
import collections
import csv
import io
import subprocess
import sys


def main(rep, top=40):
    txt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                         capture_output=True, text=True).stdout
    f, hdr = None, None
    agg = collections.Counter()
    src = {}
    execs = collections.Counter()
    cur_line = None
    for r in csv.reader(io.StringIO(txt)):
        if not r:
            continue
        if r[0] == "File Path":
            f = r[1].split("/")[-1]
            continue
        if r[0] == "Line No":
            hdr = r
            continue
        if hdr is None or len(r) != len(hdr):
            continue
        if r[0]:
            cur_line = (f, int(r[0]))
            src[cur_line] = r[1]
        s = r[4].replace(",", "")
        e = r[7].replace(",", "")
        if cur_line and s.replace(".", "").isdigit():
            agg[cur_line] += float(s)
        if cur_line and e.replace(".", "").isdigit():
            execs[cur_line] += float(e)
    tot = sum(agg.values()) or 1
    for (fl, ln), v in agg.most_common(top):
        print(f"{100 * v / tot:5.1f}%  {fl}:{ln:<5d} inst={execs[(fl, ln)]:>12.0f}  {src[(fl, ln)].strip()[:90]}")


if __name__ == "__main__":
    main(sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else 40)

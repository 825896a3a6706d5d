#!/usr/bin/env python
"""Per-kind summaries of the round's ncu captures (tools/profile_r2.sh): profiles/<tag>_ncu_<kind>.txt
(headline metrics, stall reasons, hot source lines) and profiles/ncu_kinds.json (DRAM bytes and
duration per launch, which bench.py's roofline reports beside the algorithmic-bytes fraction)."""
import contextlib
import io
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, os.path.join(ROOT, "tools"))
import ncu_lines  # noqa: E402
import ncu_summary  # noqa: E402

KINDS = ("sssp", "sswp", "ssnp", "viterbi", "bfs", "reach")
OUT = os.environ.get("NCU_OUT", os.path.join(ROOT, "profiles"))


def num(v):
    return float(str(v).replace(",", ""))


def main(tag="r2"):
    out = {}
    for k in KINDS:
        rep = os.path.join(os.environ.get("NCU_DIR", os.path.join(ROOT, "gpurun_out")), f"{tag}_ncu_{k}.ncu-rep")
        if not os.path.exists(rep):
            continue
        rows = ncu_summary.raw(rep)
        if not rows:
            continue
        r = rows[0]
        unit_scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}
        tscale = {"nsecond": 1e-6, "usecond": 1e-3, "msecond": 1.0, "second": 1e3, "ns": 1e-6, "us": 1e-3, "ms": 1.0,
                  "s": 1e3}
        rd = num(r["dram__bytes_read.sum"][0]) * unit_scale[r["dram__bytes_read.sum"][1]]
        wr = num(r["dram__bytes_write.sum"][0]) * unit_scale[r["dram__bytes_write.sum"][1]]
        ms = num(r["gpu__time_duration.sum"][0]) * tscale[r["gpu__time_duration.sum"][1]]
        out[k] = {"dram_bytes": rd + wr, "dram_read": rd, "dram_write": wr, "ms": ms,
                  "report": f"profiles/{tag}_ncu_{k}.txt"}
        buf = io.StringIO()
        with contextlib.redirect_stdout(buf):
            print(f"# ncu --set full --clock-control none --import-source on (NVTX range 'prof'): one "
                  f"batch_kernel launch, kind {k}, 32 sources, CG-2Phase, config c2.  tools/profile_r2.sh {tag}")
            ncu_summary.main(rep)
            print("\nstall samples per source line:")
            ncu_lines.main(rep, 40)
        with open(os.path.join(OUT, f"{tag}_ncu_{k}.txt"), "w") as f:
            f.write(buf.getvalue())
        print(k, round(ms, 3), "ms", round((rd + wr) / 1e9, 3), "GB", round((rd + wr) / (ms / 1e3) / 1e9, 1), "GB/s")
    path = os.path.join(OUT, "ncu_kinds.json")
    d = {}
    if os.path.exists(path):
        d = json.load(open(path))
    d["c2-livejournal-rmat"] = {"kinds": out, "how": f"ncu --set full --clock-control none, one batch_kernel launch "
                                f"per kind (32 sources, CG-2Phase), dram__bytes_read.sum + dram__bytes_write.sum and "
                                f"gpu__time_duration.sum; captures {tag} (tools/profile_r2.sh)"}
    json.dump(d, open(path, "w"), indent=1)


if __name__ == "__main__":
    main(*(sys.argv[1:] or ["r2"]))

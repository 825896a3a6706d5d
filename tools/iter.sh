#!/bin/bash
# quick GPU iteration: parity tests, C2 bench (no CPU baseline / e2e), per-iteration traces
tag=${1:-it}
mkdir -p gpurun_out
timeout 600 python -m pytest tests -m gpu -x -q --timeout 200 > gpurun_out/${tag}_pytest.txt 2>&1; tail -3 gpurun_out/${tag}_pytest.txt
timeout 400 python bench.py --config c2 --steps 5 --no-cpu-baseline --no-e2e > gpurun_out/${tag}_bench.json 2> gpurun_out/${tag}_bench.err
python - "$tag" <<'PY'
import json,sys
t=sys.argv[1]
try:
    d=json.loads(open(f"gpurun_out/{t}_bench.json").read().strip().splitlines()[-1])
    print("qps", round(d["value"],1), "full", round(d["full"]["value"],1), "frac", round(d["roofline"]["frac"],4))
    for k,v in d["per_kind"].items(): print(k, round(v["ms_2phase"],3), round(v["ms_full"],3), round(v["alg_GBps"]))
except Exception as e:
    print("bench failed", e, open(f"gpurun_out/{t}_bench.err").read()[-1500:])
PY
for k in ${KINDS:-sssp bfs}; do
  CG_TRACE=1 timeout 120 python tools/profile_query.py --config c2 --kind $k --mode 2phase --batch 32 --repeat 2 2> gpurun_out/${tag}_trace_${k}.txt > gpurun_out/${tag}_ev_${k}.txt
done

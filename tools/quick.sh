#!/bin/bash
# quick GPU iteration: parity tests, per-iteration trace, bench for both register budgets
timeout 400 python -m pytest tests -m gpu -x -q --timeout 120 2>&1 | tail -3
bash tools/trace_run.sh ${1:-c2}
for mb in 1 2; do CG_MINB=$mb timeout 240 python bench.py --config ${1:-c2} --steps 5 --no-cpu-baseline --no-e2e > gpurun_out/bench_${1:-c2}_minb$mb.json 2>&1; done
python - <<'PY'
import json,sys
for mb in (1,2):
    try:
        d=json.loads(open("gpurun_out/bench_%s_minb%d.json"%(sys.argv[1] if len(sys.argv)>1 else "c2",mb)).read().strip().splitlines()[-1])
    except Exception as e:
        print(mb, "failed", e); continue
    print(mb, round(d["value"],1), round(d["full"]["value"],1), round(d["roofline"]["frac"],4), {k:(round(v["ms_2phase"],2),round(v["ms_full"],2)) for k,v in d["per_kind"].items()})
PY

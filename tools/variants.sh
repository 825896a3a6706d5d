#!/bin/bash
# bench several library variants x register budgets: tools/variants.sh c2 "default u8" "1 2"
cfg=${1:-c2}; libs=${2:-default}; minbs=${3:-"1 2"}
for lib in $libs; do
  for mb in $minbs; do
    if [ "$lib" = default ]; then unset CGB_LIB; else export CGB_LIB=$PWD/paper_conf_eurosys_0002a0a024_b200/libcg_$lib.so; fi
    CG_MINB=$mb timeout 240 python bench.py --config $cfg --steps 5 --no-cpu-baseline --no-e2e > gpurun_out/v_${cfg}_${lib}_$mb.json 2> gpurun_out/v_${cfg}_${lib}_$mb.err
    python - "$cfg" "$lib" "$mb" <<'PY'
import json,sys
cfg,lib,mb=sys.argv[1:]
try:
    d=json.loads(open(f"gpurun_out/v_{cfg}_{lib}_{mb}.json").read().strip().splitlines()[-1])
    print(lib, mb, round(d["value"],1), round(d["full"]["value"],1), round(d["roofline"]["frac"],4), {k:(round(v["ms_2phase"],2),round(v["ms_full"],2)) for k,v in d["per_kind"].items()})
except Exception as e:
    print(lib, mb, "FAILED", e, open(f"gpurun_out/v_{cfg}_{lib}_{mb}.err").read()[-500:])
PY
  done
done
unset CGB_LIB

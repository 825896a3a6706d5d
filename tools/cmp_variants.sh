#!/bin/bash
# bench several library variants (paper_conf_eurosys_0002a0a024_b200/libcg_<name>.so, "default" = product lib)
for v in ${VARIANTS:-default}; do
  if [ "$v" = default ]; then unset CGB_LIB; else export CGB_LIB=$PWD/paper_conf_eurosys_0002a0a024_b200/libcg_$v.so; fi
  timeout 300 python bench.py --config ${CFG:-c2} --steps 5 --no-cpu-baseline --no-e2e > gpurun_out/cmp_$v.json 2> gpurun_out/cmp_$v.err
  python -c "
import json; d=json.loads(open('gpurun_out/cmp_$v.json').read().strip().splitlines()[-1])
print('$v', round(d['value'],1), round(d['full']['value'],1), {k:(round(x['ms_2phase'],2), round(x['ms_full'],2)) for k,x in d['per_kind'].items()})" || tail -3 gpurun_out/cmp_$v.err
done

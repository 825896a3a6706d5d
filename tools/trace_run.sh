#!/bin/bash
# per-iteration trace of one query batch per kind (CG_TRACE) on a config
cfg=${1:-c2}
for minb in 1 2; do
  CG_MINB=$minb CG_TRACE=1 timeout 120 python tools/profile_query.py --config $cfg --kind sssp --mode 2phase --batch 2 2> gpurun_out/trace_${cfg}_sssp_minb${minb}.txt
done

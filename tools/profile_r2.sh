#!/bin/bash
# Round-2 evidence (run from the repo root under gpurun): one `ncu --set full` capture of the batched
# query kernel per kind (C2, CG-2Phase, 32 sources, one launch inside the NVTX range "prof"), and the
# ncu launch list of the bench command.  Summaries are written by tools/ncu_kinds.py afterwards.
tag=${1:-r2}
mkdir -p gpurun_out
for k in ${KINDS:-sssp sswp ssnp viterbi bfs reach}; do
  timeout 900 ncu --set full --nvtx --nvtx-include "prof/" --clock-control none --import-source on -f \
    --kernel-name regex:"batch_kernel" -o ${NCU_DIR:-gpurun_out}/${tag}_ncu_${k} \
    python tools/profile_query.py --config c2 --kind $k --mode 2phase --batch 32 > gpurun_out/${tag}_ncu_${k}.log 2>&1
  tail -1 gpurun_out/${tag}_ncu_${k}.log
done
if [ -z "$NO_LAUNCHES" ]; then
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --kernel-name regex:"batch_kernel|query_kernel" -c 400 --csv \
  --log-file gpurun_out/${tag}_launches_c2.csv python bench.py --config c2 --steps 2 --warmup 3 --no-cpu-baseline --no-e2e \
  --no-c1 --no-c3 > gpurun_out/${tag}_launches_bench.log 2>&1
fi
python tools/ncu_kinds.py $tag

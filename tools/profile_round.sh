#!/bin/bash
# One GPU call's worth of evidence for the current library (run from the repo root under gpurun):
#   GPU parity tests, bench line (c2), per-iteration trace, ncu launch list of the bench command,
#   one ncu --set full capture of the batched query kernel (SSSP, CG-2Phase, c2, 32 sources).
tag=${1:-r1}
mkdir -p gpurun_out
timeout 600 python -m pytest tests -m gpu -x -q --timeout 200 > gpurun_out/${tag}_pytest_gpu.txt 2>&1; tail -3 gpurun_out/${tag}_pytest_gpu.txt
timeout 500 python bench.py --config c2 > gpurun_out/${tag}_bench_c2.json 2> gpurun_out/${tag}_bench_c2.err; tail -c 400 gpurun_out/${tag}_bench_c2.json
for k in sssp bfs reach; do
  CG_TRACE=1 timeout 120 python tools/profile_query.py --config c2 --kind $k --mode 2phase --batch 32 2> gpurun_out/${tag}_trace_c2_${k}.txt >/dev/null
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --kernel-name regex:"batch_kernel|query_kernel" -c 400 --csv \
  --log-file gpurun_out/${tag}_launches_c2_raw.csv python bench.py --config c2 --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/${tag}_launches_bench.log 2>&1
timeout 900 ncu --set full --nvtx --nvtx-include "prof/" --clock-control none --import-source on -f \
  -o gpurun_out/${tag}_ncu_sssp_2phase_c2 python tools/profile_query.py --config c2 --kind sssp --mode 2phase --batch 32 > gpurun_out/${tag}_ncu.log 2>&1
tail -3 gpurun_out/${tag}_ncu.log

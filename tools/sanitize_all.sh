#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck / initcheck over tools/sanitize_run.py
# (only this library's kernels are instrumented); logs -> gpurun_out/sanitize_<tool>.txt
mkdir -p gpurun_out
for tool in ${TOOLS:-memcheck racecheck synccheck initcheck}; do
  extra=""
  timeout 2400 compute-sanitizer --tool $tool $extra --kernel-name kns=cgb \
    --print-limit 50 python tools/sanitize_run.py > gpurun_out/sanitize_$tool.txt 2>&1
  echo "$tool rc=$? $(tail -2 gpurun_out/sanitize_$tool.txt | tr '\n' ' ')"
done

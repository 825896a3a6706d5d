#!/bin/bash
# bench library variants: tools/libbench.sh c2 "default mf cg" [extra env]
cfg=$1; libs=$2; shift 2
for lib in $libs; do
  if [ "$lib" = default ]; then L=""; else L="CGB_LIB=$PWD/paper_conf_eurosys_0002a0a024_b200/libcg_$lib.so"; fi
  bash tools/envbench.sh $cfg "$L $* CGB_TAG=$lib" 2>&1 | sed "s/^/$lib: /"
done

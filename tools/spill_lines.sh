#!/bin/bash
# Source lines of the local-memory (spill) instructions of one batch_kernel instantiation:
#   tools/spill_lines.sh 'batch_kernelILi0ELb1ENS0_7Lanes16ILi0EEEEEvNS0_7BParamsE'
d=$(mktemp -d)
root=$(cd "$(dirname "$0")/.." && pwd); (cd $d && cuobjdump -xelf all "$root/paper_conf_eurosys_0002a0a024_b200/build/libcoregraph_b200.so/engine_batch.cu.o" >/dev/null 2>&1 && nvdisasm -g -c engine_batch.sm_100a.cubin > all.sass 2>/dev/null)
n=$(grep -n "^\.text.*$1:" $d/all.sass | head -1 | cut -d: -f1)
awk -v s=$n 'NR>=s' $d/all.sass | awk '/^\/\/-----/{if(started)exit} {started=1; print}' |
  awk '/\/\/## File/{loc=$0} /LDL|STL/{print loc}' | grep -oE '[a-z_]+\.cu[h]?", line [0-9]+' | sort | uniq -c | sort -rn | head -${2:-12}
rm -rf $d

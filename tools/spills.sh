#!/bin/bash
# ptxas register / spill report of the batched engine's kernels (sm_100a), one line per instantiation
cd "$(dirname "$0")/../paper_conf_eurosys_0002a0a024_b200"
/usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC \
  --expt-relaxed-constexpr -Xptxas -v -I ../include "$@" -c csrc/${SRC:-engine_batch.cu} -o /tmp/spills.o 2>&1 |
python3 -c '
import sys,re,subprocess
cur=None
for line in sys.stdin:
    m=re.search(r"Compiling entry function .(_Z\w+).", line)
    if m: cur=subprocess.run(["c++filt",m.group(1)],capture_output=True,text=True).stdout.strip(); continue
    m=re.search(r"(\d+) bytes spill stores, (\d+) bytes spill loads", line)
    if m and cur: st=(m.group(1),m.group(2)); continue
    m=re.search(r"Used (\d+) registers", line)
    if m and cur:
        name=re.sub(r"cgb::\(anonymous namespace\)::","",cur)
        print(f"regs={m.group(1):>3} spill st/ld={st[0]}/{st[1]}  {name[:150]}")
        cur=None
'

#!/bin/bash
# bench under several environment settings: tools/envbench.sh c2 "CG_FRESH=3" "CG_FRESH=2" ...
# (C2 headline only; per-kind ms 2Phase / FULL)
cfg=$1; shift
for envs in "$@"; do
  tag=$(echo "$envs" | sed "s|[^A-Za-z0-9_]|_|g" | tail -c 60)
  env $envs timeout 300 python bench.py --config $cfg --steps ${STEPS:-5} --no-cpu-baseline --no-e2e --no-c1 --no-c3 \
      > gpurun_out/eb_${cfg}_$tag.json 2> gpurun_out/eb_${cfg}_$tag.err
  python - "$cfg" "$tag" <<'PY'
import json,sys
cfg,tag=sys.argv[1:]
try:
    d=json.loads(open(f"gpurun_out/eb_{cfg}_{tag}.json").read().strip().splitlines()[-1])
    print(tag, round(d["value"],1), round(d["full"]["value"],1), {k:(round(v["ms_2phase"],3),round(v["ms_full"],3)) for k,v in d["per_kind"].items()}, "wcc", round(d["wcc"]["ms_2phase"],3) if d.get("wcc") else None, flush=True)
except Exception as e:
    print(tag, "FAILED", e, open(f"gpurun_out/eb_{cfg}_{tag}.err").read()[-800:])
PY
done

#!/bin/bash
# headline run-to-run on one box: value vs host preads per step (B14 split activity), 3 runs each
# with the default split threshold and with splitting off
cd "$GRAFT_REPO_ROOT" || exit 1
O=gpurun_out
for sk in 128 0 128 0 128; do
  GSYS_SPLIT_KB=$sk timeout 300 python bench.py --steps 5 --warmup 3 --no-extras --no-cpu-baseline > $O/r02sv.json 2>/dev/null
  python - "$sk" <<'PY' >> $O/r02_split_var.jsonl
import json,sys
d=json.loads(open("gpurun_out/r02sv.json").read().strip().splitlines()[-1])
print(json.dumps({"split_kb":int(sys.argv[1]),"GBps":round(d["value"],2),"host_preads_per_step":d["service"]["host_preads_per_step"],"bundles":d["service"]["bundles_per_step"]}))
PY
done
cat $O/r02_split_var.jsonl

#!/bin/bash
# host-side bound probe: LLC size, host DRAM bandwidth, and the wordcount at several bounce-ring
# sizes (GSYS_BOUNCE_MB per worker) x chunk sizes -- does an LLC-resident bounce cut host DRAM traffic?
cd "$GRAFT_REPO_ROOT" || exit 1
O=gpurun_out
lscpu > $O/r02b_lscpu.txt 2>&1
gcc -O2 -pthread -o /tmp/host_membw tools/probes/host_membw.c && /tmp/host_membw > $O/r02b_membw.txt 2>&1
for mb in 32 8 4 2; do for ck in 256 128 64; do
  GSYS_BOUNCE_MB=$mb timeout 300 python bench.py --steps 5 --warmup 3 --no-extras --no-cpu-baseline --chunk-kib $ck > $O/r02b_${mb}_${ck}.json 2>$O/r02b_${mb}_${ck}.err
  python - "$mb" "$ck" "$O/r02b_${mb}_${ck}.json" <<'PY' >> $O/r02b_sweep.jsonl
import json,sys
try:
    d=json.loads(open(sys.argv[3]).read().strip().splitlines()[-1])
    print(json.dumps({"bounce_mb":int(sys.argv[1]),"chunk_kib":int(sys.argv[2]),"GBps":d["value"],"frac":d["roofline"]["frac"],"h2d":d["roofline"]["peak"],"service":d["service"],"parity":d.get("parity")}))
except Exception as e:
    print(json.dumps({"bounce_mb":int(sys.argv[1]),"chunk_kib":int(sys.argv[2]),"error":str(e)}))
PY
done; done
cat $O/r02b_sweep.jsonl

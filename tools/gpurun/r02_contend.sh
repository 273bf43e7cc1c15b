#!/bin/bash
# host-DRAM contention A/B: the wordcount with the default bounce ring (32 MiB per worker, 256 KiB
# chunks) vs small LLC-sized rings (2-4 MiB per worker, 64-128 KiB chunks), first alone, then while
# T hog threads stream memcpy through host DRAM (a box whose host memory is busier).
cd "$GRAFT_REPO_ROOT" || exit 1
O=gpurun_out
gcc -O2 -pthread -o /tmp/membw_hog tools/probes/membw_hog.c || exit 1
run() {  # tag bounce_mb chunk_kib [threads]
  local th=${4:-}
  GSYS_BOUNCE_MB=$2 ${th:+GSYS_THREADS=$th} timeout 300 python bench.py --steps 5 --warmup 3 --no-extras --no-cpu-baseline --chunk-kib $3 > $O/r02x.json 2>$O/r02x.err
  python - "$1" "$2" "$3" "$th" <<'PY' >> $O/r02_contend.jsonl
import json,sys
try:
    d=json.loads(open("gpurun_out/r02x.json").read().strip().splitlines()[-1])
    print(json.dumps({"hog":sys.argv[1],"bounce_mb":int(sys.argv[2]),"chunk_kib":int(sys.argv[3]),"service_threads":sys.argv[4] or 14,"GBps":round(d["value"],2),"ok":d["parity"]}))
except Exception as e:
    print(json.dumps({"hog":sys.argv[1],"error":str(e)}))
PY
}
for hog in 0 2 4; do
  if [ $hog -gt 0 ]; then /tmp/membw_hog $hog & HP=$!; sleep 2; fi
  for rep in 1 2; do
    run "hog$hog" 32 256; run "hog$hog" 2 64; run "hog$hog" 4 128
  done
  if [ $hog -gt 0 ]; then kill $HP; wait $HP 2>/dev/null; fi
done
cat $O/r02_contend.jsonl

#!/bin/bash
python -c "import inputs; inputs.make_corpus(512, 16<<20)" > /dev/null 2>&1
go() { rm -f /dev/shm/mix_go; sleep 25; touch /dev/shm/mix_go; }
# singles
for cfg in "host 0 256 256 296" "device 256 256 1024 296"; do
  set -- $cfg; (go &) ; GSYS_THREADS=14 timeout 120 python tools/mix_probe.py $1 $2 $3 $4 $5 8 >> gpurun_out/mix51.jsonl 2>>gpurun_out/mix51.err
  echo '---' >> gpurun_out/mix51.jsonl
done
# mixes: host-staged + device-staged processes at once (7 service threads each)
for dcfg in "1024 296" "1024 64" "4096 64"; do
  set -- $dcfg
  rm -f /dev/shm/mix_go
  GSYS_THREADS=7 timeout 120 python tools/mix_probe.py host 0 256 256 296 8 >> gpurun_out/mix51.jsonl 2>>gpurun_out/mix51.err &
  GSYS_THREADS=7 timeout 120 python tools/mix_probe.py device 256 256 $1 $2 8 >> gpurun_out/mix51.jsonl 2>>gpurun_out/mix51.err &
  sleep 30; touch /dev/shm/mix_go; wait
  echo '---' >> gpurun_out/mix51.jsonl
done

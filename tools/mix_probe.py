"""Steady-state wordcount throughput of one process for ~D seconds (for concurrent-process mixes).
Usage: python tools/mix_probe.py host|device first_file nfiles chunk_kib blocks seconds"""
import json, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import inputs
from paper_conf_isca_veselybblor18_b200 import gsys as G
from paper_conf_isca_veselybblor18_b200 import workloads as W
st, f0, nf, ck, blocks, secs = sys.argv[1], int(sys.argv[2]), int(sys.argv[3]), int(sys.argv[4]), int(sys.argv[5]), float(sys.argv[6])
c = inputs.make_corpus(512, 16 << 20)
paths = c.paths[f0:f0 + nf]
words, pats = inputs.dictionary(), inputs.patterns()
W.ensure_init()
of = W.OpenFiles(paths).__enter__()
s = torch.cuda.Stream()
h = torch.zeros(64, dtype=torch.int64, device="cuda")
hits = torch.zeros(len(paths), dtype=torch.int32, device="cuda")
stg = G.STAGE_HOST if st == "host" else G.STAGE_DEVICE
gf = G.WG | G.BLOCKING | G.RELAXED
def run():
    G.gsys_wordcount(of.fds, of.sizes, ck << 10, words, pats, h, hits, None, gf, blocks, 256, s, stg)
    G.gsys_wait(s)
with torch.cuda.stream(s):
    run()
    # wait for the start signal file so concurrent processes overlap
    while not os.path.exists("/dev/shm/mix_go"):
        time.sleep(0.001)
    t0 = time.perf_counter(); n = 0
    while time.perf_counter() - t0 < secs:
        run(); n += 1
    s.synchronize()
    dt = time.perf_counter() - t0
print(json.dumps({"staging": st, "files": nf, "chunk_kib": ck, "blocks": blocks, "iters": n,
                  "GBps": n * sum(of.sizes) / dt / 1e9}), flush=True)

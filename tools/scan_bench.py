"""Standalone HBM scan (row a8) timing + parity on 1 GiB of corpus text (64 x 16 MiB files).
Usage: python tools/scan_bench.py [threads] [chunk_kib] [reps]"""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import inputs
from paper_conf_isca_veselybblor18_b200 import gsys as G

threads = int(sys.argv[1]) if len(sys.argv) > 1 else 512
chunk = (int(sys.argv[2]) if len(sys.argv) > 2 else 256) << 10
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 20
c = inputs.make_corpus(64, 16 << 20)
text = torch.cat([torch.from_file(p, dtype=torch.uint8, size=os.path.getsize(p)) for p in c.paths]).cuda()
n = text.numel()
words, pats = inputs.dictionary(), inputs.patterns()
hist = torch.zeros(64, dtype=torch.int64, device="cuda")
hit = torch.zeros(1, dtype=torch.int32, device="cuda")
G.gsys_scan_device(text, n, chunk, words, pats, hist, hit, 0, threads)
torch.cuda.synchronize()
ok = np.array_equal(hist.cpu().numpy().astype(np.uint64), c.census)
for _ in range(3):
    G.gsys_scan_device(text, n, chunk, words, pats, hist, hit, 0, threads)
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(reps):
    G.gsys_scan_device(text, n, chunk, words, pats, hist, hit, 0, threads)
e1.record()
e1.synchronize()
t = e0.elapsed_time(e1) / 1e3 / reps
print(json.dumps({"threads": threads, "chunk": chunk, "ms": t * 1e3, "GBps": n / t / 1e9, "parity": bool(ok),
                  "grep_hit": int(hit.item())}))

"""Standalone HBM scan (row a8): token-level vs byte-DFA implementation, timing + parity on 1 GiB of
corpus text (64 x 16 MiB files) in HBM.  One JSON line per (impl, threads, chunk).
Usage: python tools/scan_ab.py [reps]"""
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import inputs  # noqa: E402
from paper_conf_isca_veselybblor18_b200 import gsys as G  # noqa: E402

reps = int(sys.argv[1]) if len(sys.argv) > 1 else 20
c = inputs.make_corpus(64, 16 << 20)
text = torch.cat([torch.from_file(p, dtype=torch.uint8, size=os.path.getsize(p)) for p in c.paths]).cuda()
n = text.numel()
words, pats = inputs.dictionary(), inputs.patterns()
want_hit = int(any(c.pmasks[:64]))
IMPL = {"token": G.SCAN_TOKEN, "dfa_tma": G.SCAN_DFA_TMA, "dfa": G.SCAN_DFA}
# SCAN_AB_CELLS="token:768:256,dfa:704:256" (impl:threads:chunk_kib) picks the cells
cells = [(IMPL[i], int(t), int(k)) for i, t, k in (x.split(":") for x in os.environ.get(
    "SCAN_AB_CELLS", "token:768:256,dfa_tma:704:256,dfa:704:256").split(","))]
for impl, threads, ck in cells:
    G.gsys_set_scan(impl)
    chunk = ck << 10
    hist = torch.zeros(64, dtype=torch.int64, device="cuda")
    hit = torch.zeros(1, dtype=torch.int32, device="cuda")
    G.gsys_scan_device(text, n, chunk, words, pats, hist, hit, 0, threads)
    torch.cuda.synchronize()
    ok = bool(np.array_equal(hist.cpu().numpy().astype(np.uint64), c.census)) and int(hit.item()) == want_hit
    for _ in range(3):
        G.gsys_scan_device(text, n, chunk, words, pats, hist, hit, 0, threads)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        G.gsys_scan_device(text, n, chunk, words, pats, hist, hit, 0, threads)
    e1.record()
    e1.synchronize()
    t = e0.elapsed_time(e1) / 1e3 / reps
    print(json.dumps({"impl": {G.SCAN_TOKEN: "token", G.SCAN_DFA_TMA: "dfa_tma", G.SCAN_DFA: "dfa_ldgsts"}[impl],
                      "threads": threads, "chunk": chunk,
                      "ms": t * 1e3, "GBps": n / t / 1e9, "parity": ok}), flush=True)
G.gsys_set_scan(G.SCAN_DFA)

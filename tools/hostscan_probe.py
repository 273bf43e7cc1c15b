"""How fast can work-groups scan text sitting in pinned host memory (no syscalls)?  gsys_scan_device
over a 16 MiB pinned host-mapped buffer (zero-copy, the host-staging read pattern) vs the same bytes
in HBM, at 64 and 148 work-groups; plus config 1 with the non-blocking double-buffered prefetch."""
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import inputs  # noqa: E402
from paper_conf_isca_veselybblor18_b200 import gsys as G  # noqa: E402
from paper_conf_isca_veselybblor18_b200 import workloads as W  # noqa: E402

W.ensure_init()
words, pats = inputs.dictionary(), inputs.patterns()
p = "/dev/shm/gsys_config1_16MiB.txt"
census, _ = inputs.write_file(p, inputs.SEED_FILE16M, 0, 16 << 20)
host = torch.from_file(p, dtype=torch.uint8, size=16 << 20).pin_memory()
dev = host.cuda()
for where, buf in (("pinned_host", host), ("hbm", dev)):
    for blocks in (64, 148):
        for chunk in (256 << 10, 64 << 10):
            hist = torch.zeros(64, dtype=torch.int64, device="cuda")
            for _ in range(3):
                G.gsys_scan_device(buf, 16 << 20, chunk, words, pats, hist, None, blocks, 256)
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            for _ in range(10):
                G.gsys_scan_device(buf, 16 << 20, chunk, words, pats, hist, None, blocks, 256)
            e1.record()
            e1.synchronize()
            ms = e0.elapsed_time(e1) / 10
            print(json.dumps({"probe": "scan", "where": where, "blocks": blocks, "chunk": chunk, "ms": ms,
                              "GBps": (16 << 20) / ms / 1e6}), flush=True)
fd = os.open(p, os.O_RDONLY)
h = torch.zeros(64, dtype=torch.int64, device="cuda")
for nb in (False, True):
    for chunk in (256 << 10, 64 << 10):
        ts = []
        for rep in range(20):
            h.zero_()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            G.gsys_wordcount([fd], [16 << 20], chunk, words, pats, h, None, None,
                             G.WG | (G.NONBLOCKING if nb else G.BLOCKING) | G.STRONG, 64, 256, None, G.STAGE_HOST)
            e1.record()
            G.gsys_wait(None)
            e1.synchronize()
            if rep >= 5:
                ts.append(e0.elapsed_time(e1))
        ts.sort()
        ok = bool((h.cpu().numpy().astype("uint64") == census).all())
        print(json.dumps({"probe": "config1", "nonblocking_prefetch": nb, "chunk": chunk, "ms_median": ts[len(ts) // 2],
                          "parity": ok}), flush=True)
os.close(fd)

"""Zero-copy scan of the 16 MiB config-1 file from pinned host memory (gsys_scan_device, no
syscalls) at 64 / 148 work-groups x 256 / 512 / 768 threads x 256 / 64 / 16 KiB chunks."""
import json, os, sys, torch
sys.path.insert(0, os.getcwd())
import inputs
from paper_conf_isca_veselybblor18_b200 import gsys as G
from paper_conf_isca_veselybblor18_b200 import workloads as W
W.ensure_init()
words, pats = inputs.dictionary(), inputs.patterns()
p = "/dev/shm/gsys_config1_16MiB.txt"
census, _ = inputs.write_file(p, inputs.SEED_FILE16M, 0, 16 << 20)
host = torch.from_file(p, dtype=torch.uint8, size=16 << 20).pin_memory()
for blocks in (64, 148):
    for threads in (256, 512, 768):
        for chunk in (256 << 10, 64 << 10, 16 << 10):
            hist = torch.zeros(64, dtype=torch.int64, device="cuda")
            for _ in range(3):
                G.gsys_scan_device(host, 16 << 20, chunk, words, pats, hist, None, blocks, threads)
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            for _ in range(10):
                G.gsys_scan_device(host, 16 << 20, chunk, words, pats, hist, None, blocks, threads)
            e1.record(); e1.synchronize()
            ms = e0.elapsed_time(e1) / 10
            print(json.dumps({"blocks": blocks, "threads": threads, "chunk": chunk, "ms": round(ms, 4), "GBps": round((16 << 20) / ms / 1e6, 1)}), flush=True)

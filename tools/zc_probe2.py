"""Zero-copy read variants: static vs freshly CPU-written host buffer, ld.nc vs ld.cg."""
import json, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import inputs
from paper_conf_isca_veselybblor18_b200 import gsys as G
words, pats = inputs.dictionary(), inputs.patterns()
n = 256 << 20
buf, _, _ = inputs.gen_bytes(2, 0, 64 << 20)
src = torch.from_numpy(buf)
host = torch.empty(n, dtype=torch.uint8).pin_memory()
fresh = torch.empty(n, dtype=torch.uint8)
for i in range(n // buf.size):
    host[i * buf.size:(i + 1) * buf.size].copy_(src)
    fresh[i * buf.size:(i + 1) * buf.size].copy_(src)
hist = torch.zeros(64, dtype=torch.int64, device="cuda")
pol = os.environ.get("GSYS_SCAN_LD", "0")
for blocks in (148, 296):
    for rewrite in (False, True):
        ts = []
        for it in range(4):
            if rewrite:
                host.copy_(fresh)          # CPU writes the whole buffer (like pread into staging)
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            G.gsys_scan_device(host, n, 256 << 10, words, pats, hist, None, blocks, 256)
            e1.record(); e1.synchronize()
            ts.append(e0.elapsed_time(e1) / 1e3)
        print(json.dumps({"ld": pol, "blocks": blocks, "cpu_rewrite": rewrite, "GBps": n / min(ts[1:]) / 1e9}), flush=True)

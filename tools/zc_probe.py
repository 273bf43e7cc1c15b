"""Zero-copy (host-mapped) read bandwidth probes: the scan kernel and a copy over pinned host text."""
import json, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import inputs
from paper_conf_isca_veselybblor18_b200 import gsys as G
words, pats = inputs.dictionary(), inputs.patterns()
n = 1 << 30
buf, _, _ = inputs.gen_bytes(2, 0, 64 << 20)
host = torch.empty(n, dtype=torch.uint8).pin_memory()
src = torch.from_numpy(buf)
for i in range(n // buf.size):
    host[i * buf.size:(i + 1) * buf.size].copy_(src)
dev = host.to("cuda")
hist = torch.zeros(64, dtype=torch.int64, device="cuda")
for name, t in [("hbm", dev), ("host_mapped", host)]:
    for blocks in (592, 1184):
        G.gsys_scan_device(t, n, 256 << 10, words, pats, hist, None, blocks, int(os.environ.get("ZC_THREADS", "512")))
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(3):
            G.gsys_scan_device(t, n, 256 << 10, words, pats, hist, None, blocks, int(os.environ.get("ZC_THREADS", "512")))
        e1.record(); e1.synchronize()
        print(json.dumps({"scan": name, "blocks": blocks, "GBps": 3 * n / (e0.elapsed_time(e1) / 1e3) / 1e9}), flush=True)
# plain torch copy host->device via SM reads? use a reduction that reads host memory directly
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
d2 = torch.empty_like(dev)
e0.record(); d2.copy_(host, non_blocking=True); e1.record(); e1.synchronize()
print(json.dumps({"ce_copy_1GiB_GBps": n / (e0.elapsed_time(e1) / 1e3) / 1e9}))

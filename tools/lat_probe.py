"""Single-caller round-trip latency (GPU-observed, %globaltimer) of blocking getrusage / 4 KiB pread
(host buffer) at WI and WG granularity, plus the loaded WG getrusage rate.  Env knobs are read at
gsys_init (GSYS_POLL_NS_HOST, GSYS_POLL_NS_MAX)."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_isca_veselybblor18_b200 import gsys as G
from paper_conf_isca_veselybblor18_b200 import workloads as W
W.ensure_init()
p = "/dev/shm/lat_probe.bin"
with open(p, "wb") as f:
    f.write(os.urandom(1 << 20))
fd = os.open(p, os.O_RDONLY)
hbuf = torch.empty(1 << 20, dtype=torch.uint8).pin_memory()
out = {"poll_ns_host": os.environ.get("GSYS_POLL_NS_HOST", "4096")}
for name, kind, gran, th, ln, buf, extra in [("getrusage_wi", "getrusage", G.WI, 1, 0, None, 0),
                                              ("getrusage_wg", "getrusage", G.WG, 256, 0, None, 0),
                                              ("pread4k_wg_hostbuf", "pread", G.WG, 256, 4096, hbuf, G.HOSTBUF)]:
    for _ in range(2):   # warm the learned sleep hints
        n, ret, lat, _, rc = W.bench_calls(kind, gran | G.BLOCKING | G.STRONG | extra, 1, th, 400, fd, ln, 1 << 20, buf)
    l = lat.double().cpu()[50:] / 1e3
    out[name] = {"p50_us": float(l.median()), "p10_us": float(l.quantile(0.1)), "p99_us": float(l.quantile(0.99)),
                 "ok": bool((ret >= 0).all())}
import time
t0 = time.perf_counter()
n, ret, lat, _, rc = W.bench_calls("getrusage", G.WG | G.BLOCKING | G.STRONG, 592, 256, 20)
torch.cuda.synchronize()
dt = time.perf_counter() - t0
out["getrusage_wg_loaded"] = {"calls_per_s": n * 20 / dt, "p50_us": float(lat.double().cpu().median() / 1e3)}
print(json.dumps(out), flush=True)

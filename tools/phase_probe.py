"""Where does a blocking GPU call's time go as concurrency grows?  GSYS_DIAG_PHASES=1 phase sums
(claim, publish, wait, copy+release) plus the service's time per call, for WG getrusage and WG
4 KiB preads (host buffer and pulled device buffer) at 1..592 callers.  JSON lines."""
import json
import os
import sys
import time

os.environ["GSYS_DIAG_PHASES"] = "1"
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_isca_veselybblor18_b200 import gsys as G  # noqa: E402
from paper_conf_isca_veselybblor18_b200 import workloads as W  # noqa: E402

W.ensure_init()
path = "/dev/shm/probe_pread.bin"
if not os.path.exists(path) or os.path.getsize(path) != (64 << 20):
    with open(path, "wb") as f:
        f.write(os.urandom(64 << 20))
fd = os.open(path, os.O_RDONLY)
hbuf = torch.zeros(592 * 4096, dtype=torch.uint8).pin_memory()
dbuf = torch.zeros(592 * 4096, dtype=torch.uint8, device="cuda")
for kind, extra, buf in (("getrusage", 0, None), ("pread", G.HOSTBUF, hbuf), ("pread", 0, dbuf)):
    for blocks, iters in ((1, 2000), (8, 500), (64, 200), (148, 100), (296, 60), (592, 40)):
        flags = G.WG | G.BLOCKING | G.RELAXED | extra
        kw = dict(fd=fd, length=4096, size=64 << 20, d_buf=buf) if kind == "pread" else {}
        W.bench_calls(kind, flags, blocks, 256, 2, **kw)
        G.gsys_diag_phases(True)
        G.gsys_stats_reset()
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        n, ret, lat, _, rc = W.bench_calls(kind, flags, blocks, 256, iters, **kw)
        dt = time.perf_counter() - t0
        ph = G.gsys_diag_phases(True)
        st = G.gsys_stats()
        calls = blocks * iters
        print(json.dumps({"kind": kind, "buffer": "host" if extra else ("device" if buf is not None else "-"),
                          "callers": blocks, "calls_per_s": calls / dt, "lat_p50_us": float(lat.double().median() / 1e3),
                          **ph, "svc_busy_us_per_call": st["ns_busy"] / 1e3 / calls,
                          "svc_sys_us_per_call": st["ns_syscall"] / 1e3 / calls,
                          "bundles_per_call": st["bundles"] / calls, "busy_frac": st["ns_busy"] / 1e9 / dt / st["threads"]}),
              flush=True)
os.close(fd)

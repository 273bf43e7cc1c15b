"""Syscall-path probe: getrusage / pread at WG granularity with varying concurrency; prints
calls/s, GPU-observed latency and the host service's time breakdown (one JSON line per point)."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

from paper_conf_isca_veselybblor18_b200 import gsys as G  # noqa: E402
from paper_conf_isca_veselybblor18_b200 import workloads as W  # noqa: E402

W.ensure_init()
kinds = sys.argv[1:] or ["getrusage"]
path = "/dev/shm/probe_pread.bin"
if not os.path.exists(path) or os.path.getsize(path) != (64 << 20):
    with open(path, "wb") as f:
        f.write(os.urandom(64 << 20))
fd = os.open(path, os.O_RDONLY)
for kind in kinds:
    for gran in (G.WG, G.WI):
        for blocks, iters in [(1, 2000), (8, 500), (64, 100), (592, 20)]:
            if gran == G.WI and blocks > 64:
                continue
            threads = 32 if gran == G.WI else 256
            flags = gran | G.BLOCKING | (G.STRONG if gran == G.WI else G.RELAXED) | int(os.environ.get("PROBE_FLAGS", "0"))
            length = 4096
            callers = blocks * threads if gran == G.WI else blocks if gran == G.WG else 1
            buf = torch.zeros(callers * length, dtype=torch.uint8, device="cuda") if kind == "pread" else None
            args = (kind, flags, blocks, threads, 2)
            kw = dict(fd=fd, length=length, size=64 << 20, d_buf=buf) if kind == "pread" else {}
            W.bench_calls(*args, **kw)
            G.gsys_stats_reset()
            req0 = G.gsys_stats()["requests"]
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            n, ret, lat, _, rc = W.bench_calls(kind, flags, blocks, threads, iters, **kw)
            dt = time.perf_counter() - t0
            st = G.gsys_stats()
            lat_us = lat.double().cpu() / 1e3
            calls = st["requests"] - req0
            print(json.dumps({"kind": kind, "gran": {1: "wi", 2: "wg", 4: "kernel"}[gran], "blocks": blocks,
                              "callers": n, "iters": iters, "calls": calls, "calls_per_s": calls / dt,
                              "lat_p50_us": float(lat_us.median()), "lat_p99_us": float(lat_us.quantile(0.99)),
                              "busy_frac": st["ns_busy"] / 1e9 / dt / st["threads"],
                              "sys_us_per_call": st["ns_syscall"] / 1e3 / max(calls, 1),
                              "cuda_us_per_call": st["ns_cuda"] / 1e3 / max(calls, 1),
                              "busy_us_per_call": st["ns_busy"] / 1e3 / max(calls, 1),
                              "bundles": st["bundles"], "ok": bool((ret >= 0).all())}), flush=True)
os.close(fd)

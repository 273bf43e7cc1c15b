"""Where 4 KiB work-group preads spend their time, per buffer kind and blocking mode: rate, service
CPU time per request (busy / inside pread / CUDA API / bounce waits) and, with GSYS_DIAG_PHASES=1,
the GPU-side phases of blocking calls.  One JSON line per cell."""
import json
import os
import sys
import time

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_isca_veselybblor18_b200 import gsys as G  # noqa: E402
from paper_conf_isca_veselybblor18_b200 import workloads as W  # noqa: E402

W.ensure_init()
path = "/dev/shm/gsys_pp_probe.bin"
if not os.path.exists(path):
    with open(path, "wb") as f:
        f.write(os.urandom(64 << 20))
size = os.path.getsize(path)
fd = os.open(path, os.O_RDONLY)
blocks, threads, iters = 592, 256, int(os.environ.get("PP_ITERS", "1000"))
dbuf = torch.empty(blocks * 4096, dtype=torch.uint8, device="cuda")
hbuf = torch.empty(blocks * 4096, dtype=torch.uint8, pin_memory=True)
diag = os.environ.get("GSYS_DIAG_PHASES") == "1"
for name, flags, buf in (("wg_b_strong_host", G.WG | G.BLOCKING | G.HOSTBUF, hbuf),
                         ("wg_b_strong_device", G.WG | G.BLOCKING, dbuf),
                         ("wg_nb_strong_host", G.WG | G.NONBLOCKING | G.HOSTBUF, hbuf),
                         ("wg_nb_strong_device", G.WG | G.NONBLOCKING, dbuf),
                         ("wg_nb_relaxed_device", G.WG | G.NONBLOCKING | G.RELAXED, dbuf)):
    for rep in range(2):
        G.gsys_stats_reset()
        if diag:
            G.gsys_diag_phases(True)
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        _, ret, _, _, rc = W.bench_calls("pread", flags, blocks, threads, iters, fd, 4096, size, buf)
        dt = time.perf_counter() - t0
    st = G.gsys_stats()
    n = blocks * iters
    row = {"cell": name, "calls_per_s": n / dt, "rc": rc, "threads": st["threads"],
           "busy_us_per_req": st["ns_busy"] / n / 1e3, "syscall_us_per_req": st["ns_syscall"] / n / 1e3,
           "cuda_us_per_req": st["ns_cuda"] / n / 1e3, "bounce_wait_us_per_req": st["ns_bounce_wait"] / n / 1e3,
           "bundles": st["bundles"], "deferred": st["deferred"], "flushed": st["flushed"],
           "service_busy_frac": st["ns_busy"] / (st["threads"] * dt * 1e9)}
    if diag and not (flags & G.NONBLOCKING):
        row["gpu_phases"] = G.gsys_diag_phases(True)
    print(json.dumps(row), flush=True)
os.close(fd)

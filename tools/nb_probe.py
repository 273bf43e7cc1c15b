"""Non-blocking device-buffer preads (deferred pulls, reading B15): rate vs calls per caller, WG and
WI granularity, with the service counters.  One JSON line per cell."""
import json
import os
import sys
import time

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_isca_veselybblor18_b200 import gsys as G  # noqa: E402
from paper_conf_isca_veselybblor18_b200 import workloads as W  # noqa: E402

W.ensure_init()
path = "/dev/shm/gsys_nb_probe.bin"
if not os.path.exists(path):
    with open(path, "wb") as f:
        f.write(os.urandom(64 << 20))
size = os.path.getsize(path)
fd = os.open(path, os.O_RDONLY)
for gran, blocks, threads, iters_list in ((G.WG, 592, 256, (20, 200, 1000)), (G.WI, 592, 256, (1, 2, 4))):
    callers = blocks if gran == G.WG else blocks * threads
    dbuf = torch.empty(callers * 4096, dtype=torch.uint8, device="cuda")
    for iters in iters_list:
        G.gsys_stats_reset()
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        _, ret, _, _, rc = W.bench_calls("pread", gran | G.NONBLOCKING, blocks, threads, iters, fd, 4096, size, dbuf)
        dt = time.perf_counter() - t0
        st = G.gsys_stats()
        print(json.dumps({"gran": "wg" if gran == G.WG else "wi", "iters": iters, "calls": callers * iters,
                          "seconds": dt, "calls_per_s": callers * iters / dt, "rc": rc, "deferred": st["deferred"],
                          "flushed": st["flushed"], "ns_cuda": st["ns_cuda"]}), flush=True)
os.close(fd)

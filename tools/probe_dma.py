"""Where does a device-buffer (DMA-path) pread spend host-service time?  WI / WG non-blocking
4 KiB preads into device memory; prints rate and the service's per-call time breakdown."""
import json
import os
import sys
import time

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
for name, flags, blocks, threads, iters in [("wi_b", G.WI | G.BLOCKING, 64, 256, 4), ("wi_nb", G.WI | G.NONBLOCKING, 64, 256, 4),
                                            ("wg_nb", G.WG | G.NONBLOCKING, 592, 256, 100),
                                            ("wg_b_64k", G.WG | G.BLOCKING, 592, 256, 20)]:
    length = (64 << 10) if name.endswith("64k") else 4096
    callers = blocks * threads if flags & G.WI else blocks
    buf = torch.zeros(callers * length, dtype=torch.uint8, device="cuda")
    kw = dict(fd=fd, length=length, size=64 << 20, d_buf=buf)
    W.bench_calls("pread", flags, blocks, threads, 1, **kw)
    G.gsys_stats_reset()
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    n, ret, lat, _, rc = W.bench_calls("pread", flags, blocks, threads, iters, **kw)
    dt = time.perf_counter() - t0
    st = G.gsys_stats()
    calls = st["requests"]
    print(json.dumps({"case": name, "calls": calls, "calls_per_s": calls / dt, "rc": rc,
                      **{k: (v / 1e3 / max(calls, 1) if k.startswith("ns_") else v) for k, v in st.items()
                         if k != "per_nr"}}), flush=True)
os.close(fd)

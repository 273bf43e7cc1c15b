"""One bench_kernel launch for ncu (application replay): 592 work-groups x 256 threads, blocking
WG getrusage or 4 KiB device-buffer preads (pull path), 50 calls each."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_isca_veselybblor18_b200 import gsys as G  # noqa: E402
from paper_conf_isca_veselybblor18_b200 import workloads as W  # noqa: E402

kind = sys.argv[1] if len(sys.argv) > 1 else "getrusage"
W.ensure_init()
if kind == "getrusage":
    n, ret, lat, _, rc = W.bench_calls("getrusage", G.WG | G.BLOCKING | G.RELAXED, 592, 256, 50)
else:
    path = "/dev/shm/prof_calls.bin"
    if not os.path.exists(path):
        with open(path, "wb") as f:
            f.write(os.urandom(64 << 20))
    fd = os.open(path, os.O_RDONLY)
    buf = torch.zeros(592 * 4096, dtype=torch.uint8, device="cuda")
    n, ret, lat, _, rc = W.bench_calls("pread", G.WG | G.BLOCKING | G.RELAXED, 592, 256, 50, fd, 4096, 64 << 20, buf)
    os.close(fd)
print("ok", rc, int((ret >= 0).sum()))

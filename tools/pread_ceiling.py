"""Host pread ceiling for the wordcount's pattern (C threads, 256 KiB preads of the config-3 corpus
into the 296 pinned host-mapped lines the host-staging path uses), alone and while the copy engine
streams H2D.  Diagnostic only; prints JSON lines."""
import ctypes
import json
import os
import subprocess
import sys
import threading

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import inputs  # noqa: E402

HERE = os.path.dirname(os.path.abspath(__file__))
so = os.path.join(HERE, "probes", "libpread_probe.so")
subprocess.check_call(["gcc", "-O2", "-shared", "-fPIC", "-pthread", "-o", so, os.path.join(HERE, "probes", "pread_probe.c")])
lib = ctypes.CDLL(so)
lib.pread_probe.restype = ctypes.c_double
lib.pread_probe.argtypes = [ctypes.c_void_p, ctypes.c_int, ctypes.c_uint64, ctypes.c_void_p, ctypes.c_uint64,
                            ctypes.c_int, ctypes.c_int, ctypes.c_double]
corpus = inputs.make_corpus(512, 16 << 20)
fds = (ctypes.c_int * 512)(*[os.open(p, os.O_RDONLY) for p in corpus.paths])
chunk, nlines = 256 << 10, 296
lines = torch.empty(nlines * chunk, dtype=torch.uint8).pin_memory()
src = torch.empty(1 << 30, dtype=torch.uint8).pin_memory()
dst = torch.empty(1 << 30, dtype=torch.uint8, device="cuda")
for t in (1, 4, 8, 12, 14, 16):
    g = lib.pread_probe(fds, 512, 16 << 20, lines.data_ptr(), chunk, nlines, t, 1.5)
    print(json.dumps({"case": "pread_alone", "threads": t, "GBps": g / 1e9}), flush=True)
res = {}
th = threading.Thread(target=lambda: res.setdefault("g", lib.pread_probe(fds, 512, 16 << 20, lines.data_ptr(), chunk,
                                                                         nlines, 14, 2.0)))
s = torch.cuda.Stream()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
th.start()
with torch.cuda.stream(s):
    e0.record(s)
    for _ in range(60):
        dst.copy_(src, non_blocking=True)
    e1.record(s)
e1.synchronize()
th.join()
print(json.dumps({"case": "pread_14_plus_ce", "pread_GBps": res["g"] / 1e9,
                  "ce_GBps": 60 * (1 << 30) / (e0.elapsed_time(e1) / 1e3) / 1e9}), flush=True)

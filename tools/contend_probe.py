"""Is the ~49 GB/s wordcount ceiling the PCIe link or the host?  Measures, on the config-3 corpus:
(a) host preads alone (T threads, 256 KiB reads into distinct pinned lines -- what the service
does), (b) copy-engine H2D of a static pinned buffer alone, (c) both at once.  One JSON line per
case.  Diagnostic only (not part of the hot path)."""
import json
import os
import sys
import threading
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import inputs  # noqa: E402

corpus = inputs.make_corpus(512, 16 << 20)
CH = 256 << 10
NT = int(os.environ.get("T", "14"))
lines = torch.empty(NT * 8 * CH, dtype=torch.uint8).pin_memory()
import numpy as np  # noqa: E402
L = lines.numpy()
fds = [os.open(p, os.O_RDONLY) for p in corpus.paths]
stop = threading.Event()
count = [0] * NT


def reader(t):
    k = t
    nch = (16 << 20) // CH
    mv = memoryview(L)
    while not stop.is_set():
        f, c = divmod(k % (512 * nch), nch)
        slot = (t * 8 + (k // NT) % 8) * CH
        count[t] += os.preadv(fds[f], [mv[slot:slot + CH]], c * CH)
        k += NT


def run_preads(secs):
    for i in range(NT):
        count[i] = 0
    stop.clear()
    ths = [threading.Thread(target=reader, args=(t,)) for t in range(NT)]
    t0 = time.perf_counter()
    for th in ths:
        th.start()
    time.sleep(secs)
    stop.set()
    for th in ths:
        th.join()
    return sum(count) / (time.perf_counter() - t0) / 1e9


src = torch.empty(1 << 30, dtype=torch.uint8).pin_memory()
dst = torch.empty(1 << 30, dtype=torch.uint8, device="cuda")
s = torch.cuda.Stream()


def run_ce(reps):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with torch.cuda.stream(s):
        e0.record(s)
        for _ in range(reps):
            dst.copy_(src, non_blocking=True)
        e1.record(s)
    e1.synchronize()
    return reps * src.numel() / (e0.elapsed_time(e1) / 1e3) / 1e9


run_ce(2)
print(json.dumps({"case": "preads_alone", "threads": NT, "GBps": run_preads(2.0)}), flush=True)
print(json.dumps({"case": "ce_alone", "GBps": run_ce(40)}), flush=True)
res = {}
th = threading.Thread(target=lambda: res.setdefault("pr", run_preads(2.0)))
th.start()
time.sleep(0.2)
ce = run_ce(40)
th.join()
print(json.dumps({"case": "both", "threads": NT, "ce_GBps": ce, "preads_GBps": res["pr"]}), flush=True)

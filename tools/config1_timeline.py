"""Config 1 timeline from the protocol trace (timestamped slot transitions, gsys_set_trace +
gsys_clock_sync): per request the queueing (READY -> PROCESSING), host pread (PROCESSING ->
FINISHED), GPU notice (FINISHED -> FREE) and, per work-group, the scan gap until its next READY.
Usage: python tools/config1_timeline.py [chunk_kib] [staging host|device]"""
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import inputs  # noqa: E402
from paper_conf_isca_veselybblor18_b200 import gsys as G  # noqa: E402
from paper_conf_isca_veselybblor18_b200 import workloads as W  # noqa: E402

ck = int(sys.argv[1]) if len(sys.argv) > 1 else 256
staging = G.STAGE_DEVICE if (len(sys.argv) > 2 and sys.argv[2] == "device") else G.STAGE_HOST
W.ensure_init()
path = "/dev/shm/gsys_config1_16MiB.txt"
if not os.path.exists(path) or os.path.getsize(path) != (16 << 20):
    inputs.write_file(path, inputs.SEED_FILE16M, 0, 16 << 20)
fd = os.open(path, os.O_RDONLY)
words, pats = inputs.dictionary(), inputs.patterns()
h = torch.zeros(64, dtype=torch.int64, device="cuda")


def run():
    G.gsys_wordcount([fd], [16 << 20], ck << 10, words, pats, h, None, None, G.WG | G.BLOCKING | G.STRONG, 64, 256,
                     None, staging)
    G.gsys_wait(None)


for _ in range(3):
    run()
off, unc = G.gsys_clock_sync(256)
G.gsys_set_trace(True, 1 << 16)
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
run()
e1.record()
e1.synchronize()
gtr, htr = G.gsys_trace_read()
G.gsys_set_trace(False)
t = {}
for r in gtr + htr:
    ts = r[7] + (off if r[4] == "gpu" else 0)
    t.setdefault((r[0], r[1]), {})[(r[2], r[3])] = ts
reqs = [v for v in t.values() if len(v) == 5]
t0 = min(v[(0, 1)] for v in reqs)
q = [(v[(2, 3)] - v[(1, 2)]) / 1e3 for v in reqs]
pr = [(v[(3, 4)] - v[(2, 3)]) / 1e3 for v in reqs]
nt = [(v[(4, 0)] - v[(3, 4)]) / 1e3 for v in reqs]
ready = sorted((v[(1, 2)] - t0) / 1e3 for v in reqs)
fin = sorted((v[(3, 4)] - t0) / 1e3 for v in reqs)
free = sorted((v[(4, 0)] - t0) / 1e3 for v in reqs)


def st(x):
    return {"p50": statistics.median(x), "max": max(x), "mean": statistics.mean(x)}


print(json.dumps({"chunk_kib": ck, "staging": "host" if staging == G.STAGE_HOST else "device",
                  "device_ms": e0.elapsed_time(e1), "requests": len(reqs), "clock_unc_us": unc / 1e3,
                  "queue_us": st(q), "pread_us": st(pr), "gpu_notice_us": st(nt),
                  "first_ready_us": ready[0], "last_ready_us": ready[-1], "first_finished_us": fin[0],
                  "last_finished_us": fin[-1], "last_free_us": free[-1]}))
os.close(fd)

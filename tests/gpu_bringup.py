"""Step-by-step GPU bring-up of libgsys (run under gpurun with a timeout; not collected by pytest)."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import inputs  # noqa: E402
import oracle  # noqa: E402
from oracle import plan  # noqa: E402
from paper_conf_isca_veselybblor18_b200 import gsys as G  # noqa: E402
from paper_conf_isca_veselybblor18_b200 import workloads as W  # noqa: E402


def step(name):
    print(f"=== {name}", flush=True)


step("init")
t = time.time()
W.ensure_init()
print("init s", time.time() - t, G.gsys_stats(), flush=True)

step("getrusage WG blocking 1x1")
callers, r, lat, _, rc = W.bench_calls("getrusage", G.WG, 1, 32, 1)
torch.cuda.synchronize()
print(callers, r.cpu().tolist(), lat.cpu().tolist(), rc, G.gsys_stats(), flush=True)

step("getrusage WG blocking 148x4 blocks x 10 iters")
t = time.time()
callers, r, lat, _, rc = W.bench_calls("getrusage", G.WG, 592, 256, 10)
dt = time.time() - t
print(callers, "all0", bool((r == 0).all()), "calls/s", callers * 10 / dt, "lat p50 us",
      lat.float().median().item() / 1e3, flush=True)

d = "/dev/shm/gsys_dbg"
os.makedirs(d, exist_ok=True)
p = os.path.join(d, "f16m.txt")
inputs.write_file(p, 1, 0, 16 << 20)
step("pread WG blocking")
fd = os.open(p, os.O_RDONLY)
buf = torch.zeros(64 * 4096, dtype=torch.uint8, device="cuda")
callers, r, lat, s, rc = W.bench_calls("pread", G.WG, 64, 128, 3, fd, 4096, 16 << 20, buf, want_sum=True)
data = open(p, "rb").read()
exp_ret = [plan.expected_pread_ret(16 << 20, ((c * 3 + i) * 4096) % (16 << 20), 4096) for c in range(64) for i in range(3)]
exp_sum = [sum(data[((c * 3 + i) * 4096) % (16 << 20):][:4096]) for c in range(64) for i in range(3)]
print("ret ok", r.cpu().tolist() == exp_ret, "sum ok", s.cpu().tolist() == exp_sum, rc, flush=True)

step("wordcount 16 MiB, 64 WGs")
words, pats = inputs.dictionary(), inputs.patterns()
t = time.time()
res = W.wordcount_files([p], words, pats)
dt = time.time() - t
hist_o = oracle.count_tokens(data, words)
print("hist ok", [int(x) for x in res.hist.tolist()] == [int(x) for x in hist_o], "rc", res.wait_rc, "s", dt, flush=True)
print("req_ret", res.req_ret[:4].tolist(), res.req_ret[-2:].tolist(), flush=True)
for i in range(3):
    torch.cuda.synchronize()
    t = time.time()
    res = W.wordcount_files([p], words, pats)
    dt = time.time() - t
    print(f"wordcount e2e {16 / 1024 / dt:.2f} GB/s ({dt * 1e3:.2f} ms)", flush=True)
print(G.gsys_stats(), flush=True)
G.gsys_shutdown()
print("done", flush=True)

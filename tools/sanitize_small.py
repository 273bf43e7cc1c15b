"""Small end-to-end run of every kernel for compute-sanitizer (memcheck / racecheck / synccheck)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import inputs
from paper_conf_isca_veselybblor18_b200 import gsys as G
from paper_conf_isca_veselybblor18_b200 import workloads as W
words, pats = inputs.dictionary(), inputs.patterns()
d = "/dev/shm/gsys_san"
os.makedirs(d, exist_ok=True)
p = os.path.join(d, "f.txt")
inputs.write_file(p, 1, 0, (1 << 20) + 77, grep_plants=True)
for st in (G.STAGE_HOST, G.STAGE_DEVICE, G.STAGE_MIXED(5)):
    r = W.wordcount_files([p], words, pats, chunk=64 << 10, staging=st, blocks=8)
    print("wc", st, int(r.hist.sum()), r.wait_rc)
# pull path (reading B12): 4113-byte work-group preads into unaligned device lines
r = W.wordcount_files([p], words, pats, chunk=4096, staging=G.STAGE_DEVICE, blocks=8)
print("wc-pull", int(r.hist.sum()), r.wait_rc)
fd = os.open(p, os.O_RDONLY)
dbuf = torch.zeros(64 * 1000 + 64, dtype=torch.uint8, device="cuda")
for fl, ln in ((G.WG | G.BLOCKING, 1000), (G.WI | G.BLOCKING, 200), (G.KERNEL | G.BLOCKING | G.RELAXED, 100)):
    n, ret, lat, sm, rc = W.bench_calls("pread", fl, 4, 64, 2, fd, ln, (1 << 20), dbuf[1:], want_sum=True)
    print("pull", fl, rc, int((ret == ln).sum()))
os.close(fd)
buf, _, _ = inputs.gen_bytes(2, 0, (1 << 20) + 5)
t = torch.zeros(buf.size + 64, dtype=torch.uint8, device="cuda")
t[:buf.size].copy_(torch.from_numpy(buf))
h = torch.zeros(64, dtype=torch.int64, device="cuda")
G.gsys_scan_device(t, buf.size, 4096, words, pats, h, None, 8, 512)
torch.cuda.synchronize()
print("scan", int(h.sum()))
for fl in (G.WI | G.BLOCKING, G.WG | G.NONBLOCKING | G.RELAXED, G.KERNEL | G.BLOCKING | G.RELAXED):
    n, ret, lat, _, rc = W.bench_calls("getrusage", fl, 4, 64, 2)
    print("calls", fl, rc, int((ret == 0).sum()))
# round 2: pull completion from the bounce (default; large chunks), non-blocking prefetch waiting on
# explicit tokens, token-level scan, split large preads, both completion modes of device staging
for ck in (256 << 10, 64 << 10):
    r = W.wordcount_files([p], words, pats, chunk=ck, staging=G.STAGE_DEVICE, blocks=4)
    print("wc-pullb", ck, int(r.hist.sum()), r.wait_rc)
    r = W.wordcount_files([p], words, pats, chunk=ck, staging=G.STAGE_DEVICE, blocks=4,
                          gflags=G.WG | G.NONBLOCKING | G.RELAXED)
    print("wc-prefetch", ck, int(r.hist.sum()), r.wait_rc)
prev = G.gsys_set_scan(G.SCAN_TOKEN)
r = W.wordcount_files([p], words, pats, chunk=64 << 10, staging=G.STAGE_DEVICE, blocks=4)
print("wc-token", int(r.hist.sum()), r.wait_rc)
h.zero_()
G.gsys_scan_device(t, buf.size, 4096, words, pats, h, None, 8, 512)
torch.cuda.synchronize()
print("scan-token", int(h.sum()))
G.gsys_set_scan(prev)
G.gsys_set_completion(G.COMPLETION_MEMOP)
r = W.wordcount_files([p], words, pats, chunk=64 << 10, staging=G.STAGE_DEVICE, blocks=4)
print("wc-memop", int(r.hist.sum()), r.wait_rc)
G.gsys_set_completion(G.COMPLETION_PULL)
fd = os.open(p, os.O_RDONLY)
big = torch.zeros((1 << 20) + 64, dtype=torch.uint8, device="cuda")
n, ret, lat, sm, rc = W.bench_calls("pread", G.WG | G.BLOCKING, 1, 128, 1, fd, 1 << 20, (1 << 20) + 77, big, want_sum=True)
print("split", rc, int(ret[0]))
# deferred pulls (B15): non-blocking device-buffer preads landed by gsys_wait's flush kernel
small = torch.zeros(8 * 4096, dtype=torch.uint8, device="cuda")
n, ret, lat, sm, rc = W.bench_calls("pread", G.WG | G.NONBLOCKING, 8, 64, 2, fd, 4096, (1 << 20) + 77, small)
print("deferred", rc, G.gsys_stats()["deferred"])
# warp-copied work-item pulls, block-copied kernel-scope pulls, warp-consumed deferred pulls,
# a stream-scoped flush
mid = torch.zeros(4 * 64 * 5000, dtype=torch.uint8, device="cuda")
for fl, ln in ((G.WI | G.BLOCKING, 5000), (G.KERNEL | G.BLOCKING | G.RELAXED, 100000), (G.WI | G.NONBLOCKING, 4096)):
    n, ret, lat, sm, rc = W.bench_calls("pread", fl, 4, 64, 2, fd, ln, (1 << 20) + 77, mid)
    print("coop", fl, rc, int((ret >= 0).sum()))
side = torch.cuda.Stream()
n, ret, lat, sm, rc = W.bench_calls("pread", G.WG | G.NONBLOCKING, 8, 64, 2, fd, 4096, (1 << 20) + 77, small, stream=side)
print("stream-flush", rc)
os.close(fd)
print("ok")

"""Parameter sweep of the GPU-syscall wordcount on the config-3 corpus (one process per point,
since GSYS_THREADS / GSYS_BOUNCE_MB are read at gsys_init).  Prints one JSON line."""
import argparse
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import inputs  # noqa: E402
from paper_conf_isca_veselybblor18_b200 import gsys as G  # noqa: E402
from paper_conf_isca_veselybblor18_b200 import workloads as W  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--files", type=int, default=512)
ap.add_argument("--file-mib", type=int, default=16)
ap.add_argument("--chunk-kib", type=int, default=256)
ap.add_argument("--blocks", type=int, default=0)
ap.add_argument("--threads", type=int, default=256)
ap.add_argument("--order", default="relaxed")
ap.add_argument("--nonblocking", type=int, default=0, help="1: WG non-blocking prefetch pipeline")
ap.add_argument("--cmax", type=int, default=8)
ap.add_argument("--window", type=int, default=0)
ap.add_argument("--merge", type=int, default=1)
ap.add_argument("--steps", type=int, default=3)
ap.add_argument("--staging", default="device", choices=["device", "host", "mixed"])
ap.add_argument("--dev16", type=int, default=4)
a = ap.parse_args()

corpus = inputs.make_corpus(a.files, a.file_mib << 20)
words, pats = inputs.dictionary(), inputs.patterns()
W.ensure_init()
G.gsys_set_profile(True)
G.gsys_set_coalesce_max(a.cmax)
G.gsys_set_coalesce_window(a.window)
G.gsys_set_merge(a.merge)
gflags = G.WG | (G.NONBLOCKING if a.nonblocking else G.BLOCKING) | (G.RELAXED if a.order == "relaxed" else G.STRONG)
of = W.OpenFiles(corpus.paths).__enter__()
s = torch.cuda.Stream()
h = torch.zeros(64, dtype=torch.int64, device="cuda")
hits = torch.zeros(len(of.fds), dtype=torch.int32, device="cuda")
with torch.cuda.stream(s):
    stg = {"host": G.STAGE_HOST, "device": G.STAGE_DEVICE}.get(a.staging) or G.STAGE_MIXED(a.dev16)
    G.gsys_wordcount(of.fds, of.sizes, a.chunk_kib << 10, words, pats, h, hits, None, gflags, a.blocks, a.threads, s,
                     stg)
    G.gsys_wait(s)
    G.gsys_stats_reset()
    G.gsys_read_profile(True)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    t0 = time.perf_counter()
    e0.record(s)
    for _ in range(a.steps):
        h.zero_()
        G.gsys_wordcount(of.fds, of.sizes, a.chunk_kib << 10, words, pats, h, hits, None, gflags, a.blocks,
                         a.threads, s, stg)
        G.gsys_wait(s)
    e1.record(s)
    e1.synchronize()
    wall = time.perf_counter() - t0
ok = bool((h.cpu().numpy().astype("uint64") == corpus.census).all())
st = G.gsys_stats()
pf = G.gsys_read_profile(True)
dt = e0.elapsed_time(e1) / 1e3
print(json.dumps({"GBps": corpus.total_bytes * a.steps / dt / 1e9, "wall_GBps": corpus.total_bytes * a.steps / wall / 1e9,
                  "ok": ok, "threads_env": os.environ.get("GSYS_THREADS"), **vars(a),
                  "bundles": st["bundles"] / a.steps, "host_preads": st["host_preads"] / a.steps,
                  "merged": st["merged"] / a.steps, "service_threads": st["threads"],
                  "busy_s": st["ns_busy"] / 1e9 / a.steps, "sys_s": st["ns_syscall"] / 1e9 / a.steps,
                  "cuda_s": st["ns_cuda"] / 1e9 / a.steps, "bwait_s": st["ns_bounce_wait"] / 1e9 / a.steps,
                  "step_s": dt / a.steps, "wg_wait_us": pf["wait_ns"] / max(pf["chunks"], 1) / 1e3,
                  "wg_scan_us": pf["scan_ns"] / max(pf["chunks"], 1) / 1e3}), flush=True)

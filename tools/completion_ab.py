"""A/B of the completion paths for blocking work-group preads into device memory
(include/gsys.h GSYS_COMPLETION_*): config 1 with device staging, the 8 GiB corpus with device
staging, and WG 64 KiB device-buffer preads.  One JSON line per (mode, case)."""
import json
import os
import sys
import time

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import inputs  # noqa: E402
from paper_conf_isca_veselybblor18_b200 import gsys as G  # noqa: E402
from paper_conf_isca_veselybblor18_b200 import workloads as W  # noqa: E402


def dev_time(fn, reps, warm=2):
    s = torch.cuda.current_stream()
    for _ in range(warm):
        fn()
    ts = []
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        fn()
        e1.record(s)
        e1.synchronize()
        ts.append(e0.elapsed_time(e1))
    ts.sort()
    return ts[len(ts) // 2]


def main():
    W.ensure_init()
    words, pats = inputs.dictionary(), inputs.patterns()
    nfiles = int(os.environ.get("AB_FILES", "512"))
    corpus = inputs.make_corpus(nfiles, 16 << 20)
    p1 = "/dev/shm/gsys_config1_16MiB.txt"
    if not os.path.exists(p1):
        inputs.write_file(p1, inputs.SEED_FILE16M, 0, 16 << 20)
    fd1 = os.open(p1, os.O_RDONLY)
    of = W.OpenFiles(corpus.paths).__enter__()
    h = torch.zeros(64, dtype=torch.int64, device="cuda")
    hits = torch.zeros(nfiles, dtype=torch.int32, device="cuda")
    dbuf = torch.empty(592 * 65536, dtype=torch.uint8, device="cuda")
    for mode, name in ((G.COMPLETION_MEMOP, "memop"), (G.COMPLETION_HOST, "host"), (G.COMPLETION_PULL, "pull")):
        G.gsys_set_completion(mode)
        for strong in (True, False):
            fl = G.WG | G.BLOCKING | (G.STRONG if strong else G.RELAXED)

            def c1():
                h.zero_()
                G.gsys_wordcount([fd1], [16 << 20], 256 << 10, words, pats, h, None, None, fl, 0, 256, None,
                                 G.STAGE_DEVICE)
                G.gsys_wait(None)
            ms = dev_time(c1, 15)
            print(json.dumps({"mode": name, "case": "config1_device", "strong": strong, "ms": ms,
                              "GBps": (16 << 20) / ms / 1e6}), flush=True)

        def big():
            h.zero_()
            hits.zero_()
            G.gsys_wordcount(of.fds, of.sizes, 256 << 10, words, pats, h, hits, None, G.WG | G.BLOCKING | G.RELAXED,
                             148, 256, None, G.STAGE_DEVICE)
            G.gsys_wait(None)
        ms = dev_time(big, 3, 1)
        ok = bool((h.cpu().numpy().astype("uint64") == corpus.census).all())
        print(json.dumps({"mode": name, "case": "corpus_device_148wg", "ms": ms,
                          "GBps": corpus.total_bytes / ms / 1e6, "parity": ok}), flush=True)
        t0 = time.perf_counter()
        _, ret, lat, _, rc = W.bench_calls("pread", G.WG | G.BLOCKING | G.RELAXED, 592, 256, 20, fd1, 65536,
                                           16 << 20, dbuf)
        dt = time.perf_counter() - t0
        print(json.dumps({"mode": name, "case": "wg_pread64k_device", "calls_per_s": 592 * 20 / dt,
                          "GBps": 592 * 20 * 65536 / dt / 1e9, "ok": bool((ret == 65536).all()) and rc == 0}),
              flush=True)
    G.gsys_set_completion(G.COMPLETION_PULL)
    of.__exit__()
    os.close(fd1)


if __name__ == "__main__":
    main()

"""Config 1 (16 MiB, 64 WGs, WG + blocking + strong): where the time goes per chunk size, WG size and staging --
per-chunk time in the call vs scanning (gsys_set_profile), kernel vs launch overheads."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import inputs  # noqa: E402
from paper_conf_isca_veselybblor18_b200 import gsys as G  # noqa: E402
from paper_conf_isca_veselybblor18_b200 import workloads as W  # noqa: E402

W.ensure_init()
path = "/dev/shm/gsys_config1_16MiB.txt"
if not os.path.exists(path) or os.path.getsize(path) != (16 << 20):
    inputs.write_file(path, inputs.SEED_FILE16M, 0, 16 << 20)
fd = os.open(path, os.O_RDONLY)
words, pats = inputs.dictionary(), inputs.patterns()
s = torch.cuda.Stream()
h = torch.zeros(64, dtype=torch.int64, device="cuda")
G.gsys_set_profile(True)
cells = [(t, ck, st) for st in (G.STAGE_HOST, G.STAGE_DEVICE) for ck in (256, 128, 64) for t in (256, 128)]
for threads, ck, staging in cells:
    res = []
    for rep in range(13):
        G.gsys_read_profile(True)
        G.gsys_stats_reset()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        G.gsys_wordcount([fd], [16 << 20], ck << 10, words, pats, h, None, None, G.WG | G.BLOCKING | G.STRONG, 64,
                         threads, s, staging)
        e1.record(s)
        G.gsys_wait(s)
        e1.synchronize()
        pf = G.gsys_read_profile(True)
        st = G.gsys_stats()
        if rep >= 3:
            res.append({"ms": e0.elapsed_time(e1), "wait_us_per_chunk": pf["wait_ns"] / max(pf["chunks"], 1) / 1e3,
                        "scan_us_per_chunk": pf["scan_ns"] / max(pf["chunks"], 1) / 1e3, "bundles": st["bundles"],
                        "svc_sys_us_per_call": st["ns_syscall"] / 1e3 / 64})
    res.sort(key=lambda r: r["ms"])
    print(json.dumps({"threads": threads, "chunk_kib": ck, "staging": "host" if staging == G.STAGE_HOST else "device",
                      "chunks": (16 << 10) // ck, **res[len(res) // 2]}), flush=True)
os.close(fd)

"""Phase sums (GSYS_DIAG_PHASES) of the memcached GPU server's blocking calls (recvfrom + sendto)
at 32 and 128 work-groups; JSON lines."""
import json
import os
import sys

os.environ["GSYS_DIAG_PHASES"] = "1"
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

from inputs import mc as MC  # noqa: E402
from paper_conf_isca_veselybblor18_b200 import gsys as G  # noqa: E402
from paper_conf_isca_veselybblor18_b200 import workloads as W  # noqa: E402

W.ensure_init()
keys, vals = MC.dataset(64 * 16 * 3 // 4, vlen=1024)
pkts = [MC.encode_get(i, k) for i, k in enumerate(MC.requests(keys, 30000))]
for nwg, cthr, win in ((32, 4, 8), (128, 8, 32)):
    G.gsys_diag_phases(True)
    G.gsys_stats_reset()
    resp, lat, secs, st = W.mc_serve_run(keys, vals, pkts, nwg=nwg, nbuckets=64, bucket_cap=32, client_threads=cthr,
                                         window=win, send_gflags=G.WG | G.BLOCKING | G.RELAXED)
    ph = G.gsys_diag_phases(True)
    s = G.gsys_stats()
    print(json.dumps({"work_groups": nwg, "in_flight": cthr * win, "req_per_s": len(pkts) / secs,
                      "lat_p50_us": float(np.median(np.array(lat) / 1e3)), **ph,
                      "svc_busy_us_per_call": s["ns_busy"] / 1e3 / max(ph["calls"], 1),
                      "svc_sys_us_per_call": s["ns_syscall"] / 1e3 / max(ph["calls"], 1)}), flush=True)

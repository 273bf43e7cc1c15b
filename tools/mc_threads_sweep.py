"""Config 4 under high offered load (8 client threads x 32 in flight, 128 work-groups) for one
service-thread count (env GSYS_THREADS, read at gsys_init): the load generator and the service
share the host's cores.  One JSON line per send mode."""
import json
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from inputs import mc as MC  # noqa: E402
from oracle import mc as OM  # noqa: E402
from paper_conf_isca_veselybblor18_b200 import gsys as G  # noqa: E402
from paper_conf_isca_veselybblor18_b200 import workloads as W  # noqa: E402

W.ensure_init()
keys, vals = MC.dataset(64 * 16 * 3 // 4, vlen=1024)
table = dict(zip(keys, vals))
pkts = [MC.encode_get(i, k) for i, k in enumerate(MC.requests(keys, 60000))]
nwg = int(os.environ.get("MC_WGS", "128"))
for send in ("blocking", "nonblocking"):
    sg = G.WG | G.RELAXED | (G.NONBLOCKING if send == "nonblocking" else G.BLOCKING)
    resp, lat, secs, _ = W.mc_serve_run(keys, vals, pkts, nwg=nwg, nbuckets=64, bucket_cap=32, client_threads=8,
                                        window=32, send_gflags=sg)
    ok = sum(1 for p, r in zip(pkts, resp) if r == OM.expected_response(p, table))
    lat_us = np.array(lat, dtype=np.float64) / 1e3
    print(json.dumps({"service_threads": G.gsys_stats()["threads"], "work_groups": nwg, "sendto": send,
                      "req_per_s": len(pkts) / secs, "lat_p50_us": float(np.median(lat_us)),
                      "exact": ok == len(pkts)}), flush=True)

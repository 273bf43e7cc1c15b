"""Config-4 load sweep: GPU memcached server (work-group recvfrom/sendto) vs the CPU oracle server
at increasing client concurrency (client threads x window = requests in flight).  JSON lines."""
import ctypes
import json
import os
import sys
import threading

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
from inputs import mc as MC  # noqa: E402
from oracle import mc as OM  # noqa: E402
from paper_conf_isca_veselybblor18_b200 import gsys as G  # noqa: E402
from paper_conf_isca_veselybblor18_b200 import workloads as W  # noqa: E402

W.ensure_init()
per_bucket, nbuckets = 16, 64
keys, vals = MC.dataset(nbuckets * per_bucket * 3 // 4, vlen=1024)
reqs = MC.requests(keys, 60000)
pkts = [MC.encode_get(i, k) for i, k in enumerate(reqs)]
table = dict(zip(keys, vals))
want = [OM.expected_response(p, table) for p in pkts]
kb, ko, kl, vb, vo, vl = MC.pack(keys, vals)
for cthr, win in ((4, 8), (4, 32), (8, 32)):
    for nwg in (32, 64, 128):
        for send in ("blocking", "nonblocking"):
            sg = G.WG | G.RELAXED | (G.NONBLOCKING if send == "nonblocking" else G.BLOCKING)
            resp, lat, secs, st = W.mc_serve_run(keys, vals, pkts, nwg=nwg, nbuckets=nbuckets,
                                                 bucket_cap=per_bucket * 2, client_threads=cthr, window=win,
                                                 send_gflags=sg)
            ok = sum(1 for r, w in zip(resp, want) if r == w)
            print(json.dumps({"server": "gpu", "in_flight": cthr * win, "client_threads": cthr, "work_groups": nwg,
                              "sendto": send, "req_per_s": len(pkts) / secs,
                              "lat_p50_us": float(np.median(np.array(lat) / 1e3)), "exact": ok, "n": len(pkts)}),
                  flush=True)
    for sthr in (4, 8):
        sock = MC.udp_server_socket()
        stop = ctypes.c_int(0)
        th = threading.Thread(target=lambda: oracle.lib().oracle_mc_serve(
            sock.fileno(), sthr, kb.ctypes.data, ko.ctypes.data, kl.ctypes.data, vb.ctypes.data, vo.ctypes.data,
            vl.ctypes.data, len(keys), nbuckets, ctypes.addressof(stop)))
        th.start()
        try:
            resp, lat, secs = MC.run_client(sock.getsockname()[1], pkts, nthreads=cthr, window=win)
        finally:
            stop.value = 1
            th.join()
            sock.close()
        ok = sum(1 for r, w in zip(resp, want) if r == w)
        print(json.dumps({"server": "cpu-oracle", "in_flight": cthr * win, "client_threads": cthr, "threads": sthr,
                          "req_per_s": len(pkts) / secs, "lat_p50_us": float(np.median(np.array(lat) / 1e3)),
                          "exact": ok, "n": len(pkts)}), flush=True)

"""Config 4 plumbing without a GPU: the load generator + the oracle's CPU server reproduce the
protocol definition (oracle/mc.py) for every request, including misses."""
import ctypes
import threading

import numpy as np

import oracle
from inputs import mc as MC
from oracle import mc as OM


def test_cpu_server_matches_definition():
    keys, vals = MC.dataset(2000, vlen=(64, 1500))
    reqs = MC.requests(keys, 3000)
    pkts = [MC.encode_get(i, k) for i, k in enumerate(reqs)]
    kb, ko, kl, vb, vo, vl = MC.pack(keys, vals)
    sock = MC.udp_server_socket()
    stop = ctypes.c_int(0)
    res = {}

    def serve():
        res["served"] = oracle.lib().oracle_mc_serve(sock.fileno(), 2, kb.ctypes.data, ko.ctypes.data, kl.ctypes.data,
                                                      vb.ctypes.data, vo.ctypes.data, vl.ctypes.data, len(keys), 16,
                                                      ctypes.addressof(stop))
    th = threading.Thread(target=serve)
    th.start()
    try:
        resp, lat, secs = MC.run_client(sock.getsockname()[1], pkts, nthreads=2, window=8)
    finally:
        stop.value = 1
        th.join()
        sock.close()
    table = dict(zip(keys, vals))
    for p, r in zip(pkts, resp):
        assert r == OM.expected_response(p, table)
    assert res["served"] == len(pkts)
    assert sum(1 for k in reqs if k not in table) > 0


def test_expected_response_format():
    table = {b"k" * 16: b"v" * 100}
    p = MC.encode_get(7, b"k" * 16)
    r = OM.expected_response(p, table)
    assert r[8] == 0x81 and r[14:16] == b"\0\0" and r[-100:] == b"v" * 100 and len(r) == 36 + 100
    r = OM.expected_response(MC.encode_get(8, b"x" * 20), table)
    assert r[15] == 1 and r.endswith(b"Not found")
    assert OM.expected_response(b"\0" * 40, table) is None

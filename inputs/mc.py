"""Seeded memcached-style key/value data and UDP request traffic (config 4, sec. VIII-D).

Input construction only: the key/value set, the request stream and the request packets (memcached
binary protocol over UDP: an 8-byte UDP frame header + the 24-byte binary request header + key).
The load generator that sends them and collects the replies is ``mc_client.c`` (compiled with gcc).
"""
from __future__ import annotations

import ctypes
import os
import struct
import subprocess
import threading

import numpy as np

SEED_MC = 8
OPAQUE_BASE = 0x10000000

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "mc_client.c")
_LIB = os.path.join(_HERE, "libmcclient.so")
_lock = threading.Lock()
_lib = None


def dataset(nkeys: int, seed: int = SEED_MC, klen=(16, 32), vlen=(64, 4096)):
    """nkeys unique alphanumeric keys (klen bytes) and values (vlen bytes; an int fixes the size)."""
    rng = np.random.default_rng(seed)
    alpha = np.frombuffer(b"abcdefghijklmnopqrstuvwxyzABCDEFGHIJKLMNOPQRSTUVWXYZ0123456789", dtype=np.uint8)
    keys, seen = [], set()
    while len(keys) < nkeys:
        L = int(rng.integers(klen[0], klen[1] + 1))
        k = alpha[rng.integers(0, len(alpha), size=L)].tobytes()
        if k not in seen:
            seen.add(k)
            keys.append(k)
    if isinstance(vlen, int):
        lens = np.full(nkeys, vlen)
    else:
        lens = rng.integers(vlen[0], vlen[1] + 1, size=nkeys)
    vals = [rng.integers(0, 256, size=int(n), dtype=np.uint8).tobytes() for n in lens]
    return keys, vals


def requests(keys, nreq: int, seed: int = SEED_MC + 1, miss_frac: float = 0.1, zipf_s: float = 0.99):
    """Requested keys: Zipf-popular existing keys, plus miss_frac keys that do not exist."""
    rng = np.random.default_rng(seed)
    n = len(keys)
    w = 1.0 / np.arange(1, n + 1) ** zipf_s
    w /= w.sum()
    idx = rng.choice(n, size=nreq, p=w)
    out = [keys[i] for i in idx]
    for j in np.nonzero(rng.random(nreq) < miss_frac)[0]:
        out[j] = b"miss-" + rng.integers(0, 10, size=14).astype(np.uint8).tobytes().translate(
            bytes.maketrans(bytes(range(10)), b"0123456789"))
    return out


def encode_get(index: int, key: bytes) -> bytes:
    """UDP frame header (request id, seq 0, total 1, reserved) + binary GET request.
    The opaque field carries OPAQUE_BASE + index so replies match requests one to one."""
    frame = struct.pack(">HHHH", index & 0xFFFF, 0, 1, 0)
    hdr = struct.pack(">BBHBBHIIQ", 0x80, 0x00, len(key), 0, 0, 0, len(key), OPAQUE_BASE + index, 0)
    return frame + hdr + key


def build() -> str:
    if (not os.path.exists(_LIB)) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-shared", "-fPIC", "-pthread", "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


def _client():
    global _lib
    with _lock:
        if _lib is None:
            build()
            L = ctypes.CDLL(_LIB)
            L.mc_client_run.restype = ctypes.c_int
            L.mc_client_run.argtypes = [ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p,
                                        ctypes.c_uint32, ctypes.c_int, ctypes.c_int, ctypes.c_void_p,
                                        ctypes.c_uint32, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_double,
                                        ctypes.c_void_p]
            _lib = L
    return _lib


def run_client(port: int, packets, nthreads: int = 4, window: int = 16, resp_stride: int = 4200,
               timeout_s: float = 30.0):
    """Send every packet to 127.0.0.1:port from nthreads sockets keeping <= window requests in
    flight per socket; return (responses list (bytes or None), latencies ns, wall seconds)."""
    n = len(packets)
    blob = b"".join(packets)
    off = np.zeros(n, dtype=np.uint32)
    ln = np.array([len(p) for p in packets], dtype=np.uint32)
    if n:
        off[1:] = np.cumsum(ln)[:-1]
    src = np.frombuffer(blob, dtype=np.uint8).copy() if blob else np.zeros(1, dtype=np.uint8)
    resp = np.zeros(n * resp_stride, dtype=np.uint8)
    rlen = np.zeros(n, dtype=np.uint32)
    lat = np.zeros(n, dtype=np.uint64)
    secs = ctypes.c_double(0)
    rc = _client().mc_client_run(port, src.ctypes.data, off.ctypes.data, ln.ctypes.data, n, nthreads, window,
                                 resp.ctypes.data, resp_stride, rlen.ctypes.data, lat.ctypes.data, timeout_s,
                                 ctypes.addressof(secs))
    if rc < 0:
        raise OSError(-rc, "mc_client_run")
    out = [bytes(resp[i * resp_stride: i * resp_stride + rlen[i]]) if rlen[i] else None for i in range(n)]
    return out, lat, secs.value


def pack(keys, vals):
    """Flat arrays for the C/CUDA side: (key blob, key offsets u32, key lengths u8, value blob,
    value offsets u64, value lengths u32)."""
    kb = b"".join(keys)
    ko = np.zeros(len(keys), dtype=np.uint32)
    kl = np.array([len(k) for k in keys], dtype=np.uint8)
    if len(keys):
        ko[1:] = np.cumsum(kl.astype(np.uint64))[:-1]
    vb = b"".join(vals)
    vo = np.zeros(len(vals), dtype=np.uint64)
    vl = np.array([len(v) for v in vals], dtype=np.uint32)
    if len(vals):
        vo[1:] = np.cumsum(vl.astype(np.uint64))[:-1]
    return (np.frombuffer(kb, dtype=np.uint8).copy(), ko, kl, np.frombuffer(vb, dtype=np.uint8).copy(), vo, vl)


def udp_server_socket(rcvbuf: int = 8 << 20, timeout_s: float = 0.02):
    """A UDP socket bound to 127.0.0.1:<ephemeral> with a receive timeout (for the servers)."""
    import socket
    s = socket.socket(socket.AF_INET, socket.SOCK_DGRAM)
    s.setsockopt(socket.SOL_SOCKET, socket.SO_RCVBUF, rcvbuf)
    s.setsockopt(socket.SOL_SOCKET, socket.SO_SNDBUF, rcvbuf)
    s.bind(("127.0.0.1", 0))
    sec = int(timeout_s)
    s.setsockopt(socket.SOL_SOCKET, socket.SO_RCVTIMEO, struct.pack("ll", sec, int((timeout_s - sec) * 1e6)))
    return s

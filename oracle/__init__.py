"""CPU ORACLE for the GENESYS hot path -- TEST INFRASTRUCTURE ONLY.

Only tests/, ``__graft_entry__.smoke()`` and bench.py's ``cpu_baseline`` / ``--impl reference``
leg may import this package.  It shares no code with the CUDA path
(``paper_conf_isca_veselybblor18_b200``) and never imports it; the only thing the two sides
share is the seeded input generator in ``inputs/`` (input construction, no method arithmetic).

Contents (each function cites the PAPER.md passage it follows):
  * ``oracle.c``  -- plain C: direct pread(2), scalar whole-token wordcount, grep -F -l, direct
    syscall rates (compiled with plain ``gcc -O2``; never tuned).
  * ``protocol.py`` -- the slot state machine of PAPER.md:24 sec. VI and a trace checker.
  * ``plan.py``   -- request plans: which (fd, off, len) each GPU caller issues per granularity.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lock = threading.Lock()
_lib = None

DSTRIDE = 17


def build() -> str:
    """Compile oracle.c with plain gcc -O2 (the checker is built, never used, by build())."""
    if (not os.path.exists(_LIB)) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-shared", "-fPIC", "-pthread", "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


def lib():
    global _lib
    with _lock:
        if _lib is None:
            build()
            L = ctypes.CDLL(_LIB)
            L.oracle_pread.restype = ctypes.c_int64
            L.oracle_pread.argtypes = [ctypes.c_int, ctypes.c_void_p, ctypes.c_uint64, ctypes.c_int64]
            L.oracle_exec_plan.argtypes = [ctypes.c_int] + [ctypes.c_void_p] * 6
            L.oracle_count_tokens.argtypes = [ctypes.c_void_p, ctypes.c_uint64, ctypes.c_char_p,
                                              ctypes.c_void_p, ctypes.c_int, ctypes.c_void_p]
            L.oracle_grep.argtypes = [ctypes.c_void_p, ctypes.c_uint64, ctypes.c_char_p, ctypes.c_void_p,
                                      ctypes.c_int]
            L.oracle_read_file_plan.argtypes = [ctypes.c_int, ctypes.c_uint64, ctypes.c_uint64,
                                                ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p]
            L.oracle_corpus.argtypes = [ctypes.c_void_p, ctypes.c_int, ctypes.c_int, ctypes.c_uint64,
                                        ctypes.c_char_p, ctypes.c_void_p, ctypes.c_int,
                                        ctypes.c_char_p, ctypes.c_void_p, ctypes.c_int,
                                        ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p]
            L.oracle_syscall_rate.restype = ctypes.c_double
            L.oracle_syscall_rate.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_uint64, ctypes.c_int,
                                              ctypes.c_uint64, ctypes.c_uint64]
            L.oracle_mc_serve.restype = ctypes.c_int64
            L.oracle_mc_serve.argtypes = [ctypes.c_int, ctypes.c_int] + [ctypes.c_void_p] * 6 + [
                ctypes.c_uint32, ctypes.c_uint32, ctypes.c_void_p]
            L.oracle_count_key.restype = ctypes.c_uint64
            L.oracle_count_key.argtypes = [ctypes.c_void_p, ctypes.c_uint64, ctypes.c_char_p, ctypes.c_uint64]
            L.oracle_pread_only.restype = ctypes.c_double
            L.oracle_pread_only.argtypes = [ctypes.c_void_p, ctypes.c_int, ctypes.c_int, ctypes.c_uint64]
            _lib = L
    return _lib


def _pack(words):
    buf = bytearray(DSTRIDE * len(words))
    lens = np.zeros(len(words), dtype=np.uint8)
    for i, w in enumerate(words):
        assert len(w) <= 16
        buf[DSTRIDE * i: DSTRIDE * i + len(w)] = w
        lens[i] = len(w)
    return bytes(buf), lens


def pread(fd: int, n: int, off: int):
    """Direct pread(2) -> (ret, bytes).  ret is >= 0 or -errno (raw-syscall convention)."""
    buf = np.zeros(max(n, 1), dtype=np.uint8)
    r = lib().oracle_pread(fd, buf.ctypes.data, n, off)
    return int(r), bytes(buf[: max(r, 0)])


def exec_plan(fds, offs, lens):
    """Run a request plan directly from one host thread -> (rets int64[n], list of reply bytes)."""
    n = len(fds)
    fd = np.asarray(fds, dtype=np.int32)
    off = np.asarray(offs, dtype=np.int64)
    ln = np.asarray(lens, dtype=np.uint64)
    dst = np.zeros(n, dtype=np.uint64)
    if n:
        dst[1:] = np.cumsum(ln)[:-1]
    base = np.zeros(int(ln.sum()) + 1, dtype=np.uint8)
    ret = np.zeros(n, dtype=np.int64)
    lib().oracle_exec_plan(n, fd.ctypes.data, off.ctypes.data, ln.ctypes.data, base.ctypes.data,
                           dst.ctypes.data, ret.ctypes.data)
    out = [bytes(base[int(dst[i]): int(dst[i]) + max(int(ret[i]), 0)]) for i in range(n)]
    return ret, out


def count_tokens(text: bytes | np.ndarray, dict_words) -> np.ndarray:
    """Whole-token counts of each dictionary word in text (reading A9)."""
    arr = np.frombuffer(text, dtype=np.uint8) if isinstance(text, (bytes, bytearray)) else text
    d, dl = _pack(dict_words)
    hist = np.zeros(len(dict_words), dtype=np.uint64)
    lib().oracle_count_tokens(arr.ctypes.data, arr.size, d, dl.ctypes.data, len(dict_words), hist.ctypes.data)
    return hist


def grep(text: bytes | np.ndarray, pats) -> bool:
    arr = np.frombuffer(text, dtype=np.uint8) if isinstance(text, (bytes, bytearray)) else text
    p, pl = _pack(pats)
    return bool(lib().oracle_grep(arr.ctypes.data, arr.size, p, pl.ctypes.data, len(pats)))


def read_file_plan(path: str, chunk: int):
    """Read a file through the work-group halo pread plan -> (bytes, rets per chunk)."""
    size = os.path.getsize(path)
    nch = (size + chunk - 1) // chunk
    out = np.zeros(max(size, 1), dtype=np.uint8)
    scratch = np.zeros(chunk + 64, dtype=np.uint8)
    rets = np.zeros(max(nch, 1), dtype=np.int64)
    fd = os.open(path, os.O_RDONLY)
    try:
        r = lib().oracle_read_file_plan(fd, size, chunk, out.ctypes.data, scratch.ctypes.data, rets.ctypes.data)
    finally:
        os.close(fd)
    if r:
        raise OSError(-r, "oracle_read_file_plan")
    return bytes(out[:size]), rets[:nch]


def corpus(paths, dict_words, pats, chunk: int = 256 << 10, nthreads: int | None = None):
    """Wordcount + grep -F -l over files -> (hist uint64[64], file_hits uint32[F], seconds, threads)."""
    nthreads = nthreads or len(os.sched_getaffinity(0))
    arr = (ctypes.c_char_p * len(paths))(*[p.encode() for p in paths])
    d, dl = _pack(dict_words)
    p, pl = _pack(pats)
    hist = np.zeros(len(dict_words), dtype=np.uint64)
    hits = np.zeros(len(paths), dtype=np.uint32)
    secs = ctypes.c_double(0)
    r = lib().oracle_corpus(ctypes.cast(arr, ctypes.c_void_p), len(paths), nthreads, chunk,
                            d, dl.ctypes.data, len(dict_words), p, pl.ctypes.data, len(pats),
                            hist.ctypes.data, hits.ctypes.data, ctypes.addressof(secs))
    if r:
        raise OSError(-r, "oracle_corpus")
    return hist, hits, secs.value, nthreads


def syscall_rate(kind: str, nthreads: int, iters: int, fd: int = -1, length: int = 4096, size: int = 0) -> float:
    """Direct host syscalls/s: kind 'getrusage' or 'pread'."""
    k = {"getrusage": 0, "pread": 1}[kind]
    r = lib().oracle_syscall_rate(k, nthreads, iters, fd, length, size)
    if r < 0:
        raise OSError(int(-r), "oracle_syscall_rate")
    return r


def pread_only(paths, nthreads: int, chunk: int = 256 << 10) -> float:
    """Host pread ceiling in bytes/s: nthreads threads pread the files in chunk-byte calls."""
    arr = (ctypes.c_char_p * len(paths))(*[p.encode() for p in paths])
    r = lib().oracle_pread_only(ctypes.cast(arr, ctypes.c_void_p), len(paths), nthreads, chunk)
    if r < 0:
        raise OSError(int(-r), "oracle_pread_only")
    return r


def count_key(data, key: bytes) -> int:
    """Overlapping occurrences of key in data (signal-search lookup, sec. VIII-B)."""
    arr = np.frombuffer(data, dtype=np.uint8) if isinstance(data, (bytes, bytearray)) else data
    return int(lib().oracle_count_key(arr.ctypes.data, arr.size, key, len(key)))

"""Thin ctypes binding of libgsys (include/gsys.h).  Argument marshalling only: every step of the
hot path runs in the library's C++ service and sm_100a kernels.  The library must exist (built by
``build()``); there is no CPU fallback -- a missing extension raises.

PyTorch is used only for device memory (tensor.data_ptr()) and streams (cuda_stream handles).
"""
from __future__ import annotations

import ctypes
import os

from . import build as _build

WI, WG, KERNEL = 0x01, 0x02, 0x04
BLOCKING, NONBLOCKING = 0x00, 0x08
STRONG, RELAXED = 0x00, 0x10
HOSTBUF = 0x20
WEAK = RELAXED
FREE, POPULATING, READY, PROCESSING, FINISHED = 0, 1, 2, 3, 4
NR_PREAD64, NR_PWRITE64, NR_GETRUSAGE = 17, 18, 98


def SITE(k: int) -> int:
    return (k & 63) << 24


class GsysError(OSError):
    pass


class Stats(ctypes.Structure):
    _fields_ = [("requests", ctypes.c_uint64), ("completed", ctypes.c_uint64), ("bundles", ctypes.c_uint64),
                ("max_bundle", ctypes.c_uint64), ("host_preads", ctypes.c_uint64), ("merged", ctypes.c_uint64),
                ("bytes_read", ctypes.c_uint64), ("bytes_h2d", ctypes.c_uint64), ("errors", ctypes.c_uint64),
                ("per_nr", ctypes.c_uint64 * 8), ("ns_busy", ctypes.c_uint64), ("ns_syscall", ctypes.c_uint64),
                ("ns_cuda", ctypes.c_uint64), ("ns_bounce_wait", ctypes.c_uint64),
                ("threads", ctypes.c_uint32), ("slots", ctypes.c_uint32),
                ("coalesce_max", ctypes.c_uint32), ("coalesce_window_us", ctypes.c_uint32),
                ("split", ctypes.c_uint64), ("deferred", ctypes.c_uint64), ("flushed", ctypes.c_uint64)]

    def as_dict(self):
        d = {k: getattr(self, k) for k, _ in self._fields_ if k != "per_nr"}
        d["per_nr"] = dict(zip(["pread", "pwrite", "madvise", "sendto", "recvfrom", "getrusage", "sigqueue",
                                "other"], list(self.per_nr)))
        return d


class TraceRec(ctypes.Structure):
    _fields_ = [("slot", ctypes.c_uint32), ("seq", ctypes.c_uint32), ("frm", ctypes.c_uint8),
                ("to", ctypes.c_uint8), ("actor", ctypes.c_uint8), ("blocking", ctypes.c_uint8),
                ("nr", ctypes.c_uint32), ("t_ns", ctypes.c_uint64)]


_P = ctypes.c_void_p
_U32 = ctypes.c_uint32
_U64 = ctypes.c_uint64
_I32 = ctypes.c_int32
_I64 = ctypes.c_int64

# name -> (restype, argtypes); mirrors include/gsys.h
SIGNATURES = {
    "gsys_init": (ctypes.c_int, [_U32, _U32]),
    "gsys_set_coalesce_max": (ctypes.c_int, [_U32]),
    "gsys_set_coalesce_window": (ctypes.c_int, [_U32]),
    "gsys_set_merge": (ctypes.c_int, [ctypes.c_int]),
    "gsys_set_fault": (ctypes.c_int, [ctypes.c_int32, ctypes.c_int64]),
    "gsys_diag_phases": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_int]),
    "gsys_set_trace": (ctypes.c_int, [ctypes.c_int, _U32]),
    "gsys_launch": (ctypes.c_int, [_P, _U32, _U32, _U32, _U32, _U32, _U32, _P, ctypes.c_size_t, _P]),
    "gsys_launch_cu": (ctypes.c_int, [_P, _U32, _U32, _U32, _U32, _U32, _U32, _P, ctypes.c_size_t, _P]),
    "gsys_launch_begin": (ctypes.c_int, [_U64, _P]),
    "gsys_wait": (ctypes.c_int, [_P]),
    "gsys_shutdown": (ctypes.c_int, []),
    "gsys_device_ctx": (_P, []),
    "gsys_stats": (ctypes.c_int, [_P]),
    "gsys_stats_reset": (ctypes.c_int, []),
    "gsys_trace_read": (ctypes.c_int, [_P, _U32, _P, _P, _U32, _P]),
    "gsys_clock_sync": (ctypes.c_int, [_U32, _P, _P]),
    "gsys_set_poll_timeout": (ctypes.c_int, [_U32]),
    "gsys_set_fault_drop": (ctypes.c_int, [_I64]),
    "gsys_set_completion": (ctypes.c_int, [_U32]),
    "gsys_set_scan": (ctypes.c_int, [ctypes.c_int]),
    "gsys_watchdog_read": (ctypes.c_int, [_P, _P, _U32]),
    "gsys_abi_info": (ctypes.c_int, [_P, _P, _P]),
    "gsys_plan_merge": (ctypes.c_int, [_U32, _P, _P, _P, _U64, _P, _P, _P, _P, _P]),
    "gsys_split_result": (_I64, [_I64, _U64, _U64]),
    "gsys_selftest_bounce": (ctypes.c_int, [_U64, _U32, _U64]),
    "gsys_set_profile": (ctypes.c_int, [ctypes.c_int]),
    "gsys_amr_release": (ctypes.c_int, [_U64, _U32, _U64, _P, _U32, _I32, _U64, _U64, _P, _U32, _P, _P, _P, _P, _U32,
                                        _P]),
    "gsys_signal_search": (ctypes.c_int, [_P, _U32, _U64, ctypes.c_char_p, _U32, _I32, _I32, _I32, _P, _U32, _P]),
    "gsys_sigsink_install": (ctypes.c_int, [_I32, _U32]),
    "gsys_mc_entries_bytes": (_U64, [_U32, _U32]),
    "gsys_perm_pwrite": (ctypes.c_int, [_P, _P, _U32, _U32, _U32, _P, _I32, _U64, _U32, _U32, _P]),
    "gsys_poll_storm": (ctypes.c_int, [_P, _U32, _U32, _U64, _P, _P]),
    "gsys_mc_build": (ctypes.c_int, [_P, _P, _P, _P, _P, _P, _U32, _U32, _U32, _P, _P, _P, _U64]),
    "gsys_mc_serve": (ctypes.c_int, [_I32, _P, _P, _P, _U32, _U32, _U32, _P, _P, _P, _U32, _U32, _P]),
    "gsys_sigsink_read": (ctypes.c_int, [_P, _P, _U32]),
    "gsys_read_profile": (ctypes.c_int, [_P, ctypes.c_int]),
    "gsys_wordcount": (ctypes.c_int, [_P, _P, _U32, _U32, ctypes.c_char_p, _P, _U32, ctypes.c_char_p, _P, _U32,
                                      _P, _P, _P, _U32, _U32, _U32, _U32, _P]),
    "gsys_scan_device": (ctypes.c_int, [_P, _U64, _U32, ctypes.c_char_p, _P, _U32, ctypes.c_char_p, _P, _U32,
                                        _P, _P, _U32, _U32, _P]),
    "gsys_bench_calls": (ctypes.c_int, [_U32, _U32, _U32, _U32, _U32, _I32, _U64, _U64, _P, _P, _P, _P, _P]),
}

_lib = None


def lib():
    """Load libgsys.so (building it in-tree if stale).  Raises if it cannot be built/loaded."""
    global _lib
    if _lib is None:
        path = os.environ.get("GSYS_LIB") or _build.LIB   # GSYS_LIB: a diagnostic variant (tools/)
        if path == _build.LIB and (not os.path.exists(path) or os.environ.get("GSYS_REBUILD")):
            _build.build()
        L = ctypes.CDLL(path)
        for name, (res, args) in SIGNATURES.items():
            fn = getattr(L, name)
            fn.restype = res
            fn.argtypes = args
        _lib = L
    return _lib


def _check(rc: int, what: str) -> int:
    if rc < 0:
        raise GsysError(-rc, f"{what}: {os.strerror(-rc)}")
    return rc


def _stream(stream) -> int | None:
    if stream is None:
        return None
    if isinstance(stream, int):
        return stream
    return stream.cuda_stream


def gsys_init(slots: int = 0, coalesce_window_us: int = 0) -> int:
    return _check(lib().gsys_init(slots, coalesce_window_us), "gsys_init")


def gsys_set_coalesce_max(n: int) -> int:
    return _check(lib().gsys_set_coalesce_max(n), "gsys_set_coalesce_max")


def gsys_set_coalesce_window(us: int) -> int:
    return _check(lib().gsys_set_coalesce_window(us), "gsys_set_coalesce_window")


def gsys_set_merge(on: bool) -> int:
    return _check(lib().gsys_set_merge(int(bool(on))), "gsys_set_merge")


def gsys_diag_phases(reset: bool = True) -> dict:
    """Per-call phase sums of blocking calls (needs GSYS_DIAG_PHASES=1 at init)."""
    out = (ctypes.c_uint64 * 8)()
    _check(lib().gsys_diag_phases(out, int(bool(reset))), "gsys_diag_phases")
    n = max(out[4], 1)
    return {"calls": out[4], "claim_us": out[0] / n / 1e3, "publish_us": out[1] / n / 1e3,
            "wait_us": out[2] / n / 1e3, "copy_release_us": out[7] / n / 1e3, "hint_sleep_us": out[5] / n / 1e3,
            "polls_per_call": out[6] / n}


def gsys_set_fault(err: int, offset: int = -1) -> int:
    """Test hook: preads at `offset` fail with -err (err 0 = off)."""
    return _check(lib().gsys_set_fault(err, offset), "gsys_set_fault")


def gsys_set_trace(on: bool, capacity: int = 0) -> int:
    return _check(lib().gsys_set_trace(int(bool(on)), capacity), "gsys_set_trace")


def gsys_wait(stream=None) -> int:
    """Drain: returns the first non-blocking -errno, -ETIMEDOUT after a watchdog expiry, or 0;
    raises only on CUDA errors."""
    rc = lib().gsys_wait(_stream(stream))
    if rc < 0 and -rc in (5,):   # EIO from CUDA
        raise GsysError(-rc, "gsys_wait")
    return rc


def gsys_shutdown() -> int:
    return lib().gsys_shutdown()


def gsys_device_ctx() -> int:
    return lib().gsys_device_ctx() or 0


def gsys_stats() -> dict:
    s = Stats()
    _check(lib().gsys_stats(ctypes.byref(s)), "gsys_stats")
    return s.as_dict()


def gsys_stats_reset() -> int:
    return _check(lib().gsys_stats_reset(), "gsys_stats_reset")


def gsys_trace_read(cap: int = 1 << 20):
    """Both sides' trace records as tuples (slot, seq, from, to, actor, blocking, nr, t_ns); GPU
    t_ns is %globaltimer, host t_ns CLOCK_MONOTONIC (relate them with gsys_clock_sync)."""
    g = (TraceRec * cap)()
    h = (TraceRec * cap)()
    ng = ctypes.c_uint32(0)
    nh = ctypes.c_uint32(0)
    _check(lib().gsys_trace_read(g, cap, ctypes.byref(ng), h, cap, ctypes.byref(nh)), "gsys_trace_read")
    conv = lambda arr, n: [(r.slot, r.seq, r.frm, r.to, "gpu" if r.actor == 0 else "cpu", bool(r.blocking),  # noqa: E731
                            r.nr, r.t_ns) for r in arr[: min(n, cap)]]
    return conv(g, ng.value), conv(h, nh.value)


def gsys_clock_sync(samples: int = 256):
    """(offset_ns, uncertainty_ns): host CLOCK_MONOTONIC = GPU %globaltimer + offset, +- uncertainty."""
    off = ctypes.c_int64(0)
    unc = ctypes.c_uint64(0)
    _check(lib().gsys_clock_sync(samples, ctypes.byref(off), ctypes.byref(unc)), "gsys_clock_sync")
    return off.value, unc.value


def gsys_set_poll_timeout(ms: int) -> int:
    return _check(lib().gsys_set_poll_timeout(ms), "gsys_set_poll_timeout")


COMPLETION_MEMOP, COMPLETION_HOST, COMPLETION_PULL = 0, 1, 2
SCAN_TOKEN, SCAN_DFA, SCAN_DFA_TMA = 0, 1, 2


def gsys_set_scan(impl: int) -> int:
    """Scan implementation (include/gsys.h GSYS_SCAN_*); returns the previous one."""
    return _check(lib().gsys_set_scan(impl), "gsys_set_scan")


def gsys_set_completion(mode: int) -> int:
    """Completion path of blocking device-buffer calls (include/gsys.h GSYS_COMPLETION_*)."""
    return _check(lib().gsys_set_completion(mode), "gsys_set_completion")


def gsys_set_fault_drop(offset: int) -> int:
    """Test hook: the pread at `offset` is served but its completion is never written (-1 = off)."""
    return _check(lib().gsys_set_fault_drop(offset), "gsys_set_fault_drop")


def gsys_watchdog_read(cap: int = 64):
    """(count, [(slot, seq, nr, phase)]) of the last gsys_wait that returned -ETIMEDOUT."""
    cnt = ctypes.c_uint32(0)
    recs = (ctypes.c_uint32 * (4 * cap))()
    k = _check(lib().gsys_watchdog_read(ctypes.byref(cnt), recs, cap), "gsys_watchdog_read")
    return cnt.value, [tuple(recs[4 * i: 4 * i + 4]) for i in range(k)]


def gsys_set_profile(on: bool) -> int:
    return _check(lib().gsys_set_profile(int(bool(on))), "gsys_set_profile")


def gsys_read_profile(reset: bool = True) -> dict:
    out = (ctypes.c_uint64 * 3)()
    _check(lib().gsys_read_profile(out, int(bool(reset))), "gsys_read_profile")
    return {"wait_ns": out[0], "scan_ns": out[1], "chunks": out[2]}


def gsys_abi_info():
    a, b, c = ctypes.c_uint32(), ctypes.c_uint32(), ctypes.c_uint32()
    lib().gsys_abi_info(ctypes.byref(a), ctypes.byref(b), ctypes.byref(c))
    return a.value, b.value, c.value


def gsys_plan_merge(fds, offs, lens, max_union: int):
    import numpy as np
    n = len(fds)
    fd = np.asarray(fds, dtype=np.int32)
    off = np.asarray(offs, dtype=np.int64)
    ln = np.asarray(lens, dtype=np.uint64)
    order = np.zeros(n, dtype=np.uint32)
    group = np.zeros(n, dtype=np.uint32)
    oig = np.zeros(n, dtype=np.uint64)
    goff = np.zeros(max(n, 1), dtype=np.int64)
    glen = np.zeros(max(n, 1), dtype=np.uint64)
    ng = _check(lib().gsys_plan_merge(n, fd.ctypes.data, off.ctypes.data, ln.ctypes.data, max_union,
                                      order.ctypes.data, group.ctypes.data, oig.ctypes.data, goff.ctypes.data,
                                      glen.ctypes.data), "gsys_plan_merge")
    return order, group, oig, goff[:ng], glen[:ng]


def gsys_split_result(r: int, offset_in_group: int, length: int) -> int:
    return lib().gsys_split_result(r, offset_in_group, length)


def pack_words(words):
    buf = bytearray(17 * len(words))
    lens = (ctypes.c_uint8 * max(len(words), 1))()
    for i, w in enumerate(words):
        if not 1 <= len(w) <= 16:
            raise ValueError("words must be 1..16 bytes")
        buf[17 * i: 17 * i + len(w)] = w
        lens[i] = len(w)
    return bytes(buf), lens


STAGE_DEVICE, STAGE_HOST = 0, 1


def STAGE_MIXED(n: int) -> int:
    """GSYS_STAGE_MIXED(n): n of every 16 chunks take the device line (copy-engine DMA), the rest
    the host line (SM zero-copy reads)."""
    if not 1 <= n <= 15:
        raise ValueError("mixed staging share must be 1..15 (of 16)")
    return 0x100 | n


def gsys_wordcount(fds, sizes, chunk: int, dict_words, patterns, d_hist, d_file_hits=None, d_req_ret=None,
                   gflags: int = WG | BLOCKING | STRONG, blocks: int = 0, threads: int = 0, stream=None,
                   staging: int = STAGE_DEVICE) -> int:
    """Launch the GPU-syscall wordcount/grep (asynchronous; gsys_wait(stream) before reading).
    d_hist: device uint64 tensor [ndict] (added into); d_file_hits: device int32 [nfiles] or None;
    d_req_ret: device int64 [chunks] or None."""
    n = len(fds)
    fd_arr = (ctypes.c_int32 * n)(*fds)
    sz_arr = (ctypes.c_uint64 * n)(*sizes)
    d, dl = pack_words(dict_words)
    p, pl = pack_words(patterns)
    rc = lib().gsys_wordcount(fd_arr, sz_arr, n, chunk, d, dl, len(dict_words), p, pl, len(patterns),
                              d_hist.data_ptr(), d_file_hits.data_ptr() if d_file_hits is not None else None,
                              d_req_ret.data_ptr() if d_req_ret is not None else None, gflags, staging, blocks,
                              threads, _stream(stream))
    return _check(rc, "gsys_wordcount")


def gsys_scan_device(d_text, n: int, chunk: int, dict_words, patterns, d_hist, d_hit=None, blocks: int = 0,
                     threads: int = 0, stream=None) -> int:
    d, dl = pack_words(dict_words)
    p, pl = pack_words(patterns)
    rc = lib().gsys_scan_device(d_text.data_ptr(), n, chunk, d, dl, len(dict_words), p, pl, len(patterns),
                                d_hist.data_ptr(), d_hit.data_ptr() if d_hit is not None else None, blocks, threads,
                                _stream(stream))
    return _check(rc, "gsys_scan_device")


def gsys_bench_calls(kind: str, gflags: int, blocks: int, threads: int, iters: int, fd: int = -1, length: int = 0,
                     size: int = 0, d_buf=None, d_ret=None, d_lat=None, d_sum=None, stream=None) -> int:
    k = {"getrusage": 0, "pread": 1, "pwrite": 2}[kind]
    ptr = lambda t: t.data_ptr() if t is not None else None  # noqa: E731
    rc = lib().gsys_bench_calls(k, gflags, blocks, threads, iters, fd, length, size, ptr(d_buf), ptr(d_ret),
                                ptr(d_lat), ptr(d_sum), _stream(stream))
    return _check(rc, "gsys_bench_calls")


def gsys_amr_release(host_mesh: int, nblocks: int, block_bytes: int, d_levels, iters: int, statm_fd: int,
                     watermark_bytes: int, page_bytes: int, d_field, field_words: int, statm_buf, d_released, d_rss,
                     d_maxrss, gflags: int = WG | NONBLOCKING | RELAXED, stream=None) -> int:
    rc = lib().gsys_amr_release(host_mesh, nblocks, block_bytes, d_levels.data_ptr(), iters, statm_fd,
                                watermark_bytes, page_bytes, d_field.data_ptr(), field_words, statm_buf.data_ptr(),
                                d_released.data_ptr(), d_rss.data_ptr(), d_maxrss.data_ptr(), gflags, _stream(stream))
    return _check(rc, "gsys_amr_release")


def gsys_signal_search(d_data, nblocks: int, block_bytes: int, key: bytes, tgid: int, sig: int, uid: int, counts,
                       gflags: int = WG | NONBLOCKING, stream=None) -> int:
    rc = lib().gsys_signal_search(d_data.data_ptr(), nblocks, block_bytes, key, len(key), tgid, sig, uid,
                                  counts.data_ptr(), gflags, _stream(stream))
    return _check(rc, "gsys_signal_search")


def header_functions(path: str | None = None) -> list[str]:
    """Names of the functions declared in include/gsys.h (for the export test)."""
    import re
    path = path or os.path.join(_build.INCLUDE, "gsys.h")
    src = open(path).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"^\s*(?:const\s+)?[\w\s\*]+?\b(gsys_\w+)\s*\(", src, flags=re.M)))

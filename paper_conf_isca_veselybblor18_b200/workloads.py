"""High-level drivers of the hot path over the C-ABI (argument marshalling + result readback).

These are the "public API" calls a user makes (and what bench.py's e2e leg times):
  * wordcount_files(): open files, launch the GPU-syscall wordcount/grep (gsys_wordcount), drain
    (gsys_wait), return host copies of the histogram, per-file grep hits and per-chunk pread
    returns.
  * bench_calls(): the granularity x blocking x ordering microbenchmark (gsys_bench_calls).
Everything that touches file bytes or computes counts runs in libgsys (C++ service + sm_100a
kernels); nothing here falls back to the CPU.
"""
from __future__ import annotations

import os
from dataclasses import dataclass

import torch

from . import gsys as G

_inited: set[int] = set()


def ensure_init(slots: int = 0, window_us: int = 0) -> None:
    """gsys_init() once per device of this process."""
    if not torch.cuda.is_available():
        raise RuntimeError("libgsys needs a CUDA device (no CPU fallback)")
    dev = torch.cuda.current_device()
    if dev in _inited:
        return
    G.lib()
    rc = G.lib().gsys_init(slots, window_us)
    if rc not in (0, -114):          # -EALREADY is fine
        raise G.GsysError(-rc, "gsys_init")
    _inited.add(dev)
    import atexit
    atexit.register(_shutdown_all)


def _shutdown_all():
    for dev in list(_inited):
        try:
            torch.cuda.set_device(dev)
            G.gsys_shutdown()
        except Exception:   # noqa: BLE001  (interpreter teardown)
            pass
    _inited.clear()


@dataclass
class WordcountResult:
    hist: "torch.Tensor"          # uint64-as-int64 [ndict] (host)
    file_hits: "torch.Tensor"     # int32 [nfiles] (host)
    req_ret: "torch.Tensor | None"  # int64 [chunks] (host)
    wait_rc: int


class OpenFiles:
    """Context manager holding read-only fds for a list of paths."""

    def __init__(self, paths):
        self.paths = list(paths)
        self.fds = []

    def __enter__(self):
        self.fds = [os.open(p, os.O_RDONLY) for p in self.paths]
        self.sizes = [os.fstat(fd).st_size for fd in self.fds]
        return self

    def __exit__(self, *exc):
        for fd in self.fds:
            os.close(fd)
        self.fds = []


def nchunks(sizes, chunk: int) -> int:
    return sum((s + chunk - 1) // chunk for s in sizes)


def wordcount_fds(fds, sizes, dict_words, patterns, chunk: int = 256 << 10, gflags: int = G.WG | G.BLOCKING | G.STRONG,
                  blocks: int = 0, threads: int = 0, stream=None, want_ret: bool = True,
                  d_hist=None, d_hits=None, d_ret=None, staging: int = G.STAGE_DEVICE):
    """Launch + drain on device tensors (no host copies).  Returns (d_hist, d_hits, d_ret, rc)."""
    ensure_init()
    dev = torch.device("cuda", torch.cuda.current_device())
    if d_hist is None:
        d_hist = torch.zeros(len(dict_words), dtype=torch.int64, device=dev)
    if d_hits is None and patterns:
        d_hits = torch.zeros(len(fds), dtype=torch.int32, device=dev)
    if d_ret is None and want_ret:
        d_ret = torch.full((max(nchunks(sizes, chunk), 1),), -(1 << 40), dtype=torch.int64, device=dev)
    stream = stream or torch.cuda.current_stream()
    G.gsys_wordcount(fds, sizes, chunk, dict_words, patterns, d_hist, d_hits, d_ret, gflags, blocks, threads, stream,
                     staging)
    rc = G.gsys_wait(stream)
    return d_hist, d_hits, d_ret, rc


def wordcount_files(paths, dict_words, patterns, chunk: int = 256 << 10, gflags: int = G.WG | G.BLOCKING | G.STRONG,
                    blocks: int = 0, threads: int = 0, stream=None, staging: int = G.STAGE_DEVICE) -> WordcountResult:
    """The public end-to-end call: files in, host histogram / grep hits / pread returns out."""
    with OpenFiles(paths) as of:
        h, hits, ret, rc = wordcount_fds(of.fds, of.sizes, dict_words, patterns, chunk, gflags, blocks, threads,
                                         stream, staging=staging)
        out = WordcountResult(h.cpu(), hits.cpu() if hits is not None else None,
                              ret.cpu() if ret is not None else None, rc)
    return out


def bench_calls(kind: str, gflags: int, blocks: int, threads: int, iters: int, fd: int = -1, length: int = 0,
                size: int = 0, d_buf=None, want_ret=True, want_lat=True, want_sum=False, stream=None):
    """Run the microbenchmark kernel; returns (callers, d_ret, d_lat, d_sum) after gsys_wait."""
    ensure_init()
    dev = torch.device("cuda", torch.cuda.current_device())
    gran = gflags & 7
    callers = blocks * threads if gran == G.WI else blocks if gran == G.WG else 1
    n = callers * iters
    d_ret = torch.full((n,), -(1 << 40), dtype=torch.int64, device=dev) if want_ret else None
    d_lat = torch.zeros(n, dtype=torch.int64, device=dev) if want_lat else None
    d_sum = torch.zeros(n, dtype=torch.int64, device=dev) if want_sum else None
    stream = stream or torch.cuda.current_stream()
    G.gsys_bench_calls(kind, gflags, blocks, threads, iters, fd, length, size, d_buf, d_ret, d_lat, d_sum, stream)
    rc = G.gsys_wait(stream)
    return callers, d_ret, d_lat, d_sum, rc

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
    if stream is None:
        stream = torch.cuda.current_stream()
    else:   # the outputs were initialised on the current stream
        stream.wait_stream(torch.cuda.current_stream())
    G.gsys_bench_calls(kind, gflags, blocks, threads, iters, fd, length, size, d_buf, d_ret, d_lat, d_sum, stream)
    rc = G.gsys_wait(stream)
    return callers, d_ret, d_lat, d_sum, rc


# ---------------------------------------------------------------------------- config 5 (next rows)
class HostMesh:
    """Private anonymous, page-aligned, pageable host memory (mmap) for the AMR mirror."""

    def __init__(self, nbytes: int):
        import mmap
        self.mm = mmap.mmap(-1, nbytes, flags=mmap.MAP_PRIVATE | mmap.MAP_ANONYMOUS)
        import ctypes
        self._c = ctypes.c_char.from_buffer(self.mm)
        self.addr = ctypes.addressof(self._c)
        self.nbytes = nbytes

    def view(self):
        import numpy as np
        return np.frombuffer(self.mm, dtype=np.uint8)


def amr_run(levels, block_bytes: int = 64 << 10, watermark_bytes: int = 0, field_words: int = 4096,
            gflags: int = G.WG | G.NONBLOCKING | G.RELAXED, fill: int = 0xA5, stream=None):
    """Config 5a: GPU-issued madvise/getrusage/pread(/proc/self/statm) over an AMR-style mesh.
    Returns (released[b] host array, rss[t], maxrss_kib[t], mesh, wait_rc)."""
    import numpy as np
    ensure_init()
    dev = torch.device("cuda", torch.cuda.current_device())
    lv = np.ascontiguousarray(levels, dtype=np.uint8)
    iters, nblocks = lv.shape
    mesh = HostMesh(nblocks * block_bytes)
    mesh.view()[:] = fill
    d_levels = torch.from_numpy(lv).to(dev)
    d_field = torch.rand(2 * nblocks * field_words, device=dev)
    statm = torch.zeros(nblocks * 128, dtype=torch.uint8).pin_memory()
    d_rel = torch.zeros(nblocks, dtype=torch.int32, device=dev)
    d_rss = torch.zeros(iters, dtype=torch.int64, device=dev)
    d_max = torch.zeros(iters, dtype=torch.int64, device=dev)
    fd = os.open("/proc/self/statm", os.O_RDONLY)
    try:
        stream = stream or torch.cuda.current_stream()
        G.gsys_amr_release(mesh.addr, nblocks, block_bytes, d_levels, iters, fd, watermark_bytes,
                           os.sysconf("SC_PAGE_SIZE"), d_field, field_words, statm, d_rel, d_rss, d_max, gflags,
                           stream)
        rc = G.gsys_wait(stream)
    finally:
        os.close(fd)
    return d_rel.cpu().numpy(), d_rss.cpu().numpy(), d_max.cpu().numpy(), mesh, rc


def signal_search_run(data_dev, nblocks: int, block_bytes: int, key: bytes, sig: int | None = None,
                      consumer=None, gflags: int = G.WG | G.NONBLOCKING, stream=None, timeout_s: float = 60.0):
    """Config 5b: GPU work-groups search their block and signal the host with rt_sigqueueinfo;
    `consumer(block_id)` runs on the host for each signal as it arrives.
    Returns (counts[b], received ids in arrival order, arrival times ns, wait_rc)."""
    import ctypes
    import signal as _signal
    import time
    import numpy as np
    ensure_init()
    sig = sig or (_signal.SIGRTMIN + 3)
    L = G.lib()
    rc = L.gsys_sigsink_install(sig, max(1024, 2 * nblocks))
    if rc:
        raise G.GsysError(-rc, "gsys_sigsink_install")
    counts = torch.zeros(nblocks, dtype=torch.int32).pin_memory()
    stream = stream or torch.cuda.current_stream()
    G.gsys_signal_search(data_dev, nblocks, block_bytes, key, os.getpid(), sig, os.getuid(), counts, gflags, stream)
    got, ts = [], []
    vals = (ctypes.c_int32 * 4096)()
    tns = (ctypes.c_uint64 * 4096)()
    t_end = time.time() + timeout_s
    while len(got) < nblocks and time.time() < t_end:
        n = L.gsys_sigsink_read(vals, tns, 4096)
        for i in range(max(n, 0)):
            got.append(int(vals[i]))
            ts.append(int(tns[i]))
            if consumer is not None:
                consumer(int(vals[i]))
        if n <= 0:
            time.sleep(0.0002)
    rc = G.gsys_wait(stream)
    return counts.numpy().copy(), got, ts, rc


# ---------------------------------------------------------------------------- config 4 (next row)
def mc_serve_run(keys, vals, packets, nwg: int = 8, nbuckets: int = 64, bucket_cap: int = 1024,
                 gflags: int = G.WG | G.BLOCKING | G.RELAXED, client_threads: int = 4, window: int = 8,
                 stream=None, send_gflags: int | None = None, idle_s: float = 0.0):
    """Config 4: memcached-style GET server on the GPU (recvfrom/sendto issued by work-groups)
    driven by the UDP load generator (after `idle_s` seconds without traffic).  Returns
    (responses, latencies ns, client seconds, stats [requests, misses, malformed, recv EAGAINs])."""
    import ctypes
    import numpy as np

    from inputs import mc as MC
    ensure_init()
    dev = torch.device("cuda", torch.cuda.current_device())
    L = G.lib()
    kb, ko, kl, vb, vo, vl = MC.pack(keys, vals)
    ent = torch.zeros(int(L.gsys_mc_entries_bytes(nbuckets, bucket_cap)), dtype=torch.uint8, device=dev)
    bn = torch.zeros(nbuckets, dtype=torch.int32, device=dev)
    heap = torch.zeros(max(vb.size, 1), dtype=torch.uint8, device=dev)
    rc = L.gsys_mc_build(kb.ctypes.data, ko.ctypes.data, kl.ctypes.data, vb.ctypes.data, vo.ctypes.data,
                         vl.ctypes.data, len(keys), nbuckets, bucket_cap, ent.data_ptr(), bn.data_ptr(),
                         heap.data_ptr(), heap.numel())
    if rc:
        raise G.GsysError(-rc, "gsys_mc_build")
    io = torch.zeros(nwg * 8192, dtype=torch.uint8).pin_memory()
    stop = torch.zeros(1, dtype=torch.int32).pin_memory()
    stats = torch.zeros(4, dtype=torch.int64, device=dev)
    sock = MC.udp_server_socket()
    port = sock.getsockname()[1]
    s = torch.cuda.Stream(device=dev) if stream is None else stream
    try:
        rc = L.gsys_mc_serve(sock.fileno(), ent.data_ptr(), bn.data_ptr(), heap.data_ptr(), nbuckets, bucket_cap, nwg,
                             io.data_ptr(), stop.data_ptr(), stats.data_ptr(), gflags,
                             gflags if send_gflags is None else send_gflags, s.cuda_stream)
        if rc:
            raise G.GsysError(-rc, "gsys_mc_serve")
        if idle_s > 0:
            import time
            time.sleep(idle_s)
        resp, lat, secs = MC.run_client(port, packets, nthreads=client_threads, window=window) if packets else \
            ([], [], 0.0)
    finally:
        stop[0] = 1
        G.gsys_wait(s)
        sock.close()
    return resp, lat, secs, stats.cpu().tolist()


# ---------------------------------------------------------------------------- row f3 (Fig. 8)
def perm_pwrite_run(data, perm, iters: int, path: str, gflags: int, block_bytes: int = 8192, grid: int = 0,
                    stream=None):
    """Permute every block `iters` times on the GPU and pwrite it from the work-group.
    Returns (device seconds from launch to drained, wait rc)."""
    import numpy as np
    ensure_init()
    dev = torch.device("cuda", torch.cuda.current_device())
    nb = len(data) // block_bytes
    d_in = torch.from_numpy(np.ascontiguousarray(data)).to(dev)
    d_perm = torch.from_numpy(np.ascontiguousarray(perm, dtype=np.uint16).view(np.int16)).to(dev)
    staging = torch.zeros(nb * block_bytes, dtype=torch.uint8).pin_memory()
    fd = os.open(path, os.O_RDWR | os.O_CREAT, 0o644)
    try:
        os.ftruncate(fd, nb * block_bytes)
        s = stream or torch.cuda.current_stream()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        rc = G.lib().gsys_perm_pwrite(d_in.data_ptr(), d_perm.data_ptr(), nb, block_bytes, iters,
                                      staging.data_ptr(), fd, 0, gflags, grid, s.cuda_stream)
        if rc:
            raise G.GsysError(-rc, "gsys_perm_pwrite")
        wrc = G.gsys_wait(s)
        e1.record(s)
        e1.synchronize()
    finally:
        os.close(fd)
    return e0.elapsed_time(e1) / 1e3, wrc

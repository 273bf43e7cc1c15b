"""Request plans: which calls each GPU caller issues -- TEST INFRASTRUCTURE ONLY.

A plan is a pure function of (workload, file sizes, grid shape, granularity); the oracle executes
it with direct host syscalls and the GPU results are compared per request id (reading A18).

  * wordcount / grep (sec. VIII-C, P32.7: "work-group granularity with blocking and
    weak-ordering"): one pread per work-group chunk; chunk c of a file covers [s, e) =
    [c*C, min((c+1)*C, size)) and its request is the halo read pread(off=max(s-1,0),
    len=(e+16)-off) (reading A10) -- the reply is short at end of file (reading A11).
  * granularity microbenchmark (sec. VII, P26.5-16, Fig. 7): caller c (work-item:
    global thread id; work-group: block id; kernel: 0) issues R preads of `length` bytes at
    off = ((c*R + r) * length) mod size, r = 0..R-1.
"""
from __future__ import annotations

HALO_BEFORE = 1
HALO_AFTER = 16     # longest dictionary word / grep pattern (16 B), reading A10


def wordcount_chunk_requests(size: int, chunk: int):
    """[(chunk_index, s, e, off, len)] for one file."""
    out = []
    nch = (size + chunk - 1) // chunk
    for c in range(nch):
        s = c * chunk
        e = min(s + chunk, size)
        off = s - HALO_BEFORE if s else 0
        out.append((c, s, e, off, e + HALO_AFTER - off))
    return out


def expected_pread_ret(size: int, off: int, length: int, cap: int = 0x7FFFF000) -> int:
    """POSIX pread on a regular file of stable size: min(len, size-off, per-call cap), >= 0."""
    return max(0, min(length, size - off, cap))


def microbench_requests(granularity: str, n_blocks: int, block_threads: int, R: int, length: int,
                        size: int):
    """[(caller, r, off, len)] for the granularity microbenchmark."""
    if granularity == "wi":
        callers = n_blocks * block_threads
    elif granularity == "wg":
        callers = n_blocks
    elif granularity == "kernel":
        callers = 1
    else:
        raise ValueError(granularity)
    out = []
    for c in range(callers):
        for r in range(R):
            off = ((c * R + r) * length) % size
            out.append((c, r, off, length))
    return out


def amr_released(levels, rss_ok=None):
    """Config 5a rule (sec. VIII-A: "When the RSS exceeds a watermark, madvise
    relinquishes memory"; a block is released when it is coarsened): block b is released at the
    first iteration t with levels[t][b] == 0 and RSS >= watermark (rss_ok[t], default always),
    once.  Returns released[b] = t+1, or 0 if never."""
    iters, nblocks = len(levels), len(levels[0]) if len(levels) else 0
    out = [0] * nblocks
    for t in range(iters):
        if rss_ok is not None and not rss_ok[t]:
            continue
        for b in range(nblocks):
            if out[b] == 0 and levels[t][b] == 0:
                out[b] = t + 1
    return out


def permuted_blocks(data, perm, iters: int, block_bytes: int):
    """Fig. 8 (PAPER.md:26 P26.21-27): each block permuted `iters` times, out[i] = in[perm[i]] (a
    DES-style gather, reading A20) -- the bytes the GPU work-groups must have written to the file
    (numpy fancy indexing, one step at a time).  Pinned by the hand-worked example in
    tests/golden/fig8_permutation_tiny.json."""
    import numpy as np
    blocks = np.asarray(data).reshape(-1, block_bytes)
    out = blocks.copy()
    for _ in range(iters):
        out = out[:, perm]
    return out.reshape(-1)

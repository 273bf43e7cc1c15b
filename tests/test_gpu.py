"""GPU parity tests (B200, via gpurun): the CUDA path through the C-ABI vs the CPU oracle.

All data is integer: histograms, pread return values, byte sums and file contents must match the
oracle bit-exactly.  Inputs are the seeded generator's files on tmpfs."""
import errno
import os

import numpy as np
import pytest
import torch

import inputs
import oracle
from oracle import plan, protocol
from paper_conf_isca_veselybblor18_b200 import gsys as G
from paper_conf_isca_veselybblor18_b200 import workloads as W

pytestmark = pytest.mark.gpu

WORDS = None
PATS = None


@pytest.fixture(scope="module", autouse=True)
def gsys_instance():
    global WORDS, PATS
    if not torch.cuda.is_available():
        pytest.skip("needs a GPU")
    W.ensure_init()
    WORDS, PATS = inputs.dictionary(), inputs.patterns()
    yield


@pytest.fixture(scope="module")
def file16m(tmpdir_shm):
    p = os.path.join(tmpdir_shm, "config1_16MiB.txt")
    census, _ = inputs.write_file(p, inputs.SEED_FILE16M, 0, 16 << 20)
    return p, census


@pytest.fixture(scope="module")
def ragged_corpus(tmpdir_shm):
    sizes = [0, 1, 15, 4095, 4096 + 17, (256 << 10) - 1, 256 << 10, (256 << 10) + 1, (1 << 20) + 333, 777777,
             65536, 3 * 4096]
    return inputs.make_corpus(len(sizes), sizes, seed=inputs.SEED_CORPUS, root=tmpdir_shm, tag="ragged")


def oracle_hist_hits(paths):
    h, hits, _, _ = oracle.corpus(paths, WORDS, PATS, nthreads=4)
    return h, hits


def as_u64(t):
    return t.cpu().numpy().astype(np.uint64)


# ---------------------------------------------------------------------------- wordcount (rows a1-a8)
@pytest.mark.parametrize("staging", [G.STAGE_DEVICE, G.STAGE_HOST, G.STAGE_MIXED(5)])
@pytest.mark.parametrize("order", [G.STRONG, G.RELAXED])
def test_wordcount_config1_parity(file16m, order, staging):
    """Config 1: 16 MiB file, 64 work-groups, WG + blocking (+ strong / relaxed), device or
    host-mapped (zero-copy) staging."""
    p, census = file16m
    res = W.wordcount_files([p], WORDS, PATS, chunk=256 << 10, gflags=G.WG | G.BLOCKING | order, staging=staging)
    assert res.wait_rc == 0
    data = open(p, "rb").read()
    want = oracle.count_tokens(data, WORDS)
    assert np.array_equal(as_u64(res.hist), want)
    assert np.array_equal(want, census)
    reqs = plan.wordcount_chunk_requests(len(data), 256 << 10)
    assert len(reqs) == 64
    _, rets = oracle.read_file_plan(p, 256 << 10)
    assert res.req_ret.tolist() == rets.tolist()
    assert res.req_ret.tolist() == [plan.expected_pread_ret(len(data), r[3], r[4]) for r in reqs]
    assert bool(res.file_hits[0]) == oracle.grep(data, PATS)


@pytest.mark.parametrize("staging", [G.STAGE_DEVICE, G.STAGE_HOST, G.STAGE_MIXED(5)])
@pytest.mark.parametrize("chunk,blocks,threads", [(4096, 7, 64), (256 << 10, 0, 256), (64 << 10, 3, 256),
                                                  (1 << 20, 1, 128)])
def test_wordcount_ragged_corpus(ragged_corpus, scan_impl, chunk, blocks, threads, staging):
    c = ragged_corpus
    res = W.wordcount_files(c.paths, WORDS, PATS, chunk=chunk, blocks=blocks, threads=threads,
                            gflags=G.WG | G.BLOCKING | G.RELAXED, staging=staging)
    h, hits = oracle_hist_hits(c.paths)
    assert res.wait_rc == 0
    assert np.array_equal(as_u64(res.hist), h)
    assert np.array_equal(h, c.census)
    assert res.file_hits.tolist() == hits.tolist()
    want = []
    for s in c.sizes:
        want += [plan.expected_pread_ret(s, r[3], r[4]) for r in plan.wordcount_chunk_requests(s, chunk)]
    assert res.req_ret.tolist() == want


@pytest.mark.parametrize("trial", range(20))
def test_wordcount_fuzz(tmpdir_shm, trial):
    """Seeded random launch shapes through the public call: file count and sizes (incl. 0, 1 and
    sizes next to chunk multiples), chunk, work-groups, threads per work-group, staging, ordering,
    blocking or non-blocking prefetch, scan implementation.  Counts, per-file grep hits and (when
    blocking) every per-chunk pread return equal the oracle's."""
    rng = np.random.default_rng(1000 + trial)
    chunk = int(rng.choice([4096, 8192, 4096 * 5 + 16 * 3, 65536, 256 << 10]))
    nfiles = int(rng.integers(1, 7))
    sizes = []
    for _ in range(nfiles):
        kind = int(rng.integers(4))
        if kind == 0:
            sizes.append(int(rng.choice([0, 1, 16, 17])))
        elif kind == 1:
            sizes.append(chunk * int(rng.integers(1, 5)) + int(rng.integers(-17, 18)))
        else:
            sizes.append(int(rng.integers(1, 3 << 20)))
    sizes = [max(s, 0) for s in sizes]
    c = inputs.make_corpus(nfiles, sizes, seed=inputs.SEED_CORPUS + trial, root=tmpdir_shm, tag=f"fuzz{trial}")
    blocks = int(rng.choice([0, 1, 3, 37, 148, 300]))
    threads = int(rng.choice([32, 64, 96, 128, 256]))
    staging = [G.STAGE_DEVICE, G.STAGE_HOST, G.STAGE_MIXED(int(rng.integers(1, 16)))][int(rng.integers(3))]
    order = G.STRONG if rng.integers(2) else G.RELAXED
    blk = G.BLOCKING if rng.integers(3) else G.NONBLOCKING
    prev = G.gsys_set_scan([G.SCAN_DFA, G.SCAN_TOKEN][int(rng.integers(2))])
    try:
        res = W.wordcount_files(c.paths, WORDS, PATS, chunk=chunk, blocks=blocks, threads=threads,
                                gflags=G.WG | blk | order, staging=staging)
    finally:
        G.gsys_set_scan(prev)
    shape = (chunk, sizes, blocks, threads, staging, order, blk)
    h, hits = oracle_hist_hits(c.paths)
    assert res.wait_rc == 0, shape
    assert np.array_equal(as_u64(res.hist), h), shape
    assert np.array_equal(h, c.census), shape
    assert res.file_hits.tolist() == hits.tolist(), shape
    if blk == G.BLOCKING:
        want = []
        for sz in sizes:
            want += [plan.expected_pread_ret(sz, r[3], r[4]) for r in plan.wordcount_chunk_requests(sz, chunk)]
        assert res.req_ret.tolist()[:len(want)] == want, shape


@pytest.mark.parametrize("words,pats", [([], []), ([b"the"], []), ([], [b"the "])], ids=["none", "no-pats", "no-words"])
def test_wordcount_degenerate_dictionaries(ragged_corpus, scan_impl, words, pats):
    """The GPU-issued pread path with an empty dictionary and / or no grep patterns: counts and
    per-file hits equal the oracle's (zeros where there is nothing to look for), every pread return
    still equals the plan's."""
    c = ragged_corpus
    res = W.wordcount_files(c.paths, words, pats, chunk=64 << 10, gflags=G.WG | G.BLOCKING | G.RELAXED)
    assert res.wait_rc == 0
    h, hits, _, _ = oracle.corpus(c.paths, words, pats, nthreads=4)
    assert np.array_equal(as_u64(res.hist)[:len(words)], np.asarray(h)[:len(words)])
    assert int(as_u64(res.hist)[len(words):].sum()) == 0
    if pats:
        assert res.file_hits.tolist() == hits.tolist()
    else:   # no patterns: no per-file hit vector (the oracle's is all zero)
        assert res.file_hits is None and int(hits.sum()) == 0
    want = []
    for s in c.sizes:
        want += [plan.expected_pread_ret(s, r[3], r[4]) for r in plan.wordcount_chunk_requests(s, 64 << 10)]
    assert res.req_ret.tolist() == want


def test_wordcount_grep_corpus(tmpdir_shm):
    c = inputs.make_corpus(48, 128 << 10, seed=inputs.SEED_CORPUS, root=tmpdir_shm, tag="grep48")
    res = W.wordcount_files(c.paths, WORDS, PATS, chunk=32 << 10)
    assert res.file_hits.tolist() == [1 if m else 0 for m in c.pmasks]
    assert np.array_equal(as_u64(res.hist), c.census)


@pytest.mark.parametrize("window,cmax,merge", [(0, 1, 0), (0, 8, 1), (5, 8, 1), (50, 64, 1), (50, 64, 0)])
def test_wordcount_coalescing_invariance(ragged_corpus, window, cmax, merge):
    """Results are identical with and without coalescing / merging (reading A8), bundles <= max."""
    c = ragged_corpus
    G.gsys_set_coalesce_window(window)
    G.gsys_set_coalesce_max(cmax)
    G.gsys_set_merge(merge)
    G.gsys_stats_reset()
    try:
        res = W.wordcount_files(c.paths, WORDS, PATS, chunk=16 << 10)
        st = G.gsys_stats()
    finally:
        G.gsys_set_coalesce_window(0)
        G.gsys_set_coalesce_max(8)
        G.gsys_set_merge(1)
    h, hits = oracle_hist_hits(c.paths)
    assert np.array_equal(as_u64(res.hist), h)
    assert res.file_hits.tolist() == hits.tolist()
    want = []
    for s in c.sizes:
        want += [plan.expected_pread_ret(s, r[3], r[4]) for r in plan.wordcount_chunk_requests(s, 16 << 10)]
    assert res.req_ret.tolist() == want
    assert st["max_bundle"] <= cmax
    if not merge:
        assert st["merged"] == 0


@pytest.fixture(params=[G.SCAN_TOKEN, G.SCAN_DFA, G.SCAN_DFA_TMA], ids=["token", "dfa", "dfa_tma"])
def scan_impl(request):
    prev = G.gsys_set_scan(request.param)
    yield request.param
    G.gsys_set_scan(prev)


def test_scan_device_parity(scan_impl):
    """Scan of HBM-resident text (no syscalls), ragged size, several chunk sizes."""
    for fid, size in [(0, (8 << 20) + 13), (1, 4097), (2, 100)]:
        buf, census, _ = inputs.gen_bytes(inputs.SEED_CORPUS, fid, size, grep_plants=True)
        d_text = torch.zeros(size + 64, dtype=torch.uint8, device="cuda")
        d_text[:size].copy_(torch.from_numpy(buf))
        for chunk in (16, 4096, 1 << 20):
            hist = torch.zeros(64, dtype=torch.int64, device="cuda")
            hit = torch.zeros(1, dtype=torch.int32, device="cuda")
            G.gsys_scan_device(d_text, size, chunk, WORDS, PATS, hist, hit)
            torch.cuda.synchronize()
            assert np.array_equal(as_u64(hist), oracle.count_tokens(buf, WORDS))
            assert bool(hit.item()) == oracle.grep(buf, PATS)


def _scan_dev(buf, words, pats, chunk, threads=0):
    size = len(buf)
    d_text = torch.zeros(size + 64, dtype=torch.uint8, device="cuda")
    d_text[:size].copy_(torch.from_numpy(np.frombuffer(bytes(buf), dtype=np.uint8)))
    hist = torch.zeros(64, dtype=torch.int64, device="cuda")
    hit = torch.zeros(1, dtype=torch.int32, device="cuda")
    G.gsys_scan_device(d_text, size, chunk, words, pats, hist, hit, 0, threads)
    torch.cuda.synchronize()
    return as_u64(hist)[:len(words)], bool(hit.item())


@pytest.mark.parametrize("threads", [0, 256])
def test_scan_device_high_bytes(scan_impl, threads):
    """Text mixing every byte value: 64-byte spans with a byte >= 0x80 leave the raw-byte fast path
    of the 129-column table for the clamped one (and the grep prefilter sees false candidates)."""
    rng = np.random.default_rng(11)
    words = [b"ab", b"b", b"\xc3", b"a" * 16, b"Zq_9", b"q"]
    pats = [b"\xc3\xa9ab", b"b q", b"Zq_9 "]
    alpha = np.frombuffer(b"ab q_Z9\n\xc3\xa9\xff\x80", dtype=np.uint8)
    for trial in range(4):
        n = int(rng.integers(100_000, 400_000))
        text = alpha[rng.integers(0, len(alpha), size=n)]
        text[rng.integers(0, n, size=n // 3)] = rng.integers(0, 256, size=n // 3, dtype=np.uint8)
        for chunk in (64, 4096, 256 << 10):
            hist, hit = _scan_dev(text, words, pats, chunk, threads)
            assert np.array_equal(hist, oracle.count_tokens(text, words)[:len(words)]), (trial, chunk)
            assert hit == oracle.grep(text, pats)


@pytest.mark.parametrize("words,pats", [
    ([], []),                                                    # nothing to count or find
    ([b"the", b"a", b"the", b"x y", b"a-b", b"_", b"9", b"A"], [b"q"]),   # duplicate (first wins),
    # words with a non-word byte (never a whole token), one-byte words, case sensitivity
    ([b"abcdefghijklmnop", b"abcdefghijklmno", b"abcdefgh", b"abcdefghi"], [b"abcdefghijklmnop"]),
], ids=["empty", "dup-nonword-short", "shared-prefixes"])
@pytest.mark.parametrize("size", [0, 1, 15, 16, 17, 63, 64, 65, 2047, 2048, 2049, 70_001])
def test_scan_device_degenerate(scan_impl, words, pats, size):
    """Degenerate dictionaries (empty; a duplicate word, which counts once -- the oracle's first
    match wins; words containing a non-word byte, which never equal a token; 1-byte and 16-byte
    words; words that are prefixes of one another) on texts of 0..70 KB around the 16-byte step,
    the 64-byte lane span and the 2 KiB warp tile."""
    rng = np.random.default_rng(size + 7 * len(words))
    vocab = [b"the", b"a", b"_", b"9", b"A", b"x", b"y", b"ab", b"abcdefgh", b"abcdefghi", b"abcdefghijklmno",
             b"abcdefghijklmnop", b"abcdefghijklmnopq", b"The", b"a_b"]
    seps = [b" ", b"-", b"\n", b" y ", b"--"]
    out = bytearray()
    while len(out) < size:
        out += vocab[int(rng.integers(len(vocab)))] + seps[int(rng.integers(len(seps)))]
    text = bytes(out[:size])
    hist, hit = _scan_dev(text, words, pats, 4096 if size > 4096 else 16)
    arr = np.frombuffer(text, dtype=np.uint8)
    assert np.array_equal(hist, oracle.count_tokens(arr, words)[:len(words)])
    assert hit == oracle.grep(arr, pats)


@pytest.mark.parametrize("pattern", [b"a ", b" a", b"ab ", b"a b c d e f g h ", b"aaaaaaaaaaaaaaaaa ", b"9_"])
def test_scan_device_dense_tokens(scan_impl, pattern):
    """Token-dense text: one token per 2 bytes fills the warp-cooperative scan's start list to its
    1024-entry maximum per 2 KiB tile; 1-byte words at every start, 17-byte tokens (too long to
    match) at the other extreme; ragged sizes around the tile and the chunk."""
    words = [b"a", b"b", b"ab", b"h", b"9_", b"aaaaaaaaaaaaaaaa"]
    for size in (2048, 2049, 4095, (1 << 20) + 3):
        text = (pattern * (size // len(pattern) + 1))[:size]
        arr = np.frombuffer(text, dtype=np.uint8)
        for chunk in (16, 2048, 256 << 10):
            hist, hit = _scan_dev(text, words, [b"b c"], chunk)
            assert np.array_equal(hist, oracle.count_tokens(arr, words)[:len(words)]), (pattern, size, chunk)
            assert hit == oracle.grep(arr, [b"b c"])


def test_scan_device_staging_paths_agree(tmp_path):
    """The HBM DFA scan stages whole-row tiles by swizzled tensor copies and the rest by the lanes;
    with GSYS_SCAN_SWZ=0 (a fresh process: read at load) every tile goes through the lanes.  Both
    equal the oracle on a 3 MiB + 37 B text at 64-byte-aligned and unaligned chunk sizes."""
    import subprocess
    import sys
    code = f"""
import os, sys, numpy as np, torch
sys.path.insert(0, {repr(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))})
import inputs, oracle
from paper_conf_isca_veselybblor18_b200 import gsys as G, workloads as W
W.ensure_init()
words, pats = inputs.dictionary(), inputs.patterns()
size = (3 << 20) + 37
buf, census, _ = inputs.gen_bytes(inputs.SEED_CORPUS, 5, size, grep_plants=True)
t = torch.zeros(size + 64, dtype=torch.uint8, device='cuda')
t[:size].copy_(torch.from_numpy(buf))
want = oracle.count_tokens(buf, words)
for chunk in (48, 4096, 1 << 20):
    h = torch.zeros(64, dtype=torch.int64, device='cuda')
    hit = torch.zeros(1, dtype=torch.int32, device='cuda')
    G.gsys_scan_device(t, size, chunk, words, pats, h, hit)
    torch.cuda.synchronize()
    assert np.array_equal(h.cpu().numpy().astype(np.uint64), want), chunk
    assert bool(hit.item()) == oracle.grep(buf, pats), chunk
print('ok')
"""
    for swz in ("1", "0"):
        env = dict(os.environ, GSYS_SCAN_SWZ=swz)
        out = subprocess.run([sys.executable, "-c", code], env=env, capture_output=True, text=True, timeout=300)
        assert out.returncode == 0 and "ok" in out.stdout, (swz, out.stderr[-3000:])


def test_scan_device_large_trie_uses_narrow_table(scan_impl):
    """A dictionary whose 129-column table no longer fits next to 16 warps' staging (482 trie
    states + 30 emission states) runs on the 77-column table: same counts."""
    words = [bytes([ord("A") + i % 26 if i < 26 else ord("a") + i - 26]) + bytes((97 + (i * 7 + k) % 26) for k in range(15))
             for i in range(30)]
    buf, _, _ = inputs.gen_bytes(inputs.SEED_CORPUS, 5, 1 << 20)
    text = bytearray(buf.tobytes())
    for i, w in enumerate(words):                 # plant every word a few times, whole-token
        for r in range(3):
            at = 1000 + 30_000 * (i * 3 + r) % (len(text) - 40)
            text[at:at + 18] = b" " + w + b" "
    hist, _ = _scan_dev(bytes(text), words, [], 4096)
    exp = oracle.count_tokens(np.frombuffer(bytes(text), dtype=np.uint8), words)[:len(words)]
    assert np.array_equal(hist, exp) and exp.sum() >= 30


def test_scan_device_trie_too_large_is_e2big(scan_impl):
    """The byte DFA caps the trie at 512 states (-E2BIG); the token scan has no such limit."""
    alpha = b"ABCDEFGHIJKLMNOPQRSTUVWXYZabcdefghijklmnopqrstuvwxyz0123456789"
    words = [alpha[i:i + 1] + b"x" * 15 for i in range(40)]       # 40 x 16 + 2 = 642 trie states > 512
    text = b" ".join(words[::3]) + b" abc " + words[1] + b"x " + words[7]
    if scan_impl != G.SCAN_TOKEN:
        with pytest.raises(OSError) as ei:
            _scan_dev(text, words, [], 4096)
        assert ei.value.errno == errno.E2BIG
    else:
        hist, _ = _scan_dev(text, words, [], 4096)
        assert np.array_equal(hist, oracle.count_tokens(np.frombuffer(text, dtype=np.uint8), words)[:len(words)])


def assert_call_sums(sm, reqs, data, gran, iters, ctx=None):
    """Per-call byte sums read back by the calling scope.  A kernel-scope producer call has no
    barrier before it (relaxed only, P20.33): a block done with call r may issue call r+1 into the
    same buffer while a slower block still sums call r's bytes, so for that granularity only the
    last call's sum is defined."""
    got = sm.tolist()
    assert len(got) == len(reqs), ctx
    for i, r in enumerate(reqs):
        if gran == G.KERNEL and r[1] != iters - 1:
            continue
        assert got[i] == sum(data[r[2]: r[2] + r[3]]), (ctx, i)


# ---------------------------------------------------------------------------- microbenchmark matrix
VALID_CELLS = [(G.WI, G.BLOCKING, G.STRONG), (G.WI, G.NONBLOCKING, G.STRONG),
               (G.WG, G.BLOCKING, G.STRONG), (G.WG, G.BLOCKING, G.RELAXED),
               (G.WG, G.NONBLOCKING, G.STRONG), (G.WG, G.NONBLOCKING, G.RELAXED),
               (G.KERNEL, G.BLOCKING, G.RELAXED), (G.KERNEL, G.NONBLOCKING, G.RELAXED)]


@pytest.fixture(scope="module")
def file1m(tmpdir_shm):
    p = os.path.join(tmpdir_shm, "mb_1MiB.txt")
    inputs.write_file(p, 7, 0, (1 << 20) + 100)
    return p


def test_concurrent_granularities_on_streams(file1m):
    """Four call kernels in flight at once on their own streams -- work-item non-blocking and
    blocking device preads, work-group non-blocking relaxed device preads, kernel-scope blocking
    preads -- sharing the slots, the service, the bounce rings and the deferred store; one
    device-wide gsys_wait.  Every blocking return and byte sum equals the direct read, every
    buffer ends with its caller's last read."""
    size = os.path.getsize(file1m)
    data = open(file1m, "rb").read()
    cells = [(G.WI | G.NONBLOCKING, 4, 128, 3, 3000), (G.WI | G.BLOCKING, 3, 96, 2, 4096),
             (G.WG | G.NONBLOCKING | G.RELAXED, 24, 128, 4, 8192), (G.KERNEL | G.BLOCKING | G.RELAXED, 5, 64, 3, 70000)]
    fd = os.open(file1m, os.O_RDONLY)
    runs = []
    try:
        for fl, blocks, threads, iters, length in cells:
            gran = fl & 7
            callers = blocks * threads if gran == G.WI else blocks if gran == G.WG else 1
            n = callers * iters
            buf = torch.zeros(callers * length + 64, dtype=torch.uint8, device="cuda")
            ret = torch.full((n,), -(1 << 40), dtype=torch.int64, device="cuda")
            sm = torch.zeros(n, dtype=torch.int64, device="cuda")
            runs.append((fl, blocks, threads, iters, length, callers, buf, ret, sm, torch.cuda.Stream()))
        torch.cuda.synchronize()
        for fl, blocks, threads, iters, length, callers, buf, ret, sm, st in runs:
            G.gsys_bench_calls("pread", fl, blocks, threads, iters, fd, length, size, buf, ret, None, sm, st)
        assert G.gsys_wait() == 0
    finally:
        os.close(fd)
    for fl, blocks, threads, iters, length, callers, buf, ret, sm, st in runs:
        gran = {G.WI: "wi", G.WG: "wg", G.KERNEL: "kernel"}[fl & 7]
        reqs = plan.microbench_requests(gran, blocks, threads, iters, length, size)
        if not (fl & G.NONBLOCKING):
            assert ret.tolist() == [plan.expected_pread_ret(size, r[2], r[3]) for r in reqs], gran
            assert_call_sums(sm, reqs, data, fl & 7, iters, gran)
        else:
            assert ret.tolist() == [0] * len(reqs), gran
        host = buf.cpu().numpy()
        for c in range(callers):
            off = ((c * iters + iters - 1) * length) % size
            want = data[off: off + length]
            assert bytes(host[c * length: c * length + len(want)]) == want, (gran, c)


@pytest.mark.parametrize("trial", range(32))
def test_bench_pread_fuzz(file1m, trial):
    """Seeded random cells of the pread microbenchmark: granularity x blocking x ordering, read
    length across the inline / pull-area / bounce / warp-copy / DMA limits, device or host
    buffer, grid shape and calls per caller.  Blocking returns and byte sums equal the direct
    read; after the drain every buffer holds its caller's last read."""
    rng = np.random.default_rng(500 + trial)
    gran, blk, order = VALID_CELLS[int(rng.integers(len(VALID_CELLS)))]
    length = int(rng.choice([1, 255, 256, 257, 4095, 4096, 16384, 16385, 65536, 65537, 200_000]))
    blocks = int(rng.integers(1, 9))
    threads = int(rng.choice([32, 64, 96, 128]))
    iters = int(rng.integers(1, 4))
    hostbuf = bool(rng.integers(2))
    size = os.path.getsize(file1m)
    data = open(file1m, "rb").read()
    callers = {G.WI: blocks * threads, G.WG: blocks, G.KERNEL: 1}[gran]
    if gran == G.WI and length > 16384:
        length = 16384 + int(rng.integers(0, 3))   # keep the work-item buffers small
    nbytes = callers * length + 64
    buf = (torch.zeros(nbytes, dtype=torch.uint8).pin_memory() if hostbuf
           else torch.zeros(nbytes, dtype=torch.uint8, device="cuda"))
    fd = os.open(file1m, os.O_RDONLY)
    try:
        ncall, ret, lat, sm, rc = W.bench_calls("pread", gran | blk | order | (G.HOSTBUF if hostbuf else 0), blocks,
                                                threads, iters, fd, length, size, buf, want_sum=True)
    finally:
        os.close(fd)
    shape = (gran, blk, order, length, blocks, threads, iters, hostbuf)
    assert rc == 0 and ncall == callers, shape
    reqs = plan.microbench_requests({G.WI: "wi", G.WG: "wg", G.KERNEL: "kernel"}[gran], blocks, threads, iters,
                                    length, size)
    if blk == G.BLOCKING:
        assert ret.tolist() == [plan.expected_pread_ret(size, r[2], r[3]) for r in reqs], shape
        assert_call_sums(sm, reqs, data, gran, iters, shape)
    else:
        assert ret.tolist() == [0] * len(reqs), shape
    host = buf.cpu().numpy()
    for c in range(callers):
        off = ((c * iters + iters - 1) * length) % size
        want = data[off: off + length]
        assert bytes(host[c * length: c * length + len(want)]) == want, (shape, c)


@pytest.mark.parametrize("gran,blk,order", VALID_CELLS)
def test_bench_pread_matrix(file1m, gran, blk, order):
    size = os.path.getsize(file1m)
    data = open(file1m, "rb").read()
    blocks, threads, iters, length = 6, 64, 3, 1000
    callers = {G.WI: blocks * threads, G.WG: blocks, G.KERNEL: 1}[gran]
    d_buf = torch.zeros(callers * length + 64, dtype=torch.uint8, device="cuda")
    fd = os.open(file1m, os.O_RDONLY)
    G.gsys_stats_reset()
    try:
        ncall, ret, lat, sm, rc = W.bench_calls("pread", gran | blk | order, blocks, threads, iters, fd, length,
                                                size, d_buf, want_sum=True)
    finally:
        os.close(fd)
    st = G.gsys_stats()
    assert rc == 0 and ncall == callers
    assert st["per_nr"]["pread"] == callers * iters == protocol.requests_per_call(
        {G.WI: "wi", G.WG: "wg", G.KERNEL: "kernel"}[gran], blocks * threads, blocks) * iters
    reqs = plan.microbench_requests({G.WI: "wi", G.WG: "wg", G.KERNEL: "kernel"}[gran], blocks, threads, iters,
                                    length, size)
    if blk == G.BLOCKING:
        assert ret.tolist() == [plan.expected_pread_ret(size, r[2], r[3]) for r in reqs]
        assert_call_sums(sm, reqs, data, gran, iters)
    else:
        assert ret.tolist() == [0] * len(reqs)
    # after the drain the buffers hold the last iteration's bytes
    host = d_buf.cpu().numpy()
    for c in range(callers):
        off = ((c * iters + iters - 1) * length) % size
        want = data[off: off + length]
        assert bytes(host[c * length: c * length + len(want)]) == want


@pytest.mark.parametrize("gran,blk,order", VALID_CELLS)
def test_bench_getrusage_matrix(gran, blk, order):
    G.gsys_stats_reset()
    ncall, ret, lat, _, rc = W.bench_calls("getrusage", gran | blk | order, 5, 96, 2)
    st = G.gsys_stats()
    assert rc == 0
    assert st["per_nr"]["getrusage"] == ncall * 2
    assert ret.tolist() == [0] * (ncall * 2)
    if blk == G.BLOCKING:
        assert int(lat.min()) > 0


def test_kernel_strong_is_einval(file1m):
    G.gsys_stats_reset()
    _, ret, _, _, rc = W.bench_calls("getrusage", G.KERNEL | G.BLOCKING | G.STRONG, 4, 64, 2)
    assert ret.tolist() == [-errno.EINVAL] * 2
    assert G.gsys_stats()["per_nr"]["getrusage"] == 0


def test_kernel_granularity_larger_than_residency(file1m):
    """Kernel-scope producer calls must not deadlock when the grid exceeds co-residency."""
    size = os.path.getsize(file1m)
    fd = os.open(file1m, os.O_RDONLY)
    d_buf = torch.zeros(4096, dtype=torch.uint8, device="cuda")
    try:
        _, ret, _, _, rc = W.bench_calls("pread", G.KERNEL | G.BLOCKING | G.RELAXED, 148 * 40, 256, 3, fd, 4000,
                                         size, d_buf)
    finally:
        os.close(fd)
    assert rc == 0
    assert ret.tolist() == [plan.expected_pread_ret(size, (r * 4000) % size, 4000) for r in range(3)]


def test_errors_surface(file1m):
    d_buf = torch.zeros(1 << 16, dtype=torch.uint8, device="cuda")
    _, ret, _, _, rc = W.bench_calls("pread", G.WG | G.BLOCKING, 2, 32, 1, -1, 100, 1000, d_buf)
    assert ret.tolist() == [-errno.EBADF] * 2 and rc == 0
    _, ret, _, _, rc = W.bench_calls("pread", G.WG | G.NONBLOCKING, 2, 32, 1, -1, 100, 1000, d_buf)
    assert ret.tolist() == [0, 0] and rc == -errno.EBADF        # reading A4
    assert G.gsys_wait() == 0                                     # cleared


# ---------------------------------------------------------------------------- watchdog
@pytest.mark.parametrize("gran,length", [(G.WG, 4096), (G.WG, 100000), (G.WI, 100)])
def test_watchdog_lost_completion(file1m, gran, length):
    """A completion the host never writes (gsys_set_fault_drop) must not hang the GPU: the caller's
    wait expires with -ETIMEDOUT (PAPER.md:30 P30.0, PAPER.md:22 P22.0), gsys_wait reports it with
    the slot / request / phase, the slot is returned to free, and the next launch is unaffected."""
    import time
    size = os.path.getsize(file1m)
    fd = os.open(file1m, os.O_RDONLY)
    blocks, threads, iters = 2, (32 if gran == G.WI else 64), 2
    callers = blocks * threads if gran == G.WI else blocks
    d_buf = torch.zeros(callers * length, dtype=torch.uint8, device="cuda")
    lost = (1 * length) % size                  # caller 0, second call
    try:
        G.gsys_set_poll_timeout(300)
        G.gsys_set_fault_drop(lost)
        t0 = time.time()
        _, ret, _, _, rc = W.bench_calls("pread", gran | G.BLOCKING, blocks, threads, iters, fd, length, size, d_buf)
        dt = time.time() - t0
        G.gsys_set_fault_drop(-1)
        assert rc == -errno.ETIMEDOUT
        cnt, recs = G.gsys_watchdog_read()
        assert cnt == 1 and recs[0][2] == G.NR_PREAD64 and recs[0][3] == 3, (cnt, recs)
        want = [plan.expected_pread_ret(size, (i * length) % size, length) for i in range(callers * iters)]
        want[1] = -errno.ETIMEDOUT
        assert ret.tolist() == want
        assert dt < 10, dt
        # the poisoned slot was freed: the same calls now all complete
        _, ret, _, _, rc = W.bench_calls("pread", gran | G.BLOCKING, blocks, threads, iters, fd, length, size, d_buf)
        assert rc == 0 and ret.tolist() == [plan.expected_pread_ret(size, (i * length) % size, length)
                                            for i in range(callers * iters)]
    finally:
        G.gsys_set_fault_drop(-1)
        G.gsys_set_poll_timeout(20000)
        os.close(fd)


# ---------------------------------------------------------------------------- ordering semantics
@pytest.mark.parametrize("gran,blk,order", [(G.WG, G.BLOCKING, G.STRONG), (G.WG, G.BLOCKING, G.RELAXED),
                                            (G.WG, G.NONBLOCKING, G.RELAXED), (G.WI, G.BLOCKING, G.STRONG),
                                            (G.KERNEL, G.BLOCKING, G.RELAXED)])
def test_pwrite_consumer_barrier(tmpdir_shm, gran, blk, order):
    """Consumer calls keep Bar1 (P22.42): every thread's share of the buffer must reach the file."""
    blocks, threads, length = 4, 256, 8192
    callers = {G.WI: blocks * threads, G.WG: blocks, G.KERNEL: 1}[gran]
    if gran == G.WI:
        length = 64
    size = callers * length
    p = os.path.join(tmpdir_shm, f"pw_{gran}_{blk}_{order}.bin")
    open(p, "wb").write(b"\0" * size)
    fd = os.open(p, os.O_RDWR)
    d_buf = torch.zeros(size, dtype=torch.uint8, device="cuda")
    try:
        _, ret, _, _, rc = W.bench_calls("pwrite", gran | blk | order, blocks, threads, 1, fd, length, size, d_buf)
    finally:
        os.close(fd)
    assert rc == 0
    got = open(p, "rb").read()
    for c in range(callers):
        want = bytes(((c * 131 + i * 7 + 13) & 0xFF) for i in range(length))
        assert got[c * length: (c + 1) * length] == want, c


@pytest.mark.parametrize("trial", range(16))
def test_bench_pwrite_fuzz(tmpdir_shm, trial):
    """Seeded random pwrite cells (consumer calls): granularity x blocking x ordering, length
    (1 B .. 64 KiB + 1), device or host buffer, grid shape, calls per caller (one where the scope
    does not wait for the host before rewriting its buffer: non-blocking and kernel-scope calls).
    Every call's bytes reach the file at its offset; every return is the length."""
    rng = np.random.default_rng(900 + trial)
    gran, blk, order = VALID_CELLS[int(rng.integers(len(VALID_CELLS)))]
    length = int(rng.choice([1, 17, 256, 4096, 5000, 16385, 65537]))
    blocks = int(rng.integers(1, 6))
    threads = int(rng.choice([32, 64, 128]))
    iters = 1 if (blk == G.NONBLOCKING or gran == G.KERNEL) else int(rng.integers(1, 4))
    hostbuf = bool(rng.integers(2))
    callers = {G.WI: blocks * threads, G.WG: blocks, G.KERNEL: 1}[gran]
    if gran == G.WI:
        length = min(length, 4096)
    size = callers * iters * length
    p = os.path.join(tmpdir_shm, f"pwf_{trial}.bin")
    open(p, "wb").write(b"\0" * size)
    buf = (torch.zeros(callers * length + 64, dtype=torch.uint8).pin_memory() if hostbuf
           else torch.zeros(callers * length + 64, dtype=torch.uint8, device="cuda"))
    fd = os.open(p, os.O_RDWR)
    try:
        _, ret, _, _, rc = W.bench_calls("pwrite", gran | blk | order | (G.HOSTBUF if hostbuf else 0), blocks,
                                         threads, iters, fd, length, size, buf)
    finally:
        os.close(fd)
    shape = (gran, blk, order, length, blocks, threads, iters, hostbuf)
    assert rc == 0, shape
    if blk == G.BLOCKING and gran != G.KERNEL:
        assert ret.tolist() == [length] * (callers * iters), shape
    elif blk == G.BLOCKING:   # kernel-scope consumer: the last block to arrive calls, nobody waits (A6)
        assert set(ret.tolist()) <= {0, length}, shape
    got = np.frombuffer(open(p, "rb").read(), dtype=np.uint8)
    i = np.arange(length, dtype=np.uint64)
    for idx in range(callers * iters):
        want = ((idx * 131 + i * 7 + 13) & 0xFF).astype(np.uint8)
        assert np.array_equal(got[idx * length: (idx + 1) * length], want), (shape, idx)


# ---------------------------------------------------------------------------- protocol trace (rows a2-a5, a7)
def _traced(run):
    """Run `run()` with protocol tracing on; return (records, eps): records are (req=(slot, seq),
    slot, from, to, actor, t) from both logs, unsorted, GPU times mapped onto the host clock with
    gsys_clock_sync taken before and after; eps = the clock relation's error bound."""
    off0, unc0 = G.gsys_clock_sync(256)
    G.gsys_set_trace(True, 1 << 16)
    try:
        run()
        assert G.gsys_wait() == 0
        gtr, htr = G.gsys_trace_read()
    finally:
        G.gsys_set_trace(False)
    off1, unc1 = G.gsys_clock_sync(256)
    off = (off0 + off1) // 2
    eps = max(unc0, unc1) + abs(off1 - off0) // 2 + 1
    recs = [((r[0], r[1]), r[0], r[2], r[3], r[4], r[7] + (off if r[4] == "gpu" else 0)) for r in gtr + htr]
    blocking = {}
    for r in gtr + htr:
        blocking.setdefault((r[0], r[1]), r[5])
    return recs, blocking, eps, gtr, htr


def test_clock_sync_is_tight():
    off, unc = G.gsys_clock_sync(256)
    assert 0 < unc < 20000, unc          # a PCIe round trip: a few microseconds
    off2, unc2 = G.gsys_clock_sync(256)
    assert abs(off2 - off) <= unc + unc2 + 2000


def test_protocol_trace_validates(file1m):
    """Rows a2-a5/a7 against oracle/protocol.check_trace: the GPU and host logs as recorded
    (never reordered), every request's path in timestamp order, one live request per slot,
    sequence numbers growing per slot -- at WG, WI and kernel granularity, blocking and
    non-blocking (WG non-blocking calls reuse their slot back to back: P24.11, A15)."""
    size = os.path.getsize(file1m)
    fd = os.open(file1m, os.O_RDONLY)
    d_buf = torch.zeros(64 * 2000, dtype=torch.uint8, device="cuda")

    def run():
        W.bench_calls("pread", G.WG | G.BLOCKING, 8, 64, 3, fd, 2000, size, d_buf)
        W.bench_calls("getrusage", G.WG | G.NONBLOCKING | G.RELAXED, 8, 64, 2)
        W.bench_calls("getrusage", G.WI | G.BLOCKING, 2, 64, 1)
        W.bench_calls("getrusage", G.KERNEL | G.BLOCKING | G.RELAXED, 4, 64, 4)
        W.bench_calls("pread", G.KERNEL | G.NONBLOCKING | G.RELAXED, 2, 64, 3, fd, 2000, size, d_buf)
        W.bench_calls("pread", G.WI | G.NONBLOCKING, 1, 32, 2, fd, 2000, size, d_buf)
    try:
        recs, blocking, eps, gtr, htr = _traced(run)
    finally:
        os.close(fd)
    assert eps < 20000, eps
    n_req = 8 * 3 + 8 * 2 + 2 * 64 + 4 + 3 + 32 * 2
    assert len(blocking) == n_req
    assert protocol.check_trace(recs, blocking.__getitem__, eps=eps, seq_of=lambda r: r[1]) == n_req
    # the host-visible state word is returned to free by the GPU for blocking calls (A3) and by
    # the host for non-blocking ones (P24.34)
    assert sum(1 for r in gtr if r[3] == protocol.FREE) == sum(1 for b in blocking.values() if b)
    assert sum(1 for r in htr if r[3] == protocol.FREE) == sum(1 for b in blocking.values() if not b)


@pytest.mark.parametrize("trial", range(6))
def test_protocol_trace_fuzz(file1m, trial):
    """Seeded random mixes of three call cells (getrusage / pread into device or host buffers, any
    valid granularity x blocking x ordering, lengths across the pull limits) traced together:
    check_trace accepts the raw logs -- one live request per slot, every request's path in
    timestamp order -- and the request count is the plan's."""
    rng = np.random.default_rng(77 + trial)
    size = os.path.getsize(file1m)
    fd = os.open(file1m, os.O_RDONLY)
    cells = []
    for _ in range(3):
        gran, blk, order = VALID_CELLS[int(rng.integers(len(VALID_CELLS)))]
        kind = "getrusage" if rng.integers(3) == 0 else "pread"
        blocks, threads, iters = int(rng.integers(1, 5)), int(rng.choice([32, 64])), int(rng.integers(1, 4))
        length = int(rng.choice([100, 4096, 20000]))
        hostbuf = kind == "pread" and bool(rng.integers(2))
        cells.append((kind, gran | blk | order | (G.HOSTBUF if hostbuf else 0), blocks, threads, iters, length,
                      hostbuf))
    bufs = [(torch.zeros(8 * 64 * 20000, dtype=torch.uint8).pin_memory() if c[6]
             else torch.zeros(8 * 64 * 20000, dtype=torch.uint8, device="cuda")) for c in cells]

    def run():
        for (kind, fl, blocks, threads, iters, length, _), b in zip(cells, bufs):
            if kind == "pread":
                W.bench_calls("pread", fl, blocks, threads, iters, fd, length, size, b)
            else:
                W.bench_calls("getrusage", fl, blocks, threads, iters)
    try:
        recs, blocking, eps, gtr, htr = _traced(run)
    finally:
        os.close(fd)
    n_req = sum({G.WI: bl * th, G.WG: bl, G.KERNEL: 1}[fl & 7] * it for _, fl, bl, th, it, _, _ in cells)
    assert len(blocking) == n_req, cells
    assert protocol.check_trace(recs, blocking.__getitem__, eps=eps, seq_of=lambda r: r[1]) == n_req, cells


def test_protocol_trace_catches_a_reordered_log(file1m):
    """The checker is not vacuous on real logs: moving one host pick-up before its GPU publish
    by more than the clock error fails."""
    recs, blocking, eps, _, _ = _traced(lambda: W.bench_calls("getrusage", G.WG | G.BLOCKING, 4, 64, 2))
    assert protocol.check_trace(recs, blocking.__getitem__, eps=eps) == 8
    ready = {r[0]: r[5] for r in recs if r[3] == protocol.READY}
    bad = [r if r[3] != protocol.PROCESSING else r[:5] + (ready[r[0]] - eps - 1,) for r in recs]
    with pytest.raises(AssertionError):
        protocol.check_trace(bad, blocking.__getitem__, eps=eps)


# ---------------------------------------------------------------------------- full size (config 3 shape)
@pytest.mark.slow
@pytest.mark.parametrize("staging", [G.STAGE_DEVICE, G.STAGE_HOST, G.STAGE_MIXED(5)])
def test_full_size_corpus_census(tmpdir_shm, staging):
    """8 GiB, 512 x 16 MiB files, the bench launch configuration: whole-corpus histogram equals
    the generator's census and grep hits equal the planted set; 4 sampled files through the oracle."""
    import shutil
    free = shutil.disk_usage(tmpdir_shm).free
    if free < (10 << 30):
        pytest.skip("tmpfs too small for the 8 GiB corpus")
    c = inputs.make_corpus(512, 16 << 20, seed=inputs.SEED_CORPUS, root=tmpdir_shm, tag="full8g")
    for chunk, blocks in ((256 << 10, 148), (1 << 20, 0)):   # 148 x 256 KiB: the bench's launch
        res = W.wordcount_files(c.paths, WORDS, PATS, chunk=chunk, blocks=blocks, gflags=G.WG | G.BLOCKING | G.RELAXED,
                                staging=staging)
        assert np.array_equal(as_u64(res.hist), c.census)
    assert res.file_hits.tolist() == [1 if m else 0 for m in c.pmasks]
    assert (res.req_ret > 0).all()
    for f in (0, 101, 255, 511):
        h, hits = oracle_hist_hits([c.paths[f]])
        r1 = W.wordcount_files([c.paths[f]], WORDS, PATS, chunk=256 << 10, staging=staging)
        assert np.array_equal(as_u64(r1.hist), h) and r1.file_hits.tolist() == hits.tolist()


# ---------------------------------------------------------------------------- pull path (reading B12)
@pytest.mark.parametrize("gran,length", [(G.WG, n) for n in (1, 15, 16, 255, 256, 257, 1000, 4096, 16383, 16384,
                                                             16385, 65536)] +
                         [(G.WI, n) for n in (1, 100, 256, 257)] + [(G.KERNEL, n) for n in (200, 3000)])
@pytest.mark.parametrize("shift", [0, 1, 4, 8])
def test_pread_pull_sizes(file1m, gran, length, shift):
    """Blocking preads into device memory: <= 256 B (any caller) and work-group preads of up to
    the slot's pull area (16 KiB) are read by the host into a host-mapped pull area and copied by
    the GPU; longer ones take the DMA path.  Every size and destination alignment must give the
    file's bytes, the POSIX return and the byte sums the scope computes right after the call."""
    size = os.path.getsize(file1m)
    data = open(file1m, "rb").read()
    blocks, threads, iters = 3, 96, 2
    callers = {G.WI: blocks * threads, G.WG: blocks, G.KERNEL: 1}[gran]
    order = G.RELAXED if gran == G.KERNEL else G.STRONG
    d_all = torch.zeros(callers * length + 64, dtype=torch.uint8, device="cuda")
    d_buf = d_all[shift:]
    fd = os.open(file1m, os.O_RDONLY)
    try:
        ncall, ret, _, sm, rc = W.bench_calls("pread", gran | G.BLOCKING | order, blocks, threads, iters, fd, length,
                                              size, d_buf, want_sum=True)
    finally:
        os.close(fd)
    assert rc == 0 and ncall == callers
    reqs = plan.microbench_requests({G.WI: "wi", G.WG: "wg", G.KERNEL: "kernel"}[gran], blocks, threads, iters,
                                    length, size)
    assert ret.tolist() == [plan.expected_pread_ret(size, r[2], r[3]) for r in reqs]
    assert_call_sums(sm, reqs, data, gran, iters)
    host = d_all.cpu().numpy()
    assert not host[:shift].any()
    for c in range(callers):
        off = ((c * iters + iters - 1) * length) % size
        want = data[off: off + length]
        assert bytes(host[shift + c * length: shift + c * length + len(want)]) == want


# ---------------------------------------------------------------------------- fault injection
from ownership import owned_counts  # noqa: E402


@pytest.mark.parametrize("staging", [G.STAGE_DEVICE, G.STAGE_HOST])
def test_wordcount_injected_eio(file16m, staging):
    """A failing pread (EIO injected by the service on chunk 37's request) reaches the work-group
    as -EIO (POSIX convention), that chunk is not scanned, every other chunk is: the histogram
    equals the oracle's whole-file counts minus the counts the failed chunk owns."""
    p, census = file16m
    data = open(p, "rb").read()
    chunk = 256 << 10
    k = 37
    s = k * chunk
    G.gsys_set_fault(5, s - 1)       # chunk k's request is [s - 1, e + 16)
    try:
        res = W.wordcount_files([p], WORDS, PATS, chunk=chunk, gflags=G.WG | G.BLOCKING | G.STRONG, staging=staging)
    finally:
        G.gsys_set_fault(0, -1)
    rets = res.req_ret.tolist()
    assert rets[k] == -5
    reqs = plan.wordcount_chunk_requests(len(data), chunk)
    assert [r for i, r in enumerate(rets) if i != k] == [plan.expected_pread_ret(len(data), r[3], r[4])
                                                         for i, r in enumerate(reqs) if i != k]
    want = oracle.count_tokens(data, WORDS) - owned_counts(data, s, min(s + chunk, len(data)), WORDS)
    assert np.array_equal(as_u64(res.hist), want)
    # the fault is off again: a clean run equals the census
    res2 = W.wordcount_files([p], WORDS, PATS, chunk=chunk, staging=staging)
    assert np.array_equal(as_u64(res2.hist), census)


# ---------------------------------------------------------------------------- non-blocking prefetch
@pytest.mark.parametrize("staging", [G.STAGE_DEVICE, G.STAGE_HOST, G.STAGE_MIXED(5)])
@pytest.mark.parametrize("chunk,blocks,threads", [(4096, 7, 64), (256 << 10, 0, 256), (1 << 20, 1, 128)])
def test_wordcount_nonblocking_prefetch(ragged_corpus, chunk, blocks, threads, staging):
    """WG + non-blocking: each work-group prefetches its next chunk before scanning the current one
    (two lines, ordered by the slot's one-request rule); histogram and grep set equal the oracle,
    every call returns 0 (reading A4) and gsys_wait reports no error."""
    c = ragged_corpus
    res = W.wordcount_files(c.paths, WORDS, PATS, chunk=chunk, blocks=blocks, threads=threads,
                            gflags=G.WG | G.NONBLOCKING | G.RELAXED, staging=staging)
    h, hits = oracle_hist_hits(c.paths)
    assert res.wait_rc == 0
    assert np.array_equal(as_u64(res.hist), h)
    assert res.file_hits.tolist() == hits.tolist()
    assert set(res.req_ret.tolist()) <= {0}


def test_wordcount_nonblocking_full_corpus(tmpdir_shm):
    """The bench corpus (8 GiB) through the prefetching configuration."""
    import shutil
    if shutil.disk_usage(tmpdir_shm).free < (10 << 30) and not os.path.exists(os.path.join(tmpdir_shm, "full8g")):
        pytest.skip("tmpfs too small for the 8 GiB corpus")
    c = inputs.make_corpus(512, 16 << 20, seed=inputs.SEED_CORPUS, root=tmpdir_shm, tag="full8g")
    res = W.wordcount_files(c.paths, WORDS, PATS, chunk=256 << 10, blocks=296,
                            gflags=G.WG | G.NONBLOCKING | G.RELAXED, staging=G.STAGE_HOST)
    assert res.wait_rc == 0
    assert np.array_equal(as_u64(res.hist), c.census)
    assert res.file_hits.tolist() == [1 if m else 0 for m in c.pmasks]


# ---------------------------------------------------------------------------- the per-call read cap
@pytest.mark.parametrize("hostbuf", [False, True])
def test_pread_per_call_cap_from_gpu(tmpdir_shm, hostbuf):
    """Reading A11: one GPU-issued pread returns what one POSIX pread returns -- a 2 GiB read is
    capped at 0x7ffff000 bytes (Fig. 7's kernel-level read).  Device buffers are served piecewise
    through the bounce ring and must stop at exactly the same byte; host buffers are read in place."""
    cap = 0x7FFFF000
    path = os.path.join(tmpdir_shm, "sparse_2g.bin")
    with open(path, "wb") as f:
        f.truncate((1 << 31) + 4096)
        for off, val in ((0, 0x11), (1 << 20, 0x22), (cap - 1, 0x33), (cap, 0x44)):
            f.seek(off)
            f.write(bytes([val]))
    n = 1 << 31
    if hostbuf:
        buf = torch.zeros(n + 16, dtype=torch.uint8).pin_memory()
        flags = G.KERNEL | G.BLOCKING | G.RELAXED | G.HOSTBUF
    else:
        buf = torch.zeros(n + 16, dtype=torch.uint8, device="cuda")
        flags = G.KERNEL | G.BLOCKING | G.RELAXED
    fd = os.open(path, os.O_RDONLY)
    try:
        _, ret, _, _, rc = W.bench_calls("pread", flags, 1, 32, 1, fd, n, (1 << 31) + 4096, buf)
    finally:
        os.close(fd)
        os.unlink(path)
    assert rc == 0
    assert ret.tolist() == [cap] == [plan.expected_pread_ret((1 << 31) + 4096, 0, n)]
    probe = torch.tensor([0, 1 << 20, cap - 1, cap], dtype=torch.int64)
    got = buf[probe.to(buf.device)].cpu().tolist()
    assert got == [0x11, 0x22, 0x33, 0]      # the byte at the cap was not read


# ---------------------------------------------------------------------------- boundary: external kernels
@pytest.fixture(scope="module")
def ext_lib(tmpdir_shm):
    """tests/native/ext_kernel.cu compiled as its own module (own CUDA runtime), against
    include/gsys_device.cuh only."""
    import ctypes
    import subprocess
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    out = os.path.join(tmpdir_shm, "libext_kernel.so")
    subprocess.check_call(["/usr/local/cuda/bin/nvcc", "-O2", "-std=c++17", "-shared", "-Xcompiler", "-fPIC",
                           "-gencode", "arch=compute_100a,code=sm_100a", "-I", os.path.join(root, "include"),
                           os.path.join(root, "tests", "native", "ext_kernel.cu"), "-o", out])
    L = ctypes.CDLL(out)
    L.ext_function.argtypes = [ctypes.c_void_p]
    return L


@pytest.mark.parametrize("nwarps,length", [(4, 3000), (8, 65536)])
def test_external_kernel_tokens(file1m, ext_lib, nwarps, length):
    """A kernel from another module, launched with gsys_launch_cu: non-blocking work-item preads
    issued one after the other by different warps, each waited for by ANOTHER thread through its
    explicit (slot, seq) token (no reliance on hardware-slot reuse, P24.11 / P20.34-38), plus a
    blocking work-group pread; every return value and byte sum equals the direct read."""
    import ctypes
    size = os.path.getsize(file1m)
    data = np.fromfile(file1m, dtype=np.uint8)
    fn = ctypes.c_void_p(0)
    assert ext_lib.ext_function(ctypes.byref(fn)) == 0 and fn.value

    class ExtArgs(ctypes.Structure):
        _fields_ = [("ctx", ctypes.c_void_p), ("dbuf", ctypes.c_void_p), ("ret", ctypes.c_void_p),
                    ("sum", ctypes.c_void_p), ("size", ctypes.c_uint64), ("len", ctypes.c_uint32),
                    ("fd", ctypes.c_int32)]
    blocks = 6
    n = blocks * (nwarps + 1)
    dbuf = torch.zeros(n * length, dtype=torch.uint8, device="cuda")
    ret = torch.full((n,), -(1 << 40), dtype=torch.int64, device="cuda")
    sm = torch.zeros(n, dtype=torch.int64, device="cuda")
    fd = os.open(file1m, os.O_RDONLY)
    try:
        a = ExtArgs(G.gsys_device_ctx(), dbuf.data_ptr(), ret.data_ptr(), sm.data_ptr(), size, length, fd)
        argv = (ctypes.c_void_p * 1)(ctypes.cast(ctypes.pointer(a), ctypes.c_void_p))
        rc = G.lib().gsys_launch_cu(fn, blocks, 1, 1, 32 * nwarps, 1, 1, argv, 0, None)
        assert rc == 0
        assert G.gsys_wait() == 0
    finally:
        os.close(fd)
    for i in range(n):
        off = (i * length) % size
        want = data[off: off + length]
        assert int(ret[i]) == len(want), i
        assert int(sm[i]) == int(want.astype(np.int64).sum()), i


@pytest.mark.parametrize("klen", [3000, 1 << 20, (1 << 20) + 5])
def test_warp_and_block_copied_device_preads(file1m, ext_lib, klen):
    """Blocking work-item preads into device memory from a diverged subset of lanes, with lengths
    on both sides of the warp-copy limit (64 KiB) and zero: the converged lanes copy each other's
    payloads (B13).  Then a kernel-scope pread that the first-arriving block copies (<= 1 MiB) or
    the copy engine serves (> 1 MiB): every block sees the bytes after the call."""
    import ctypes
    size = os.path.getsize(file1m)
    data = np.fromfile(file1m, dtype=np.uint8)
    fn = ctypes.c_void_p(0)
    ext_lib.ext_function_mixed.argtypes = [ctypes.c_void_p]
    assert ext_lib.ext_function_mixed(ctypes.byref(fn)) == 0 and fn.value

    class MixArgs(ctypes.Structure):
        _fields_ = [("ctx", ctypes.c_void_p), ("dbuf", ctypes.c_void_p), ("ret", ctypes.c_void_p),
                    ("sum", ctypes.c_void_p), ("lens", ctypes.c_void_p), ("kbuf", ctypes.c_void_p),
                    ("kret", ctypes.c_void_p), ("ksum", ctypes.c_void_p), ("size", ctypes.c_uint64),
                    ("stride", ctypes.c_uint64), ("klen", ctypes.c_uint64), ("fd", ctypes.c_int32)]
    lens_h = [0, 1, 15, 16, 17, 100, 4096, 5000, 16384, 16385, 65535, 65536, 65537, 70000, 256, 257] * 2
    blocks, threads, stride = 5, 96, 70016
    nt = blocks * threads
    lens = torch.tensor(lens_h, dtype=torch.int32, device="cuda")
    dbuf = torch.zeros(nt * stride, dtype=torch.uint8, device="cuda")
    ret = torch.full((nt,), -(1 << 40), dtype=torch.int64, device="cuda")
    sm = torch.zeros(nt, dtype=torch.int64, device="cuda")
    kbuf = torch.zeros(klen, dtype=torch.uint8, device="cuda")
    kret = torch.zeros(blocks, dtype=torch.int64, device="cuda")
    ksum = torch.zeros(blocks, dtype=torch.int64, device="cuda")
    torch.cuda.synchronize()
    fd = os.open(file1m, os.O_RDONLY)
    try:
        a = MixArgs(G.gsys_device_ctx(), dbuf.data_ptr(), ret.data_ptr(), sm.data_ptr(), lens.data_ptr(),
                    kbuf.data_ptr(), kret.data_ptr(), ksum.data_ptr(), size, stride, klen, fd)
        argv = (ctypes.c_void_p * 1)(ctypes.cast(ctypes.pointer(a), ctypes.c_void_p))
        assert G.lib().gsys_launch_cu(fn, blocks, 1, 1, threads, 1, 1, argv, 0, None) == 0
        assert G.gsys_wait() == 0
    finally:
        os.close(fd)
    ret_h, sm_h = ret.cpu().numpy(), sm.cpu().numpy()
    for t in range(nt):
        if t % 3 == 0:
            assert ret_h[t] == -(1 << 40), t
            continue
        off = (t * 4099) % size
        want = data[off: off + lens_h[t % 32]]
        assert ret_h[t] == len(want), (t, ret_h[t], len(want))
        assert sm_h[t] == int(want.astype(np.int64).sum()), t
    kwant = data[12345: 12345 + klen]
    assert kret.cpu().tolist() == [len(kwant)] * blocks
    assert ksum.cpu().tolist() == [int(kwant.astype(np.int64).sum())] * blocks


# ---------------------------------------------------------------------------- completion paths (B13)
@pytest.fixture
def completion_mode(request):
    G.gsys_set_completion(request.param)
    yield request.param
    G.gsys_set_completion(G.COMPLETION_PULL)


@pytest.mark.parametrize("completion_mode", [G.COMPLETION_MEMOP, G.COMPLETION_HOST, G.COMPLETION_PULL], indirect=True)
@pytest.mark.parametrize("chunk,blocks,threads,nb", [(4096, 7, 64, False), (256 << 10, 0, 256, False),
                                                     (64 << 10, 3, 256, True), (1 << 20, 1, 128, False)])
def test_wordcount_device_staging_completion_modes(ragged_corpus, completion_mode, chunk, blocks, threads, nb):
    """Device staging under each completion path: a stream memop after the DMA, a host store after
    the DMA, and the work-group copying its pulled bytes out of the service's host-mapped bounce
    (reading B13, the default)."""
    c = ragged_corpus
    res = W.wordcount_files(c.paths, WORDS, PATS, chunk=chunk, blocks=blocks, threads=threads,
                            gflags=G.WG | (G.NONBLOCKING if nb else G.BLOCKING) | G.RELAXED, staging=G.STAGE_DEVICE)
    h, hits = oracle_hist_hits(c.paths)
    assert res.wait_rc == 0
    assert np.array_equal(as_u64(res.hist), h)
    assert res.file_hits.tolist() == hits.tolist()
    if not nb:
        want = []
        for s in c.sizes:
            want += [plan.expected_pread_ret(s, r[3], r[4]) for r in plan.wordcount_chunk_requests(s, chunk)]
        assert res.req_ret.tolist() == want


@pytest.mark.parametrize("completion_mode", [G.COMPLETION_PULL], indirect=True)
@pytest.mark.parametrize("length", [16385, 100000, 1 << 20])
@pytest.mark.parametrize("order", [G.STRONG, G.RELAXED])
def test_pread_pull_bounce(file1m, completion_mode, length, order):
    """WG blocking preads into device memory past the pull areas, copied out of the bounce by the
    work-group: every return value and the byte sum every thread computes after the call."""
    size = os.path.getsize(file1m)
    data = np.fromfile(file1m, dtype=np.uint8)
    blocks, iters = 6, 3
    d_buf = torch.zeros(blocks * length, dtype=torch.uint8, device="cuda")
    fd = os.open(file1m, os.O_RDONLY)
    try:
        _, ret, _, sm, rc = W.bench_calls("pread", G.WG | G.BLOCKING | order, blocks, 128, iters, fd, length, size,
                                          d_buf, want_sum=True)
    finally:
        os.close(fd)
    assert rc == 0
    for i in range(blocks * iters):
        off = (i * length) % size
        b = data[off: off + length]
        assert int(ret[i]) == len(b) and int(sm[i]) == int(b.astype(np.int64).sum()), i


def test_wordcount_calls_on_two_streams(ragged_corpus):
    """Back-to-back launches on two streams share the workspace safely: both results
    equal the oracle."""
    c = ragged_corpus
    h, hits = oracle_hist_hits(c.paths)
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
    outs = []
    with W.OpenFiles(c.paths) as of:
        for s in (s1, s2, s1, s2):
            d_hist = torch.zeros(64, dtype=torch.int64, device="cuda")
            d_hits = torch.zeros(len(c.paths), dtype=torch.int32, device="cuda")
            G.gsys_wordcount(of.fds, of.sizes, 16 << 10, WORDS, PATS, d_hist, d_hits, None,
                             G.WG | G.BLOCKING | G.RELAXED, 5, 128, s, G.STAGE_DEVICE)
            outs.append((d_hist, d_hits))
        assert G.gsys_wait() == 0
    for d_hist, d_hits in outs:
        assert np.array_equal(as_u64(d_hist), h)
        assert d_hits.cpu().tolist() == hits.tolist()


def test_kernel_call_sites(file1m):
    """Kernel-scope call sites are GSYS_SITE(0..7); a larger site id is -EINVAL (it used
    to alias site k mod 8)."""
    _, ret, _, _, rc = W.bench_calls("getrusage", G.KERNEL | G.BLOCKING | G.RELAXED | G.SITE(7), 4, 64, 3)
    assert rc == 0 and ret.tolist() == [0, 0, 0]
    _, ret, _, _, rc = W.bench_calls("getrusage", G.KERNEL | G.BLOCKING | G.RELAXED | G.SITE(9), 4, 64, 2)
    assert ret.tolist() == [-errno.EINVAL] * 2


# ---------------------------------------------------------------------------- deferred pulls (B15)
@pytest.mark.parametrize("side_stream", [False, True])
def test_nonblocking_device_preads_are_deferred_and_land(file1m, side_stream):
    """Non-blocking WG and WI preads into device memory are served as deferred pulls (no
    copy-engine transfer per request): each lands when its caller's next call claims the slot, the
    last ones by gsys_wait's flush -- device-wide, or scoped to a side stream (every GPU copier
    claims a record first, reading B15); every buffer holds the bytes of the caller's last read,
    as with the DMA path."""
    size = os.path.getsize(file1m)
    data = open(file1m, "rb").read()
    stream = torch.cuda.Stream() if side_stream else None
    for gran, blocks, threads in ((G.WG, 32, 128), (G.WI, 2, 64)):
        iters, length = 3, 4096
        callers = blocks if gran == G.WG else blocks * threads
        d_buf = torch.zeros(callers * length, dtype=torch.uint8, device="cuda")
        fd = os.open(file1m, os.O_RDONLY)
        G.gsys_stats_reset()
        try:
            _, ret, _, _, rc = W.bench_calls("pread", gran | G.NONBLOCKING, blocks, threads, iters, fd, length, size,
                                             d_buf, stream=stream)
        finally:
            os.close(fd)
        st = G.gsys_stats()
        torch.cuda.synchronize()
        assert rc == 0 and ret.tolist() == [0] * (callers * iters)
        # earlier pulls land when the caller's next call claims the slot, the last ones by the flush
        assert st["deferred"] == callers * iters and 0 < st["flushed"] <= callers * iters, st
        host = d_buf.cpu().numpy()
        for c in range(callers):
            off = ((c * iters + iters - 1) * length) % size
            want = data[off: off + length]
            assert bytes(host[c * length: c * length + len(want)]) == want, c


def test_deferred_pull_ring_overflow_falls_back(tmpdir_shm, file1m):
    """With a 1 MiB deferred range store per worker, 64 KiB non-blocking preads overflow it: the
    rest take the overflow store (GSYS_DEFER_GROW_MB, allocated on the first overflow) and then the
    copy-engine path, each after any pending pull into the same buffer has landed; every buffer
    still ends with the caller's last read (fresh processes: the sizes are fixed at init)."""
    import subprocess
    import sys
    code = f"""
import os, sys, numpy as np, torch
sys.path.insert(0, {repr(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))})
from paper_conf_isca_veselybblor18_b200 import gsys as G, workloads as W
W.ensure_init()
p = {file1m!r}
size = os.path.getsize(p); data = open(p, 'rb').read()
blocks, iters, length = 64, 2, 65536
d = torch.zeros(blocks * length, dtype=torch.uint8, device='cuda')
fd = os.open(p, os.O_RDONLY)
_, ret, _, _, rc = W.bench_calls('pread', G.WG | G.NONBLOCKING, blocks, 64, iters, fd, length, size, d)
os.close(fd)
st = G.gsys_stats()
h = d.cpu().numpy()
for c in range(blocks):
    off = ((c * iters + iters - 1) * length) % size
    want = data[off: off + length]
    got = bytes(h[c * length: c * length + len(want)])
    which = [r for r in range(iters) if got == data[((c * iters + r) * length) % size:][:len(want)]]
    assert got == want, (c, which, st)
assert rc == 0 and 0 < st['deferred'] < blocks * iters and st['flushed'] > 0, st
print('ok', st['deferred'], st['flushed'])
"""
    env = dict(os.environ, GSYS_DEFER_MB="1", GSYS_DEFER_GROW_MB="0", GSYS_THREADS="4")
    out = subprocess.run([sys.executable, "-c", code], env=env, capture_output=True, text=True, timeout=300)
    assert out.returncode == 0 and "ok" in out.stdout, out.stderr[-3000:]
    # with a 1 MiB overflow store allocated on the first overflow: deferred pulls land in both
    # stores, the copy engine takes what neither holds, every buffer still ends with the last read
    env = dict(os.environ, GSYS_DEFER_MB="1", GSYS_DEFER_GROW_MB="1", GSYS_THREADS="4")
    out = subprocess.run([sys.executable, "-c", code], env=env, capture_output=True, text=True, timeout=300)
    assert out.returncode == 0 and "ok" in out.stdout, out.stderr[-3000:]
    # a store large enough for everything: no copy-engine overflow at all
    code_all = code.replace("0 < st['deferred'] < blocks * iters", "st['deferred'] == blocks * iters")
    env = dict(os.environ, GSYS_DEFER_MB="1", GSYS_DEFER_GROW_MB="16", GSYS_THREADS="4")
    out = subprocess.run([sys.executable, "-c", code_all], env=env, capture_output=True, text=True, timeout=300)
    assert out.returncode == 0 and "ok" in out.stdout, out.stderr[-3000:]

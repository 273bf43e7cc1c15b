"""Pins for the CPU oracle (no GPU).  Each test ties the oracle to something other than itself:
hand-derived fixtures, brute force on tiny inputs (Python ``re``/``bytes.find``), POSIX facts
checked through Python's own file reads, closed forms, and by-construction counts recorded by the
input generator (which never tokenizes)."""
import collections
import errno
import itertools
import json
import os
import re

import numpy as np
import pytest

import inputs
import oracle
from oracle import plan, protocol

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")
WORD_RE = re.compile(rb"[A-Za-z0-9_]+")


def brute_counts(text: bytes, words):
    c = collections.Counter(WORD_RE.findall(text))
    return [c.get(w, 0) for w in words]


def test_golden_tiny_wordcount():
    g = json.load(open(os.path.join(GOLDEN, "wordcount_tiny.json")))
    words = [w.encode() for w in g["dict"]]
    got = oracle.count_tokens(g["text"].encode(), words)
    assert list(got) == g["counts"]
    assert oracle.grep(g["text"].encode(), [p.encode() for p in g["grep_patterns"]]) == g["grep_hit"]


def test_exhaustive_tiny_strings():
    """Every string of length <= 7 over {a, b, ' ', '\\n', ','} with dictionary {a,b,ab,ba,aab}."""
    alpha = b"ab \n,"
    words = [b"a", b"b", b"ab", b"ba", b"aab"]
    n = 0
    for L in range(0, 8):
        for tup in itertools.product(alpha, repeat=L):
            s = bytes(tup)
            assert list(oracle.count_tokens(s, words)) == brute_counts(s, words), s
            n += 1
    assert n == sum(5 ** L for L in range(8))


def test_grep_brute_force_random():
    rng = np.random.default_rng(11)
    pats = [b"ab", b"bca", b"aaaa"]
    for _ in range(3000):
        L = int(rng.integers(0, 24))
        s = bytes(rng.choice(list(b"abc "), size=L).tolist())
        want = any(s.find(p) >= 0 for p in pats)
        assert oracle.grep(s, pats) == want, s


def test_token_edges():
    words = [b"x" * 16, b"_", b"A1"]
    # 16-byte word at start and at end of text; a 17-byte token never equals a <=16 B word
    s = b"x" * 16 + b" " + b"x" * 17 + b" _ A1" + b"," + b"x" * 16
    assert list(oracle.count_tokens(s, words)) == [2, 1, 1]
    assert list(oracle.count_tokens(b"", words)) == [0, 0, 0]


@pytest.mark.parametrize("size", [1, 4095, 4096, 4097, (1 << 20) + 777, 3 * (256 << 10) + 5])
def test_generator_census_pins_oracle(size):
    """The generator records each dictionary word it inserted (input construction, no tokenizer);
    the oracle's whole-token counts must equal that census exactly, at any size."""
    words = inputs.dictionary()
    buf, census, _ = inputs.gen_bytes(inputs.SEED_FILE16M, 0, size)
    got = oracle.count_tokens(buf, words)
    assert np.array_equal(got, census)
    assert got[48:].sum() == 0          # absent + adversarial prefix/suffix words: closed-form 0
    if size > 100000:
        assert brute_counts(bytes(buf), words) == [int(x) for x in got]


def test_generator_dictionary_properties():
    words = inputs.dictionary()
    assert len(words) == 64 and len(set(words)) == 64
    assert all(1 <= len(w) <= 16 for w in words)
    assert any(len(w) == 16 for w in words)
    assert all(w.startswith(b"Z") for w in words[48:56])
    pats = inputs.patterns()
    assert len(pats) == 8 and all(12 <= len(p) <= 16 and p[:1].isdigit() for p in pats)


def test_adversarial_words_are_substrings_but_not_tokens():
    """Readings A9: prefixes/suffixes of frequent words occur as substrings but never as tokens."""
    words = inputs.dictionary()
    buf, census, _ = inputs.gen_bytes(inputs.SEED_FILE16M, 0, 1 << 20)
    text = bytes(buf)
    for w in words[56:]:
        assert text.find(w) >= 0
    assert list(oracle.count_tokens(text, words[56:])) == [0] * 8


def test_pread_posix_pins(tmpdir_shm):
    p = os.path.join(tmpdir_shm, "pread.bin")
    data = os.urandom(100000)
    open(p, "wb").write(data)
    fd = os.open(p, os.O_RDONLY)
    try:
        for off, n in [(0, 10), (99990, 100), (100000, 5), (200000, 5), (12345, 0), (1, 99999)]:
            r, b = oracle.pread(fd, n, off)
            assert r == plan.expected_pread_ret(len(data), off, n)
            assert b == data[off: off + n]
    finally:
        os.close(fd)
    r, _ = oracle.pread(fd, 10, 0)          # closed fd
    assert r == -errno.EBADF
    fd = os.open(p, os.O_RDONLY)
    try:
        r, _ = oracle.pread(fd, 10, -1)
        assert r == -errno.EINVAL
    finally:
        os.close(fd)


@pytest.mark.slow
def test_pread_per_call_cap(tmpdir_shm):
    """Linux caps one read at 0x7ffff000 bytes (reading A11; Fig. 7's 2 GB kernel-level pread)."""
    p = os.path.join(tmpdir_shm, "sparse.bin")
    with open(p, "wb") as f:
        f.truncate((1 << 31) + 4096)
    fd = os.open(p, os.O_RDONLY)
    try:
        r, _ = oracle.pread(fd, 1 << 31, 0)
    finally:
        os.close(fd)
        os.unlink(p)
    assert r == 0x7FFFF000 == plan.expected_pread_ret((1 << 31) + 4096, 0, 1 << 31)


@pytest.mark.parametrize("chunk", [1000, 4096, 256 << 10])
def test_read_file_plan_reassembles(tmpdir_shm, chunk):
    size = (1 << 20) + 333
    p = os.path.join(tmpdir_shm, f"plan{chunk}.txt")
    inputs.write_file(p, 5, 1, size)
    got, rets = oracle.read_file_plan(p, chunk)
    assert got == open(p, "rb").read()
    reqs = plan.wordcount_chunk_requests(size, chunk)
    assert len(rets) == len(reqs)
    for (c, s, e, off, ln), r in zip(reqs, rets):
        assert r == plan.expected_pread_ret(size, off, ln)
    assert rets[-1] < reqs[-1][4]      # the last halo request is a short read at EOF


def test_exec_plan_matches_python_reads(tmpdir_shm):
    size = 70000
    p = os.path.join(tmpdir_shm, "mb.txt")
    inputs.write_file(p, 6, 0, size)
    data = open(p, "rb").read()
    reqs = plan.microbench_requests("wg", 5, 64, 3, 4096, size)
    fd = os.open(p, os.O_RDONLY)
    try:
        rets, outs = oracle.exec_plan([fd] * len(reqs), [r[2] for r in reqs], [r[3] for r in reqs])
    finally:
        os.close(fd)
    for (c, r, off, ln), ret, out in zip(reqs, rets, outs):
        assert ret == plan.expected_pread_ret(size, off, ln)
        assert out == data[off: off + ln]


def test_corpus_oracle_pins(tmpdir_shm):
    sizes = [300000, 65536, 1 << 20, 4096 * 5 + 17, 0, 1]
    c = inputs.make_corpus(len(sizes), sizes, seed=9, root=tmpdir_shm, tag="c1")
    words, pats = inputs.dictionary(), inputs.patterns()
    h1, hits1, _, _ = oracle.corpus(c.paths, words, pats, chunk=4096, nthreads=1)
    h4, hits4, _, _ = oracle.corpus(c.paths, words, pats, chunk=256 << 10, nthreads=4)
    assert np.array_equal(h1, c.census) and np.array_equal(h4, c.census)
    assert list(hits1) == list(hits4) == [1 if m else 0 for m in c.pmasks]


def test_grep_plants_known_by_construction(tmpdir_shm):
    c = inputs.make_corpus(24, 64 << 10, seed=2, root=tmpdir_shm, tag="c2")
    words, pats = inputs.dictionary(), inputs.patterns()
    _, hits, _, _ = oracle.corpus(c.paths, words, pats, nthreads=2)
    assert any(c.pmasks) and not all(c.pmasks)
    for f, path in enumerate(c.paths):
        text = open(path, "rb").read()
        per = [text.find(p) >= 0 for p in pats]
        assert per == [bool(c.pmasks[f] >> k & 1) for k in range(8)]
        assert hits[f] == (1 if c.pmasks[f] else 0)


def test_syscall_rate_positive(tmpdir_shm):
    assert oracle.syscall_rate("getrusage", 1, 2000) > 1000
    p = os.path.join(tmpdir_shm, "rate.bin")
    open(p, "wb").write(b"\0" * (1 << 20))
    fd = os.open(p, os.O_RDONLY)
    try:
        assert oracle.syscall_rate("pread", 2, 1000, fd, 4096, 1 << 20) > 1000
    finally:
        os.close(fd)


# ---------------------------------------------------------------- protocol reference model
def test_paper_constants_closed_forms():
    g = json.load(open(os.path.join(GOLDEN, "paper_constants.json")))
    assert g["area_bytes"]["value"] // g["slot_bytes"]["value"] == 20480
    assert 20480 % g["slots_per_hwid"]["value"] == 0 and 20480 // 64 == 320
    assert 1024 // g["wavefront_width"]["value"] == g["wavefronts_per_1024_wg"]["value"]
    assert [protocol.NAMES[s] for s in range(5)] == g["states"]["value"]


def test_protocol_model_paths():
    m = protocol.SlotMachine(4)
    reqs = [(0, 0, True), (1, 1, False), (2, 0, True), (3, 1, False), (4, 3, True)]
    tr = m.run(reqs)
    assert protocol.check_trace(tr, lambda r: dict((a, c) for a, _, c in reqs)[r], 4) == 5
    assert m.state == [protocol.FREE] * 4
    assert len(tr) == sum(len(protocol.expected_path(b)) for _, _, b in reqs)
    # the checker takes the two actors' logs in any order: concatenated GPU log + host log
    gpu = [r for r in tr if r[4] == "gpu"]
    cpu = [r for r in tr if r[4] == "cpu"]
    assert protocol.check_trace(cpu + gpu, lambda r: dict((a, c) for a, _, c in reqs)[r], 4) == 5


def _interleaved_two_slots():
    """A valid concurrent schedule: requests 0 (slot 0, blocking) and 1 (slot 1, non-blocking)
    overlap in time; then request 2 reuses slot 1 after the host freed it."""
    m = protocol.SlotMachine(2)
    m.claim(0, 0); m.claim(1, 1); m.publish(1, 1); m.publish(0, 0)
    m.pick_up(0, 0); m.pick_up(1, 1); m.complete(1, 1, False); m.complete(0, 0, True)
    assert not m.claim(2, 0)                  # slot 0 still finished: the caller is delayed (P24.11)
    m.claim(2, 1); m.consume(0, 0); m.publish(2, 1); m.pick_up(2, 1); m.complete(2, 1, True); m.consume(2, 1)
    return m.trace, {0: True, 1: False, 2: True}


def test_protocol_interleaved_schedule_is_valid():
    tr, blk = _interleaved_two_slots()
    assert protocol.check_trace(tr, blk.__getitem__, 2) == 3


def _retime(tr, req, edge, t):
    return [r if (r[0], r[2], r[3]) != (req,) + edge else r[:5] + (t,) for r in tr]


def test_protocol_model_rejects_violations():
    m = protocol.SlotMachine(2)
    assert m.claim(0, 0)
    assert not m.claim(1, 0)                          # P24.11: slot not free -> delayed
    with pytest.raises(AssertionError):
        m.process(0, 0, True)                          # populating -> processing is illegal
    good = protocol.SlotMachine(1).run([(7, 0, True)])
    blk = lambda r: True  # noqa: E731
    with pytest.raises(AssertionError):                # dropped edge
        protocol.check_trace(good[:-1], blk)
    with pytest.raises(AssertionError):                # duplicated edge
        protocol.check_trace(good + [good[2]], blk)
    with pytest.raises(AssertionError):                # wrong actor
        bad = list(good)
        bad[2] = bad[2][:4] + ("gpu",) + bad[2][5:]
        protocol.check_trace(bad, blk)
    with pytest.raises(AssertionError):                # non-blocking request that waited for finished
        protocol.check_trace(good, lambda r: False)


def test_protocol_rejects_host_pickup_before_ready():
    tr, blk = _interleaved_two_slots()
    t_ready = [r for r in tr if r[0] == 0 and r[3] == protocol.READY][0][5]
    bad = _retime(tr, 0, (protocol.READY, protocol.PROCESSING), t_ready - 3)
    with pytest.raises(AssertionError, match="precedes"):
        protocol.check_trace(bad, blk.__getitem__)
    # within the cross-actor clock error it is accepted, beyond it not
    assert protocol.check_trace(bad, blk.__getitem__, eps=3) == 3
    with pytest.raises(AssertionError, match="precedes"):
        protocol.check_trace(bad, blk.__getitem__, eps=2)


def test_protocol_rejects_consume_before_finish():
    tr, blk = _interleaved_two_slots()
    t_fin = [r for r in tr if r[0] == 2 and r[3] == protocol.FINISHED][0][5]
    bad = _retime(tr, 2, (protocol.FINISHED, protocol.FREE), t_fin - 1)
    with pytest.raises(AssertionError, match="precedes"):
        protocol.check_trace(bad, blk.__getitem__)


def test_protocol_rejects_two_live_requests_on_one_slot():
    # request 2 claims slot 1 while request 1 (non-blocking) is still being processed there
    m = protocol.SlotMachine(2)
    tr, blk = _interleaved_two_slots()
    t_free1 = [r for r in tr if r[0] == 1 and r[3] == protocol.FREE][0][5]
    bad = _retime(tr, 2, (protocol.FREE, protocol.POPULATING), t_free1 - 2)
    with pytest.raises(AssertionError, match="live"):
        protocol.check_trace(bad, blk.__getitem__)
    # the same overlap on the blocking slot: two requests on slot 0, the second claimed before
    # the first was consumed (both GPU edges: no clock slack applies)
    trace = m.run([(10, 0, True)]) + [(11, 0, protocol.FREE, protocol.POPULATING, "gpu", 4),
                                     (11, 0, protocol.POPULATING, protocol.READY, "gpu", 6),
                                     (11, 0, protocol.READY, protocol.PROCESSING, "cpu", 7),
                                     (11, 0, protocol.PROCESSING, protocol.FINISHED, "cpu", 8),
                                     (11, 0, protocol.FINISHED, protocol.FREE, "gpu", 9)]
    with pytest.raises(AssertionError, match="live"):
        protocol.check_trace(trace, lambda r: True, eps=100)
    ok = [r if r[0] == 10 else r[:5] + (r[5] + 10,) for r in trace]
    assert protocol.check_trace(ok, lambda r: True, eps=0) == 2


def test_protocol_rejects_sequence_going_backwards():
    trace = protocol.SlotMachine(1).run([((0, 5), 0, True), ((0, 4), 0, True)])
    with pytest.raises(AssertionError, match="sequence"):
        protocol.check_trace(trace, lambda r: True, seq_of=lambda r: r[1])
    trace = protocol.SlotMachine(1).run([((0, 4), 0, True), ((0, 5), 0, False)])
    assert protocol.check_trace(trace, lambda r: r[1] == 4, seq_of=lambda r: r[1]) == 2


def test_request_count_closed_forms():
    assert protocol.requests_per_call("wi", 148 * 4 * 256, 148 * 4) == 151552
    assert protocol.requests_per_call("wg", 151552, 592) == 592
    assert protocol.requests_per_call("kernel", 151552, 592) == 1
    assert len(plan.microbench_requests("wi", 3, 64, 2, 4096, 1 << 20)) == 3 * 64 * 2
    assert len(plan.microbench_requests("kernel", 3, 64, 5, 4096, 1 << 20)) == 5


def test_count_key_brute_force():
    rng = np.random.default_rng(4)
    for _ in range(500):
        n = int(rng.integers(0, 60))
        d = bytes(rng.choice(list(b"ab"), size=n).tolist())
        k = bytes(rng.choice(list(b"ab"), size=int(rng.integers(1, 4))).tolist())
        assert oracle.count_key(d, k) == sum(1 for i in range(len(d) - len(k) + 1) if d[i:i + len(k)] == k)


def test_amr_release_rule():
    lv = [[1, 0, 2, 3], [0, 0, 1, 3], [2, 2, 0, 3]]
    assert plan.amr_released(lv) == [2, 1, 3, 0]
    assert plan.amr_released(lv, rss_ok=[False, True, True]) == [2, 2, 3, 0]


def test_owned_counts_partition_sums_to_whole():
    """tests/ownership.owned_counts (used by the GPU fault-injection test) is pinned here: for any
    chunking, the per-chunk owned counts add up to the whole-text counts."""
    from ownership import owned_counts
    rng = np.random.default_rng(11)
    words = [b"a", b"ab", b"ba", b"b_1", b"abc"]
    for _ in range(300):
        n = int(rng.integers(0, 60))
        text = bytes(rng.choice(list(b"ab_1 ,\n"), size=n).tolist())
        whole = oracle.count_tokens(text, words)
        chunk = int(rng.integers(1, 12))
        tot = np.zeros(len(words), dtype=np.uint64)
        for s in range(0, n, chunk):
            tot += owned_counts(text, s, min(s + chunk, n), words)
        assert np.array_equal(tot, whole), (text, chunk)


def test_permuted_blocks_hand_worked_example():
    """plan.permuted_blocks (Fig. 8, PAPER.md:26 P26.21-27) against a hand-derived 4-block example
    (tests/golden/fig8_permutation_tiny.json): gather direction (reading A20), one step per
    iteration, blocks independent; the scatter direction is rejected."""
    g = json.load(open(os.path.join(GOLDEN, "fig8_permutation_tiny.json")))
    data = np.array(g["data"], dtype=np.uint8)
    perm = np.array(g["perm"])
    for k, want in g["expected"].items():
        got = plan.permuted_blocks(data, perm, int(k), g["block_bytes"])
        assert got.tolist() == want, k
    assert plan.permuted_blocks(data, perm, 1, 4).tolist() != g["scatter_reading_1_step"]


def test_permuted_blocks_group_properties():
    """Iterations compose (p^a then p^b = p^(a+b)) and the permutation's order restores the input."""
    rng = np.random.default_rng(5)
    bs = 64
    perm = rng.permutation(bs)
    data = rng.integers(0, 256, size=4 * bs, dtype=np.uint8)
    for a, b in [(1, 2), (3, 5), (0, 4)]:
        once = plan.permuted_blocks(plan.permuted_blocks(data, perm, a, bs), perm, b, bs)
        assert np.array_equal(once, plan.permuted_blocks(data, perm, a + b, bs))
    # order of the permutation = lcm of its cycle lengths
    import math
    seen, lcm = np.zeros(bs, bool), 1
    for i in range(bs):
        if not seen[i]:
            n, j = 0, i
            while not seen[j]:
                seen[j] = True
                j = perm[j]
                n += 1
            lcm = lcm * n // math.gcd(lcm, n)
    assert np.array_equal(plan.permuted_blocks(data, perm, lcm, bs), data)
    if lcm > 1:
        assert not np.array_equal(plan.permuted_blocks(data, perm, 1, bs), data)

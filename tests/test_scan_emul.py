"""CPU checks of the CUDA path's scan logic (no GPU): tests/native/scan_emul.cu compiles the same
csrc/scan_core.cuh (byte DFA) and csrc/tokscan.cuh (token-level scan) the sm_100a kernels use into a
host library that walks the chunks/lane spans sequentially; results must equal the oracle
bit-exactly."""
import ctypes
import os
import subprocess

import numpy as np
import pytest

import inputs
import oracle
from paper_conf_isca_veselybblor18_b200.gsys import pack_words

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
SRC = os.path.join(HERE, "native", "scan_emul.cu")
LIB = os.path.join(HERE, "native", "libscanemul.so")
DEPS = [SRC, os.path.join(ROOT, "paper_conf_isca_veselybblor18_b200", "csrc", "scan_core.cuh"),
        os.path.join(ROOT, "paper_conf_isca_veselybblor18_b200", "csrc", "tokscan.cuh")]


@pytest.fixture(scope="module")
def emul():
    if not os.path.exists(LIB) or any(os.path.getmtime(d) > os.path.getmtime(LIB) for d in DEPS):
        subprocess.check_call(["g++", "-O2", "-std=c++17", "-x", "c++", "-fPIC", "-shared",
                               "-I", os.path.join(ROOT, "paper_conf_isca_veselybblor18_b200", "csrc"),
                               "-I", os.path.join(ROOT, "include"), "-I", "/usr/local/cuda/include",
                               "-o", LIB, SRC])
    L = ctypes.CDLL(LIB)
    P = ctypes.c_void_p
    L.scan_emul2.argtypes = [P, ctypes.c_uint64, ctypes.c_uint32, ctypes.c_char_p, P, ctypes.c_uint32,
                             ctypes.c_char_p, P, ctypes.c_uint32, P, P, ctypes.c_int]

    def run(text, words, pats, chunk):
        h0, g0 = run2(text, words, pats, chunk, 0)
        for mode in (1, 2, 3, 4):
            # 1: wc_kernel's 64-byte lane spans (77-column table); 2: scan_kernel's lane spans (129
            # columns, raw-byte fast path); 3: 16-byte reference steps on the 129-column table;
            # 4: the warp-cooperative token scan (tokscan.cuh tokw_*: per-tile start lists, then
            # lookups)
            h, g = run2(text, words, pats, chunk, mode)
            assert np.array_equal(h0, h) and g0 == g, mode
        return h0, g0

    def run2(text, words, pats, chunk, pairs):
        arr = np.frombuffer(text, dtype=np.uint8) if isinstance(text, (bytes, bytearray)) else text
        d, dl = pack_words(words)
        p, pl = pack_words(pats) if pats else (b"", None)
        hist = np.zeros(len(words), dtype=np.uint64)
        hit = ctypes.c_uint32(0)
        rc = L.scan_emul2(arr.ctypes.data, arr.size, chunk, d, dl, len(words), p, pl, len(pats), hist.ctypes.data,
                          ctypes.byref(hit), pairs)
        assert rc == 0
        return hist, bool(hit.value)
    return run


@pytest.mark.parametrize("size", [1, 15, 16, 17, 31, 33, 4095, 4097, 12345, (1 << 20) + 7])
@pytest.mark.parametrize("chunk", [16, 48, 4096, 256 << 10])
def test_scan_emul_matches_oracle_generated(emul, size, chunk):
    words, pats = inputs.dictionary(), inputs.patterns()
    buf, census, _ = inputs.gen_bytes(inputs.SEED_FILE16M, 3, size)
    hist, hit = emul(buf, words, pats, chunk)
    assert np.array_equal(hist, oracle.count_tokens(buf, words))
    assert np.array_equal(hist, census)
    assert hit == oracle.grep(buf, pats)


def test_scan_emul_grep_positive_files(emul):
    words, pats = inputs.dictionary(), inputs.patterns()
    seen = 0
    for fid in range(40):
        buf, census, pm = inputs.gen_bytes(inputs.SEED_CORPUS, fid, 64 << 10, grep_plants=True)
        for chunk in (4096, 256 << 10):
            hist, hit = emul(buf, words, pats, chunk)
            assert hit == bool(pm) == oracle.grep(buf, pats)
            assert np.array_equal(hist, census)
        seen += bool(pm)
    assert seen > 0


def test_scan_emul_random_small_alphabet(emul):
    """Dense adversarial text: tokens of every length, dictionary with prefixes/suffixes."""
    rng = np.random.default_rng(5)
    words = [b"a", b"b", b"ab", b"ba", b"aab", b"_", b"A9", b"a" * 16, b"b" * 15, b"ab" * 8]
    pats = [b"aab", b"b_a", b"9 ", b"ab" * 8]
    alpha = np.frombuffer(b"ab _,\n9A", dtype=np.uint8)
    for trial in range(30):
        n = int(rng.integers(1, 3000))
        p = np.array([0.3, 0.3, 0.15, 0.05, 0.05, 0.05, 0.05, 0.05])
        text = alpha[rng.choice(len(alpha), size=n, p=p)]
        for chunk in (16, 32, 64, 1024):
            hist, hit = emul(text, words, pats, chunk)
            assert np.array_equal(hist, oracle.count_tokens(text, words)), (trial, chunk)
            assert hit == oracle.grep(text, pats)


def test_scan_emul_long_tokens_and_high_bytes(emul):
    words = [b"x" * 16, b"y", b"\xc3"[:0] + b"z"]
    text = (b"x" * 16 + b" " + b"x" * 17 + b"\xc3\xa9y y\xffz " + b"x" * 16) * 50
    for chunk in (16, 32, 4096):
        hist, _ = emul(text, words, [], chunk)
        assert np.array_equal(hist, oracle.count_tokens(text, words))


def test_scan_emul_duplicate_and_nonword_dictionary_entries(emul):
    words = [b"ab", b"ab", b"a-b", b"x", b"x_y", b"Q"]
    text = b"ab a-b ab, x x_y xQ Q ab_ a b " * 20
    for chunk in (16, 64):
        hist, _ = emul(text, words, [], chunk)
        assert np.array_equal(hist, oracle.count_tokens(text, words))
        assert hist[1] == 0 and hist[2] == 0


@pytest.mark.parametrize("pattern", [b"a ", b" a", b"ab ", b"a b c d e f g h ", b"aaaaaaaaaaaaaaaaa ", b"9_"])
def test_scan_emul_dense_tokens(emul, pattern):
    """One token per 2 bytes (the token scan's per-tile start list at its 1024-entry maximum),
    1-byte and 16-byte words, 17-byte tokens; every scan form equals the oracle."""
    words = [b"a", b"b", b"ab", b"h", b"9_", b"aaaaaaaaaaaaaaaa"]
    for size in (2048, 2049, 4095, 70_001):
        text = (pattern * (size // len(pattern) + 1))[:size]
        arr = np.frombuffer(text, dtype=np.uint8)
        for chunk in (16, 2048, 256 << 10):
            h, g = emul(arr, words, [b"b c"], chunk)
            assert np.array_equal(h, oracle.count_tokens(arr, words)[:len(words)]), (pattern, size, chunk)
            assert g == oracle.grep(arr, [b"b c"])

"""Seeded synthetic text corpus (input construction only -- none of the method's arithmetic).

The byte-level recipe lives in ``gen_corpus.c`` (see its header and DESIGN.md "Input recipe").
This module compiles it with gcc on first use, and writes files to a directory (tmpfs by
default, like the paper's pread microbenchmark on tmpfs, sec. VII, P26.5).

Seeds: 16 MiB file seed 1, corpus seed 2 (file i keyed by (2, i)),
dictionary seed 3, grep-plant seed 4.
"""
from __future__ import annotations

import ctypes
import hashlib
import json
import os
import subprocess
import threading
from dataclasses import dataclass, field

import numpy as np

NDICT = 64
NPAT = 8
SEED_FILE16M = 1
SEED_CORPUS = 2
SEED_DICT = 3
SEED_PLANTS = 4

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "gen_corpus.c")
_LIB = os.path.join(_HERE, "libgsysgen.so")
_lock = threading.Lock()
_lib = None
_inited_seed = None


def build() -> str:
    """Compile gen_corpus.c -> libgsysgen.so (plain gcc; no GPU needed)."""
    if (not os.path.exists(_LIB)) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-shared", "-fPIC", "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


def _load(dict_seed: int = SEED_DICT):
    global _lib, _inited_seed
    with _lock:
        if _lib is None:
            build()
            lib = ctypes.CDLL(_LIB)
            lib.gen_init.argtypes = [ctypes.c_uint64]
            lib.gen_dict.argtypes = [ctypes.c_char_p, ctypes.c_void_p]
            lib.gen_patterns.argtypes = [ctypes.c_char_p, ctypes.c_void_p]
            lib.gen_dict_rank.argtypes = [ctypes.c_int]
            lib.gen_file.argtypes = [ctypes.c_uint64, ctypes.c_uint64, ctypes.c_uint64, ctypes.c_int,
                                     ctypes.c_void_p, ctypes.c_uint64, ctypes.c_void_p, ctypes.c_void_p]
            _lib = lib
        if _inited_seed != dict_seed:
            rc = _lib.gen_init(dict_seed)
            if rc != 0:
                raise RuntimeError(f"gen_init({dict_seed}) failed: {rc}")
            _inited_seed = dict_seed
    return _lib


def _table(fn, n, dict_seed):
    lib = _load(dict_seed)
    buf = ctypes.create_string_buffer(17 * n)
    lens = (ctypes.c_uint8 * n)()
    getattr(lib, fn)(buf, ctypes.addressof(lens))
    raw = buf.raw
    return [raw[17 * i: 17 * i + lens[i]] for i in range(n)]


def dictionary(dict_seed: int = SEED_DICT) -> list[bytes]:
    """The 64 wordcount strings (P32.6)."""
    return _table("gen_dict", NDICT, dict_seed)


def patterns(dict_seed: int = SEED_DICT) -> list[bytes]:
    """The 8 grep -F patterns (P30.27)."""
    return _table("gen_patterns", NPAT, dict_seed)


def dict_ranks(dict_seed: int = SEED_DICT) -> list[int]:
    lib = _load(dict_seed)
    return [lib.gen_dict_rank(j) for j in range(NDICT)]


def gen_bytes(seed: int, file_id: int, size: int, grep_plants: bool = False,
              plant_seed: int = SEED_PLANTS, dict_seed: int = SEED_DICT):
    """Generate one file in memory -> (uint8 ndarray, census uint64[64], pattern bitmask)."""
    lib = _load(dict_seed)
    buf = np.empty(size, dtype=np.uint8)
    census = np.zeros(NDICT, dtype=np.uint64)
    pmask = ctypes.c_uint32(0)
    rc = lib.gen_file(seed, file_id, plant_seed, int(grep_plants), buf.ctypes.data, size,
                      census.ctypes.data, ctypes.addressof(pmask))
    if rc != 0:
        raise RuntimeError("gen_file failed")
    return buf, census, int(pmask.value)


def write_file(path: str, seed: int, file_id: int, size: int, grep_plants: bool = False,
               plant_seed: int = SEED_PLANTS, dict_seed: int = SEED_DICT):
    buf, census, pmask = gen_bytes(seed, file_id, size, grep_plants, plant_seed, dict_seed)
    tmp = path + ".tmp"
    with open(tmp, "wb") as f:
        f.write(memoryview(buf))
    os.replace(tmp, path)
    return census, pmask


@dataclass
class Corpus:
    root: str
    paths: list[str]
    sizes: list[int]
    census: np.ndarray            # uint64[64] summed over files (emissions by construction)
    pmasks: list[int]             # grep patterns planted per file (bitmask over 8 patterns)
    seed: int
    meta: dict = field(default_factory=dict)

    @property
    def total_bytes(self) -> int:
        return int(sum(self.sizes))

    def grep_files(self) -> list[int]:
        """Files containing at least one planted pattern (the grep -F -l answer by construction)."""
        return [i for i, m in enumerate(self.pmasks) if m]


def default_root() -> str:
    base = "/dev/shm" if os.path.isdir("/dev/shm") else "/tmp"
    return os.path.join(base, "gsys_corpus")


def make_corpus(nfiles: int, file_size, seed: int = SEED_CORPUS, grep_plants: bool = True,
                root: str | None = None, threads: int | None = None,
                plant_seed: int = SEED_PLANTS, dict_seed: int = SEED_DICT,
                tag: str | None = None) -> Corpus:
    """Write (or reuse) nfiles seeded files.  file_size may be an int or a list of ints."""
    sizes = list(file_size) if isinstance(file_size, (list, tuple)) else [int(file_size)] * nfiles
    assert len(sizes) == nfiles
    key = hashlib.sha1(json.dumps([nfiles, sizes, seed, grep_plants, plant_seed, dict_seed]).encode()).hexdigest()[:12]
    root = root or default_root()
    d = os.path.join(root, tag or f"c{key}")
    os.makedirs(d, exist_ok=True)
    manifest = os.path.join(d, "manifest.json")
    paths = [os.path.join(d, f"f{i:05d}.txt") for i in range(nfiles)]
    if os.path.exists(manifest):
        with open(manifest) as f:
            m = json.load(f)
        if m.get("key") == key and all(os.path.exists(p) and os.path.getsize(p) == s for p, s in zip(paths, sizes)):
            return Corpus(d, paths, sizes, np.array(m["census"], dtype=np.uint64), m["pmasks"], seed, m)
    _load(dict_seed)
    census = np.zeros((nfiles, NDICT), dtype=np.uint64)
    pmasks = [0] * nfiles
    nthr = threads or min(32, len(os.sched_getaffinity(0)))
    nxt = [0]
    lk = threading.Lock()

    def work():
        while True:
            with lk:
                i = nxt[0]
                nxt[0] += 1
            if i >= nfiles:
                return
            c, pm = write_file(paths[i], seed, i, sizes[i], grep_plants, plant_seed, dict_seed)
            census[i] = c
            pmasks[i] = pm

    ts = [threading.Thread(target=work) for _ in range(nthr)]
    for t in ts:
        t.start()
    for t in ts:
        t.join()
    tot = census.sum(axis=0, dtype=np.uint64)
    m = {"key": key, "census": [int(x) for x in tot], "pmasks": pmasks, "sizes": sizes, "seed": seed}
    with open(manifest, "w") as f:
        json.dump(m, f)
    return Corpus(d, paths, sizes, tot, pmasks, seed, m)


# ---------------------------------------------------------------------------- config 5 inputs
SEED_AMR = 6
SEED_SIGNAL = 7


def amr_levels(iters: int, nblocks: int, seed: int = SEED_AMR, p_coarsen: float = 0.04):
    """Refinement level per (iteration, block) for the AMR-style mesh (config 5a, PAPER.md:28
    sec. VIII-A: "when lower resolution is possible ... miniamr reduces memory"): level 1..3, and 0
    (block coarsened, its host mirror may be released) with probability p_coarsen."""
    rng = np.random.default_rng(seed)
    lv = rng.integers(1, 4, size=(iters, nblocks), dtype=np.uint8)
    lv[rng.random((iters, nblocks)) < p_coarsen] = 0
    return lv


def signal_blocks(nblocks: int, block_bytes: int, seed: int = SEED_SIGNAL):
    """Data array for signal-search (config 5b, sec. VIII-B): synthetic text blocks."""
    buf, _, _ = gen_bytes(seed, 0, nblocks * block_bytes)
    return buf


SEED_PERM = 9


def perm_inputs(nblocks: int, block_bytes: int = 8192, seed: int = SEED_PERM):
    """Fig. 8 inputs (sec. VII: "The input data array is preloaded with random values
    and divided into 8KB blocks"): random bytes and a fixed random permutation of block positions."""
    rng = np.random.default_rng(seed)
    data = rng.integers(0, 256, size=nblocks * block_bytes, dtype=np.uint8)
    perm = rng.permutation(block_bytes).astype(np.uint16)
    return data, perm

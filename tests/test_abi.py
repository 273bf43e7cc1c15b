"""C-ABI checks that need no GPU: libgsys builds for sm_100a, loads, exports every function
include/gsys.h declares, reports the paper's slot layout, and its coalescing planner (reading A8)
is correct against brute force."""
import errno
import os
import subprocess

import numpy as np
import pytest

from paper_conf_isca_veselybblor18_b200 import build as B
from paper_conf_isca_veselybblor18_b200 import gsys as G


def test_library_exports_header_functions():
    L = G.lib()
    names = G.header_functions()
    assert len(names) >= 15
    missing = [n for n in names if not hasattr(L, n)]
    assert not missing
    assert set(G.SIGNATURES) == set(names)


def test_sass_is_sm100a():
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", B.LIB], capture_output=True, text=True)
    assert "sm_100a" in out.stdout


def test_slot_layout_matches_paper():
    import json
    g = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "paper_constants.json")))
    slot, inline, nstates = G.gsys_abi_info()
    assert slot == g["slot_bytes"]["value"] == 64          # P24.7
    assert nstates == len(g["states"]["value"]) == 5       # P24.10-34
    assert inline >= 144                                   # struct rusage


def test_calls_without_gpu_fail_cleanly():
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    L = G.lib()
    assert L.gsys_init(0, 0) == -errno.ENODEV
    assert L.gsys_wait(None) == -errno.ENODEV
    assert L.gsys_shutdown() == 0
    assert L.gsys_init(1 << 25, 0) == -errno.EINVAL


def brute_groups(fds, offs, lens, max_union):
    order = sorted(range(len(fds)), key=lambda i: (fds[i], offs[i]))
    groups = []
    for i in order:
        if groups:
            g = groups[-1]
            u0, u1, fd = g["u0"], g["u1"], g["fd"]
            if fds[i] == fd and offs[i] <= u1 and max(u1, offs[i] + lens[i]) - u0 <= max_union and lens[i] > 0:
                g["m"].append(i)
                g["u1"] = max(u1, offs[i] + lens[i])
                continue
        groups.append({"fd": fds[i], "u0": offs[i], "u1": offs[i] + lens[i], "m": [i]})
    return groups


def test_plan_merge_random_vs_brute():
    rng = np.random.default_rng(3)
    for _ in range(300):
        n = int(rng.integers(1, 12))
        fds = rng.integers(3, 5, size=n).tolist()
        offs = rng.integers(0, 200, size=n).tolist()
        lens = rng.integers(0, 60, size=n).tolist()
        mu = int(rng.integers(30, 400))
        order, group, oig, goff, glen = G.gsys_plan_merge(fds, offs, lens, mu)
        want = brute_groups(fds, offs, lens, mu)
        assert len(goff) == len(want)
        for gi, g in enumerate(want):
            assert goff[gi] == g["u0"] and glen[gi] == g["u1"] - g["u0"]
            for i in g["m"]:
                assert group[i] == gi and oig[i] == offs[i] - g["u0"]


def test_split_result_equals_individual_pread(tmpdir_shm):
    """A merged union read split with clamp(r - (off_i - u0), 0, len_i) returns exactly what each
    pread would have returned on a regular file of stable size (reading A8), incl. EOF."""
    p = os.path.join(tmpdir_shm, "split.bin")
    data = os.urandom(5000)
    open(p, "wb").write(data)
    fd = os.open(p, os.O_RDONLY)
    try:
        rng = np.random.default_rng(1)
        for _ in range(200):
            n = int(rng.integers(2, 8))
            offs = np.sort(rng.integers(0, 5200, size=n)).tolist()
            lens = rng.integers(1, 900, size=n).tolist()
            order, group, oig, goff, glen = G.gsys_plan_merge([fd] * n, offs, lens, 1 << 20)
            for gi in range(len(goff)):
                u = os.pread(fd, int(glen[gi]), int(goff[gi]))
                for i in range(n):
                    if group[i] != gi:
                        continue
                    r = G.gsys_split_result(len(u), int(oig[i]), lens[i])
                    want = os.pread(fd, lens[i], offs[i])
                    assert r == len(want)
                    assert u[int(oig[i]): int(oig[i]) + r] == want
    finally:
        os.close(fd)
    assert G.gsys_split_result(-errno.EIO, 5, 10) == -errno.EIO


@pytest.mark.parametrize("seed", [1, 2, 3, 12345])
@pytest.mark.parametrize("cap", [4096, 1 << 20, 32 << 20])
def test_bounce_ring_never_overlaps_inflight(seed, cap):
    """Regression for the wrap bug: a wrapped allocation must wait for the previous lap's tail
    and for the current lap's oldest regions before reusing bounce memory."""
    assert G.lib().gsys_selftest_bounce(seed, 20000, cap) == 0

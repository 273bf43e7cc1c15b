"""N > 1 plumbing on CPU (gloo, world_size 2): file sharding + the single all_reduce produce the
whole-corpus answer.  Each rank computes its shard with the CPU oracle as a stand-in for the GPU
kernel (the GPU path itself is covered by the -m gpu tests)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import inputs
import oracle
from paper_conf_isca_veselybblor18_b200 import dist as D


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, paths, out_dir):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    words, pats = inputs.dictionary(), inputs.patterns()
    lo, hi = D.shard_range(len(paths), rank, world)
    if hi > lo:
        h, hits, _, _ = oracle.corpus(paths[lo:hi], words, pats, nthreads=2)
    else:
        h, hits = np.zeros(64, dtype=np.uint64), np.zeros(0, dtype=np.uint32)
    v = D.pack_result(torch.from_numpy(h.astype(np.int64)), torch.from_numpy(hits.astype(np.int64)), lo, hi,
                      len(paths))
    D.reduce_result(v)
    np.save(os.path.join(out_dir, f"r{rank}.npy"), v.numpy())
    dist.destroy_process_group()


@pytest.mark.parametrize("nfiles", [7, 12])
def test_sharded_allreduce_equals_whole_corpus(tmpdir_shm, tmp_path, nfiles):
    c = inputs.make_corpus(nfiles, [50000 + 4099 * i for i in range(nfiles)], seed=inputs.SEED_CORPUS,
                           root=tmpdir_shm, tag=f"dist{nfiles}")
    world = 2
    mp.start_processes(_worker, args=(world, _free_port(), c.paths, str(tmp_path)), nprocs=world,
                       start_method="spawn", join=True)
    v0 = np.load(tmp_path / "r0.npy")
    v1 = np.load(tmp_path / "r1.npy")
    assert np.array_equal(v0, v1)                      # every rank holds the reduced answer
    assert np.array_equal(v0[:64].astype(np.uint64), c.census)
    assert v0[64:].tolist() == [1 if m else 0 for m in c.pmasks]


def test_shard_ranges_partition():
    for n in (0, 1, 5, 512):
        for w in (1, 2, 3, 8):
            rs = [D.shard_range(n, r, w) for r in range(w)]
            assert rs[0][0] == 0 and rs[-1][1] == n
            assert all(a[1] == b[0] for a, b in zip(rs, rs[1:]))
            assert max(h - l for l, h in rs) - min(h - l for l, h in rs) <= 1

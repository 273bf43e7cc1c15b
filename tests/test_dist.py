"""N > 1 plumbing on CPU (gloo, world_size 2): file sharding + the single all_reduce produce the
whole-corpus answer.  Each rank computes its shard with the CPU oracle as a stand-in for the GPU
kernel; the same plumbing around the real GPU path is tests/test_gpu_dist.py (-m gpu).  Also the
bench launcher: `--gpus N` spawns N ranks, and a rank count other than --gpus is refused."""
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


def _bench(args, env=None, timeout=600):
    import json
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    out = subprocess.run([sys.executable, os.path.join(root, "bench.py"), *args], env=env, capture_output=True,
                         text=True, timeout=timeout, cwd=root)
    lines = [json.loads(ln) for ln in out.stdout.splitlines() if ln.startswith("{")]
    return out, lines


def test_bench_spawns_ranks_itself(tmpdir_shm):
    """`bench.py --gpus 2` outside torchrun re-launches itself as 2 ranks (here the CPU reference
    arm: rank 0 times the oracle and prints the one line, rank 1 exits 0)."""
    env = {k: v for k, v in os.environ.items() if k not in ("WORLD_SIZE", "RANK", "LOCAL_RANK")}
    out, lines = _bench(["--impl", "reference", "--gpus", "2", "--files", "2", "--file-mib", "1", "--steps", "1",
                         "--warmup", "1", "--root", os.path.join(tmpdir_shm, "bref")], env=env)
    assert out.returncode == 0, out.stderr[-2000:]
    assert len(lines) == 1 and lines[0]["impl"] == "reference" and lines[0]["n_gpus"] == 2


def test_bench_rejects_world_mismatch(tmpdir_shm):
    """A launch whose rank count differs from --gpus fails loudly instead of timing something else."""
    env = dict(os.environ, WORLD_SIZE="1", RANK="0", LOCAL_RANK="0")
    out, _ = _bench(["--gpus", "2", "--files", "2", "--file-mib", "1", "--steps", "1", "--warmup", "3",
                     "--no-extras", "--no-cpu-baseline", "--root", os.path.join(tmpdir_shm, "bench_mm")], env=env)
    assert out.returncode != 0 and "--gpus 2" in (out.stderr + out.stdout)

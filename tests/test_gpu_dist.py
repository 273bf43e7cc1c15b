"""Multi-rank GPU path (row a9) on the one-GPU test box: N ranks, each with
its own libgsys instance on cuda:0, shard the corpus by whole files, run the real GPU path and
all-reduce over gloo (NCCL refuses two ranks on one device); the reduced histogram and grep
vector equal the CPU oracle's over the whole corpus, element by element.  Plus the bench launcher:
`bench.py --gpus 2` spawns its ranks itself."""
import json
import os
import socket
import subprocess
import sys

import numpy as np
import pytest
import torch

import inputs
import oracle

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


@pytest.fixture(scope="module", autouse=True)
def need_gpu():
    if not torch.cuda.is_available():
        pytest.skip("needs a GPU")


@pytest.mark.parametrize("world,staging,chunk", [(2, "device", 256 << 10), (2, "host", 64 << 10),
                                                 (3, "device", 16 << 10)])
def test_sharded_gpu_path_equals_oracle(tmpdir_shm, tmp_path, world, staging, chunk):
    sizes = [(1 << 20) + 4099 * i for i in range(9)] + [0, 17]
    c = inputs.make_corpus(len(sizes), sizes, seed=inputs.SEED_CORPUS, root=tmpdir_shm, tag=f"gdist{world}")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={world}",
           "--master-addr=127.0.0.1", f"--master-port={_port()}", os.path.join(ROOT, "tests", "dist_gpu_worker.py"),
           str(tmp_path), staging, str(chunk), *c.paths]
    subprocess.run(cmd, check=True, timeout=600, cwd=ROOT)
    vs = [np.load(tmp_path / f"r{r}.npy") for r in range(world)]
    for v in vs[1:]:
        assert np.array_equal(v, vs[0])                   # every rank holds the reduced answer
    h, hits, _, _ = oracle.corpus(c.paths, inputs.dictionary(), inputs.patterns(), nthreads=4)
    assert np.array_equal(vs[0][:64].astype(np.uint64), h)
    assert vs[0][64:].tolist() == hits.astype(np.int64).tolist()


def test_bench_spawns_ranks(tmpdir_shm):
    """`python bench.py --gpus 2` (no torchrun around it) launches 2 ranks and prints one line whose
    reduced result matches the generator census and planted grep set."""
    env = dict(os.environ, GSYS_BENCH_ONE_GPU="1")
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "2", "--files", "8",
                          "--file-mib", "2", "--steps", "2", "--warmup", "3", "--no-extras", "--no-cpu-baseline",
                          "--root", os.path.join(tmpdir_shm, "bench2")], env=env, capture_output=True, text=True,
                         timeout=900, cwd=ROOT)
    assert out.returncode == 0, out.stderr[-3000:]
    lines = [ln for ln in out.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, out.stdout
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["parity"]["hist_equals_generator_census"]
    assert d["parity"]["grep_hits_equal_plants"]
    assert len(d["per_rank"]) == 2 and sum(r["bytes"] for r in d["per_rank"]) == d["config"]["bytes"]

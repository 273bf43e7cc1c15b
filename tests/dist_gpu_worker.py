"""One rank of the sharded GPU path (row a9 / SURVEY.md sec. 8e), launched by
tests/test_gpu_dist.py under torch.distributed.run: the rank's contiguous file range goes through
the real GPU path (GPU-issued preads + scan on cuda:0 -- the test box has one GPU, so the ranks
share it and use gloo), then the path's single all_reduce; every rank saves the reduced vector.

    python -m torch.distributed.run --nproc-per-node N tests/dist_gpu_worker.py OUT STAGING CHUNK PATH...
"""
import os
import sys

import numpy as np
import torch
import torch.distributed as dist

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import inputs  # noqa: E402
from paper_conf_isca_veselybblor18_b200 import dist as D  # noqa: E402
from paper_conf_isca_veselybblor18_b200 import gsys as G  # noqa: E402
from paper_conf_isca_veselybblor18_b200 import workloads as W  # noqa: E402


def main():
    out, staging, chunk, paths = sys.argv[1], sys.argv[2], int(sys.argv[3]), sys.argv[4:]
    rank, world = int(os.environ["RANK"]), int(os.environ["WORLD_SIZE"])
    torch.cuda.set_device(0)
    dist.init_process_group("gloo")
    lo, hi = D.shard_range(len(paths), rank, world)
    st = G.STAGE_DEVICE if staging == "device" else G.STAGE_HOST
    res = W.wordcount_files(paths[lo:hi], inputs.dictionary(), inputs.patterns(), chunk=chunk, staging=st,
                            gflags=G.WG | G.BLOCKING | G.RELAXED) if hi > lo else None
    hist = res.hist if res is not None else torch.zeros(64, dtype=torch.int64)
    hits = res.file_hits if res is not None else None
    v = D.pack_result(hist.cpu(), hits.cpu() if hits is not None else None, lo, hi, len(paths))
    D.reduce_result(v)
    np.save(os.path.join(out, f"r{rank}.npy"), v.numpy())
    if res is not None:
        assert res.wait_rc == 0
    dist.destroy_process_group()


if __name__ == "__main__":
    main()

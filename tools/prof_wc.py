"""Single wordcount launch for ncu (application replay): the first N (default 64) of the bench's
512 x 16 MiB files; argv[1] = device (default pull completion) | host staging."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import inputs
from paper_conf_isca_veselybblor18_b200 import gsys as G
from paper_conf_isca_veselybblor18_b200 import workloads as W
staging = G.STAGE_DEVICE if (len(sys.argv) > 1 and sys.argv[1] == "device") else G.STAGE_HOST
nf = int(sys.argv[2]) if len(sys.argv) > 2 else 64
c = inputs.make_corpus(512, 16 << 20)
paths = c.paths[:nf]
res = W.wordcount_files(paths, inputs.dictionary(), inputs.patterns(), chunk=256 << 10,
                        gflags=G.WG | G.BLOCKING | G.RELAXED, blocks=148, staging=staging)
print("ok", int(res.hist.sum()))

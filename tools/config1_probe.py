import sys, os, json
sys.path.insert(0, os.getcwd())
import bench, torch, inputs
from paper_conf_isca_veselybblor18_b200 import gsys as G
from paper_conf_isca_veselybblor18_b200 import workloads as W
W.ensure_init()
print(json.dumps(bench.config1_latency(G, W, torch.device("cuda", 0), inputs.dictionary(), inputs.patterns(), None)))

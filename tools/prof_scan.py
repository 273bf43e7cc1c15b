"""scan_kernel (or, with argv[1] == token, scan_tok_kernel) over 1 GiB HBM-resident corpus text
(for ncu kernel replay)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import inputs
from paper_conf_isca_veselybblor18_b200 import gsys as G
c = inputs.make_corpus(512, 16 << 20)
text = torch.cat([torch.from_file(p, dtype=torch.uint8, size=os.path.getsize(p)) for p in c.paths[:64]]).cuda()
hist = torch.zeros(64, dtype=torch.int64, device="cuda")
hit = torch.zeros(1, dtype=torch.int32, device="cuda")
tok = len(sys.argv) > 1 and sys.argv[1] == "token"
if tok:
    G.gsys_set_scan(G.SCAN_TOKEN)
for _ in range(3):   # the bench's launch: 1 block/SM x 1024 threads, grep on
    G.gsys_scan_device(text, text.numel(), 256 << 10, inputs.dictionary(), inputs.patterns(), hist, hit, 0,
                       1024)
torch.cuda.synchronize()
print("ok")

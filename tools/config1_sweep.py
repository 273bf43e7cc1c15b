"""Config 1 (16 MiB, 64 work-groups, WG + blocking + strong): device time vs chunk size and
staging / completion path.  One JSON line per cell."""
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import inputs  # noqa: E402
from paper_conf_isca_veselybblor18_b200 import gsys as G  # noqa: E402
from paper_conf_isca_veselybblor18_b200 import workloads as W  # noqa: E402


def main():
    W.ensure_init()
    words, pats = inputs.dictionary(), inputs.patterns()
    p = "/dev/shm/gsys_config1_16MiB.txt"
    census, _ = inputs.write_file(p, inputs.SEED_FILE16M, 0, 16 << 20)
    fd = os.open(p, os.O_RDONLY)
    s = torch.cuda.Stream()
    h = torch.zeros(64, dtype=torch.int64, device="cuda")
    chunks = [int(x) << 10 for x in os.environ.get("C1_CHUNKS", "256,128,64,32,16").split(",")]
    for st_name, st in (("host", G.STAGE_HOST), ("device_pull", G.STAGE_DEVICE)):
        for chunk in chunks:
            ts = []
            ok = True
            for rep in range(25):
                h.zero_()
                torch.cuda.synchronize()
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(s)
                G.gsys_wordcount([fd], [16 << 20], chunk, words, pats, h, None, None, G.WG | G.BLOCKING | G.STRONG,
                                 64, 256, s, st)
                e1.record(s)
                G.gsys_wait(s)
                e1.synchronize()
                if rep >= 5:
                    ts.append(e0.elapsed_time(e1))
                ok = ok and bool((h.cpu().numpy().astype("uint64") == census).all())
            ts.sort()
            print(json.dumps({"staging": st_name, "chunk": chunk, "blocks": 64, "ms_median": ts[len(ts) // 2],
                              "ms_min": ts[0], "GBps": (16 << 20) / ts[len(ts) // 2] / 1e6, "parity": ok}),
                  flush=True)
    os.close(fd)


if __name__ == "__main__":
    main()

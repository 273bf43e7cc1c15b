"""Condense `ncu --csv --page raw` outputs into profiles/<name>.json: {label: {metric: value}} for
the kernel rows (metrics with '__' in their name, device attributes dropped).
Usage: python tools/ncu_raw_to_json.py OUT.json LABEL=raw.csv [LABEL=raw.csv ...]"""
import csv
import json
import sys


def rows(path):
    lines = [ln for ln in open(path) if ln.startswith('"')]
    r = list(csv.reader(lines))
    return [dict(zip(r[0], x)) for x in r[1:]]


out = {}
for arg in sys.argv[2:]:
    label, path = arg.split("=", 1)
    for d in rows(path):
        if "wc_kernel" in d.get("Kernel Name", "") or "scan" in d.get("Kernel Name", ""):
            out[label] = {"kernel": d.get("Kernel Name"), "source": path.split("/")[-1],
                          **{k: v for k, v in d.items() if "__" in k and not k.startswith(("device__", "nvlink__",
                                                                                             "c2clink__", "numa__"))}}
json.dump(out, open(sys.argv[1], "w"), indent=1, sort_keys=True)
print(sys.argv[1], list(out))

"""Summarise an ncu report: key raw metrics + instruction-count hot blocks from the SASS page.
Usage: python tools/ncu_summary.py report.ncu-rep [nblocks]"""
import csv, io, subprocess, sys

rep = sys.argv[1]
nb = int(sys.argv[2]) if len(sys.argv) > 2 else 12
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
r = list(csv.reader(io.StringIO(raw)))
h, v = r[0], r[2]
want = ["Kernel Name", "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum", "smsp__inst_executed.sum",
        "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
        "l1tex__throughput.avg.pct_of_peak_sustained_active", "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum",
        "l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum", "l1tex__data_pipe_lsu_wavefronts_mem_shared_op_atom.sum",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum", "smsp__thread_inst_executed_per_inst_executed.ratio",
        "sm__warps_active.avg.per_cycle_active", "launch__registers_per_thread", "launch__occupancy_limit_shared_mem",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed", "syslts__t_sectors_aperture_sysmem_lookup_miss.sum"]
out = {}
for w in want:
    if w in h:
        out[w] = v[h.index(w)]
for i, x in enumerate(h):
    if x.startswith("smsp__pcsamp_warps_issue_stalled_") and not x.endswith("_not_issued") and v[i] not in ("", "0"):
        out[x] = v[i]
for k, x in out.items():
    print(f"{k:75s} {x}")
src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"], capture_output=True,
                     text=True).stdout
rows = list(csv.reader(io.StringIO(src)))
hh = rows[1]
data = rows[2:]
ia, iss, isrc = hh.index("Instructions Executed"), hh.index("Warp Stall Sampling (All Samples)"), hh.index("Source")
tot = sum(float(r[ia] or 0) for r in data)
blocks, cur = [], None
for r in data:
    c = float(r[ia] or 0)
    op = r[isrc].split()[0] if r[isrc] else ""
    if cur and abs(c - cur["c"]) <= 0.02 * max(c, 1):
        cur["n"] += 1; cur["s"] += float(r[iss] or 0); cur["ops"].append(op)
    else:
        cur = {"c": c, "n": 1, "s": float(r[iss] or 0), "ops": [op]}; blocks.append(cur)
blocks.sort(key=lambda b: -b["c"] * b["n"])
print(f"instructions executed: {tot:.0f}")
for b in blocks[:nb]:
    print(f"{int(b['c']):>9d} x {b['n']:>4d} = {b['c'] * b['n'] / tot * 100:5.1f}%  stall-samples {int(b['s']):>6d}  "
          + " ".join(b["ops"][:10]))

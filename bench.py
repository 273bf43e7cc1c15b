#!/usr/bin/env python
"""bench.py -- headline benchmark of the GENESYS hot path on B200.

Metric (BASELINE.json): "GPU-issued syscalls/sec (WG granularity) and pread-wordcount GB/s at
1/2/4/8 B200".  One step = one pass of the whole hot path over the config-3 workload: every
work-group of the wordcount/grep kernel issues GPU-side preads of its 256 KiB chunks (rows
a1-a6), the host service drains/coalesces/executes them and DMAs the bytes (a7), the kernel scans
them (a8), the per-rank histogram + grep hits are all-reduced over NCCL (a9, N > 1 only) and the
service is drained (a10).  The workload is 512 synthetic 16 MiB text files (8 GiB) on tmpfs,
sharded by whole files across ranks (fixed total: strong scaling).  `value` = corpus GB/s
(device-timed, CUDA events on the launch stream, max over ranks); `e2e` = the same through the
public Python API (files in -> host histogram out, wall clock); the WG syscall rate is reported
in `secondary`.  `--impl reference` times the CPU oracle on a bounded sample.

    python bench.py [--gpus N --steps K --warmup W] [--impl reference]
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "GPU-issued syscalls/sec (WG granularity) and pread-wordcount GB/s at 1/2/4/8 B200"


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="gsys", choices=["gsys", "reference"])
    ap.add_argument("--files", type=int, default=512)
    ap.add_argument("--file-mib", type=int, default=16)
    ap.add_argument("--chunk-kib", type=int, default=256)
    ap.add_argument("--order", default="relaxed", choices=["strong", "relaxed"])
    ap.add_argument("--blocks", type=int, default=148, help="work-groups (1 per SM: 0.8 %% above 2 per SM, profiles/r01_blocks_ab.jsonl)")
    ap.add_argument("--threads", type=int, default=256)
    ap.add_argument("--staging", default="device", choices=["device", "host", "mixed"],
                    help="device: preads land in HBM lines (default completion: the work-group pulls them "
                         "from the service's host-mapped bounce, reading B13); host: zero-copy host lines")
    ap.add_argument("--dev16", type=int, default=4, help="mixed staging: chunks per 16 on the device (DMA) path")
    ap.add_argument("--cmax", type=int, default=8, help="coalescing max bundle (P22.13)")
    ap.add_argument("--window", type=int, default=0, help="coalescing window us (P22.13)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cell-ms", type=float, default=100.0, help="syscalls mode: target ms of calls per cell")
    ap.add_argument("--no-extras", action="store_true", help="skip scan roofline / syscall-rate extras")
    ap.add_argument("--root", default=None, help="corpus directory (default /dev/shm/gsys_corpus)")
    ap.add_argument("--mode", default="wordcount", choices=["wordcount", "syscalls", "memcached", "mm", "fig8", "fig9"],
                    help="syscalls: config-2 sweep; memcached: config 4; mm: config 5 (one JSON line each)")
    return ap.parse_args()


class Clocks:
    """nvidia-smi sampling during the timed region (B200_PROFILING.md clocks line)."""

    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.proc = None
        self.lines = []

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", f"--id={self.index}", f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except OSError:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except subprocess.TimeoutExpired:
            self.proc.kill()
        sm, smax, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            f = [x.strip() for x in ln.split(",")]
            if len(f) < 9:
                continue
            try:
                sm.append(float(f[1]))
                smax.append(float(f[2]))
            except ValueError:
                continue
            for n, v in zip(names, f[5:9]):
                if v.lower() in ("active", "0x1", "yes"):
                    reasons.add(n)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(smax) if smax else None,
                "reasons": sorted(reasons), "samples": len(sm)}


def dist_env():
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return rank, world, local


def host_cores() -> int:
    return len(os.sched_getaffinity(0))


def cpu_model() -> str:
    try:
        for ln in open("/proc/cpuinfo"):
            if ln.startswith("model name"):
                return ln.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


def workload_config(a, nbytes, world):
    return {
        "workload": f"config3: pread-driven grep + wordcount, {a.files} x {a.file_mib} MiB synthetic text files "
                    f"({nbytes / 2**30:.2f} GiB) on tmpfs, WG granularity, blocking + {a.order}, "
                    f"{a.chunk_kib} KiB chunks, {a.staging} staging, files sharded across {world} GPU(s), "
                    f"NCCL histogram all-reduce",
        "files": a.files, "bytes": nbytes, "chunk": a.chunk_kib << 10, "blocks": a.blocks or "2/SM",
        "staging": a.staging, "coalesce_max": a.cmax, "coalesce_window_us": a.window,
        "threads_per_wg": a.threads, "dictionary_words": 64, "grep_patterns": 8,
        "l2": "inputs larger than L2 (8 GiB corpus streamed from the host every step)",
        "input_residency": ("host page cache (tmpfs); inside the timed region the GPU-issued preads bring it "
                            "into HBM staging lines (device staging) or the scan reads it from pinned host "
                            "lines over PCIe (host staging)"),
        "parallelism": f"files/{world}",
    }


def run_reference(a):
    """--impl reference: the CPU oracle (plain C, all host cores) on a bounded sample per step."""
    rank, world, local = dist_env()
    if rank != 0:
        return 0
    import inputs
    import oracle
    corpus = inputs.make_corpus(a.files, a.file_mib << 20, root=a.root)
    words, pats = inputs.dictionary(), inputs.patterns()
    # each step a bounded sample of the workload: the next 32 files of the corpus (rotating, so K
    # steps cover K x 32 different files; ~0.7 s per step on 16 host threads)
    per = max(1, min(len(corpus.paths), 32))
    nthr = host_cores()
    for _ in range(a.warmup):
        oracle.corpus(corpus.paths[:2], words, pats, chunk=a.chunk_kib << 10, nthreads=nthr)
    times, done = [], 0
    for i in range(a.steps):
        sample = [corpus.paths[(i * per + j) % len(corpus.paths)] for j in range(per)]
        _, _, secs, _ = oracle.corpus(sample, words, pats, chunk=a.chunk_kib << 10, nthreads=nthr)
        times.append(secs)
        done += sum(os.path.getsize(p) for p in sample)
    t = sum(times)
    sbytes = done / a.steps
    value = done / t / 1e9
    out = {"impl": "reference", "metric": METRIC, "value": value, "unit": "GB/s", "n_gpus": world,
           "steps": a.steps, "warmup": a.warmup, "ms_per_step": t / a.steps * 1e3, "higher_is_better": True,
           "scaling": "strong", "vs_baseline": None, "dtype": "u8", "data": "synthetic",
           "config": {**workload_config(a, corpus.total_bytes, world),
                      "reference_sample": f"each step times the oracle on {per} of the {a.files} files "
                                          f"(bounded sample); value = sampled bytes / oracle time"},
           "cpu_baseline": {"value": value, "unit": "GB/s", "cores": nthr, "kind": "oracle",
                            "sample": f"{per} of the {a.files} files ({sbytes / 2**20:.0f} MiB) per step, the next "
                                      f"{per} each step (rotating): pread + scalar wordcount + grep, {nthr} "
                                      f"pthreads, {cpu_model()}"},
           "e2e": {"value": value, "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(out), flush=True)
    return 0


def spawn_ranks(a) -> int | None:
    """`--gpus N` without a torchrun environment: re-launch this command as N ranks (one process per
    GPU) under torch.distributed.run on 127.0.0.1, and return its exit code; None when already
    inside a launch (or N == 1)."""
    if a.gpus <= 1 or "WORLD_SIZE" in os.environ:
        return None
    import socket
    sk = socket.socket()
    sk.bind(("127.0.0.1", 0))
    port = sk.getsockname()[1]
    sk.close()
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={a.gpus}",
           "--master-addr=127.0.0.1", f"--master-port={port}", os.path.abspath(__file__), *sys.argv[1:]]
    return subprocess.call(cmd)


def check_world(a, world):
    """The launch must match --gpus, one GPU per rank (GSYS_BENCH_ONE_GPU=1, test only: every
    rank on cuda:0)."""
    import torch
    if a.gpus != world:
        raise SystemExit(f"bench.py: --gpus {a.gpus} but the launch has {world} rank(s)")
    if os.environ.get("GSYS_BENCH_ONE_GPU") != "1" and torch.cuda.device_count() < world:
        raise SystemExit(f"bench.py: {world} ranks but only {torch.cuda.device_count()} visible GPU(s)")


def main():
    a = parse()
    rc = spawn_ranks(a)
    if rc is not None:
        return rc
    if a.impl == "reference":
        return run_reference(a)
    if a.mode == "syscalls":
        return run_syscalls(a)
    if a.mode == "memcached":
        return run_memcached(a)
    if a.mode == "mm":
        return run_mm(a)
    if a.mode == "fig8":
        return run_fig8(a)
    if a.mode == "fig9":
        return run_fig9(a)
    import torch
    import torch.distributed as dist

    import inputs
    from paper_conf_isca_veselybblor18_b200 import gsys as G
    from paper_conf_isca_veselybblor18_b200 import workloads as W

    rank, world, local = dist_env()
    check_world(a, world)
    # GSYS_BENCH_ONE_GPU=1 (test only): every rank on cuda:0 with gloo, to exercise the N > 1 path
    # on a one-GPU box (NCCL refuses two ranks on one device)
    one_gpu = os.environ.get("GSYS_BENCH_ONE_GPU") == "1"
    dev_idx = 0 if one_gpu else local
    torch.cuda.set_device(dev_idx)
    dev = torch.device("cuda", dev_idx)
    if world > 1:
        if one_gpu:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=dev)

    def barrier():
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()

    def max_over_ranks(x: float) -> float:
        if world == 1:
            return x
        t = torch.tensor([x], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    # corpus: local rank 0 writes it once per node; everyone shards by whole files
    if local == 0:
        corpus = inputs.make_corpus(a.files, a.file_mib << 20, root=a.root)
    barrier()
    corpus = inputs.make_corpus(a.files, a.file_mib << 20, root=a.root)
    words, pats = inputs.dictionary(), inputs.patterns()
    from paper_conf_isca_veselybblor18_b200 import dist as D
    lo, hi = D.shard_range(a.files, rank, world)
    mine = corpus.paths[lo:hi]
    chunk = a.chunk_kib << 10
    gflags = G.WG | G.BLOCKING | (G.RELAXED if a.order == "relaxed" else G.STRONG)

    W.ensure_init()
    G.gsys_set_coalesce_max(a.cmax)
    G.gsys_set_coalesce_window(a.window)
    staging = {"host": G.STAGE_HOST, "device": G.STAGE_DEVICE}.get(a.staging) or G.STAGE_MIXED(a.dev16)
    stream = torch.cuda.Stream(device=dev)
    of = W.OpenFiles(mine).__enter__()
    my_bytes = sum(of.sizes)
    nf = len(mine)
    d_hist = torch.zeros(64, dtype=torch.int64, device=dev)
    d_hits = torch.zeros(max(nf, 1), dtype=torch.int32, device=dev)
    d_all = [None]

    def step():
        d_hist.zero_()
        d_hits.zero_()
        G.gsys_wordcount(of.fds, of.sizes, chunk, words, pats, d_hist, d_hits, None, gflags, a.blocks, a.threads,
                         stream, staging)
        G.gsys_wait(stream)
        if world > 1:   # row a9: the path's only collective
            d_all[0] = D.reduce_result(D.pack_result(d_hist, d_hits[:nf], lo, hi, a.files))

    with torch.cuda.stream(stream):
        for _ in range(a.warmup):
            step()
        barrier()
        clk = Clocks(dev_idx)
        clk.start()
        ev0 = torch.cuda.Event(enable_timing=True)
        ev1 = torch.cuda.Event(enable_timing=True)
        G.gsys_stats_reset()
        req0 = G.gsys_stats()["requests"]   # the drained-request counter is cumulative
        barrier()
        ev0.record(stream)
        for _ in range(a.steps):
            step()
        ev1.record(stream)
        ev1.synchronize()
        barrier()
        clocks = clk.stop()
        st = G.gsys_stats()
        st["requests"] -= req0
    my_s = ev0.elapsed_time(ev1) / 1e3
    dev_s = max_over_ranks(my_s)
    value = corpus.total_bytes * a.steps / dev_s / 1e9
    # per-rank rate (own bytes / own device time) and, measured by every rank at once after the
    # timed region, the concurrent pinned H2D rate of each rank's link: the host-side ceiling of a
    # scaling curve (all ranks share the host's page cache, DRAM and cores)
    per_rank_local = [float(rank), my_bytes * a.steps / my_s / 1e9, float(my_bytes)]
    if world > 1:
        barrier()
        conc_h2d = measure_h2d(dev)
        t = torch.tensor(per_rank_local + [conc_h2d], dtype=torch.float64, device=dev)
        gathered = [torch.zeros_like(t) for _ in range(world)]
        dist.all_gather(gathered, t)
        per_rank = [{"rank": int(g[0]), "GBps": float(g[1]), "bytes": int(g[2]),
                     "concurrent_h2d_GBps": float(g[3])} for g in (x.cpu() for x in gathered)]
    else:
        per_rank = [{"rank": 0, "GBps": per_rank_local[1], "bytes": my_bytes}]
    # parity of the last step against the generator census (cheap, exact)
    if world > 1:
        red = d_all[0].cpu().numpy()
        hist_ok = bool((red[:64].astype("uint64") == corpus.census).all())
        hits_ok = red[64:].tolist() == [1 if m else 0 for m in corpus.pmasks]
    else:
        hist_ok = bool((d_hist.cpu().numpy().astype("uint64") == corpus.census).all())
        hits_ok = d_hits[:nf].cpu().tolist() == [1 if m else 0 for m in corpus.pmasks]

    # ---- e2e through the public API (files in -> host histogram out), wall clock
    barrier()
    e2e_t = []
    for _ in range(max(1, min(a.steps, 3))):
        barrier()
        t0 = time.perf_counter()
        res = W.wordcount_files(mine, words, pats, chunk=chunk, gflags=gflags, blocks=a.blocks, threads=a.threads,
                                stream=stream, staging=staging)
        if world > 1:
            D.reduce_result(D.pack_result(res.hist.to(dev), res.file_hits.to(dev), lo, hi, a.files)).cpu()
        e2e_t.append(max_over_ranks(time.perf_counter() - t0))
    e2e_s = statistics.median(e2e_t)
    e2e_value = corpus.total_bytes / e2e_s / 1e9

    # ---- roofline of the dominant kernel (wc_kernel): host-link bound
    extras = {}
    h2d_peak = None
    if not a.no_extras and rank == 0:   # after the timed region; rank 0 alone (shared host files)
        h2d_peak = measure_h2d(dev)
        extras["scan"] = scan_roofline(G, dev, corpus, words, pats, chunk)
        extras["syscalls"] = wg_syscall_rate(G, W, dev, corpus.paths[0])
        extras["config1"] = config1_latency(G, W, dev, words, pats, a.root)
        for v in extras["config1"].values():
            v["frac_of_h2d"] = v["GBps_median"] / h2d_peak if h2d_peak else None
        extras["fig10"] = fig10_coalescing(G, W, dev, corpus.paths[0])
    kernel_s = dev_s / a.steps
    algo_bytes = my_bytes + sum(((s + chunk - 1) // chunk) * 17 for s in of.sizes)   # chunk + halo
    rank_achieved = algo_bytes / kernel_s / 1e9
    traffic, traffic_src = None, None
    summ = os.path.join(ROOT, "profiles", "r02_ncu_summary.json")
    label = {"device": "wc_kernel_64x16MiB_device_pull", "host": "wc_kernel_64x16MiB_host_staging"}.get(a.staging)
    if label and os.path.exists(summ):   # ncu capture of wc_kernel over 64 of the files (1 GiB), scaled per launch
        wk = json.load(open(summ)).get(label, {})
        try:
            cap_bytes = 64 * (16 << 20)
            dram = float(wk["dram__bytes_read.sum"]) + float(wk["dram__bytes_write.sum"])
            traffic = dram * algo_bytes / cap_bytes
            traffic_src = f"profiles/r02_ncu_summary.json[{label}]"
        except (KeyError, ValueError):
            pass
    # the host-side co-bound: ~3 bytes of host DRAM traffic per corpus byte (pread reads the page
    # cache and writes the bounce, the GPU reads the bounce over PCIe) against the box's measured
    # memcpy bandwidth (tools/probes/host_membw.c, profiles/r02_host_membw.jsonl)
    host_mem = None
    hm = os.path.join(ROOT, "profiles", "r02_host_membw.jsonl")
    if os.path.exists(hm):
        try:
            peak_h = max(json.loads(ln)["GBps_read_plus_write"] for ln in open(hm) if ln.strip())
            host_mem = {"bound": "host DRAM (3 B per corpus byte)", "achieved": 3 * rank_achieved, "peak": peak_h,
                        "unit": "GB/s", "frac": 3 * rank_achieved / peak_h,
                        "peak_source": "profiles/r02_host_membw.jsonl (16-thread memcpy, read + write)"}
        except (ValueError, KeyError):
            pass
    roofline = {"bound": "host-link", "achieved": rank_achieved, "peak": h2d_peak, "unit": "GB/s",
                "frac": (rank_achieved / h2d_peak) if h2d_peak else None, "traffic": traffic,
                "traffic_note": f"dram__bytes_read.sum + dram__bytes_write.sum of {traffic_src} (ncu application "
                                "replay, 1 GiB) scaled to this launch: the staging lines stay in L2, so HBM "
                                "traffic is ~0; the algorithmic bytes cross the host link once",
                "kernel": "wc_kernel (GPU-issued WG preads + scan), one launch per step per rank",
                "peak_source": "measured live: pinned cudaMemcpyAsync H2D, 256 MiB x 8, this box's PCIe link "
                               "(MEASURED_PEAKS.json has no host-link figure)"}
    of.__exit__()

    cpu_baseline = None
    if rank == 0 and world == 1 and not a.no_cpu_baseline:
        cpu_baseline = cpu_baseline_leg(a, corpus, words, pats, chunk)
    if world > 1:
        dist.barrier()
    if rank == 0:
        syscalls_per_step = st["requests"] / a.steps
        if cpu_baseline and "syscalls" in extras:   # WG syscall rates against the oracle's direct rates
            for k, cell in extras["syscalls"].items():
                base = cpu_baseline["pread4k_direct_calls_per_s" if k.startswith("pread") else
                                    "getrusage_direct_calls_per_s"]
                cell["frac_of_oracle_direct"] = cell["calls_per_s"] / base if base else None
        out = {"metric": METRIC, "value": value, "unit": "GB/s", "n_gpus": world, "steps": a.steps,
               "warmup": a.warmup, "ms_per_step": dev_s / a.steps * 1e3, "higher_is_better": True,
               "scaling": "strong", "vs_baseline": None, "dtype": "u8", "data": "synthetic",
               "config": workload_config(a, corpus.total_bytes, world),
               "e2e": {"value": e2e_value, "unit": "GB/s", "h2d_bytes_per_step": my_bytes * world,
                       "d2h_bytes_per_step": (64 + a.files) * 8, "api": "workloads.wordcount_files"},
               "gpu_launches": a.steps,
               "roofline": roofline,
               "cpu_baseline": cpu_baseline,
               "clocks": clocks,
               "parity": {"hist_equals_generator_census": hist_ok, **({"grep_hits_equal_plants": hits_ok}
                                                                     if hits_ok is not None else {})},
               "per_rank": per_rank,
               "secondary": {"wg_syscalls_per_s_in_wordcount": syscalls_per_step * world / (dev_s / a.steps),
                             **({"syscalls_wg": extras["syscalls"]} if "syscalls" in extras else {}),
                             **({"config1_16MiB": extras["config1"]} if "config1" in extras else {}),
                             **({"scan_hbm": extras["scan"]} if "scan" in extras else {}),
                             **({"fig10_coalescing": extras["fig10"]} if "fig10" in extras else {}),
                             **({"host_memory_roofline": host_mem} if host_mem else {})},
               "service_path": service_path(a, st),
               "service": {"threads": st["threads"], "coalesce_max": st["coalesce_max"],
                           "window_us": st["coalesce_window_us"], "bundles_per_step": st["bundles"] / a.steps,
                           "merged_per_step": st["merged"] / a.steps,
                           "host_preads_per_step": st["host_preads"] / a.steps},
               "host": {"cores": host_cores(), "cpu": cpu_model()}}
        print(json.dumps(out), flush=True)
    if world > 1:
        dist.destroy_process_group()
    return 0


def service_path(a, st):
    """Which service path the timed steps took (from the service counters)."""
    if a.staging == "device":
        how = ("device staging, pull completion (reading B13): a service worker preads each work-group's "
               "chunk into its host-mapped bounce and completes with a host store; the work-group copies "
               "the bytes into its HBM line and scans them there; the service makes no CUDA call")
    elif a.staging == "host":
        how = ("host staging: a service worker preads each chunk straight into the work-group's pinned "
               "host-mapped line and completes with a host store; the scan reads the line over PCIe")
    else:
        how = "mixed staging: some chunks by copy-engine DMA into HBM lines, the rest zero-copy host lines"
    return {"description": how, "requests_per_step": st["requests"] / a.steps,
            "bundles_per_step": st["bundles"] / a.steps, "merged_requests_per_step": st["merged"] / a.steps,
            "merge_note": "adjacent work-group halo reads are not merged on this path: each lands in its own "
                          "bounce range that its work-group releases (merging is exercised by the coalescing "
                          "invariance tests and by fig10_coalescing)"}


def fig10_coalescing(G, W, dev, path):
    """Fig. 10 analogue (PAPER.md:28 P28.12-19) in the driver's run: WG blocking preads of 64 B and
    1 KiB into device memory, 592 work-groups x 40 calls, coalescing max 1 vs 8."""
    import torch
    size = os.path.getsize(path)
    fd = os.open(path, os.O_RDONLY)
    dbuf = torch.empty(592 * 1024, dtype=torch.uint8, device=dev)
    rows = []
    try:
        for length in (64, 1024):
            for cmax in (1, 8):
                G.gsys_set_coalesce_max(cmax)
                W.bench_calls("pread", G.WG | G.BLOCKING | G.RELAXED, 592, 256, 2, fd, length, size, dbuf)
                G.gsys_stats_reset()
                t0 = time.perf_counter()
                _, ret, _, _, rc = W.bench_calls("pread", G.WG | G.BLOCKING | G.RELAXED, 592, 256, 40, fd, length,
                                                 size, dbuf)
                dt = time.perf_counter() - t0
                st = G.gsys_stats()
                rows.append({"bytes_per_call": length, "coalesce_max": cmax, "calls_per_s": 592 * 40 / dt,
                             "ns_per_byte": dt * 1e9 / (592 * 40 * length), "bundles": st["bundles"],
                             "max_bundle": st["max_bundle"], "merged": st["merged"],
                             "ok": bool((ret == length).all()) and rc == 0})
    finally:
        G.gsys_set_coalesce_max(8)
        os.close(fd)
    return rows


def measure_h2d(dev):
    import torch
    n = 256 << 20
    h = torch.empty(n, dtype=torch.uint8).pin_memory()
    d = torch.empty(n, dtype=torch.uint8, device=dev)
    s = torch.cuda.Stream(device=dev)
    with torch.cuda.stream(s):
        for _ in range(2):
            d.copy_(h, non_blocking=True)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        for _ in range(8):
            d.copy_(h, non_blocking=True)
        e1.record(s)
        e1.synchronize()
    return n * 8 / (e0.elapsed_time(e1) / 1e3) / 1e9


def scan_roofline(G, dev, corpus, words, pats, chunk):
    """Standalone scan (row a8) over 1 GiB of corpus text resident in HBM: GB/s vs measured HBM."""
    import torch
    nb = min(len(corpus.paths), 64)
    parts = [torch.from_file(p, dtype=torch.uint8, size=os.path.getsize(p)) for p in corpus.paths[:nb]]
    text = torch.cat(parts).to(dev)
    n = text.numel()
    hist = torch.zeros(64, dtype=torch.int64, device=dev)
    hit = torch.zeros(1, dtype=torch.int32, device=dev)
    s = torch.cuda.Stream(device=dev)
    with torch.cuda.stream(s):
        for _ in range(3):
            G.gsys_scan_device(text, n, chunk, words, pats, hist, hit, 0, 1024, s)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        reps = 10
        e0.record(s)
        for _ in range(reps):
            G.gsys_scan_device(text, n, chunk, words, pats, hist, hit, 0, 1024, s)
        e1.record(s)
        e1.synchronize()
    t = e0.elapsed_time(e1) / 1e3 / reps
    # the selectable warp-cooperative token scan on the same text (GSYS_SCAN_TOKEN, 32 warps/SM)
    tok = None
    prev = G.gsys_set_scan(G.SCAN_TOKEN)
    try:
        with torch.cuda.stream(s):
            for _ in range(3):
                G.gsys_scan_device(text, n, chunk, words, pats, hist, hit, 0, 1024, s)
            t0, t1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            t0.record(s)
            for _ in range(reps):
                G.gsys_scan_device(text, n, chunk, words, pats, hist, hit, 0, 1024, s)
            t1.record(s)
            t1.synchronize()
        tok = {"kernel": "scan_tok_kernel (warp-cooperative token scan, 1 block/SM x 1024 threads)",
               "achieved": n / (t0.elapsed_time(t1) / 1e3 / reps) / 1e9, "unit": "GB/s"}
    finally:
        G.gsys_set_scan(prev)
    peak = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"] if os.path.exists(
        os.path.join(ROOT, "MEASURED_PEAKS.json")) else 6650.0
    ach = n / t / 1e9
    del text
    traffic, limiter = None, None
    summ = os.path.join(ROOT, "profiles", "r02_scan_dfa32_ncu.json")
    if os.path.exists(summ):   # ncu --set full of the same 1 GiB scan in this launch configuration (base units)
        try:
            kv = json.load(open(summ))
            traffic = (kv["dram__bytes_read.sum"]["value"] + kv["dram__bytes_write.sum"]["value"]) * n / kv["text_bytes"]
            limiter = (f"shared-memory pipe: l1tex {kv['l1tex__throughput.avg.pct_of_peak_sustained_active']['value']:.0f}% "
                       f"of peak (DFA gathers, 3.3 wavefronts per warp lookup; tiles staged by swizzled tensor copies), issue "
                       f"{kv['smsp__issue_active.avg.pct_of_peak_sustained_active']['value']:.0f}%")
        except (KeyError, ValueError, TypeError):
            pass
    # compute-side roofline: one random 16-bit shared-memory gather per byte (the DFA
    # lookup), against the measured random-gather rate of tools/probes/b200_probes.cu
    compute = None
    probes = os.path.join(ROOT, "profiles", "r02_probes.jsonl")
    if os.path.exists(probes):
        for ln in open(probes):
            try:
                r = json.loads(ln)
            except ValueError:
                continue
            if r.get("probe") == "smem" and "random gather" in r.get("op", ""):
                compute = {"bound": "smem random gather (1 DFA lookup per byte)", "achieved": n / t,
                           "peak": r["lookups_per_s"], "unit": "lookups/s", "frac": n / t / r["lookups_per_s"],
                           "peak_source": "profiles/r02_probes.jsonl (tools/probes/b200_probes.cu)"}
    return {"bound": "hbm", "achieved": ach, "peak": peak, "unit": "GB/s", "frac": ach / peak, "bytes": n,
            "traffic": traffic, "limiter": limiter, "ms": t * 1e3, "compute_roofline": compute,
            "token_scan": dict(tok, frac=tok["achieved"] / peak) if tok else None,
            "kernel": "scan_kernel (HBM-resident text, 1 block/SM x 1024 threads (32 warps), each 2 KiB warp tile one swizzled tensor copy, 129-column transposed DFA in shared memory; profiles/r02_swz.jsonl)",
            "peak_source": "MEASURED_PEAKS.json hbm_gbs (copy)", "note": "input 1 GiB > L2; read-once"}


def config1_latency(G, W, dev, words, pats, root):
    """Config 1 (BASELINE.json configs[0]): one 16 MiB file, 64 work-groups, WG + blocking + strong:
    device time per wordcount (the latency case: 64 preads in flight at once)."""
    import torch

    import inputs
    path = os.path.join(root or "/dev/shm", "gsys_config1_16MiB.txt")
    census, _ = inputs.write_file(path, inputs.SEED_FILE16M, 0, 16 << 20)
    fd = os.open(path, os.O_RDONLY)
    out = {}
    try:
        s = torch.cuda.Stream(device=dev)
        h = torch.zeros(64, dtype=torch.int64, device=dev)
        # 64 work-groups each take chunks from the file's queue: 64 KiB chunks (4 blocking preads
        # per work-group) keep the link busier than one 256 KiB read each (profiles/r02_config1_sweep.jsonl)
        for name, st, ck in (("host", G.STAGE_HOST, 64), ("host_256k", G.STAGE_HOST, 256),
                             ("device", G.STAGE_DEVICE, 64)):
            ts, ws = [], []
            for rep in range(23):
                h.zero_()
                torch.cuda.synchronize(dev)
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                t0 = time.perf_counter()
                e0.record(s)
                G.gsys_wordcount([fd], [16 << 20], ck << 10, words, pats, h, None, None,
                                 G.WG | G.BLOCKING | G.STRONG, 64, 256, s, st)
                e1.record(s)          # device time: table upload + the kernel (its 64 preads inside)
                G.gsys_wait(s)
                _ = h.cpu()           # wall time: the call until the histogram is on the host
                w = time.perf_counter() - t0
                e1.synchronize()
                if rep >= 3:
                    ts.append(e0.elapsed_time(e1))
                    ws.append(w * 1e3)
            ts.sort()
            ws.sort()
            out[name] = {"ms_median": ts[len(ts) // 2], "GBps_median": (16 << 20) / (ts[len(ts) // 2] / 1e3) / 1e9,
                         "ms_min": ts[0], "wall_ms_median": ws[len(ws) // 2], "chunk": ck << 10, "work_groups": 64,
                         "parity": bool((h.cpu().numpy().astype("uint64") == census).all())}
    finally:
        os.close(fd)
    return out


def wg_syscall_rate(G, W, dev, path):
    """The metric's other half, "GPU-issued syscalls/sec (WG granularity)": 592 work-groups
    (4/SM x 256 threads), each cell calibrated until one pass runs >= 150 ms of calls.  getrusage blocking
    and non-blocking; 4 KiB preads into device memory, blocking (the pull path, reading B12) and
    non-blocking (deferred pulls, reading B15)."""
    import torch
    blocks, threads = 592, 256
    size = os.path.getsize(path)
    fd = os.open(path, os.O_RDONLY)
    dbuf = torch.empty(blocks * 4096, dtype=torch.uint8, device=dev)
    out = {}
    try:
        for name, kind, flags in (("getrusage_blocking", "getrusage", G.WG | G.BLOCKING | G.RELAXED),
                                  ("getrusage_nonblocking", "getrusage", G.WG | G.NONBLOCKING | G.RELAXED),
                                  ("pread4k_device_blocking", "pread", G.WG | G.BLOCKING | G.RELAXED),
                                  ("pread4k_device_nonblocking", "pread", G.WG | G.NONBLOCKING | G.RELAXED)):
            kw = dict(fd=fd, length=4096, size=size, d_buf=dbuf) if kind == "pread" else {}
            iters = 20
            for _ in range(4):   # calibration passes until one pass lasts >= 150 ms (launch, ramp
                # and the final drain are then a few per cent of it)
                torch.cuda.synchronize()
                t0 = time.perf_counter()
                _, ret, lat, _, rc = W.bench_calls(kind, flags, blocks, threads, iters, **kw)
                dt = time.perf_counter() - t0
                rate = blocks * iters / dt
                if dt >= 0.15 or iters >= 4000:
                    break
                iters = int(min(max(20, rate * 0.25 / blocks), 4000))
            lat_us = (lat.double() / 1e3).cpu()
            blocking = not (flags & G.NONBLOCKING)
            ok = bool((ret == (4096 if kind == "pread" else 0)).all()) if blocking else bool((ret == 0).all())
            out[name] = {"calls_per_s": rate, "callers": blocks, "seconds": dt,
                         "lat_p50_us": float(lat_us.median()) if blocking else None,
                         "lat_p99_us": float(lat_us.quantile(0.99)) if blocking else None,
                         "all_ok": ok and rc == 0}
    finally:
        os.close(fd)
    return out


def cpu_baseline_leg(a, corpus, words, pats, chunk):
    import oracle
    nthr = host_cores()
    sample = corpus.paths[:384]   # ~6 GiB: about 10 s of the oracle on 16 threads
    sbytes = sum(os.path.getsize(p) for p in sample)
    oracle.corpus(sample[:1], words, pats, chunk=chunk, nthreads=nthr)
    _, _, secs, _ = oracle.corpus(sample, words, pats, chunk=chunk, nthreads=nthr)
    rate = oracle.syscall_rate("getrusage", nthr, 200000)
    fd = os.open(corpus.paths[0], os.O_RDONLY)
    try:
        prate = oracle.syscall_rate("pread", nthr, 100000, fd, 4096, os.path.getsize(corpus.paths[0]))
    finally:
        os.close(fd)
    _, _, secs1, _ = oracle.corpus(sample[:4], words, pats, chunk=chunk, nthreads=1)
    one_thread = sum(os.path.getsize(p) for p in sample[:4]) / secs1 / 1e9
    pread_ceiling = {str(t): oracle.pread_only(corpus.paths[:64], t, chunk) / 1e9 for t in (1, 4, 8, nthr)}
    return {"value": sbytes / secs / 1e9, "unit": "GB/s", "cores": nthr, "kind": "oracle",
            "host_pread_only_GBps_by_threads": pread_ceiling, "value_1_thread": one_thread,
            "sample": f"{len(sample)} of {a.files} files ({sbytes / 2**20:.0f} MiB): pread + scalar wordcount + grep, "
                      f"{nthr} pthreads, {cpu_model()}",
            "getrusage_direct_calls_per_s": rate, "pread4k_direct_calls_per_s": prate}


def run_syscalls(a):
    """Config 2 (BASELINE.json configs[1]): getrusage / pread microbenchmark over work-item,
    work-group and kernel granularity x blocking x ordering (sec. VII, Fig. 7/8/10),
    plus the unloaded ping-pong, a Fig-7 file-size sweep and a Fig-10 coalescing sweep.  Rates
    are calls / wall time of launch..gsys_wait; latency is GPU-observed (%globaltimer) per call."""
    import torch

    import oracle
    from paper_conf_isca_veselybblor18_b200 import gsys as G
    from paper_conf_isca_veselybblor18_b200 import workloads as W

    torch.cuda.set_device(0)
    W.ensure_init()
    gname = {G.WI: "wi", G.WG: "wg", G.KERNEL: "kernel"}
    cells = [(G.WI, G.BLOCKING, G.STRONG), (G.WI, G.NONBLOCKING, G.STRONG),
             (G.WG, G.BLOCKING, G.STRONG), (G.WG, G.BLOCKING, G.RELAXED),
             (G.WG, G.NONBLOCKING, G.STRONG), (G.WG, G.NONBLOCKING, G.RELAXED),
             (G.KERNEL, G.BLOCKING, G.RELAXED), (G.KERNEL, G.NONBLOCKING, G.RELAXED)]
    root = a.root or "/dev/shm"
    path = os.path.join(root, "gsys_mb_1GiB.bin")
    if not os.path.exists(path) or os.path.getsize(path) != (1 << 30):
        with open(path, "wb") as f:
            for _ in range(16):
                f.write(os.urandom(64 << 20))
    fd = os.open(path, os.O_RDONLY)
    size = 1 << 30
    blocks, threads = 592, 256
    out = {"mode": "syscalls", "metric": "GPU-issued syscalls/sec and GPU-observed round-trip latency",
           "grid": f"{blocks} blocks x {threads} threads", "cells": []}
    hbuf = torch.empty(blocks * threads * 4096, dtype=torch.uint8).pin_memory()
    dbuf = torch.empty(blocks * threads * 4096, dtype=torch.uint8, device="cuda")

    def run(kind, flags, bl, th, iters, length=0, sz=0, buf=None):
        W.bench_calls(kind, flags, bl, th, 1, fd, length, sz or 1, buf)
        G.gsys_stats_reset()
        r0 = G.gsys_stats()["requests"]
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        n, ret, lat, _, rc = W.bench_calls(kind, flags, bl, th, iters, fd, length, sz or 1, buf)
        dt = time.perf_counter() - t0
        st = G.gsys_stats()
        calls = st["requests"] - r0
        lat_us = lat.double().cpu() / 1e3
        blocking = not (flags & G.NONBLOCKING)
        return {"calls": calls, "seconds": dt, "calls_per_s": calls / dt, "callers": n,
                "lat_p50_us": float(lat_us.median()) if blocking else None,
                "lat_p99_us": float(lat_us.quantile(0.99)) if blocking else None,
                "issue_p50_us": None if blocking else float(lat_us.median()),
                "ok": bool((ret >= 0).all()) and rc == 0,
                "service_busy_frac": st["ns_busy"] / 1e9 / dt / st["threads"]}

    # steady state: each cell is first run with a short calibration count, then with enough
    # iterations per caller for >= a.cell_ms of calls (launch and drain are then negligible)
    link_peak = measure_h2d(0)
    nthr = host_cores()
    out["oracle_direct"] = {"cores": nthr, "getrusage_calls_per_s": oracle.syscall_rate("getrusage", nthr, 200000),
                            "pread4k_calls_per_s": oracle.syscall_rate("pread", nthr, 100000, fd, 4096, size),
                            "getrusage_1thread": oracle.syscall_rate("getrusage", 1, 200000)}
    odir = {"getrusage": out["oracle_direct"]["getrusage_calls_per_s"],
            "pread": out["oracle_direct"]["pread4k_calls_per_s"]}
    for kind, iters_by in (("getrusage", {G.WI: 2, G.WG: 20, G.KERNEL: 100}),
                           ("pread", {G.WI: 2, G.WG: 20, G.KERNEL: 100})):
        for gran, blk, order in cells:
            flags = gran | blk | order
            for bufkind in (("device", "host") if kind == "pread" else ("-",)):
                buf = None
                if kind == "pread":
                    buf = dbuf if bufkind == "device" else hbuf
                    if bufkind == "host":
                        flags |= G.HOSTBUF
                length = 4096 if kind == "pread" else 0
                r = run(kind, flags, blocks, threads, iters_by[gran], length, size, buf)
                callers = max(r["callers"], 1)
                iters = int(min(max(iters_by[gran], r["calls_per_s"] * a.cell_ms / 1e3 / callers), 4000))
                if iters > iters_by[gran]:
                    r = run(kind, flags, blocks, threads, iters, length, size, buf)
                # algorithmic host-link bytes per call: 64 B slot + 8 B doorbell + 8 B completion +
                # 8 B state + the payload that crosses the link (the 144 B rusage
                # read back from the inline buffer; 4 KiB DMA'd into a device buffer; a host-buffer
                # pread's bytes stay in host memory)
                pay = 144 if kind == "getrusage" else (4096 if bufkind == "device" else 0)
                r.update({"kind": kind, "granularity": gname[gran], "blocking": not (blk & G.NONBLOCKING),
                          "ordering": "relaxed" if order else "strong", "buffer": bufkind,
                          "bytes_per_call": 4096 if kind == "pread" else 144, "iters_per_caller": iters,
                          "link_bytes_per_call": 88 + pay,
                          "link_frac": (r["calls_per_s"] * (88 + pay) / (link_peak * 1e9)) if link_peak else None,
                          "frac_of_oracle_direct": r["calls_per_s"] / odir[kind] if odir.get(kind) else None})
                out["cells"].append(r)
    out["host_link_peak_GBps"] = link_peak
    # unloaded ping-pong (1 caller, sequential blocking calls): the intrinsic round trip
    out["pingpong_getrusage"] = run("getrusage", G.WG | G.BLOCKING, 1, 32, 2000)
    out["pingpong_pread4k_host"] = run("pread", G.WG | G.BLOCKING | G.HOSTBUF, 1, 32, 2000, 4096, size, hbuf)
    out["pingpong_pread4k_device"] = run("pread", G.WG | G.BLOCKING, 1, 32, 2000, 4096, size, dbuf)
    # Fig. 7 (left): fixed number of work-items, whole file read at each granularity
    fig7 = []
    for fsz in (16 << 20, 256 << 20, 1 << 30):
        for gran in (G.WI, G.WG, G.KERNEL):
            callers = blocks * threads if gran == G.WI else blocks if gran == G.WG else 1
            length = max(16, fsz // callers // 16 * 16)
            flags = gran | G.BLOCKING | (G.RELAXED if gran == G.KERNEL else G.STRONG) | G.HOSTBUF
            big = torch.empty(callers * length, dtype=torch.uint8).pin_memory()
            reps = [run("pread", flags, blocks, threads, 1, length, fsz, big) for _ in range(3)]
            r = sorted(reps, key=lambda x: x["seconds"])[1]     # median of 3 one-shot reads
            r.update({"file_bytes": fsz, "granularity": gname[gran], "bytes_per_call": length, "repeats": 3,
                      "GBps": callers * length / r["seconds"] / 1e9})
            fig7.append(r)
            del big
    out["fig7_granularity"] = fig7
    # Fig. 10: coalescing on/off for small preads (WG, blocking), device buffers
    fig10 = []
    for length in (64, 1024, 16384):
        for cmax, win in ((1, 0), (8, 0), (8, 20)):
            G.gsys_set_coalesce_max(cmax)
            G.gsys_set_coalesce_window(win)
            r = run("pread", G.WG | G.BLOCKING, blocks, threads, 20, length, size, dbuf)
            r.update({"bytes_per_call": length, "coalesce_max": cmax, "window_us": win,
                      "ns_per_byte": r["seconds"] * 1e9 / (r["calls"] * length)})
            fig10.append(r)
    G.gsys_set_coalesce_max(8)
    G.gsys_set_coalesce_window(0)
    out["fig10_coalescing"] = fig10
    out["service_threads"] = G.gsys_stats()["threads"]
    os.close(fd)
    print(json.dumps(out), flush=True)
    return 0


def run_memcached(a):
    """Config 4 (BASELINE.json configs[3]): memcached-style binary-UDP GET server.  GPU server =
    work-groups issuing recvfrom/sendto (WG, blocking, weak -- P32.29-30); CPU server = the
    oracle's threaded C server over the same store; same load generator, same request stream.
    Reported: requests/s and client-side latency for 16 and 1024 elements per bucket (the paper's
    large-bucket case, P32.33) with 1 KiB values."""
    import ctypes
    import threading

    import numpy as np
    import torch

    import oracle
    from inputs import mc as MC
    from oracle import mc as OM
    from paper_conf_isca_veselybblor18_b200 import gsys as G
    from paper_conf_isca_veselybblor18_b200 import workloads as W

    torch.cuda.set_device(0)
    nthr = host_cores()
    # the load generator (up to 8 client threads) runs on the same host: the service gets the
    # other cores, as the CPU server's 8 threads do -- busy-polling service threads on cores the
    # client needs would measure the oversubscription, not the server (tools/mc_threads_sweep.py)
    os.environ.setdefault("GSYS_THREADS", str(max(2, nthr - 8)))
    W.ensure_init()
    out = {"mode": "memcached", "metric": "GET requests/s (binary memcached over UDP loopback)", "cases": []}
    for per_bucket in (16, 1024):
        nbuckets = 64
        nkeys = nbuckets * per_bucket * 3 // 4
        keys, vals = MC.dataset(nkeys, vlen=1024)
        reqs = MC.requests(keys, 20000)
        pkts = [MC.encode_get(i, k) for i, k in enumerate(reqs)]
        table = dict(zip(keys, vals))
        for nwg, send in ((4, "blocking"), (12, "blocking"), (12, "nonblocking"), (32, "blocking"),
                          (32, "nonblocking"), (64, "nonblocking")):
            sg = G.WG | G.RELAXED | (G.NONBLOCKING if send == "nonblocking" else G.BLOCKING)
            resp, lat, secs, stats = W.mc_serve_run(keys, vals, pkts, nwg=nwg, nbuckets=nbuckets,
                                                    bucket_cap=per_bucket * 2, client_threads=4, window=8,
                                                    send_gflags=sg)
            ok = sum(1 for p, r in zip(pkts, resp) if r == OM.expected_response(p, table))
            lat_us = np.array(lat, dtype=np.float64) / 1e3
            out["cases"].append({"server": "gpu", "sendto": send, "elements_per_bucket": per_bucket, "work_groups": nwg,
                                 "req_per_s": len(pkts) / secs, "lat_p50_us": float(np.median(lat_us)),
                                 "lat_p99_us": float(np.quantile(lat_us, 0.99)), "exact_replies": ok,
                                 "requests": len(pkts)})
        kb, ko, kl, vb, vo, vl = MC.pack(keys, vals)
        for st in (1, 4):
            sock = MC.udp_server_socket()
            stop = ctypes.c_int(0)
            th = threading.Thread(target=lambda: oracle.lib().oracle_mc_serve(
                sock.fileno(), st, kb.ctypes.data, ko.ctypes.data, kl.ctypes.data, vb.ctypes.data, vo.ctypes.data,
                vl.ctypes.data, len(keys), nbuckets, ctypes.addressof(stop)))
            th.start()
            try:
                resp, lat, secs = MC.run_client(sock.getsockname()[1], pkts, nthreads=4, window=8)
            finally:
                stop.value = 1
                th.join()
                sock.close()
            lat_us = np.array(lat, dtype=np.float64) / 1e3
            ok = sum(1 for p, r in zip(pkts, resp) if r == OM.expected_response(p, table))
            out["cases"].append({"server": "cpu-oracle", "threads": st, "elements_per_bucket": per_bucket,
                                 "req_per_s": len(pkts) / secs, "lat_p50_us": float(np.median(lat_us)),
                                 "lat_p99_us": float(np.quantile(lat_us, 0.99)), "exact_replies": ok,
                                 "requests": len(pkts)})
    # the config's value-size mix (64 B - 4 KiB, uniform), 16 elements per bucket, 32 work-groups vs
    # the CPU server with 4 threads
    keys, vals = MC.dataset(64 * 16 * 3 // 4, vlen=(64, 4096))
    table = dict(zip(keys, vals))
    pkts = [MC.encode_get(i, k) for i, k in enumerate(MC.requests(keys, 20000))]
    resp, lat, secs, _ = W.mc_serve_run(keys, vals, pkts, nwg=32, nbuckets=64, bucket_cap=32, client_threads=4,
                                        window=8, send_gflags=G.WG | G.RELAXED | G.BLOCKING)
    ok = sum(1 for p, r in zip(pkts, resp) if r == OM.expected_response(p, table))
    lat_us = np.array(lat, dtype=np.float64) / 1e3
    out["cases"].append({"server": "gpu", "sendto": "blocking", "elements_per_bucket": 16, "work_groups": 32,
                         "value_bytes": "64-4096", "req_per_s": len(pkts) / secs,
                         "lat_p50_us": float(np.median(lat_us)), "lat_p99_us": float(np.quantile(lat_us, 0.99)),
                         "exact_replies": ok, "requests": len(pkts)})
    kb, ko, kl, vb, vo, vl = MC.pack(keys, vals)
    sock = MC.udp_server_socket()
    stop = ctypes.c_int(0)
    th = threading.Thread(target=lambda: oracle.lib().oracle_mc_serve(
        sock.fileno(), 4, kb.ctypes.data, ko.ctypes.data, kl.ctypes.data, vb.ctypes.data, vo.ctypes.data,
        vl.ctypes.data, len(keys), 64, ctypes.addressof(stop)))
    th.start()
    try:
        resp, lat, secs = MC.run_client(sock.getsockname()[1], pkts, nthreads=4, window=8)
    finally:
        stop.value = 1
        th.join()
        sock.close()
    ok = sum(1 for p, r in zip(pkts, resp) if r == OM.expected_response(p, table))
    lat_us = np.array(lat, dtype=np.float64) / 1e3
    out["cases"].append({"server": "cpu-oracle", "threads": 4, "elements_per_bucket": 16, "value_bytes": "64-4096",
                         "req_per_s": len(pkts) / secs, "lat_p50_us": float(np.median(lat_us)),
                         "lat_p99_us": float(np.quantile(lat_us, 0.99)), "exact_replies": ok,
                         "requests": len(pkts)})
    # higher offered load (8 client sockets x 32 in flight): the GPU server with 128 work-groups
    # against the CPU server with 4 and 8 threads (profiles/r01_memcached_load_sweep.jsonl)
    keys, vals = MC.dataset(64 * 16 * 3 // 4, vlen=1024)
    table = dict(zip(keys, vals))
    pkts = [MC.encode_get(i, k) for i, k in enumerate(MC.requests(keys, 60000))]
    kb, ko, kl, vb, vo, vl = MC.pack(keys, vals)
    for send in ("blocking", "nonblocking"):
        sg = G.WG | G.RELAXED | (G.NONBLOCKING if send == "nonblocking" else G.BLOCKING)
        resp, lat, secs, _ = W.mc_serve_run(keys, vals, pkts, nwg=128, nbuckets=64, bucket_cap=32, client_threads=8,
                                            window=32, send_gflags=sg)
        ok = sum(1 for p, r in zip(pkts, resp) if r == OM.expected_response(p, table))
        lat_us = np.array(lat, dtype=np.float64) / 1e3
        out["cases"].append({"server": "gpu", "sendto": send, "elements_per_bucket": 16, "work_groups": 128,
                             "in_flight": 256, "req_per_s": len(pkts) / secs, "lat_p50_us": float(np.median(lat_us)),
                             "lat_p99_us": float(np.quantile(lat_us, 0.99)), "exact_replies": ok,
                             "requests": len(pkts)})
    for st in (4, 8):
        sock = MC.udp_server_socket()
        stop = ctypes.c_int(0)
        th = threading.Thread(target=lambda: oracle.lib().oracle_mc_serve(
            sock.fileno(), st, kb.ctypes.data, ko.ctypes.data, kl.ctypes.data, vb.ctypes.data, vo.ctypes.data,
            vl.ctypes.data, len(keys), 64, ctypes.addressof(stop)))
        th.start()
        try:
            resp, lat, secs = MC.run_client(sock.getsockname()[1], pkts, nthreads=8, window=32)
        finally:
            stop.value = 1
            th.join()
            sock.close()
        lat_us = np.array(lat, dtype=np.float64) / 1e3
        ok = sum(1 for p, r in zip(pkts, resp) if r == OM.expected_response(p, table))
        out["cases"].append({"server": "cpu-oracle", "threads": st, "elements_per_bucket": 16, "in_flight": 256,
                             "req_per_s": len(pkts) / secs, "lat_p50_us": float(np.median(lat_us)),
                             "lat_p99_us": float(np.quantile(lat_us, 0.99)), "exact_replies": ok,
                             "requests": len(pkts)})
    out["host_cores"] = nthr
    out["service_threads"] = G.gsys_stats()["threads"]
    print(json.dumps(out), flush=True)
    return 0


def run_mm(a):
    """Config 5 (BASELINE.json configs[4]): (a) AMR-style mesh whose coarsened blocks are released
    with GPU-issued madvise(MADV_DONTNEED) once RSS (GPU-issued pread of /proc/self/statm) passes a
    watermark; (b) signal-search: GPU work-groups notify the host with rt_sigqueueinfo and the host
    hashes each block (SHA-512, as in the paper, P30.14) as its signal arrives vs after the kernel."""
    import hashlib

    import numpy as np
    import torch

    import inputs
    from oracle import plan
    from paper_conf_isca_veselybblor18_b200 import workloads as W

    torch.cuda.set_device(0)
    W.ensure_init()
    out = {"mode": "mm"}
    # (a) AMR: 1024 blocks x 256 KiB mirror (256 MiB), 12 iterations
    nb, bs, iters = 1024, 256 << 10, 12
    lv = inputs.amr_levels(iters, nb, p_coarsen=0.03)
    t0 = time.perf_counter()
    released, rss, maxrss, mesh, rc = W.amr_run(lv, block_bytes=bs, watermark_bytes=0)
    dt = time.perf_counter() - t0
    want = plan.amr_released(lv)
    view = mesh.view().reshape(nb, bs)
    zero_ok = all((not view[b].any()) == bool(want[b]) for b in range(nb))
    out["amr"] = {"blocks": nb, "block_bytes": bs, "iters": iters, "seconds": dt, "wait_rc": rc,
                  "released_blocks": int((released > 0).sum()), "released_equals_rule": released.tolist() == want,
                  "released_read_back_zero": zero_ok, "rss_first_MiB": float(rss[0]) / 2**20,
                  "rss_last_MiB": float(rss[-1]) / 2**20, "maxrss_last_MiB": float(maxrss[-1]) / 1024,
                  "madvise_calls": int((released > 0).sum()), "statm_preads": nb * iters, "getrusage_calls": nb * iters}
    del mesh
    # (b) signal-search: 2048 blocks x 64 KiB
    nb, bs = 2048, 64 << 10
    data = inputs.signal_blocks(nb, bs)
    d = torch.from_numpy(data).cuda()
    key = inputs.dictionary()[0]
    digests = {}

    def consume(b):
        digests[b] = hashlib.sha512(data[b * bs:(b + 1) * bs].tobytes()).hexdigest()
    t0 = time.perf_counter()
    counts, got, ts, rc = W.signal_search_run(d, nb, bs, key, consumer=consume)
    overlapped = time.perf_counter() - t0
    t0 = time.perf_counter()
    counts2, got2, _, _ = W.signal_search_run(d, nb, bs, key)
    for b in range(nb):
        hashlib.sha512(data[b * bs:(b + 1) * bs].tobytes()).hexdigest()
    serial = time.perf_counter() - t0
    out["signal_search"] = {"blocks": nb, "block_bytes": bs, "signals_received": len(got),
                            "ids_exact_once": sorted(got) == list(range(nb)), "digests": len(digests),
                            "overlapped_s": overlapped, "search_then_hash_s": serial,
                            "speedup": serial / overlapped if overlapped > 0 else None}
    print(json.dumps(out), flush=True)
    return 0


def run_fig8(a):
    """Row f3 (sec. VII, Fig. 8): blocking x ordering of a work-group pwrite after N
    permutation iterations on 8 KB blocks, 1024 work-items per work-group.  Reported: time per
    permutation iteration (lower is better) for strong/weak x block/non-block."""
    import numpy as np
    import torch

    import inputs
    from oracle import plan
    from paper_conf_isca_veselybblor18_b200 import gsys as G
    from paper_conf_isca_veselybblor18_b200 import workloads as W

    torch.cuda.set_device(0)
    W.ensure_init()
    nb, bs = 8192, 8192
    data, perm = inputs.perm_inputs(nb, bs)
    path = os.path.join(a.root or "/dev/shm", "gsys_fig8.bin")
    combos = {"strong-block": G.WG | G.BLOCKING | G.STRONG, "strong-nonblock": G.WG | G.NONBLOCKING | G.STRONG,
              "weak-block": G.WG | G.BLOCKING | G.RELAXED, "weak-nonblock": G.WG | G.NONBLOCKING | G.RELAXED}
    out = {"mode": "fig8", "blocks": nb, "block_bytes": bs, "work_items_per_wg": 1024, "grid": 296, "rows": []}
    for iters in (1, 2, 4, 8, 16, 32):
        row = {"iters": iters}
        for name, fl in combos.items():
            W.perm_pwrite_run(data[:bs * 64], perm, iters, path, fl, bs, grid=64)
            secs, rc = W.perm_pwrite_run(data, perm, iters, path, fl, bs, grid=296)
            row[name + "_us_per_perm"] = secs * 1e6 / iters
            row[name + "_ok"] = rc == 0
        got = np.fromfile(path, dtype=np.uint8)
        row["file_equals_cpu_permutation"] = bool(np.array_equal(got, plan.permuted_blocks(data, perm, iters, bs)))
        out["rows"].append(row)
    print(json.dumps(out), flush=True)
    return 0


def run_fig9(a):
    """Row f4 (sec. VII, Fig. 9): host memory-copy throughput while GPU threads poll
    N distinct 64 B lines of pinned host memory (PCIe reads) or of device memory (L2)."""
    import threading

    import numpy as np
    import torch

    from paper_conf_isca_veselybblor18_b200 import gsys as G

    torch.cuda.set_device(0)
    L = G.lib()
    src = np.ones(256 << 20, dtype=np.uint8)
    dst = np.empty_like(src)

    def host_bw(seconds):
        n, t0 = 0, time.perf_counter()
        while time.perf_counter() - t0 < seconds:
            np.copyto(dst, src)
            n += 1
        return n * src.nbytes * 2 / (time.perf_counter() - t0) / 1e9     # read + write bytes
    out = {"mode": "fig9", "baseline_host_copy_GBps": host_bw(1.0), "rows": []}
    sink = torch.zeros(2, dtype=torch.int64, device="cuda")
    for where in ("host", "device"):
        for nlines in (1, 64, 1024, 4096, 16384, 65536, 262144):
            lines = (torch.zeros(nlines * 8, dtype=torch.int64).pin_memory() if where == "host"
                     else torch.zeros(nlines * 8, dtype=torch.int64, device="cuda"))
            sink.zero_()
            ns = int(1.5e9)
            L.gsys_poll_storm(lines.data_ptr(), nlines, max(nlines, 148 * 256), ns, sink.data_ptr(), None)
            time.sleep(0.2)
            bw = host_bw(1.0)
            torch.cuda.synchronize()
            out["rows"].append({"polled": where, "lines": nlines, "gpu_threads": max(nlines, 148 * 256),
                                "host_copy_GBps": bw, "gpu_polls_per_s": int(sink[0].item()) / 1.5})
    print(json.dumps(out), flush=True)
    return 0


if __name__ == "__main__":
    sys.exit(main())

"""paper_conf_isca_veselybblor18_b200 -- GPU-issued POSIX system calls (GENESYS, ISCA 2018) on B200.

The product is the C-ABI library ``libgsys.so`` (include/gsys.h, include/gsys_device.cuh); this
package holds its sources (csrc/), the in-tree nvcc build (build.py), the thin ctypes binding
(gsys.py) and the high-level workload drivers (workloads.py).
"""
from . import gsys  # noqa: F401
from .gsys import (  # noqa: F401
    WI, WG, KERNEL, BLOCKING, NONBLOCKING, STRONG, RELAXED, WEAK, SITE,
    gsys_init, gsys_wait, gsys_shutdown, gsys_stats, gsys_stats_reset, gsys_set_coalesce_max,
    gsys_set_coalesce_window, gsys_set_merge, gsys_set_trace, gsys_trace_read, gsys_device_ctx,
    gsys_wordcount, gsys_scan_device, gsys_bench_calls, gsys_plan_merge, gsys_split_result, gsys_abi_info,
)

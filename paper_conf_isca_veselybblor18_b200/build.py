"""Build libgsys.so (host service + sm_100a kernels) in-tree with nvcc.

    python -m paper_conf_isca_veselybblor18_b200.build

nvcc cross-compiles for sm_100a without a GPU.  The CUDA runtime is linked statically and the
driver API is reached through cudaGetDriverEntryPoint, so the library loads (and its symbols can
be checked) on a machine without libcuda.
"""
from __future__ import annotations

import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
INCLUDE = os.path.join(ROOT, "include")
LIB = os.path.join(PKG, "libgsys.so")
SOURCES = [os.path.join(CSRC, "gsys_host.cpp"), os.path.join(CSRC, "gsys_kernels.cu"),
           os.path.join(CSRC, "gsys_next.cu")]
HEADERS = [os.path.join(INCLUDE, "gsys.h"), os.path.join(INCLUDE, "gsys_device.cuh"),
           os.path.join(CSRC, "gsys_internal.h"), os.path.join(CSRC, "scan_core.cuh"),
           os.path.join(CSRC, "tokscan.cuh")]
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def _stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    return any(os.path.getmtime(p) > t for p in SOURCES + HEADERS + [__file__])


def build(force: bool = False, verbose: bool = False, defines=(), out: str = "", host_flags=(), link=()) -> str:
    """Compile libgsys.so; `defines`/`out` build a diagnostic variant elsewhere (tools/)."""
    if not out and not force and not _stale():
        return LIB
    objs = []
    build_dir = os.path.join(PKG, "build" + ("_" + os.path.basename(out) if out else ""))
    os.makedirs(build_dir, exist_ok=True)
    common = ["-O3", "-std=c++17", "-lineinfo", "-Xcompiler", "-fPIC,-O3,-Wall", "-I", INCLUDE, "-I", CSRC,
              *["-D" + d for d in defines], *[x for f in host_flags for x in ("-Xcompiler", f)]]
    for src in SOURCES:
        obj = os.path.join(build_dir, os.path.basename(src) + ".o")
        cmd = [NVCC, *common, *ARCH, "-c", src, "-o", obj]
        if src.endswith(".cu"):
            cmd += ["-Xptxas", "-v"] if verbose else []
        else:
            cmd = [NVCC, "-x", "cu", *common, *ARCH, "-c", src, "-o", obj]
        subprocess.check_call(cmd)
        objs.append(obj)
    target = out or LIB
    tmp = target + f".tmp{os.getpid()}"
    subprocess.check_call([NVCC, *ARCH, "-shared", "-cudart", "static", "-o", tmp, *objs,
                           "-Xlinker", "--no-undefined", "-lpthread", "-ldl", "-lrt", *link])
    os.replace(tmp, target)
    return target


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose="-v" in sys.argv))

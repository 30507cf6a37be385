"""Build libsnp.so in-tree with nvcc for sm_100a (B200).

    nvcc -gencode arch=compute_100a,code=sm_100a -lineinfo -O3 -shared -cudart static ...

The library is a plain C-ABI shared object (include/snp.h); no torch headers.
"""
from __future__ import annotations

import glob
import os
import subprocess

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
LIB = os.path.join(PKG, "libsnp.so")
HEADER = os.path.join(ROOT, "include", "snp.h")

NVCC_FLAGS = [
    "-gencode", "arch=compute_100a,code=sm_100a",
    "-lineinfo", "-O3", "-std=c++17",
    "-Xcompiler", "-fPIC", "-shared", "-cudart", "static",
    "-Xptxas", "-warn-spills",
]


def sources():
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")))


def _inputs():
    return sources() + sorted(glob.glob(os.path.join(CSRC, "*.h")) + glob.glob(os.path.join(CSRC, "*.cuh"))) + [HEADER, __file__]


def stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    return any(os.path.getmtime(p) > t for p in _inputs())


def nvcc() -> str:
    for c in (os.environ.get("NVCC"), "/usr/local/cuda/bin/nvcc", "nvcc"):
        if c and (os.path.sep not in c or os.path.exists(c)):
            return c
    return "nvcc"


def build_library(force: bool = False, verbose: bool = False) -> str:
    """Compile csrc/*.cu (in parallel) and link libsnp.so if missing/stale (or force)."""
    if not force and not stale():
        return LIB
    import concurrent.futures as cf
    import tempfile
    objdir = tempfile.mkdtemp(prefix="snp_build_")
    compile_flags = [f for f in NVCC_FLAGS if f != "-shared"]
    jobs = []
    for src in sources():
        obj = os.path.join(objdir, os.path.basename(src) + ".o")
        jobs.append((obj, [nvcc(), *compile_flags, "-c", src, "-o", obj]))
    with cf.ThreadPoolExecutor(max_workers=min(8, len(jobs))) as ex:
        futs = [ex.submit(subprocess.run, cmd, capture_output=True, text=True) for _, cmd in jobs]
        for (obj, cmd), f in zip(jobs, futs):
            r = f.result()
            if verbose:
                print(" ".join(cmd))
            if r.stdout or r.stderr:
                print(r.stdout + r.stderr)
            if r.returncode != 0:
                raise subprocess.CalledProcessError(r.returncode, cmd)
    tmp = LIB + f".tmp{os.getpid()}"
    link = [nvcc(), "-gencode", "arch=compute_100a,code=sm_100a", "-shared", "-cudart", "static",
            "-o", tmp, *[o for o, _ in jobs]]
    if verbose:
        print(" ".join(link))
    subprocess.check_call(link)
    os.replace(tmp, LIB)
    return LIB


if __name__ == "__main__":
    print(build_library(force=True, verbose=True))

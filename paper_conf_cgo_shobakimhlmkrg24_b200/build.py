"""Build the in-tree CUDA library libaco_b200.so (sm_100a) with nvcc."""
from __future__ import annotations

import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
LIB = os.path.join(HERE, "libaco_b200.so")
SOURCES = [os.path.join(CSRC, f) for f in ("aco_kernels.cu", "aco_host.cpp")]
HEADERS = [os.path.join(CSRC, "aco_internal.h"),
           os.path.join(os.path.dirname(HERE), "include", "aco.h")]
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
FLAGS = ["-O3", "-lineinfo", "-std=c++17", "-gencode", "arch=compute_100a,code=sm_100a",
         "-Xcompiler", "-fPIC", "-Xcompiler", "-pthread", "-shared"]


def source_fingerprint() -> str:
    """sha256 over the library's sources, headers and nvcc flags: identifies a
    build (nvcc output itself is not byte-reproducible).  A profile records
    it; bench.py uses the profile's figures only for the same fingerprint."""
    import hashlib
    h = hashlib.sha256()
    for f in SOURCES + HEADERS:
        with open(f, "rb") as fh:
            h.update(fh.read())
    h.update(" ".join(FLAGS).encode())
    return h.hexdigest()


def stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    return any(os.path.getmtime(f) > t for f in SOURCES + HEADERS)


def build(force: bool = False, verbose: bool = False, variant: str = "", defines=()) -> str:
    """variant/defines: an A/B build (libaco_b200_<variant>.so) for tools/ only."""
    lib = LIB if not variant else os.path.join(HERE, f"libaco_b200_{variant}.so")
    if force or variant or stale():
        cmd = ([NVCC] + FLAGS + (["-Xptxas", "-v"] if verbose else []) + [f"-D{d}" for d in defines]
               + ["-o", lib] + SOURCES)
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            sys.stderr.write(r.stdout + r.stderr)
            raise RuntimeError("nvcc failed building libaco_b200.so")
        if verbose:
            sys.stderr.write(r.stderr)
    return lib


if __name__ == "__main__":
    # build.py [-v] [variant DEF1 DEF2 ...]
    args = [a for a in sys.argv[1:] if a != "-v"]
    print(build(force=True, verbose="-v" in sys.argv, variant=args[0] if args else "", defines=args[1:]))

"""Build the in-tree C-ABI library ``libdcb200.so`` for sm_100a with nvcc.

Usage: ``python -m paper_conf_ipps_lopez_ortizss13_b200.build [--verbose]``.
The shared library is written next to this file so that it travels with the
repo snapshot to the GPU box (it is git-ignored, not gpurun-ignored).
"""
from __future__ import annotations

import fcntl
import glob
import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
INCLUDE = os.path.join(ROOT, "include")
LIB = os.path.join(PKG, "libdcb200.so")

NVCC_FLAGS = [
    "-gencode", "arch=compute_100a,code=sm_100a",
    "-O3", "-lineinfo", "-std=c++17",
    "-Xcompiler", "-fPIC,-O2",
    "-shared", "-cudart", "static",
]


def sources() -> list[str]:
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")))


def _stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    deps = glob.glob(os.path.join(CSRC, "*")) + glob.glob(os.path.join(INCLUDE, "*.h"))
    return any(os.path.getmtime(d) > t for d in deps) or os.path.getmtime(__file__) > t


def build(force: bool = False, verbose: bool = False, out: str | None = None,
          defines: list[str] | None = None) -> str:
    """Compile libdcb200.so.  ``out``/``defines`` build tuning variants
    (e.g. DC_FAST_IT=31) next to the default library without replacing it."""
    target = out or LIB
    if out is None and not force and not _stale():
        return LIB
    # one builder at a time per target (spawned ranks of a test may all find the
    # library stale); the others wait and re-check instead of rebuilding
    with open(target + ".lock", "w") as lk:
        fcntl.flock(lk, fcntl.LOCK_EX)
        if out is None and not force and not _stale():
            return LIB
        return _compile(target, verbose, defines)


def _compile(target: str, verbose: bool, defines: list[str] | None) -> str:
    nvcc = os.environ.get("NVCC", "nvcc")
    tmp = target + ".tmp%d" % os.getpid()
    cmd = [nvcc, *NVCC_FLAGS, "-I", INCLUDE, "-I", CSRC, "-o", tmp,
           *["-D" + d for d in (defines or [])], *sources()]
    if verbose:
        cmd.insert(1, "-Xptxas=-v")
        print(" ".join(cmd), file=sys.stderr)
    subprocess.check_call(cmd)
    os.replace(tmp, target)
    return target


if __name__ == "__main__":
    import argparse

    ap = argparse.ArgumentParser()
    ap.add_argument("--verbose", action="store_true")
    ap.add_argument("--out", default=None)
    ap.add_argument("-D", dest="defines", action="append", default=[])
    a = ap.parse_args()
    print(build(force=True, verbose=a.verbose, out=a.out, defines=a.defines))

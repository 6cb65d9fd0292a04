"""Build libgrophecy.so in-tree with nvcc for sm_100a.

    python -m paper_conf_ipps_boyermk13_b200.build [--force] [--verbose]

Flags that matter for results: ``-fmad=false`` (no FMA contraction in device
code; DESIGN.md §3 N1) and ``-ffp-contract=off`` for host code (the host
precomputes per-(kernel, transformation) constants that must be bitwise the
definition's values).
"""
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
CSRC = os.path.join(HERE, "csrc")
INCLUDE = os.path.join(ROOT, "include")
LIB = os.path.join(HERE, "libgrophecy.so")
SOURCES = ["space.cpp", "plan.cpp", "project.cu", "groups.cu", "synth.cu", "pcie.cu", "nccl.cpp"]
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def _inputs():
    files = [os.path.join(CSRC, f) for f in SOURCES]
    files += [os.path.join(CSRC, "internal.h"), os.path.join(INCLUDE, "grophecy.h"),
              os.path.abspath(__file__)]
    return files


def up_to_date():
    if not os.path.exists(LIB):
        return False
    t = os.path.getmtime(LIB)
    return all(os.path.getmtime(f) <= t for f in _inputs())


def build(force=False, verbose=False):
    if not force and up_to_date():
        return LIB
    cmd = [NVCC, *ARCH, "-O3", "-lineinfo", "-std=c++17", "-fmad=false", "-shared",
           "-Xcompiler", "-fPIC,-ffp-contract=off,-fno-fast-math,-O2",
           "-I", INCLUDE, "-I", CSRC, "-o", LIB]
    if verbose:
        cmd += ["-Xptxas", "-v"]
    if os.environ.get("GROPHECY_THREADS"):
        cmd += [f"-DGROPHECY_THREADS={int(os.environ['GROPHECY_THREADS'])}"]
    for m in ("GROPHECY_CG", "GROPHECY_CMINB", "GROPHECY_AU32", "GROPHECY_SMINB", "GROPHECY_I2F_MAGIC", "GROPHECY_PHASE_TIMING", "GROPHECY_FUSED", "GROPHECY_PERM", "GROPHECY_XINF_SKIP", "GROPHECY_DISPATCH_TREE"):
        if os.environ.get(m):
            cmd += [f"-D{m}={int(os.environ[m])}"]
    if os.environ.get("GROPHECY_MINB"):
        cmd += [f"-DGROPHECY_MINB={int(os.environ['GROPHECY_MINB'])}"]
    cmd += [os.path.join(CSRC, f) for f in SOURCES] + ["-ldl"]
    subprocess.check_call(cmd)
    return LIB


if __name__ == "__main__":
    build(force="--force" in sys.argv, verbose="--verbose" in sys.argv)
    print(LIB)

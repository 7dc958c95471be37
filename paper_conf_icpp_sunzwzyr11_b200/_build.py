"""Build libcrsd.so in-tree (sm_100a) with nvcc.

Sources: csrc/builder.cpp (host builder, OpenMP), csrc/capi.cpp (C-ABI),
csrc/dist.cpp (NCCL halo exchange), csrc/spmv.cu (kernels).
NCCL headers/library come from the torch-bundled nvidia-nccl wheel so the
process loads one libnccl.so.2 (SURVEY.md §5 hazard).
"""
from __future__ import annotations

import glob
import os
import subprocess
import sys
import sysconfig

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
ROOT = os.path.dirname(HERE)
LIB = os.path.join(HERE, "libcrsd.so")
BUILD = os.path.join(HERE, "build")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def _nccl_dirs():
    cands = []
    for sp in {sysconfig.get_paths()["purelib"], sysconfig.get_paths()["platlib"]}:
        cands.append(os.path.join(sp, "nvidia", "nccl"))
    for c in cands:
        if os.path.exists(os.path.join(c, "include", "nccl.h")):
            return os.path.join(c, "include"), os.path.join(c, "lib")
    return "/usr/include", "/usr/lib/x86_64-linux-gnu"


def _sources():
    return sorted(glob.glob(os.path.join(CSRC, "*.cpp")) + glob.glob(os.path.join(CSRC, "*.cu")))


def _headers():
    return glob.glob(os.path.join(CSRC, "*.h")) + glob.glob(os.path.join(ROOT, "include", "*.h"))


def _stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    return any(os.path.getmtime(f) > t for f in _sources() + _headers() + [__file__])


def build(force: bool = False, verbose: bool = False) -> str:
    if not force and not _stale():
        return LIB
    os.makedirs(BUILD, exist_ok=True)
    inc, libdir = _nccl_dirs()
    common = ["-O3", "-std=c++17", "-lineinfo", "-Xcompiler", "-fPIC,-fopenmp,-Wall", f"-I{inc}", f"-I{os.path.join(ROOT, 'include')}"]
    objs = []
    procs = []
    for src in _sources():
        obj = os.path.join(BUILD, os.path.basename(src) + ".o")
        cmd = [NVCC] + common + ARCH + ["-c", src, "-o", obj]
        if src.endswith(".cu"):
            cmd += ["-Xptxas", "-v"]
        objs.append(obj)
        procs.append((cmd, subprocess.Popen(cmd, stdout=subprocess.PIPE, stderr=subprocess.STDOUT, text=True)))
    for cmd, p in procs:
        out, _ = p.communicate()
        if p.returncode != 0:
            sys.stderr.write(out)
            raise RuntimeError("nvcc failed: " + " ".join(cmd))
        if verbose and out:
            sys.stderr.write(out)
    link = [NVCC, "-shared"] + ARCH + ["-o", LIB] + objs + [
        f"-L{libdir}",
        "-l:libnccl.so.2",
        "-Xlinker",
        f"-rpath,{libdir}",
        "-lgomp",
        "-ldl",
    ]
    subprocess.check_call(link)
    return LIB


EXAMPLE_SRC = os.path.join(ROOT, "examples", "crsd_example.c")
EXAMPLE_BIN = os.path.join(ROOT, "examples", "crsd_example")


def build_example() -> str:
    """Plain-C consumer of the C-ABI (examples/crsd_example.c), linked
    against the in-tree libcrsd.so: proves the boundary needs no Python."""
    if os.path.exists(EXAMPLE_BIN) and os.path.getmtime(EXAMPLE_BIN) > max(
        os.path.getmtime(EXAMPLE_SRC), os.path.getmtime(LIB)
    ):
        return EXAMPLE_BIN
    cuda = os.path.dirname(os.path.dirname(NVCC))
    cmd = [
        "gcc", "-O2", "-Wall", f"-I{os.path.join(ROOT, 'include')}", f"-I{os.path.join(cuda, 'include')}",
        EXAMPLE_SRC, "-o", EXAMPLE_BIN, f"-L{HERE}", "-lcrsd", f"-L{os.path.join(cuda, 'lib64')}", "-lcudart",
        "-lm", f"-Wl,-rpath,{HERE}", f"-Wl,-rpath,{os.path.join(cuda, 'lib64')}",
    ]
    subprocess.check_call(cmd)
    return EXAMPLE_BIN


TOOL_SRC = os.path.join(ROOT, "tools", "hbm_read.cu")
TOOL_LIB = os.path.join(ROOT, "tools", "libhbmread.so")


def build_tools() -> str:
    """tools/libhbmread.so: the read-only HBM bandwidth probe bench.py reports
    as roofline context (not part of the product library)."""
    if not os.path.exists(TOOL_LIB) or os.path.getmtime(TOOL_LIB) < os.path.getmtime(TOOL_SRC):
        subprocess.check_call([NVCC, "-O3"] + ARCH + ["-Xcompiler", "-fPIC", "-shared", "-o", TOOL_LIB, TOOL_SRC])
    return TOOL_LIB


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose=True))

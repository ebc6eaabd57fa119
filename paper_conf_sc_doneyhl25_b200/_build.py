"""Builds libeim.so in-tree (nvcc, sm_100a only).  Used by __graft_entry__.build()
and by the tests; never builds anything under oracle/."""
from __future__ import annotations

import concurrent.futures as cf
import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
BUILD = os.path.join(PKG, "build")
LIB = os.path.join(PKG, "libeim.so")
INCLUDE = os.path.join(ROOT, "include")

ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
SOURCES = ["capi.cpp", "imm.cpp", "comm.cpp", "graph.cu", "sample.cu", "arena.cu", "select.cu"]


def _nccl_dirs():
    import importlib.util
    spec = importlib.util.find_spec("nvidia.nccl")
    if spec is None or not spec.submodule_search_locations:
        raise RuntimeError("NCCL (nvidia.nccl wheel) not found")
    base = list(spec.submodule_search_locations)[0]
    return os.path.join(base, "include"), os.path.join(base, "lib")


def _nvcc():
    for c in (os.environ.get("NVCC"), "/usr/local/cuda/bin/nvcc", "nvcc"):
        if c and (os.path.sep not in c or os.path.exists(c)):
            return c
    return "nvcc"


def _flags(extra_inc):
    # EIM_NVCC_DEFS: extra -D flags for tuning experiments (build with --force)
    defs = os.environ.get("EIM_NVCC_DEFS", "").split()
    return ["-O3", "-std=c++17", *ARCH, "-lineinfo", "-Xcompiler", "-fPIC,-ffp-contract=off,-fno-fast-math",
            "-I", INCLUDE, "-I", CSRC, "-I", extra_inc, "--expt-relaxed-constexpr", *defs]


def build(force: bool = False, verbose: bool = False) -> str:
    nccl_inc, nccl_lib = _nccl_dirs()
    os.makedirs(BUILD, exist_ok=True)
    headers = [os.path.join(CSRC, f) for f in os.listdir(CSRC) if f.endswith((".h", ".cuh"))]
    headers.append(os.path.join(INCLUDE, "eim.h"))
    newest_hdr = max(os.path.getmtime(h) for h in headers)
    nvcc = _nvcc()
    jobs = []
    objs = []
    for src in SOURCES:
        sp = os.path.join(CSRC, src)
        obj = os.path.join(BUILD, src + ".o")
        objs.append(obj)
        if force or not os.path.exists(obj) or os.path.getmtime(obj) < max(os.path.getmtime(sp), newest_hdr):
            cmd = [nvcc, *_flags(nccl_inc), "-c", sp, "-o", obj]
            if src.endswith(".cu"):
                cmd += ["-Xptxas", "-v"] if verbose else []
            jobs.append(cmd)

    def run(cmd):
        r = subprocess.run(cmd, capture_output=True, text=True)
        return cmd, r

    if jobs:
        with cf.ThreadPoolExecutor(max_workers=min(8, len(jobs))) as ex:
            for cmd, r in ex.map(run, jobs):
                if verbose or r.returncode != 0:
                    sys.stderr.write(r.stdout + r.stderr)
                if r.returncode != 0:
                    raise RuntimeError("nvcc failed: " + " ".join(cmd))
    if jobs or force or not os.path.exists(LIB) or os.path.getmtime(LIB) < max(os.path.getmtime(o) for o in objs):
        cmd = [nvcc, *ARCH, "-shared", "-o", LIB, *objs, "-L", nccl_lib, "-l:libnccl.so.2",
               "-Xlinker", "-rpath," + nccl_lib]
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            sys.stderr.write(r.stdout + r.stderr)
            raise RuntimeError("link failed")
    return LIB


def build_probe(force: bool = False) -> str:
    """tools/philox_roof: the Philox throughput probe bench.py uses as the ALU
    roof; tools/gather_roof: the random dependent-load probe (LT walk roof)."""
    hdr = os.path.join(CSRC, "philox.cuh")
    exe = ""
    for name, deps in (("philox_roof", [hdr]), ("gather_roof", [])):
        src = os.path.join(ROOT, "tools", name, name + ".cu")
        exe_n = os.path.join(ROOT, "tools", name, name)
        if force or not os.path.exists(exe_n) or os.path.getmtime(exe_n) < max(os.path.getmtime(p) for p in [src, *deps]):
            subprocess.check_call([_nvcc(), "-O3", "-std=c++17", *ARCH, "-lineinfo", "-o", exe_n, src])
        exe = exe or exe_n
    return exe


if __name__ == "__main__":
    build(force="--force" in sys.argv, verbose="-v" in sys.argv)
    print(LIB)

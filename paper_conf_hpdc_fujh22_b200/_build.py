"""Builds libtlp.so in-tree: nvcc for sm_100a, linked against the NCCL that
torch itself loads (the venv's nvidia-nccl 2.28), with an rpath to it."""
from __future__ import annotations

import concurrent.futures as cf
import glob
import os
import shutil
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
INCLUDE = os.path.join(ROOT, "include")
LIB = os.path.join(PKG, "libtlp.so")
BUILD = os.path.join(ROOT, "build", "tlp")

ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def nccl_dirs():
    """(include dir, lib dir) of the NCCL that torch loads."""
    import importlib.util
    spec = importlib.util.find_spec("nvidia")
    cands = []
    if spec and spec.submodule_search_locations:
        for loc in spec.submodule_search_locations:
            cands.append(os.path.join(loc, "nccl"))
    for c in cands:
        inc, lib = os.path.join(c, "include"), os.path.join(c, "lib")
        if os.path.exists(os.path.join(inc, "nccl.h")) and glob.glob(os.path.join(lib, "libnccl.so*")):
            return inc, lib
    raise RuntimeError("NCCL (nvidia-nccl wheel) not found next to torch")


def nvcc():
    p = shutil.which("nvcc") or "/usr/local/cuda/bin/nvcc"
    if not os.path.exists(p):
        raise RuntimeError("nvcc not found")
    return p


def _sources():
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")))


def _deps():
    return (_sources() + glob.glob(os.path.join(CSRC, "*.h")) + glob.glob(os.path.join(CSRC, "*.cuh"))
            + [os.path.join(INCLUDE, "tlp.h"), __file__])


def up_to_date():
    if not os.path.exists(LIB):
        return False
    t = os.path.getmtime(LIB)
    return all(os.path.getmtime(d) <= t for d in _deps())


def build(force=False, verbose=False, ptxas_verbose=False, defines=(), out=None):
    """defines: extra -D macros (tuning variants); out: alternative .so path."""
    lib = out or LIB
    if not force and not defines and out is None and up_to_date():
        return LIB
    bdir = BUILD if not defines else BUILD + "_" + "_".join(d.replace("=", "") for d in defines)
    os.makedirs(bdir, exist_ok=True)
    nccl_inc, nccl_lib = nccl_dirs()
    flags = ARCH + ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC", "-Xcompiler", "-O3",
                    "--expt-relaxed-constexpr", "-I" + INCLUDE, "-I" + CSRC, "-I" + nccl_inc]
    if ptxas_verbose:
        flags += ["-Xptxas", "-v"]
    flags += ["-D" + d for d in defines]
    objs = []

    def compile_one(src):
        obj = os.path.join(bdir, os.path.basename(src) + ".o")
        cmd = [nvcc()] + flags + ["-c", src, "-o", obj]
        if verbose:
            print(" ".join(cmd), file=sys.stderr)
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError(f"nvcc failed for {src}:\n{r.stdout}\n{r.stderr}")
        if ptxas_verbose or verbose:
            sys.stderr.write(r.stderr)
        return obj

    with cf.ThreadPoolExecutor(max_workers=min(8, os.cpu_count() or 2)) as ex:
        objs = list(ex.map(compile_one, _sources()))
    tmp = lib + ".tmp%d" % os.getpid()
    nccl_so = sorted(glob.glob(os.path.join(nccl_lib, "libnccl.so*")))[0]
    cmd = [nvcc()] + ARCH + ["-shared", "-o", tmp] + objs + [
        "-L" + nccl_lib, "-l:" + os.path.basename(nccl_so), "-Xlinker", "-rpath," + nccl_lib,
        "-cudart", "static"]
    if verbose:
        print(" ".join(cmd), file=sys.stderr)
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"link failed:\n{r.stdout}\n{r.stderr}")
    os.replace(tmp, lib)
    return lib


PROBE_SRC = os.path.join(ROOT, "bench_probe", "l2_ceiling.cu")
PROBE_LIB = os.path.join(ROOT, "bench_probe", "libl2c.so")


def build_probe(force=False):
    """bench.py's L2 gather-ceiling probe (a measurement tool, not the product)."""
    if not os.path.exists(PROBE_SRC):
        return None
    if not force and os.path.exists(PROBE_LIB) and os.path.getmtime(PROBE_LIB) >= os.path.getmtime(PROBE_SRC):
        return PROBE_LIB
    tmp = PROBE_LIB + ".tmp%d" % os.getpid()
    cmd = [nvcc()] + ARCH + ["-O3", "-lineinfo", "-shared", "-Xcompiler", "-fPIC", "-o", tmp, PROBE_SRC,
                             "-cudart", "static"]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"nvcc failed for {PROBE_SRC}:\n{r.stdout}\n{r.stderr}")
    os.replace(tmp, PROBE_LIB)
    return PROBE_LIB


if __name__ == "__main__":
    defs = [a[2:] for a in sys.argv[1:] if a.startswith("-D")]
    outs = [a[6:] for a in sys.argv[1:] if a.startswith("--out=")]
    print(build(force="--force" in sys.argv, verbose="-v" in sys.argv,
                ptxas_verbose="--ptxas" in sys.argv, defines=defs, out=outs[0] if outs else None))

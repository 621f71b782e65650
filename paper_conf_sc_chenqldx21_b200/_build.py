"""Builds libvs.so (the C-ABI library of include/vs.h) in-tree for sm_100a with nvcc.

Each csrc/*.cu is compiled to an object in parallel, then linked into
paper_conf_sc_chenqldx21_b200/libvs.so.  ptxas register/spill reports go to
build/ptxas_<file>.log.  No GPU is needed (nvcc cross-compiles)."""
from __future__ import annotations

import glob
import os
import shutil
import subprocess

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
LIB = os.path.join(PKG, "libvs.so")
BUILD_DIR = os.path.join(ROOT, "build")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
NVCC_FLAGS = ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC", "-Xptxas", "-v",
              "--expt-relaxed-constexpr", "-I" + os.path.join(ROOT, "include")]


def nvcc_path() -> str:
    for cand in (os.environ.get("NVCC"), "/usr/local/cuda/bin/nvcc", shutil.which("nvcc")):
        if cand and os.path.exists(cand):
            return cand
    raise RuntimeError("nvcc not found: cannot build libvs.so")


def _sources():
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")))


def _deps():
    return _sources() + glob.glob(os.path.join(CSRC, "*.cuh")) + [os.path.join(ROOT, "include", "vs.h")]


def up_to_date() -> bool:
    if not os.path.exists(LIB):
        return False
    t = os.path.getmtime(LIB)
    return all(os.path.getmtime(d) <= t for d in _deps())


def build(force: bool = False, verbose: bool = False, out: str = None, defines=()) -> str:
    """Builds libvs.so (or, with ``out``/``defines``, an experimental variant elsewhere)."""
    global LIB, BUILD_DIR
    if out is not None:
        saved = (LIB, BUILD_DIR)
        LIB, BUILD_DIR = out, out + ".build"
        try:
            return _build(True, verbose, list(defines))
        finally:
            LIB, BUILD_DIR = saved
    if not force and up_to_date():
        return LIB
    return _build(force, verbose, [])


def _build(force: bool, verbose: bool, defines) -> str:
    nvcc = nvcc_path()
    os.makedirs(BUILD_DIR, exist_ok=True)
    procs = []
    objs = []
    for src in _sources():
        name = os.path.splitext(os.path.basename(src))[0]
        obj = os.path.join(BUILD_DIR, name + ".o")
        log = open(os.path.join(BUILD_DIR, f"ptxas_{name}.log"), "w")
        cmd = [nvcc, *ARCH, *NVCC_FLAGS, *("-D" + d for d in defines), "-c", src, "-o", obj]
        procs.append((subprocess.Popen(cmd, stdout=log, stderr=subprocess.STDOUT), log, src))
        objs.append(obj)
    failed = []
    for p, log, src in procs:
        p.wait()
        log.close()
        if p.returncode != 0:
            failed.append(src)
    if failed:
        msgs = []
        for src in failed:
            name = os.path.splitext(os.path.basename(src))[0]
            msgs.append(open(os.path.join(BUILD_DIR, f"ptxas_{name}.log")).read()[-4000:])
        raise RuntimeError("nvcc failed for %s:\n%s" % (failed, "\n".join(msgs)))
    tmp = LIB + f".tmp{os.getpid()}"
    subprocess.run([nvcc, *ARCH, "-shared", "-o", tmp, *objs, "-lcudart"], check=True)
    os.replace(tmp, LIB)
    if verbose:
        print("built", LIB)
    return LIB


if __name__ == "__main__":
    build(force=True, verbose=True)

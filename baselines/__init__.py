"""Same-box library baselines for bench.py: cuBLAS Hgemm / GemmEx, cuSPARSE SpMM (Blocked-ELL
and scalar CSR) and SDDMM (scalar CSR).  Bench infrastructure, not the product path."""
from __future__ import annotations

import ctypes
import os
import subprocess

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "baselines.cu")
LIB = os.path.join(_HERE, "libvsbaselines.so")
_lib = None
_P = ctypes.c_void_p
_I64 = ctypes.c_int64


def build(force: bool = False) -> str:
    if not force and os.path.exists(LIB) and os.path.getmtime(LIB) >= os.path.getmtime(_SRC):
        return LIB
    nvcc = "/usr/local/cuda/bin/nvcc"
    tmp = LIB + f".tmp{os.getpid()}"
    subprocess.run([nvcc, "-gencode", "arch=compute_100a,code=sm_100a", "-O2", "-std=c++17",
                    "-Xcompiler", "-fPIC", "-shared", _SRC, "-o", tmp, "-lcublas", "-lcusparse"],
                   check=True)
    os.replace(tmp, LIB)
    return LIB


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(LIB)
        L.bl_create.restype = _P
        L.bl_destroy.argtypes = [_P]
        for f in (L.bl_hgemm, L.bl_gemmex):
            f.restype = ctypes.c_int
            f.argtypes = [_P, _I64, _I64, _I64, _P, _P, _P, _P]
        L.bl_spmm_csr_plan.restype = _P
        L.bl_spmm_csr_plan.argtypes = [_P, _I64, _I64, _I64, _I64, _P, _P, _P, _P, _P, _P,
                                       ctypes.POINTER(ctypes.c_int)]
        L.bl_spmm_bell_plan.restype = _P
        L.bl_spmm_bell_plan.argtypes = [_P, _I64, _I64, _I64, _I64, _I64, _P, _P, _P, _P, _P,
                                        ctypes.POINTER(ctypes.c_int)]
        L.bl_sddmm_csr_plan.restype = _P
        L.bl_sddmm_csr_plan.argtypes = [_P, _I64, _I64, _I64, _I64, _P, _P, _P, _P, _P,
                                        ctypes.c_int, _P, ctypes.POINTER(ctypes.c_int)]
        L.bl_plan_run.restype = ctypes.c_int
        L.bl_plan_run.argtypes = [_P]
        L.bl_plan_free.argtypes = [_P]
        _lib = L
    return _lib

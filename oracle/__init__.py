"""CPU fp64 oracle (ctypes wrapper of oracle/oracle.c).

TEST INFRASTRUCTURE ONLY: import this from tests/, __graft_entry__.smoke() and bench.py's
cpu_baseline / ``--impl reference`` legs, nowhere else.  It shares no code with the CUDA
path and never imports it.  Every function follows the plain definition in oracle.c
(Chen et al. SC'21 §4.1-4.2; §6.4).

Arrays in and out are numpy: fp16 matrices are ``np.float16`` (passed as their bit
patterns), indices ``np.int32``, results ``np.float64``.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB_PATH = os.path.join(_HERE, "liboracle.so")
_lib = None
_lock = threading.Lock()

_P = ctypes.c_void_p
_I64 = ctypes.c_int64


def build(force: bool = False) -> str:
    """Compile oracle.c with gcc (-O2 -fopenmp) into oracle/liboracle.so."""
    if (not force and os.path.exists(_LIB_PATH)
            and os.path.getmtime(_LIB_PATH) >= os.path.getmtime(_SRC)):
        return _LIB_PATH
    tmp = _LIB_PATH + f".tmp{os.getpid()}"
    cmd = ["gcc", "-O2", "-std=c99", "-fopenmp", "-fPIC", "-shared", _SRC, "-o", tmp, "-lm"]
    subprocess.run(cmd, check=True)
    os.replace(tmp, _LIB_PATH)
    return _LIB_PATH


def lib():
    global _lib
    with _lock:
        if _lib is None:
            build()
            L = ctypes.CDLL(_LIB_PATH)
            L.oracle_encode.restype = _I64
            L.oracle_encode.argtypes = [_I64, _I64, ctypes.c_int, _P, _P, _P, _P, _P]
            L.oracle_decode.restype = None
            L.oracle_decode.argtypes = [_I64, _I64, ctypes.c_int, _P, _P, _P, _P]
            L.oracle_spmm.restype = None
            L.oracle_spmm.argtypes = [_I64, _I64, _I64, ctypes.c_int, _P, _P, _P, _P, _P, _P]
            L.oracle_sddmm.restype = None
            L.oracle_sddmm.argtypes = [_I64, _I64, _I64, ctypes.c_int, _P, _P, _P, _P, _P, _P]
            L.oracle_spmm_sample.restype = None
            L.oracle_spmm_sample.argtypes = [_I64, _I64, _I64, ctypes.c_int, _P, _P, _P, _P,
                                             _I64, _P, _P, _P, _P]
            L.oracle_sddmm_sample.restype = None
            L.oracle_sddmm_sample.argtypes = [_I64, _I64, _I64, ctypes.c_int, _P, _P, _P,
                                              _I64, _P, _P, _P, _P]
            L.oracle_softmax.restype = None
            L.oracle_softmax.argtypes = [_I64, ctypes.c_int, _P, _P, ctypes.c_double, _P]
            L.oracle_half_to_double.restype = ctypes.c_double
            L.oracle_half_to_double.argtypes = [ctypes.c_uint16]
            L.oracle_time_layer.restype = _I64
            L.oracle_time_layer.argtypes = [_I64, _I64, _I64, ctypes.c_int, _P, _P, _P,
                                            ctypes.c_int, ctypes.c_int, _P]
            L.oracle_set_num_threads.restype = ctypes.c_int
            L.oracle_set_num_threads.argtypes = [ctypes.c_int]
            L.oracle_num_threads.restype = ctypes.c_int
            L.oracle_num_threads.argtypes = []
            _lib = L
    return _lib


def _ptr(a):
    return None if a is None else a.ctypes.data_as(ctypes.c_void_p)


def _f16(a):
    a = np.ascontiguousarray(a)
    assert a.dtype == np.float16, a.dtype
    return a.view(np.uint16)


def num_threads() -> int:
    return int(lib().oracle_num_threads())


def use_all_cores() -> int:
    """OpenMP team = every core this process may run on (os.sched_getaffinity), whatever
    OMP_NUM_THREADS a launcher exported (torchrun sets 1).  Returns the team size."""
    try:
        n = len(os.sched_getaffinity(0))
    except AttributeError:
        n = os.cpu_count() or 1
    return int(lib().oracle_set_num_threads(n))


def half_to_double(h: int) -> float:
    return float(lib().oracle_half_to_double(int(h) & 0xFFFF))


def encode(M: int, K: int, V: int, dense=None, mask=None, with_vals: bool = True):
    """Column-vector encoding (Fig. 8).  Returns (row_ptr int32[W+1], col_idx int32[nnz],
    vals float16[nnz*V] or None)."""
    assert dense is not None or mask is not None
    W = -(-M // V) if M > 0 else 0
    d = _f16(dense) if dense is not None else None
    m = np.ascontiguousarray(mask, dtype=np.uint8) if mask is not None else None
    if d is not None:
        assert d.shape == (M, K)
    if m is not None:
        assert m.shape == (M, K)
    row_ptr = np.zeros(W + 1, dtype=np.int32)
    nnz = lib().oracle_encode(M, K, V, _ptr(d), _ptr(m), _ptr(row_ptr), None, None)
    col_idx = np.zeros(nnz, dtype=np.int32)
    vals = np.zeros(nnz * V, dtype=np.uint16) if (with_vals and d is not None) else None
    nnz2 = lib().oracle_encode(M, K, V, _ptr(d), _ptr(m), _ptr(row_ptr), _ptr(col_idx), _ptr(vals))
    assert nnz2 == nnz
    return row_ptr, col_idx, (vals.view(np.float16) if vals is not None else None)


def decode(M: int, K: int, V: int, row_ptr, col_idx, vals) -> np.ndarray:
    out = np.zeros((M, K), dtype=np.uint16)
    lib().oracle_decode(M, K, V, _ptr(np.ascontiguousarray(row_ptr, np.int32)),
                        _ptr(np.ascontiguousarray(col_idx, np.int32)), _ptr(_f16(vals)), _ptr(out))
    return out.view(np.float16)


def transpose(M: int, K: int, V: int, row_ptr, col_idx, vals=None):
    """Column-vector encoding (grain V) of A^T [K x M] from the encoding of A [M x K]: by
    definition, the encoding of the dense transpose (Discussion: C^T "under
    column-vector sparse encoding"; §8 Case 1: "encode both W and W^T with our
    column-vector sparse encoding").  With vals None the transpose is of the pattern: every
    stored vector's rows (< M) count as nonzero.  Returns (rowT, colT, valsT or None)."""
    if vals is not None:
        dense = decode(M, K, V, row_ptr, col_idx, vals)
        return encode(K, M, V, dense=np.ascontiguousarray(dense.T))
    mask = np.zeros((M, K), dtype=np.uint8)
    W = len(row_ptr) - 1
    for w in range(W):
        for p in range(int(row_ptr[w]), int(row_ptr[w + 1])):
            for r in range(V):
                if w * V + r < M:
                    mask[w * V + r, int(col_idx[p])] = 1
    return encode(K, M, V, mask=np.ascontiguousarray(mask.T))


def spmm(M: int, K: int, N: int, V: int, row_ptr, col_idx, vals, B):
    """Returns (C64 [M,N] float64, S64 [M,N] float64 = sum |a*b|)."""
    B16 = _f16(B)
    assert B16.shape == (K, N)
    C = np.empty((M, N), dtype=np.float64)
    S = np.empty((M, N), dtype=np.float64)
    lib().oracle_spmm(M, K, N, V, _ptr(np.ascontiguousarray(row_ptr, np.int32)),
                      _ptr(np.ascontiguousarray(col_idx, np.int32)), _ptr(_f16(vals)), _ptr(B16),
                      _ptr(C), _ptr(S))
    return C, S


def sddmm(M: int, N: int, K: int, V: int, row_ptr, col_idx, A, Bt):
    """Returns (out64 [nnz*V], S64 [nnz*V])."""
    A16, Bt16 = _f16(A), _f16(Bt)
    assert A16.shape == (M, K) and Bt16.shape == (N, K)
    nnz = int(row_ptr[-1])
    out = np.empty(nnz * V, dtype=np.float64)
    S = np.empty(nnz * V, dtype=np.float64)
    lib().oracle_sddmm(M, N, K, V, _ptr(np.ascontiguousarray(row_ptr, np.int32)),
                       _ptr(np.ascontiguousarray(col_idx, np.int32)), _ptr(A16), _ptr(Bt16),
                       _ptr(out), _ptr(S))
    return out, S


def spmm_sample(M, K, N, V, row_ptr, col_idx, vals, B, rows, cols):
    """SpMM at output elements (rows[s], cols[s]).  Returns (out64, S64)."""
    rows = np.ascontiguousarray(rows, np.int64)
    cols = np.ascontiguousarray(cols, np.int64)
    out = np.empty(rows.size, np.float64)
    S = np.empty(rows.size, np.float64)
    lib().oracle_spmm_sample(M, K, N, V, _ptr(np.ascontiguousarray(row_ptr, np.int32)),
                             _ptr(np.ascontiguousarray(col_idx, np.int32)), _ptr(_f16(vals)),
                             _ptr(_f16(B)), rows.size, _ptr(rows), _ptr(cols), _ptr(out), _ptr(S))
    return out, S


def sddmm_sample(M, N, K, V, row_ptr, col_idx, A, Bt, vec_p):
    """SDDMM for the stored vectors vec_p.  Returns (out64 [n,V], S64 [n,V])."""
    vec_p = np.ascontiguousarray(vec_p, np.int64)
    rp = np.asarray(row_ptr, np.int64)
    vec_w = np.searchsorted(rp, vec_p, side="right").astype(np.int64) - 1
    out = np.empty(vec_p.size * V, np.float64)
    S = np.empty(vec_p.size * V, np.float64)
    lib().oracle_sddmm_sample(M, N, K, V, _ptr(np.ascontiguousarray(col_idx, np.int32)),
                              _ptr(_f16(A)), _ptr(_f16(Bt)), vec_p.size, _ptr(vec_p), _ptr(vec_w),
                              _ptr(out), _ptr(S))
    return out.reshape(-1, V), S.reshape(-1, V)


def time_layer(M, K, N, V, dense, X, G, threads=0, reps=3):
    """Seconds of `reps` runs of one bench layer step (encode W -> SpMM W X -> SDDMM
    (G X^T) o pattern(W)) with `threads` OpenMP threads (0 = all), timed inside oracle.c with
    the monotonic clock.  Returns (list of seconds, nnz_v)."""
    d, x, g = _f16(dense), _f16(X), _f16(G)
    assert d.shape == (M, K) and x.shape == (K, N) and g.shape == (M, N)
    secs = np.zeros(reps, np.float64)
    nnz = lib().oracle_time_layer(M, K, N, V, _ptr(d), _ptr(x), _ptr(g), int(threads), int(reps),
                                  _ptr(secs))
    if nnz < 0:
        raise MemoryError("oracle_time_layer: allocation failed")
    return secs.tolist(), int(nnz)


def softmax(M: int, V: int, row_ptr, vals, scale: float) -> np.ndarray:
    """Row softmax over the stored entries (Eq. 1).  Returns float64 [nnz*V]."""
    rp = np.ascontiguousarray(row_ptr, np.int32)
    out = np.empty(int(rp[-1]) * V, np.float64)
    lib().oracle_softmax(M, V, _ptr(rp), _ptr(_f16(vals)), float(scale), _ptr(out))
    return out


def softmax_tolerance(p64) -> np.ndarray:
    """Softmax bar: fp16 output rounding (2^-11 relative) plus fp32 exp / sum
    error, bounded by 2^-10 * p + 2^-24."""
    return 2.0 ** -10 * np.abs(np.asarray(p64, np.float64)) + 2.0 ** -24


def tolerance(S64) -> np.ndarray:
    """Acceptance bound of the north star: 2e-3 * sum|a*b| + 2^-24 per element."""
    return 2e-3 * np.asarray(S64, np.float64) + 2.0 ** -24

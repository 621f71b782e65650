"""paper_conf_sc_chenqldx21_b200 — column-vector-sparse fp16 SpMM / SDDMM for B200 (sm_100a).

Thin Python binding of the C ABI in include/vs.h (libvs.so, built in-tree by _build.py).
Argument marshalling only: torch supplies device memory and the current stream; every
step of the path runs in the library's CUDA kernels.  There is no CPU fallback — if
libvs.so is missing or the device is not sm_100 the calls raise.

Method: Chen et al., "Efficient Tensor Core-Based GPU Kernels for Structured Sparsity
under Reduced Precision", SC'21 (column-vector sparse encoding §4.2; SpMM §5
P:635-921; SDDMM §6).

Entry points (same names as the C ABI):
  vs_encode_colvec(M, K, V, dense=None, mask=None, row_ptr, col_idx=None, vals=None, ...)
  vs_spmm(M, K, N, V, row_ptr, col_idx, vals, B, C)
  vs_sddmm(M, N, K, V, row_ptr, col_idx, A, Bt, out_vals)
Conveniences that allocate outputs: encode(), spmm(), sddmm().
"""
from __future__ import annotations

import ctypes
import os
import threading

__all__ = ["VSError", "lib_path", "load", "vs_encode_colvec", "vs_spmm", "vs_spmm_scatter", "vs_sddmm",
           "vs_softmax_colvec", "vs_encode_colvec_batched", "vs_spmm_batched", "vs_sddmm_batched",
           "vs_softmax_colvec_batched", "sparse_attention",
           "encode", "spmm", "sddmm", "transpose", "transpose_pattern", "num_windows"]

_PKG = os.path.dirname(os.path.abspath(__file__))
# VS_LIB_PATH overrides the library location (used to compare kernel build variants)
lib_path = os.environ.get("VS_LIB_PATH") or os.path.join(_PKG, "libvs.so")
_lib = None
_lock = threading.Lock()

_P = ctypes.c_void_p
_I64 = ctypes.c_int64

class SpmmProblem(ctypes.Structure):
    """vs_spmm_problem_t"""
    _fields_ = [("M", ctypes.c_int64), ("K", ctypes.c_int64), ("N", ctypes.c_int64),
                ("V", ctypes.c_int32), ("reserved", ctypes.c_int32), ("row_ptr", ctypes.c_void_p),
                ("col_idx", ctypes.c_void_p), ("vals", ctypes.c_void_p), ("B", ctypes.c_void_p),
                ("C", ctypes.c_void_p)]


class SddmmProblem(ctypes.Structure):
    """vs_sddmm_problem_t"""
    _fields_ = [("M", ctypes.c_int64), ("N", ctypes.c_int64), ("K", ctypes.c_int64),
                ("V", ctypes.c_int32), ("reserved", ctypes.c_int32), ("row_ptr", ctypes.c_void_p),
                ("col_idx", ctypes.c_void_p), ("A", ctypes.c_void_p), ("Bt", ctypes.c_void_p),
                ("out_vals", ctypes.c_void_p)]


class EncodeProblem(ctypes.Structure):
    """vs_encode_problem_t"""
    _fields_ = [("M", ctypes.c_int64), ("K", ctypes.c_int64), ("V", ctypes.c_int32),
                ("reserved", ctypes.c_int32), ("dense", ctypes.c_void_p), ("mask", ctypes.c_void_p),
                ("row_ptr", ctypes.c_void_p), ("col_idx", ctypes.c_void_p), ("vals", ctypes.c_void_p)]


class SoftmaxProblem(ctypes.Structure):
    """vs_softmax_problem_t"""
    _fields_ = [("M", ctypes.c_int64), ("V", ctypes.c_int32), ("scale", ctypes.c_float),
                ("row_ptr", ctypes.c_void_p), ("vals", ctypes.c_void_p), ("out", ctypes.c_void_p)]


STATUS = {0: "VS_SUCCESS", 1: "VS_ERROR_INVALID_VALUE", 2: "VS_ERROR_NOT_SUPPORTED",
          3: "VS_ERROR_CUDA", 4: "VS_ERROR_MISALIGNED"}


class VSError(RuntimeError):
    def __init__(self, status: int, where: str):
        self.status = status
        super().__init__(f"{where}: {STATUS.get(status, status)}")


def load():
    """Loads libvs.so (raises if it has not been built)."""
    global _lib
    with _lock:
        if _lib is None:
            if not os.path.exists(lib_path):
                raise ImportError(f"{lib_path} is missing: run __graft_entry__.build() "
                                  "(nvcc -gencode arch=compute_100a,code=sm_100a)")
            L = ctypes.CDLL(lib_path)
            L.vs_status_string.restype = ctypes.c_char_p
            L.vs_status_string.argtypes = [ctypes.c_int]
            L.vs_version.restype = ctypes.c_int
            L.vs_version.argtypes = []
            L.vs_encode_colvec.restype = ctypes.c_int
            L.vs_encode_colvec.argtypes = [_I64, _I64, ctypes.c_int, _P, _P, _P, _P, _P,
                                           ctypes.POINTER(ctypes.c_int64), _P]
            L.vs_spmm.restype = ctypes.c_int
            L.vs_spmm.argtypes = [_I64, _I64, _I64, ctypes.c_int, _P, _P, _P, _P, _P, _P]
            L.vs_spmm_scatter.restype = ctypes.c_int
            L.vs_spmm_scatter.argtypes = [_I64, _I64, _I64, ctypes.c_int, _P, _P, _P, _P,
                                          ctypes.POINTER(ctypes.c_void_p), ctypes.c_int, _I64, _P]
            L.vs_sddmm.restype = ctypes.c_int
            L.vs_sddmm.argtypes = [_I64, _I64, _I64, ctypes.c_int, _P, _P, _P, _P, _P, _P]
            L.vs_transpose_colvec_workspace.restype = _I64
            L.vs_transpose_colvec_workspace.argtypes = [_I64, _I64, ctypes.c_int]
            L.vs_transpose_colvec.restype = ctypes.c_int
            L.vs_transpose_colvec.argtypes = [_I64, _I64, ctypes.c_int, _P, _P, _P, _P, _P, _P, _P,
                                              ctypes.POINTER(ctypes.c_int64), _P]
            L.vs_transpose_colvec_values.restype = ctypes.c_int
            L.vs_transpose_colvec_values.argtypes = [_I64, _I64, ctypes.c_int, _P, _P, _P, _P, _P, _P, _P]
            L.vs_softmax_colvec.restype = ctypes.c_int
            L.vs_softmax_colvec.argtypes = [_I64, ctypes.c_int, _P, _P, _P, ctypes.c_float, _P]
            for name, st in (("vs_spmm_batched", SpmmProblem), ("vs_sddmm_batched", SddmmProblem),
                             ("vs_encode_colvec_batched", EncodeProblem),
                             ("vs_softmax_colvec_batched", SoftmaxProblem)):
                f = getattr(L, name)
                f.restype = ctypes.c_int
                f.argtypes = [_I64, ctypes.POINTER(st), _P]
            _lib = L
    return _lib


def _check(st: int, where: str):
    if st != 0:
        raise VSError(st, where)


def _stream(stream):
    import torch
    if stream is None:
        stream = torch.cuda.current_stream()
    return ctypes.c_void_p(stream.cuda_stream)


def _ptr(t, dtype=None, name="tensor"):
    """Device pointer of a contiguous CUDA tensor (None -> NULL)."""
    if t is None:
        return None
    import torch
    if not isinstance(t, torch.Tensor) or not t.is_cuda:
        raise TypeError(f"{name} must be a CUDA tensor")
    if dtype is not None and t.dtype != dtype:
        raise TypeError(f"{name} must be {dtype}, got {t.dtype}")
    if not t.is_contiguous():
        raise ValueError(f"{name} must be contiguous")
    return ctypes.c_void_p(t.data_ptr()) if t.numel() > 0 else None


def _addr(t, dtype=None, name="tensor"):
    """_ptr() as a plain integer (or None) for ctypes structure fields."""
    p = _ptr(t, dtype, name)
    return None if p is None else p.value


def num_windows(M: int, V: int) -> int:
    return -(-int(M) // int(V)) if M > 0 else 0


# ------------------------------------------------------------------ C-ABI mirrors

def vs_encode_colvec(M, K, V, dense=None, mask=None, row_ptr=None, col_idx=None, vals=None,
                     want_nnz=False, stream=None):
    """Mirror of vs_encode_colvec.  Count mode when col_idx is None.  Returns nnz_v when
    ``want_nnz`` (the call then synchronises the stream), else None."""
    import torch
    nnz = ctypes.c_int64(-1)
    st = load().vs_encode_colvec(
        int(M), int(K), int(V), _ptr(dense, torch.float16, "dense"),
        _ptr(mask, torch.uint8, "mask"), _ptr(row_ptr, torch.int32, "row_ptr"),
        _ptr(col_idx, torch.int32, "col_idx"), _ptr(vals, torch.float16, "vals"),
        ctypes.byref(nnz) if want_nnz else None, _stream(stream))
    _check(st, "vs_encode_colvec")
    return int(nnz.value) if want_nnz else None


def vs_spmm(M, K, N, V, row_ptr, col_idx, vals, B, C, stream=None):
    import torch
    st = load().vs_spmm(int(M), int(K), int(N), int(V), _ptr(row_ptr, torch.int32, "row_ptr"),
                        _ptr(col_idx, torch.int32, "col_idx"), _ptr(vals, torch.float16, "vals"),
                        _ptr(B, torch.float16, "B"), _ptr(C, torch.float16, "C"), _stream(stream))
    _check(st, "vs_spmm")


def vs_spmm_scatter(M, K, N, V, row_ptr, col_idx, vals, B, dst_ptrs, ldc, stream=None):
    """Mirror of vs_spmm_scatter: ``dst_ptrs`` is a list of integer device addresses (e.g.
    symmetric-memory peer buffers offset to this rank's first column), ``ldc`` their leading
    dimension in elements."""
    import torch
    n = len(dst_ptrs)
    arr = (ctypes.c_void_p * max(n, 1))(*[int(p) for p in dst_ptrs])
    st = load().vs_spmm_scatter(int(M), int(K), int(N), int(V), _ptr(row_ptr, torch.int32, "row_ptr"),
                                _ptr(col_idx, torch.int32, "col_idx"), _ptr(vals, torch.float16, "vals"),
                                _ptr(B, torch.float16, "B"), arr, n, int(ldc), _stream(stream))
    _check(st, "vs_spmm_scatter")


def vs_sddmm(M, N, K, V, row_ptr, col_idx, A, Bt, out_vals, stream=None):
    import torch
    st = load().vs_sddmm(int(M), int(N), int(K), int(V), _ptr(row_ptr, torch.int32, "row_ptr"),
                         _ptr(col_idx, torch.int32, "col_idx"), _ptr(A, torch.float16, "A"),
                         _ptr(Bt, torch.float16, "Bt"), _ptr(out_vals, torch.float16, "out_vals"),
                         _stream(stream))
    _check(st, "vs_sddmm")


def vs_transpose_colvec_workspace(M, K, V) -> int:
    return int(load().vs_transpose_colvec_workspace(int(M), int(K), int(V)))


def vs_transpose_colvec(M, K, V, row_ptr, col_idx, vals, rowT_ptr, colT_idx=None, valsT=None,
                        workspace=None, want_nnz=False, stream=None):
    """Mirror of vs_transpose_colvec.  Count mode when colT_idx
    is None.  Returns nnzT when ``want_nnz`` (the call then synchronises), else None."""
    import torch
    nnz = ctypes.c_int64(-1)
    st = load().vs_transpose_colvec(
        int(M), int(K), int(V), _ptr(row_ptr, torch.int32, "row_ptr"),
        _ptr(col_idx, torch.int32, "col_idx"), _ptr(vals, torch.float16, "vals"),
        _ptr(rowT_ptr, torch.int32, "rowT_ptr"), _ptr(colT_idx, torch.int32, "colT_idx"),
        _ptr(valsT, torch.float16, "valsT"), _ptr(workspace, None, "workspace"),
        ctypes.byref(nnz) if want_nnz else None, _stream(stream))
    _check(st, "vs_transpose_colvec")
    return int(nnz.value) if want_nnz else None


def vs_transpose_colvec_values(M, K, V, row_ptr, col_idx, vals, rowT_ptr, valsT, workspace,
                               stream=None):
    """Mirror of vs_transpose_colvec_values: new values, same transposed pattern."""
    import torch
    st = load().vs_transpose_colvec_values(
        int(M), int(K), int(V), _ptr(row_ptr, torch.int32, "row_ptr"),
        _ptr(col_idx, torch.int32, "col_idx"), _ptr(vals, torch.float16, "vals"),
        _ptr(rowT_ptr, torch.int32, "rowT_ptr"), _ptr(valsT, torch.float16, "valsT"),
        _ptr(workspace, None, "workspace"), _stream(stream))
    _check(st, "vs_transpose_colvec_values")


def vs_softmax_colvec(M, V, row_ptr, vals, out, scale, stream=None):
    """Row softmax over the stored entries (Eq. 1)."""
    import torch
    st = load().vs_softmax_colvec(int(M), int(V), _ptr(row_ptr, torch.int32, "row_ptr"),
                                  _ptr(vals, torch.float16, "vals"), _ptr(out, torch.float16, "out"),
                                  float(scale), _stream(stream))
    _check(st, "vs_softmax_colvec")


# ------------------------------------------------------------------ batched mirrors
#
# Each takes a list of per-problem tuples in the order of the C struct fields (tensors for
# pointers, None for NULL).  Build the ctypes array once with make_*_batch() and pass it to
# the vs_*_batched() call to keep the per-call marshalling cost off a hot loop.

def make_spmm_batch(problems):
    """problems: [(M, K, N, V, row_ptr, col_idx, vals, B, C), ...]"""
    import torch
    arr = (SpmmProblem * len(problems))()
    for i, (M, K, N, V, rp, ci, va, B, C) in enumerate(problems):
        arr[i] = SpmmProblem(int(M), int(K), int(N), int(V), 0, _addr(rp, torch.int32, "row_ptr"),
                             _addr(ci, torch.int32, "col_idx"), _addr(va, torch.float16, "vals"),
                             _addr(B, torch.float16, "B"), _addr(C, torch.float16, "C"))
    return arr


def make_sddmm_batch(problems):
    """problems: [(M, N, K, V, row_ptr, col_idx, A, Bt, out_vals), ...]"""
    import torch
    arr = (SddmmProblem * len(problems))()
    for i, (M, N, K, V, rp, ci, A, Bt, out) in enumerate(problems):
        arr[i] = SddmmProblem(int(M), int(N), int(K), int(V), 0, _addr(rp, torch.int32, "row_ptr"),
                              _addr(ci, torch.int32, "col_idx"), _addr(A, torch.float16, "A"),
                              _addr(Bt, torch.float16, "Bt"), _addr(out, torch.float16, "out_vals"))
    return arr


def make_encode_batch(problems):
    """problems: [(M, K, V, dense, mask, row_ptr, col_idx, vals), ...]"""
    import torch
    arr = (EncodeProblem * len(problems))()
    for i, (M, K, V, d, m, rp, ci, va) in enumerate(problems):
        arr[i] = EncodeProblem(int(M), int(K), int(V), 0, _addr(d, torch.float16, "dense"),
                               _addr(m, torch.uint8, "mask"), _addr(rp, torch.int32, "row_ptr"),
                               _addr(ci, torch.int32, "col_idx"), _addr(va, torch.float16, "vals"))
    return arr


def make_softmax_batch(problems):
    """problems: [(M, V, scale, row_ptr, vals, out), ...]"""
    import torch
    arr = (SoftmaxProblem * len(problems))()
    for i, (M, V, sc, rp, va, out) in enumerate(problems):
        arr[i] = SoftmaxProblem(int(M), int(V), float(sc), _addr(rp, torch.int32, "row_ptr"),
                                _addr(va, torch.float16, "vals"), _addr(out, torch.float16, "out"))
    return arr


def vs_softmax_colvec_batched(batch, stream=None):
    if isinstance(batch, list):
        batch = make_softmax_batch(batch)
    _check(load().vs_softmax_colvec_batched(len(batch), batch, _stream(stream)),
           "vs_softmax_colvec_batched")


def sparse_attention(row_ptr, col_idx, Q, Kmat, Vmat, V, scale=None, nnz=None, stream=None):
    """Eq. 1 on a column-vector mask (row_ptr, col_idx) over [l x l]:
    S = (Q K^T) o C (vs_sddmm), P = softmax(scale * S) row-wise (vs_softmax_colvec),
    out = P Vmat (vs_spmm).  Q, Kmat: [l x k]; Vmat: [l x dv]; returns out [l x dv]."""
    import math
    import torch
    l, k = Q.shape
    if scale is None:
        scale = 1.0 / math.sqrt(k)
    S = sddmm(row_ptr, col_idx, Q, Kmat, V, nnz=nnz, stream=stream)
    vs_softmax_colvec(l, V, row_ptr, S, S, scale, stream=stream)
    return spmm(row_ptr, col_idx, S, Vmat, l, V, stream=stream)


def vs_spmm_batched(batch, stream=None):
    if isinstance(batch, list):
        batch = make_spmm_batch(batch)
    _check(load().vs_spmm_batched(len(batch), batch, _stream(stream)), "vs_spmm_batched")


def vs_sddmm_batched(batch, stream=None):
    if isinstance(batch, list):
        batch = make_sddmm_batch(batch)
    _check(load().vs_sddmm_batched(len(batch), batch, _stream(stream)), "vs_sddmm_batched")


def vs_encode_colvec_batched(batch, stream=None):
    if isinstance(batch, list):
        batch = make_encode_batch(batch)
    _check(load().vs_encode_colvec_batched(len(batch), batch, _stream(stream)),
           "vs_encode_colvec_batched")


# ------------------------------------------------------------------ conveniences

def encode(V, dense=None, mask=None, capacity=None, stream=None):
    """Encodes ``dense`` (fp16 [M,K]) and/or ``mask`` (uint8 [M,K]) with grain V.
    Returns (row_ptr, col_idx, vals) (vals None for a mask-only call).

    Without ``capacity`` a count-mode call sizes the outputs (one stream sync).  With a
    capacity (>= nnz_v, e.g. W*K) the encode is a single asynchronous call and the outputs
    are returned at full capacity length; row_ptr[-1] holds nnz_v."""
    import torch
    src = dense if dense is not None else mask
    M, K = src.shape
    W = num_windows(M, V)
    dev = src.device
    row_ptr = torch.empty(W + 1, dtype=torch.int32, device=dev)
    if capacity is None:
        capacity = vs_encode_colvec(M, K, V, dense, mask, row_ptr, want_nnz=True, stream=stream)
    col_idx = torch.empty(int(capacity), dtype=torch.int32, device=dev)
    vals = torch.empty(int(capacity) * V, dtype=torch.float16, device=dev) if dense is not None else None
    # with capacity 0 there is nothing to write: still produce row_ptr
    vs_encode_colvec(M, K, V, dense, mask, row_ptr,
                     col_idx if capacity > 0 else None, vals if capacity > 0 else None,
                     stream=stream)
    return row_ptr, col_idx, vals


def transpose(row_ptr, col_idx, vals, M, K, V, stream=None):
    """Column-vector encoding of A^T [K x M] from that of A [M x K] (vals None: pattern
    only).  Returns (rowT_ptr, colT_idx, valsT); one count-mode call sizes the outputs."""
    import torch
    dev = row_ptr.device
    KT = num_windows(K, V)
    rowT = torch.empty(KT + 1, dtype=torch.int32, device=dev)
    ws = torch.empty(max(vs_transpose_colvec_workspace(M, K, V), 4), dtype=torch.uint8, device=dev)
    n = vs_transpose_colvec(M, K, V, row_ptr, col_idx, vals, rowT, workspace=ws, want_nnz=True,
                            stream=stream)
    colT = torch.empty(max(n, 1), dtype=torch.int32, device=dev)
    valsT = torch.empty(max(n, 1) * V, dtype=torch.float16, device=dev) if vals is not None else None
    if n > 0:  # (n == 0: rowT is complete and there is nothing else to write)
        vs_transpose_colvec(M, K, V, row_ptr, col_idx, vals, rowT, colT, valsT, workspace=ws,
                            stream=stream)
    return rowT, colT[:n], (valsT[:n * V] if valsT is not None else None)


def transpose_pattern(row_ptr, col_idx, M, K, V, stream=None):
    """Pattern-only encoding of A^T for a layer whose values will be refreshed every step
    (vs_transpose_colvec with vals = NULL: every stored element of A has a slot, so a value
    that is +0.0 now and nonzero later is still placed; see vs.h).  Returns
    (rowT_ptr, colT_idx, valsT buffer, workspace); fill valsT with
    vs_transpose_colvec_values(M, K, V, row_ptr, col_idx, vals, rowT_ptr, valsT, workspace)."""
    import torch
    dev = row_ptr.device
    KT = num_windows(K, V)
    rowT = torch.empty(KT + 1, dtype=torch.int32, device=dev)
    ws = torch.empty(max(vs_transpose_colvec_workspace(M, K, V), 4), dtype=torch.uint8, device=dev)
    n = vs_transpose_colvec(M, K, V, row_ptr, col_idx, None, rowT, workspace=ws, want_nnz=True,
                            stream=stream)
    colT = torch.empty(max(n, 1), dtype=torch.int32, device=dev)
    if n > 0:
        vs_transpose_colvec(M, K, V, row_ptr, col_idx, None, rowT, colT, None, workspace=ws,
                            stream=stream)
    valsT = torch.empty(max(n, 1) * V, dtype=torch.float16, device=dev)
    return rowT, colT[:n], valsT[:n * V], ws


def spmm(row_ptr, col_idx, vals, B, M, V, out=None, stream=None):
    """C[M,N] = A * B for A = (row_ptr, col_idx, vals) with grain V."""
    import torch
    K, N = B.shape
    C = out if out is not None else torch.empty((M, N), dtype=torch.float16, device=B.device)
    vs_spmm(M, K, N, V, row_ptr, col_idx, vals, B, C, stream=stream)
    return C


def sddmm(row_ptr, col_idx, A, Bt, V, nnz=None, out=None, stream=None):
    """out_vals = (A Bt^T) sampled at the mask (row_ptr, col_idx); A [M,K], Bt [N,K]."""
    import torch
    M, K = A.shape
    N = Bt.shape[0]
    if out is None:
        n = int(row_ptr[-1].item()) if nnz is None else int(nnz)
        out = torch.empty(n * V, dtype=torch.float16, device=A.device)
    vs_sddmm(M, N, K, V, row_ptr, col_idx, A, Bt, out, stream=stream)
    return out

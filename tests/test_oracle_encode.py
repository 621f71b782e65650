"""Pins of the oracle's column-vector encoder (§4.2, Fig. 8).

Each test checks oracle.encode / oracle.decode against something other than the oracle:
the paper's worked example, bit-exact round trips, and two library encoders that are the
same format (scipy BSR with (V,1) blocks, torch.to_sparse_bsr)."""
import json
import os

import numpy as np
import pytest
import scipy.sparse as sp

import oracle
from synth import gen

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "fig8_encoding.json")


def test_fig8_worked_example():
    """Fig. 8: V=2, 3 windows; csrRowPtr=[0,3,4,6], csrColInd=[0,2,6,3,1,6], csrVal=[0..11]."""
    g = json.load(open(GOLDEN))
    # the 6 x 7 matrix drawn in Fig. 8 (value v at its position; everything else 0)
    X = np.zeros((6, 7), dtype=np.float16)
    X[0, 0], X[1, 0] = 0, 1      # vector (0,1): stored zero inside a kept vector
    X[0, 2], X[1, 2] = 2, 3
    X[0, 6], X[1, 6] = 4, 5
    X[2, 3], X[3, 3] = 6, 7
    X[4, 1], X[5, 1] = 8, 9
    X[4, 6], X[5, 6] = 10, 11
    row_ptr, col_idx, vals = oracle.encode(g["M"], g["K"], g["V"], dense=X)
    assert row_ptr.tolist() == g["csrRowPtr"]
    assert col_idx.tolist() == g["csrColInd"]
    assert vals.astype(np.float64).tolist() == [float(v) for v in g["csrVal"]]
    # count-only call agrees and decode inverts
    assert np.array_equal(oracle.decode(6, 7, 2, row_ptr, col_idx, vals).view(np.uint16),
                          X.view(np.uint16))


@pytest.mark.parametrize("V", [1, 2, 4, 8])
@pytest.mark.parametrize("M,K", [(1, 1), (5, 3), (13, 17), (64, 40), (67, 31)])
def test_roundtrip_bitexact(V, M, K):
    """decode(encode(X)) == X bit for bit, including -0.0 and zeros inside kept vectors."""
    rng = gen.make_rng(f"rt_{V}_{M}_{K}")
    X = gen.colvec_dense(rng, M, K, V, 0.3, inner_zero_frac=0.2, neg_zero_frac=0.05)
    rp, ci, va = oracle.encode(M, K, V, dense=X)
    W = -(-M // V)
    assert rp.shape == (W + 1,) and rp[0] == 0 and np.all(np.diff(rp) >= 0)
    for w in range(W):
        cols = ci[rp[w]:rp[w + 1]]
        assert np.all(np.diff(cols) > 0), "ascending, distinct columns per window"
    # padded rows of the last window hold +0.0 bits
    if M % V:
        pad = va.view(np.uint16).reshape(-1, V)[rp[W - 1]:rp[W], M % V:]
        assert np.all(pad == 0)
    Y = oracle.decode(M, K, V, rp, ci, va)
    assert np.array_equal(Y.view(np.uint16), X.view(np.uint16))


@pytest.mark.parametrize("V", [1, 2, 4, 8])
def test_matches_scipy_bsr(V):
    """BSR with blocksize (V,1) is the same format: indptr=row_ptr, indices=col_idx,
    data=(nnz,V,1)=vals.  Values compared as fp32 (fp16->fp32 is exact)."""
    rng = gen.make_rng(f"bsr_{V}")
    M, K = 8 * 12, 57
    X = gen.colvec_dense(rng, M, K, V, 0.25)
    rp, ci, va = oracle.encode(M, K, V, dense=X)
    B = sp.bsr_matrix(X.astype(np.float32), blocksize=(V, 1))
    B.sort_indices()
    assert np.array_equal(B.indptr, rp)
    assert np.array_equal(B.indices, ci)
    assert np.array_equal(B.data.reshape(-1), va.astype(np.float32))


@pytest.mark.parametrize("V", [1, 2, 4, 8])
def test_matches_torch_bsr(V):
    import torch
    rng = gen.make_rng(f"tbsr_{V}")
    M, K = 8 * 9, 45
    X = gen.colvec_dense(rng, M, K, V, 0.3)
    rp, ci, va = oracle.encode(M, K, V, dense=X)
    T = torch.from_numpy(X.astype(np.float32)).to_sparse_bsr((V, 1))
    assert np.array_equal(T.crow_indices().numpy(), rp)
    assert np.array_equal(T.col_indices().numpy(), ci)
    assert np.array_equal(T.values().numpy().reshape(-1), va.astype(np.float32))


@pytest.mark.parametrize("V", [1, 2, 4, 8])
def test_mask_and_value_encoding_agree(V):
    """On generator data (stored vectors have no all-zero vector) encoding by the mask and
    encoding by the values give the same pattern."""
    rng = gen.make_rng(f"mask_{V}")
    M, K = 50, 70
    X = gen.colvec_dense(rng, M, K, V, 0.2)
    mask = (X != 0).astype(np.uint8)
    rp1, ci1, _ = oracle.encode(M, K, V, dense=X)
    rp2, ci2, _ = oracle.encode(M, K, V, mask=mask)
    assert np.array_equal(rp1, rp2) and np.array_equal(ci1, ci2)


def test_mask_keeps_vectors_by_mask_not_values():
    """With a mask, the mask decides; vals are copied from dense even when all zero."""
    X = np.zeros((4, 3), np.float16)
    mask = np.zeros((4, 3), np.uint8)
    mask[1, 2] = 1
    rp, ci, va = oracle.encode(4, 3, 2, dense=X, mask=mask)
    assert rp.tolist() == [0, 1, 1] and ci.tolist() == [2]
    assert va.view(np.uint16).tolist() == [0, 0]


def test_degenerate_shapes():
    rp, ci, va = oracle.encode(0, 5, 4, dense=np.zeros((0, 5), np.float16))
    assert rp.tolist() == [0] and ci.size == 0
    rp, ci, va = oracle.encode(7, 0, 4, dense=np.zeros((7, 0), np.float16))
    assert rp.tolist() == [0, 0, 0] and ci.size == 0


def test_half_to_double_all_bit_patterns():
    """The oracle's fp16 widening equals numpy's for every finite bit pattern."""
    L = oracle.lib()
    bits = np.arange(65536, dtype=np.uint32).astype(np.uint16)
    ref = bits.view(np.float16).astype(np.float64)
    got = np.array([L.oracle_half_to_double(int(b)) for b in bits])
    fin = np.isfinite(ref)
    assert np.array_equal(got[fin], ref[fin])
    assert np.array_equal(np.signbit(got[fin]), np.signbit(ref[fin]))
    assert np.all(np.isinf(got[np.isinf(ref)])) and np.all(np.isnan(got[np.isnan(ref)]))

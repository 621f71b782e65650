"""Pins of oracle.transpose — the column-vector encoding of A^T (the
training-side operand dX = W^T dY, §8 Case 1 P:1625-1638, Discussion P:1605-1614) — against
scipy, brute force, square-block closed forms and the SpMM adjoint identity."""
import itertools

import numpy as np
import pytest
import scipy.sparse as sp

import oracle
from synth import gen


def f64(x):
    return np.asarray(x, dtype=np.float64)


@pytest.mark.parametrize("V", [1, 2, 4, 8])
def test_transpose_is_bsr_of_dense_transpose(V):
    # scipy BSR with (V,1) blocks of the dense transpose (values nonzero: no -0.0 / stored 0)
    rng = gen.make_rng(f"otr_bsr_{V}")
    M, K = 8 * V, 6 * V
    A = gen.colvec_dense(rng, M, K, V, 0.3)
    rp, ci, va = oracle.encode(M, K, V, dense=A)
    rT, cT, vT = oracle.transpose(M, K, V, rp, ci, va)
    B = sp.bsr_matrix(A.T.astype(np.float32), blocksize=(V, 1))
    B.sort_indices()
    assert np.array_equal(rT, B.indptr) and np.array_equal(cT, B.indices)
    assert np.array_equal(vT.astype(np.float32), B.data.reshape(-1))


@pytest.mark.parametrize("V", [1, 2, 4, 8])
def test_transpose_brute_force_tiny(V):
    # decode(transpose(A)) == decode(A)^T bit for bit, including -0.0 and zeros in vectors
    for M, K in itertools.product([1, 3, 8, 9, 17], [1, 2, 7, 16, 19]):
        rng = gen.make_rng(f"otr_tiny_{V}_{M}_{K}")
        A = gen.colvec_dense(rng, M, K, V, 0.4, inner_zero_frac=0.2, neg_zero_frac=0.05)
        rp, ci, va = oracle.encode(M, K, V, dense=A)
        rT, cT, vT = oracle.transpose(M, K, V, rp, ci, va)
        AT = oracle.decode(K, M, V, rT, cT, vT)
        assert np.array_equal(AT.view(np.uint16), np.ascontiguousarray(A.T).view(np.uint16))
        # every stored A^T vector has a nonzero bit pattern (keep rule R5)
        if len(cT):
            assert np.all(vT.view(np.uint16).reshape(-1, V).any(axis=1))


@pytest.mark.parametrize("V", [2, 4, 8])
def test_square_blocks_closed_form_and_involution(V):
    # square V x V blocks: each block gives exactly V vectors of A^T, and transposing twice
    # returns the original encoding
    rng = gen.make_rng(f"otr_blk_{V}")
    M, K = 12 * V, 9 * V
    A = gen.block_dense(rng, M, K, V, 0.35)
    rp, ci, va = oracle.encode(M, K, V, dense=A)
    rT, cT, vT = oracle.transpose(M, K, V, rp, ci, va)
    blocks = (A.reshape(M // V, V, K // V, V) != 0).any(axis=(1, 3))
    assert np.array_equal(np.diff(rT), V * blocks.sum(axis=0))
    assert int(rT[-1]) == int(rp[-1])
    r2, c2, v2 = oracle.transpose(K, M, V, rT, cT, vT)
    assert np.array_equal(r2, rp) and np.array_equal(c2, ci)
    assert np.array_equal(v2.view(np.uint16), va.view(np.uint16))


@pytest.mark.parametrize("V", [1, 2, 4, 8])
def test_adjoint_identity_spmm_transpose(V):
    # <W X, G> = <X, W^T G> with both products from oracle.spmm (W and W^T encodings)
    rng = gen.make_rng(f"otr_adj_{V}")
    M, K, N = 40, 36, 12
    A = gen.colvec_dense(rng, M, K, V, 0.3)
    X = gen.dense_operand(rng, K, N)
    G = gen.dense_operand(rng, M, N)
    rp, ci, va = oracle.encode(M, K, V, dense=A)
    rT, cT, vT = oracle.transpose(M, K, V, rp, ci, va)
    Y, _ = oracle.spmm(M, K, N, V, rp, ci, va, X)
    dX, _ = oracle.spmm(K, M, N, V, rT, cT, vT, G)
    lhs = float(np.sum(Y * f64(G)))
    rhs = float(np.sum(f64(X) * dX))
    assert abs(lhs - rhs) <= 1e-9 * max(1.0, abs(lhs))
    np.testing.assert_allclose(dX, f64(A).T @ f64(G), rtol=1e-12, atol=1e-12)


@pytest.mark.parametrize("V", [1, 4, 8])
def test_pattern_transpose(V):
    # pattern-only transpose == value transpose when no stored element is zero
    rng = gen.make_rng(f"otr_pat_{V}")
    M, K = 5 * V + 3, 7 * V + 1
    A = gen.colvec_dense(rng, M, K, V, 0.3)
    rp, ci, va = oracle.encode(M, K, V, dense=A)
    rT, cT, _ = oracle.transpose(M, K, V, rp, ci, va)
    # a kept vector's rows are all nonzero here except padding rows >= M, which the
    # pattern transpose skips too
    pT, pcT, none = oracle.transpose(M, K, V, rp, ci, None)
    assert none is None
    assert np.array_equal(pT, rT) and np.array_equal(pcT, cT)

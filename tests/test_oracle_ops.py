"""Pins of the oracle's SpMM (§4.1) and SDDMM (§4.1, §6.4).

References used here are independent of oracle.c: numpy fp64 dense products on the
generator's dense matrices (brute force), scipy CSR / BSR products, closed forms (identity
operands, integer-exact inputs), the all-ones mask = GEMM reading of P:1539-1541 and the
adjoint identity between the two ops (training equations)."""
import itertools

import numpy as np
import pytest
import scipy.sparse as sp

import oracle
from synth import gen

SIZES = [1, 2, 3, 5, 8, 9, 16]


def f64(x):
    return np.asarray(x).astype(np.float64)


# ------------------------------------------------------------------------------- SpMM

@pytest.mark.parametrize("V", [1, 2, 4, 8])
@pytest.mark.parametrize("density", [0.0, 0.3, 1.0])
def test_spmm_brute_force_tiny(V, density):
    """Every tiny shape: oracle(encode(A)) == numpy fp64 A @ B (up to fp64 rounding)."""
    for M, K, N in itertools.product(SIZES, SIZES, SIZES):
        rng = gen.make_rng(f"bf_spmm_{V}_{density}_{M}_{K}_{N}")
        A = gen.colvec_dense(rng, M, K, V, density)
        B = gen.dense_operand(rng, K, N)
        rp, ci, va = oracle.encode(M, K, V, dense=A)
        C, S = oracle.spmm(M, K, N, V, rp, ci, va, B)
        ref = f64(A) @ f64(B)
        np.testing.assert_allclose(C, ref, rtol=1e-12, atol=1e-12)
        assert np.all(S >= np.abs(C) - 1e-12)
        np.testing.assert_allclose(S, np.abs(f64(A)) @ np.abs(f64(B)), rtol=1e-12, atol=1e-12)


def test_spmm_v1_equals_scalar_csr():
    """V=1 is plain CSR: compare with scipy.sparse.csr_matrix(A) @ B."""
    rng = gen.make_rng("csr_v1")
    M, K, N = 97, 130, 33
    A = gen.colvec_dense(rng, M, K, 1, 0.1)
    B = gen.dense_operand(rng, K, N)
    rp, ci, va = oracle.encode(M, K, 1, dense=A)
    C, _ = oracle.spmm(M, K, N, 1, rp, ci, va, B)
    csr = sp.csr_matrix((f64(va), ci, rp), shape=(M, K))
    np.testing.assert_allclose(C, csr @ f64(B), rtol=1e-12, atol=1e-13)
    np.testing.assert_allclose(C, sp.csr_matrix(f64(A)) @ f64(B), rtol=1e-12, atol=1e-13)


@pytest.mark.parametrize("V", [2, 4, 8])
def test_spmm_equals_bsr(V):
    """The encoding is BSR with (V,1) blocks: bsr_matrix((vals,col_idx,row_ptr)) @ B."""
    rng = gen.make_rng(f"bsr_spmm_{V}")
    M, K, N = 8 * 11, 75, 40
    A = gen.colvec_dense(rng, M, K, V, 0.2)
    B = gen.dense_operand(rng, K, N)
    rp, ci, va = oracle.encode(M, K, V, dense=A)
    C, _ = oracle.spmm(M, K, N, V, rp, ci, va, B)
    bsr = sp.bsr_matrix((f64(va).reshape(-1, V, 1), ci, rp), shape=(M, K))
    np.testing.assert_allclose(C, bsr @ f64(B), rtol=1e-12, atol=1e-13)


@pytest.mark.parametrize("V", [1, 2, 4, 8])
def test_spmm_integer_exact(V):
    """Values in {-2,-1,1,2}: every sum is an integer, the oracle result is exact."""
    rng = gen.make_rng(f"int_spmm_{V}")
    M, K, N = 45, 64, 24
    A = gen.colvec_dense(rng, M, K, V, 0.4, exact=True)
    B = gen.dense_operand(rng, K, N, exact=True)
    rp, ci, va = oracle.encode(M, K, V, dense=A)
    C, _ = oracle.spmm(M, K, N, V, rp, ci, va, B)
    ref = A.astype(np.int64) @ B.astype(np.int64)
    assert np.array_equal(C, ref.astype(np.float64))


@pytest.mark.parametrize("V", [1, 4, 8])
def test_spmm_identity_B(V):
    """B = I_K gives C = A exactly (a pure scatter of vals)."""
    rng = gen.make_rng(f"eye_spmm_{V}")
    M, K = 37, 29
    A = gen.colvec_dense(rng, M, K, V, 0.3)
    rp, ci, va = oracle.encode(M, K, V, dense=A)
    C, _ = oracle.spmm(M, K, K, V, rp, ci, va, np.eye(K, dtype=np.float16))
    assert np.array_equal(C, f64(A))


def test_spmm_empty_windows_give_zero_rows():
    M, K, N, V = 16, 10, 5, 4
    A = np.zeros((M, K), np.float16)
    A[5, 3] = 1.5
    rp, ci, va = oracle.encode(M, K, V, dense=A)
    B = gen.dense_operand(gen.make_rng("ew"), K, N)
    C, _ = oracle.spmm(M, K, N, V, rp, ci, va, B)
    ref = np.zeros((M, N))
    ref[5] = 1.5 * f64(B[3])
    assert np.array_equal(C, ref)


def test_spmm_sample_matches_full():
    rng = gen.make_rng("samp_spmm")
    M, K, N, V = 50, 40, 30, 4
    A = gen.colvec_dense(rng, M, K, V, 0.3)
    B = gen.dense_operand(rng, K, N)
    rp, ci, va = oracle.encode(M, K, V, dense=A)
    C, S = oracle.spmm(M, K, N, V, rp, ci, va, B)
    rows = rng.integers(0, M, 200)
    cols = rng.integers(0, N, 200)
    o, s = oracle.spmm_sample(M, K, N, V, rp, ci, va, B, rows, cols)
    assert np.array_equal(o, C[rows, cols]) and np.array_equal(s, S[rows, cols])


# ------------------------------------------------------------------------------ SDDMM

def sddmm_brute(A, Bt, mask, M, N, V, rp, ci):
    """Dense fp64 A @ Bt^T gathered at the stored vectors (test-side, numpy)."""
    D = f64(A) @ f64(Bt).T
    out = []
    W = len(rp) - 1
    for w in range(W):
        for p in range(rp[w], rp[w + 1]):
            for r in range(V):
                i = w * V + r
                out.append(D[i, ci[p]] if i < M else 0.0)
    return np.array(out, np.float64)


@pytest.mark.parametrize("V", [1, 2, 4, 8])
@pytest.mark.parametrize("density", [0.0, 0.3, 1.0])
def test_sddmm_brute_force_tiny(V, density):
    for M, N, K in itertools.product(SIZES, SIZES, [1, 3, 8, 16]):
        rng = gen.make_rng(f"bf_sddmm_{V}_{density}_{M}_{N}_{K}")
        mask = gen.colvec_mask(rng, M, N, V, density)
        A = gen.dense_operand(rng, M, K)
        Bt = gen.dense_operand(rng, N, K)
        rp, ci, _ = oracle.encode(M, N, V, mask=mask)
        out, S = oracle.sddmm(M, N, K, V, rp, ci, A, Bt)
        ref = sddmm_brute(A, Bt, mask, M, N, V, rp, ci)
        np.testing.assert_allclose(out, ref, rtol=1e-12, atol=1e-12)
        assert np.all(S >= np.abs(out) - 1e-12)


@pytest.mark.parametrize("V", [1, 2, 4, 8])
def test_sddmm_all_ones_mask_is_gemm(V):
    """A dense all-ones mask C turns the sampled product into the dense A B."""
    rng = gen.make_rng(f"ones_{V}")
    M, N, K = 8 * 5, 24, 48
    mask = np.ones((M, N), np.uint8)
    A = gen.dense_operand(rng, M, K)
    Bt = gen.dense_operand(rng, N, K)
    rp, ci, _ = oracle.encode(M, N, V, mask=mask)
    out, _ = oracle.sddmm(M, N, K, V, rp, ci, A, Bt)
    G = out.reshape(M // V, N, V).transpose(0, 2, 1).reshape(M, N)
    np.testing.assert_allclose(G, f64(A) @ f64(Bt).T, rtol=1e-12, atol=1e-12)


@pytest.mark.parametrize("V", [1, 4, 8])
def test_sddmm_identity_A_is_gather(V):
    """A = I (M = K): out[pV + r] = Bt[col_idx[p]][wV + r] exactly."""
    rng = gen.make_rng(f"eye_sddmm_{V}")
    M = K = 24
    N = 31
    mask = gen.colvec_mask(rng, M, N, V, 0.4)
    Bt = gen.dense_operand(rng, N, K)
    rp, ci, _ = oracle.encode(M, N, V, mask=mask)
    out, _ = oracle.sddmm(M, N, K, V, rp, ci, np.eye(M, dtype=np.float16), Bt)
    exp = []
    for w in range(len(rp) - 1):
        for p in range(rp[w], rp[w + 1]):
            exp.extend(f64(Bt[ci[p], w * V:(w + 1) * V]))
    assert np.array_equal(out, np.array(exp))


@pytest.mark.parametrize("V", [1, 2, 4, 8])
def test_sddmm_integer_exact(V):
    rng = gen.make_rng(f"int_sddmm_{V}")
    M, N, K = 35, 40, 64
    mask = gen.colvec_mask(rng, M, N, V, 0.3)
    A = gen.dense_operand(rng, M, K, exact=True)
    Bt = gen.dense_operand(rng, N, K, exact=True)
    rp, ci, _ = oracle.encode(M, N, V, mask=mask)
    out, _ = oracle.sddmm(M, N, K, V, rp, ci, A, Bt)
    D = A.astype(np.int64) @ Bt.astype(np.int64).T
    for w in range(len(rp) - 1):
        for p in range(rp[w], rp[w + 1]):
            for r in range(V):
                i = w * V + r
                assert out[p * V + r] == (D[i, ci[p]] if i < M else 0)


def test_sddmm_v1_equals_csr_sampling():
    """V=1: out = (A Bt^T) at the CSR positions (scipy: csr.multiply(dense))."""
    rng = gen.make_rng("csr_sddmm")
    M, N, K = 60, 70, 32
    mask = gen.colvec_mask(rng, M, N, 1, 0.1)
    A = gen.dense_operand(rng, M, K)
    Bt = gen.dense_operand(rng, N, K)
    rp, ci, _ = oracle.encode(M, N, 1, mask=mask)
    out, _ = oracle.sddmm(M, N, K, 1, rp, ci, A, Bt)
    pattern = sp.csr_matrix((np.ones(ci.size), ci, rp), shape=(M, N))
    ref = pattern.multiply(f64(A) @ f64(Bt).T).tocsr()
    ref.sort_indices()
    np.testing.assert_allclose(out, ref.data, rtol=1e-12, atol=1e-13)


def test_sddmm_sample_matches_full():
    rng = gen.make_rng("samp_sddmm")
    M, N, K, V = 30, 50, 20, 8
    mask = gen.colvec_mask(rng, M, N, V, 0.3)
    A = gen.dense_operand(rng, M, K)
    Bt = gen.dense_operand(rng, N, K)
    rp, ci, _ = oracle.encode(M, N, V, mask=mask)
    out, S = oracle.sddmm(M, N, K, V, rp, ci, A, Bt)
    ps = rng.integers(0, ci.size, 40)
    o, s = oracle.sddmm_sample(M, N, K, V, rp, ci, A, Bt, ps)
    assert np.array_equal(o, out.reshape(-1, V)[ps]) and np.array_equal(s, S.reshape(-1, V)[ps])


# ------------------------------------------------------------------- SpMM <-> SDDMM

@pytest.mark.parametrize("V", [1, 2, 4, 8])
def test_adjoint_identity(V):
    """Training pair: Y = W X is SpMM, dL/dW = (dL/dY X^T) o pattern(W) is
    SDDMM; hence <SpMM(W, X), G> = <vals_W, SDDMM(pattern W; G, X)>.  Here vs_sddmm's
    A is G [M x N] and its Bt [K x N] is X (K rows of length N)."""
    rng = gen.make_rng(f"adj_{V}")
    M, K, N = 8 * 7 + 3, 45, 38
    Wd = gen.colvec_dense(rng, M, K, V, 0.3)
    X = gen.dense_operand(rng, K, N)
    G = gen.dense_operand(rng, M, N)
    rp, ci, va = oracle.encode(M, K, V, dense=Wd)
    Y, _ = oracle.spmm(M, K, N, V, rp, ci, va, X)
    dW, _ = oracle.sddmm(M, K, N, V, rp, ci, G, X)
    lhs = float(np.sum(Y * f64(G)))
    rhs = float(np.dot(f64(va), dW))
    assert abs(lhs - rhs) <= 1e-9 * max(1.0, abs(lhs))


# ---------------------------------------------------- softmax (NEXT item, Eq. 1)

def dense_masked_softmax(vals, rp, ci, M, N, V, scale):
    """numpy: scatter the stored entries into a dense [M x N] matrix filled with -inf, then
    the textbook row softmax; gathered back at the stored positions."""
    D = np.full((M, N), -np.inf)
    W = len(rp) - 1
    for w in range(W):
        for p in range(rp[w], rp[w + 1]):
            for r in range(V):
                if w * V + r < M:
                    D[w * V + r, ci[p]] = scale * f64(vals[p * V + r])
    with np.errstate(invalid="ignore"):
        E = np.exp(D - D.max(axis=1, keepdims=True))
        P = E / E.sum(axis=1, keepdims=True)
    out = []
    for w in range(W):
        for p in range(rp[w], rp[w + 1]):
            for r in range(V):
                out.append(P[w * V + r, ci[p]] if w * V + r < M else 0.0)
    return np.array(out)


@pytest.mark.parametrize("V", [1, 2, 4, 8])
def test_softmax_matches_dense_masked_softmax(V):
    rng = gen.make_rng(f"sm_{V}")
    M, N = 8 * 5 + 3, 70
    mask = gen.colvec_mask(rng, M, N, V, 0.3)
    rp, ci, _ = oracle.encode(M, N, V, mask=mask)
    vals = gen.fp16_values(rng, int(rp[-1]) * V) * np.float16(4)
    out = oracle.softmax(M, V, rp, vals, 0.125)
    np.testing.assert_allclose(out, dense_masked_softmax(vals, rp, ci, M, N, V, 0.125),
                               rtol=1e-12, atol=1e-15)


@pytest.mark.parametrize("V", [2, 8])
def test_softmax_invariants(V):
    """Rows sum to 1, a constant row is uniform, a shift of a row changes nothing, padded
    rows are 0."""
    rng = gen.make_rng(f"smi_{V}")
    M, N = 8 * 4 + 5, 50
    mask = gen.colvec_mask(rng, M, N, V, 0.4)
    rp, ci, _ = oracle.encode(M, N, V, mask=mask)
    nnz = int(rp[-1])
    vals = gen.fp16_values(rng, nnz * V)
    out = oracle.softmax(M, V, rp, vals, 1.0).reshape(-1, V)
    for w in range(len(rp) - 1):
        seg = out[rp[w]:rp[w + 1]]
        if seg.shape[0] == 0:
            continue
        for r in range(V):
            if w * V + r < M:
                assert abs(seg[:, r].sum() - 1.0) < 1e-12
            else:
                assert np.all(seg[:, r] == 0)
    const = np.full(nnz * V, np.float16(0.5))
    outc = oracle.softmax(M, V, rp, const, 3.0).reshape(-1, V)
    for w in range(len(rp) - 1):
        n = rp[w + 1] - rp[w]
        for r in range(V):
            if n and w * V + r < M:
                np.testing.assert_allclose(outc[rp[w]:rp[w + 1], r], 1.0 / n, rtol=1e-14)
    # shift invariance on values k/16 (exact in fp16 before and after the shift)
    grid = (rng.integers(-16, 16, nnz * V) / 16.0).astype(np.float16)
    shifted = (grid.astype(np.float64) - 0.5).astype(np.float16)
    assert np.array_equal(shifted.astype(np.float64) + 0.5, grid.astype(np.float64))
    np.testing.assert_allclose(oracle.softmax(M, V, rp, shifted, 1.0),
                               oracle.softmax(M, V, rp, grid, 1.0), rtol=1e-12, atol=1e-15)


@pytest.mark.parametrize("V", [1, 4, 8])
def test_softmax_minus_inf_scores(V):
    """-inf scores (entries masked by the caller): where a row has a finite score the result
    equals the dense masked softmax (exp(-inf) = 0); a row whose stored scores are all -inf
    outputs 0 (reading R23 -- the plain formula is 0/0)."""
    rng = gen.make_rng(f"sminf_{V}")
    M, N = 8 * 6 + 3, 64
    mask = gen.colvec_mask(rng, M, N, V, 0.4)
    rp, ci, _ = oracle.encode(M, N, V, mask=mask)
    nnz = int(rp[-1])
    vals = gen.fp16_values(rng, nnz * V).copy()
    vals[rng.random(nnz * V) < 0.3] = -np.inf
    v2 = vals.reshape(-1, V)
    w_all = 2                                # window 2: every row fully -inf
    v2[rp[w_all]:rp[w_all + 1], :] = -np.inf
    out = oracle.softmax(M, V, rp, vals, 0.5)
    o2 = out.reshape(-1, V)
    assert np.all(o2[rp[w_all]:rp[w_all + 1]] == 0)
    assert np.all(out[np.isneginf(vals.astype(np.float64))] == 0)
    ref = dense_masked_softmax(vals, rp, ci, M, N, V, 0.5)
    finite = ~np.isnan(ref)                  # numpy's 0/0 rows are the R23 rows
    np.testing.assert_allclose(out[finite], ref[finite], rtol=1e-12, atol=1e-15)
    assert np.all(out[~finite] == 0)


def test_attention_mask_density():
    rng = gen.make_rng("amask")
    m = gen.attention_mask(rng, 4096, 8, 0.9)   # band 256 = 6.25% < 10%: random fills the rest
    assert abs(m.mean() - 0.1) < 0.01
    # the diagonal band is dense
    assert m[1000, 1000 - 100:1000 + 100].all()

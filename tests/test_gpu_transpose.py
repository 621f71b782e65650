"""GPU parity of vs_transpose_colvec (the W^T operand of the backward pass, SURVEY §8(f)-2,
P:1625-1638) against oracle.transpose — bit-exact — and of dX = W^T dY through vs_spmm on the
transposed encoding against the fp64 oracle."""
import itertools

import numpy as np
import pytest

import oracle
from synth import gen

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")


@pytest.fixture(scope="module")
def vs():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_sc_chenqldx21_b200 as m
    m.load()
    return m


def host(t):
    return t.cpu().numpy()


def dev(x):
    return torch.from_numpy(np.ascontiguousarray(x)).cuda()


def gpu_transpose(vs, A, V, pattern=False):
    M, K = A.shape
    rp, ci, va = vs.encode(V, dense=dev(A))
    n = int(rp[-1].item())
    rT, cT, vT = vs.transpose(rp, ci[:n], None if pattern else va[:n * V], M, K, V)
    torch.cuda.synchronize()
    return (rT.cpu().numpy(), cT.cpu().numpy(),
            None if vT is None else vT.cpu().numpy())


def check_bitexact(vs, A, V, pattern=False):
    M, K = A.shape
    rT, cT, vT = gpu_transpose(vs, A, V, pattern)
    orp, oci, ova = oracle.encode(M, K, V, dense=A)
    oT, ocT, ovT = oracle.transpose(M, K, V, orp, oci, None if pattern else ova)
    assert np.array_equal(rT, oT), "rowT_ptr"
    assert np.array_equal(cT, ocT), "colT_idx"
    if not pattern:
        assert np.array_equal(vT.view(np.uint16), ovT.view(np.uint16)), "valsT"


@pytest.mark.parametrize("V", [1, 2, 4, 8])
def test_transpose_tiny_sweep_bitexact(vs, V):
    for M, K in itertools.product([1, 3, 8, 9, 17], [1, 2, 7, 16, 19]):
        rng = gen.make_rng(f"gtr_tiny_{V}_{M}_{K}")
        A = gen.colvec_dense(rng, M, K, V, 0.4, inner_zero_frac=0.2, neg_zero_frac=0.05)
        check_bitexact(vs, A, V)


@pytest.mark.parametrize("V", [1, 2, 4, 8])
@pytest.mark.parametrize("M,K,d", [(256, 256, 0.1), (67, 301, 0.3), (2048, 512, 0.02),
                                   (512, 2048, 0.5), (1000, 33, 0.9)])
def test_transpose_multitile_bitexact(vs, V, M, K, d):
    rng = gen.make_rng(f"gtr_mt_{V}_{M}_{K}_{d}")
    check_bitexact(vs, gen.colvec_dense(rng, M, K, V, d, inner_zero_frac=0.1), V)


@pytest.mark.parametrize("V", [2, 4, 8])
def test_transpose_square_blocks(vs, V):
    rng = gen.make_rng(f"gtr_blk_{V}")
    M, K = 64 * V, 48 * V
    A = gen.block_dense(rng, M, K, V, 0.2)
    check_bitexact(vs, A, V)
    rT, _, _ = gpu_transpose(vs, A, V)
    blocks = (A.reshape(M // V, V, K // V, V) != 0).any(axis=(1, 3))
    assert np.array_equal(np.diff(rT), V * blocks.sum(axis=0))


@pytest.mark.parametrize("V", [1, 4, 8])
def test_transpose_pattern_mode(vs, V):
    rng = gen.make_rng(f"gtr_pat_{V}")
    check_bitexact(vs, gen.colvec_dense(rng, 203, 77, V, 0.3), V, pattern=True)


def test_transpose_deterministic_and_empty(vs):
    rng = gen.make_rng("gtr_det")
    A = gen.colvec_dense(rng, 300, 200, 4, 0.3)
    a = gpu_transpose(vs, A, 4)
    b = gpu_transpose(vs, A, 4)
    assert all(np.array_equal(x, y) for x, y in zip(a, b))
    Z = np.zeros((16, 24), np.float16)
    rT, cT, vT = gpu_transpose(vs, Z, 4)
    assert np.array_equal(rT, np.zeros(7, np.int32)) and len(cT) == 0


@pytest.mark.parametrize("V", [1, 2, 4, 8])
@pytest.mark.parametrize("M,K,N", [(256, 256, 64), (300, 257, 200), (512, 1024, 128)])
def test_backward_dx_through_spmm(vs, V, M, K, N):
    # dX = W^T dY: vs_spmm on the transposed encoding vs the fp64 oracle on the oracle's
    # transposed encoding
    rng = gen.make_rng(f"gtr_dx_{V}_{M}_{K}_{N}")
    Wd = gen.colvec_dense(rng, M, K, V, 0.2)
    dY = gen.dense_operand(rng, M, N)
    rp, ci, va = vs.encode(V, dense=dev(Wd))
    n = int(rp[-1].item())
    rT, cT, vT = vs.transpose(rp, ci[:n], va[:n * V], M, K, V)
    dX = vs.spmm(rT, cT, vT, dev(dY), K, V)
    torch.cuda.synchronize()
    orp, oci, ova = oracle.encode(M, K, V, dense=Wd)
    oT, ocT, ovT = oracle.transpose(M, K, V, orp, oci, ova)
    X64, S64 = oracle.spmm(K, M, N, V, oT, ocT, ovT, dY)
    err = np.abs(dX.float().cpu().numpy().astype(np.float64) - X64)
    assert np.all(err <= oracle.tolerance(S64)), f"max err {err.max()}"


@pytest.mark.parametrize("V", [1, 2, 4, 8])
@pytest.mark.parametrize("blocks", [False, True])
def test_transpose_values_refresh(vs, V, blocks):
    # a training step changes W's values, not its pattern: vs_transpose_colvec_values rewrites
    # valsT in place and must equal the oracle transpose of the new values (no new zeros)
    rng = gen.make_rng(f"gtr_vals_{V}_{blocks}")
    M, K = 37 * V + 3, 29 * V + 5
    W1 = (gen.block_dense(rng, M, K, V, 0.3) if blocks else gen.colvec_dense(rng, M, K, V, 0.3))
    W2 = np.where(W1 != 0, gen.dense_operand(rng, M, K), np.float16(0)).astype(np.float16)
    rp, ci, va = vs.encode(V, dense=dev(W1))
    n = int(rp[-1].item())
    rT, cT, vT = vs.transpose(rp, ci[:n], va[:n * V], M, K, V)
    ws = torch.empty(max(vs.vs_transpose_colvec_workspace(M, K, V), 4), dtype=torch.uint8, device="cuda")
    nT = int(rT[-1].item())
    cT2 = torch.empty(max(nT, 1), dtype=torch.int32, device="cuda")
    vT2 = torch.empty(max(nT, 1) * V, dtype=torch.float16, device="cuda")
    vs.vs_transpose_colvec(M, K, V, rp, ci[:n], va[:n * V], rT, cT2, vT2, workspace=ws)
    rp2, ci2, va2 = vs.encode(V, dense=dev(W2))
    assert torch.equal(rp2, rp) and torch.equal(ci2[:n], ci[:n])
    vs.vs_transpose_colvec_values(M, K, V, rp, ci[:n], va2[:n * V], rT, vT2, ws)
    torch.cuda.synchronize()
    orp, oci, ova = oracle.encode(M, K, V, dense=W2)
    oT, ocT, ovT = oracle.transpose(M, K, V, orp, oci, ova)
    assert np.array_equal(rT.cpu().numpy(), oT) and np.array_equal(cT2[:nT].cpu().numpy(), ocT)
    assert np.array_equal(vT2[:nT * V].cpu().numpy().view(np.uint16), ovT.view(np.uint16))


@pytest.mark.parametrize("V", [1, 2, 4, 8])
def test_transpose_pattern_refresh_places_new_nonzeros(vs, V):
    """a pattern built from W's STORED pattern (vals = NULL) gives every stored
    element of W a slot, so values that were +0.0 at build time and are nonzero after the
    update reach W^T.  valsT[q*V + j] = W2[colT[q]][kw*V + j] by definition (the transposed
    element), against the oracle's pattern transpose; dX = W^T dY against the oracle."""
    rng = gen.make_rng(f"gtr_pat_{V}")
    M, K, N = 41 * V + 3, 23 * V + 5, 64
    W1 = gen.colvec_dense(rng, M, K, V, 0.3, inner_zero_frac=0.4)
    rp, ci, va = vs.encode(V, dense=dev(W1))
    n = int(rp[-1].item())
    rT, cT, vT, ws = vs.transpose_pattern(rp, ci[:n], M, K, V)
    # new values on every stored element of W1's pattern, zeros inside vectors included
    orp, oci, ova = oracle.encode(M, K, V, dense=W1)
    ova2 = gen.fp16_values(rng, n * V)
    vs.vs_transpose_colvec_values(M, K, V, rp, ci[:n], dev(ova2), rT, vT, ws)
    torch.cuda.synchronize()
    W2 = oracle.decode(M, K, V, orp, oci, ova2)
    oT, ocT, _ = oracle.transpose(M, K, V, orp, oci, None)
    assert np.array_equal(host(rT), oT) and np.array_equal(host(cT), ocT)
    KT = len(oT) - 1
    exp = np.zeros((len(ocT), V), np.float16)
    for kw in range(KT):
        for q in range(oT[kw], oT[kw + 1]):
            for j in range(V):
                if kw * V + j < K:
                    exp[q, j] = W2[ocT[q], kw * V + j]
    assert np.array_equal(host(vT).reshape(-1, V).view(np.uint16), exp.view(np.uint16))
    dY = gen.dense_operand(rng, M, N)
    dX = host(vs.spmm(rT, cT, vT, dev(dY), K, V))
    o2rp, o2ci, o2va = oracle.encode(M, K, V, dense=W2)
    tT, tcT, tvT = oracle.transpose(M, K, V, o2rp, o2ci, o2va)
    X64, S64 = oracle.spmm(K, M, N, V, tT, tcT, tvT, dY)
    err = np.abs(dX.astype(np.float64) - X64)
    assert np.all(err <= oracle.tolerance(S64)), f"max err {err.max()}"

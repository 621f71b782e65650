"""NEXT item: column-vector softmax and the sparse-attention chain of Eq. 1
(P:1535-1545): S = (Q K^T) o C (vs_sddmm), P = softmax(S / sqrt(k)) (vs_softmax_colvec),
out = P V (vs_spmm), on band + random 8x1 masks.  Each stage is checked
against the oracle on the SAME fp16 input the GPU stage received."""
import math

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


def dev(x):
    return torch.from_numpy(np.ascontiguousarray(x)).cuda()


def host(t):
    return t.cpu().numpy()


@pytest.mark.parametrize("V", [1, 2, 4, 8])
@pytest.mark.parametrize("M,N", [(37, 50), (256, 300), (1000, 1024)])
def test_softmax_parity(vs, V, M, N):
    rng = gen.make_rng(f"gsm_{V}_{M}_{N}")
    mask = gen.colvec_mask(rng, M, N, V, 0.2)
    rp, ci, _ = vs.encode(V, mask=dev(mask))
    nnz = int(rp[-1].item())
    x = gen.fp16_values(rng, nnz * V) * np.float16(8)
    xd = dev(x)
    out = torch.empty_like(xd)
    vs.vs_softmax_colvec(M, V, rp, xd, out, 0.3)
    p64 = oracle.softmax(M, V, host(rp), x, 0.3)
    err = np.abs(host(out).astype(np.float64) - p64)
    assert np.all(err <= oracle.softmax_tolerance(p64)), err.max()
    # in place gives the same bits
    vs.vs_softmax_colvec(M, V, rp, xd, xd, 0.3)
    assert torch.equal(xd.view(torch.int16), out.view(torch.int16))


@pytest.mark.parametrize("V", [1, 2, 4, 8])
def test_softmax_minus_inf_scores(vs, V):
    """-inf scores add nothing; a row whose stored scores are all -inf outputs 0 (R23), no NaN."""
    M, N = 8 * 20 + 5, 200
    rng = gen.make_rng(f"gsminf_{V}")
    mask = gen.colvec_mask(rng, M, N, V, 0.3)
    rp, ci, _ = vs.encode(V, mask=dev(mask))
    rph = host(rp)
    nnz = int(rph[-1])
    x = gen.fp16_values(rng, nnz * V).copy()
    x[rng.random(nnz * V) < 0.4] = -np.inf
    x2 = x.reshape(-1, V)
    x2[rph[3]:rph[4], :] = -np.inf           # window 3 fully masked
    x2[rph[5]:rph[6], 0] = -np.inf           # one row of window 5 fully masked
    xd = dev(x)
    out = torch.empty_like(xd)
    vs.vs_softmax_colvec(M, V, rp, xd, out, 0.7)
    g = host(out).astype(np.float64)
    assert not np.isnan(g).any()
    p64 = oracle.softmax(M, V, rph, x, 0.7)
    assert np.all(np.abs(g - p64) <= oracle.softmax_tolerance(p64))


@pytest.mark.parametrize("V", [8, 4])
def test_sparse_attention_chain(vs, V):
    l, k = 1024, 64
    rng = gen.make_rng(f"attn_{V}")
    mask = gen.attention_mask(rng, l, V, 0.9, band=128)
    Q = gen.dense_operand(rng, l, k)
    Km = gen.dense_operand(rng, l, k)
    Vm = gen.dense_operand(rng, l, k)
    rp, ci, _ = vs.encode(V, mask=dev(mask))
    nnz = int(rp[-1].item())
    scale = 1.0 / math.sqrt(k)
    # stage by stage through the C ABI
    S = vs.sddmm(rp, ci, dev(Q), dev(Km), V, nnz=nnz)
    torch.cuda.synchronize()
    s_h = host(S)
    orp, oci, _ = oracle.encode(l, l, V, mask=mask)
    assert np.array_equal(host(rp), orp) and np.array_equal(host(ci)[:nnz], oci)
    o64, s64 = oracle.sddmm(l, l, k, V, orp, oci, Q, Km)
    assert np.all(np.abs(s_h.astype(np.float64) - o64) <= oracle.tolerance(s64))
    P = torch.empty_like(S)
    vs.vs_softmax_colvec(l, V, rp, S, P, scale)
    p_h = host(P)
    p64 = oracle.softmax(l, V, orp, s_h, scale)
    assert np.all(np.abs(p_h.astype(np.float64) - p64) <= oracle.softmax_tolerance(p64))
    out = vs.spmm(rp, ci, P, dev(Vm), l, V)
    c64, c_s = oracle.spmm(l, l, k, V, orp, oci, p_h, Vm)
    assert np.all(np.abs(host(out).astype(np.float64) - c64) <= oracle.tolerance(c_s))
    # the convenience chain gives the same bits as the staged calls
    out2 = vs.sparse_attention(rp, ci, dev(Q), dev(Km), dev(Vm), V, nnz=nnz)
    assert torch.equal(out2.view(torch.int16), out.view(torch.int16))
    # and agrees with dense masked attention in fp64 within the composed fp16 error
    D = (Q.astype(np.float64) @ Km.astype(np.float64).T) * scale
    D[mask == 0] = -np.inf
    Pd = np.exp(D - D.max(axis=1, keepdims=True))
    Pd /= Pd.sum(axis=1, keepdims=True)
    ref = Pd @ Vm.astype(np.float64)
    assert np.max(np.abs(host(out).astype(np.float64) - ref)) < 2e-2


def test_softmax_batched_matches_single(vs):
    probs, singles = [], []
    for i, (M, N, V) in enumerate([(100, 80, 2), (64, 256, 8), (33, 40, 4), (128, 128, 1)]):
        rng = gen.make_rng(f"smb_{i}")
        rp, ci, _ = vs.encode(V, mask=dev(gen.colvec_mask(rng, M, N, V, 0.3)))
        nnz = int(rp[-1].item())
        x = dev(gen.fp16_values(rng, max(nnz, 1) * V))
        o1, o2 = torch.empty_like(x), torch.empty_like(x)
        vs.vs_softmax_colvec(M, V, rp, x, o1, 0.7)
        probs.append((M, V, 0.7, rp, x, o2))
        singles.append((o1, nnz * V))
    vs.vs_softmax_colvec_batched(probs)
    torch.cuda.synchronize()
    for (o1, n), p in zip(singles, probs):
        assert torch.equal(o1[:n].view(torch.int16), p[5][:n].view(torch.int16))

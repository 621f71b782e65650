"""GPU parity of the dense-tile tcgen05 path (dense_tile.cu): the B200 cost
model (dense_select.cuh) sends 128-row blocks with enough stored vectors to tensor-core dense
tiles with a sampled (SDDMM) epilogue.  Every case is checked against the fp64 oracle
(|gpu - oracle| <= 2e-3*sum|ab| + 2^-24): dense masks (every row block dense), mixed masks
(dense and sparse row blocks in one call -> both kernels), ragged M / N / K tails, K > 256
(streamed A tiles), unaligned outputs, and unsorted windows inside dense row blocks (those
stay with the gather kernel)."""
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


def assert_within(gpu_f16, o64, s64, what=""):
    g = np.asarray(gpu_f16, np.float16).astype(np.float64).reshape(o64.shape)
    err = np.abs(g - o64)
    tol = oracle.tolerance(s64)
    bad = err > tol
    assert not bad.any(), (f"{what}: {bad.sum()} of {bad.size} outside tolerance; "
                           f"max err {err.max():.4g}, worst ratio {(err / tol).max():.3g}")


def mixed_mask(rng, M, N, V, dense_d, sparse_d):
    """Row blocks of 128 rows alternate between density dense_d and sparse_d."""
    mask = np.zeros((M, N), np.uint8)
    for i0 in range(0, M, 128):
        rows = min(128, M - i0)
        d = dense_d if (i0 // 128) % 2 == 0 else sparse_d
        mask[i0:i0 + rows] = gen.colvec_mask(rng, rows, N, V, d)
    return mask


def run_sddmm(vs, mask, A, Bt, V, out_offset=0):
    M, N = mask.shape
    K = A.shape[1]
    rp, ci, _ = vs.encode(V, mask=dev(mask))
    nnz = int(rp[-1].item())
    flat = torch.full((nnz * V + out_offset + 8,), 7.0, dtype=torch.float16, device="cuda")
    out = flat[out_offset:out_offset + nnz * V]
    vs.vs_sddmm(M, N, K, V, rp, ci, dev(A), dev(Bt), out)
    torch.cuda.synchronize()
    orp, oci, _ = oracle.encode(M, N, V, mask=mask)
    o64, s64 = oracle.sddmm(M, N, K, V, orp, oci, A, Bt)
    return host(out), o64, s64


@pytest.mark.parametrize("V", [2, 4, 8])
@pytest.mark.parametrize("M,N,K", [(256, 256, 256), (300, 200, 264), (128, 640, 256), (200, 300, 512),
                                   (130, 129, 1000), (512, 1024, 320), (256, 256, 64)])
def test_sddmm_dense_blocks(vs, V, M, N, K):
    rng = gen.make_rng(f"gdense_sd_{V}_{M}_{N}_{K}")
    mask = gen.colvec_mask(rng, M, N, V, 0.6)
    A = gen.dense_operand(rng, M, K)
    Bt = gen.dense_operand(rng, N, K)
    out, o64, s64 = run_sddmm(vs, mask, A, Bt, V)
    assert_within(out, o64, s64, f"dense sddmm V{V} {M}x{N}x{K}")


@pytest.mark.parametrize("V", [2, 4, 8])
@pytest.mark.parametrize("K", [64, 256, 384, 1000])
def test_sddmm_mixed_blocks(vs, V, K):
    rng = gen.make_rng(f"gdense_mix_{V}_{K}")
    M, N = 640, 900
    mask = mixed_mask(rng, M, N, V, 0.7, 0.01)
    A = gen.dense_operand(rng, M, K)
    Bt = gen.dense_operand(rng, N, K)
    out, o64, s64 = run_sddmm(vs, mask, A, Bt, V)
    assert_within(out, o64, s64, f"mixed sddmm V{V} K{K}")


@pytest.mark.parametrize("V", [2, 8])
def test_sddmm_dense_unaligned_out_and_integer_exact(vs, V):
    """Outputs at an odd element offset (scalar stores) and integer-exact inputs: bitwise."""
    rng = gen.make_rng(f"gdense_int_{V}")
    M, N, K = 200, 300, 256
    mask = gen.colvec_mask(rng, M, N, V, 0.8)
    A = gen.dense_operand(rng, M, K, exact=True)
    Bt = gen.dense_operand(rng, N, K, exact=True)
    out, o64, _ = run_sddmm(vs, mask, A, Bt, V, out_offset=1)
    assert np.array_equal(out.astype(np.float64), o64)


@pytest.mark.parametrize("V", [2, 4, 8])
def test_sddmm_dense_padded_rows_zero(vs, V):
    rng = gen.make_rng(f"gdense_pad_{V}")
    M, N, K = 128 + 5, 256, 256  # last window of the second row block is padded for V > 1
    mask = gen.colvec_mask(rng, M, N, V, 0.9)
    A = gen.dense_operand(rng, M, K)
    Bt = gen.dense_operand(rng, N, K)
    out, o64, s64 = run_sddmm(vs, mask, A, Bt, V)
    assert_within(out, o64, s64, "pad")
    rp, _, _ = oracle.encode(M, N, V, mask=mask)
    if M % V:
        last = out.reshape(-1, V)[rp[-2]:rp[-1], M % V:]
        assert np.all(last.view(np.uint16) == 0)


@pytest.mark.parametrize("V", [2, 4, 8])
@pytest.mark.parametrize("kind", ["perm", "dup"])
def test_sddmm_dense_unsorted_windows(vs, V, kind):
    """Windows whose col_idx is not strictly ascending inside dense row blocks: the dense kernel's
    per-tile search assumes ascending windows, the gather kernel recomputes such windows in full
    after it.  Every output vs the oracle on the same (permuted / duplicated)
    arrays, per vector."""
    rng = gen.make_rng(f"gdense_unsorted_{V}_{kind}")
    M, N, K = 384, 640, 256
    mask = gen.colvec_mask(rng, M, N, V, 0.6)
    A = gen.dense_operand(rng, M, K)
    Bt = gen.dense_operand(rng, N, K)
    rp, ci, _ = oracle.encode(M, N, V, mask=mask)
    ci = ci.copy()
    W = len(rp) - 1
    for w in range(0, W, 3):  # every third window
        b, e = int(rp[w]), int(rp[w + 1])
        if e - b < 2:
            continue
        if kind == "perm":
            ci[b:e] = ci[b:e][rng.permutation(e - b)]
        else:
            ci[b + 1] = ci[b]  # a duplicate column (same output twice)
    nnz = int(rp[-1])
    out = torch.full((nnz * V,), 7.0, dtype=torch.float16, device="cuda")
    vs.vs_sddmm(M, N, K, V, dev(rp), dev(ci), dev(A), dev(Bt), out)
    torch.cuda.synchronize()
    o64, s64 = oracle.sddmm(M, N, K, V, rp, ci, A, Bt)
    assert_within(host(out), o64, s64, f"unsorted {kind} V{V}")


def test_sddmm_dense_batched_equals_single(vs):
    """vs_sddmm_batched == vs_sddmm bit for bit on problems whose row blocks take the dense-tile
    kernel (inner K >= 256), mixed with gather-only problems in the same batch; every output
    also within the oracle's tolerance."""
    rng = gen.make_rng("gdense_batched")
    cases = [(130, 300, 256, 2, 0.5), (300, 640, 320, 4, 0.4), (512, 384, 512, 8, 0.6),
             (256, 200, 256, 1, 0.3), (200, 256, 64, 4, 0.5), (384, 512, 264, 2, 0.02)]
    single, batch, ref = [], [], []
    for (M, N, K, V, dens) in cases:
        mask = gen.colvec_mask(rng, M, N, V, dens)
        A = gen.dense_operand(rng, M, K)
        Bt = gen.dense_operand(rng, N, K)
        rp, ci, _ = oracle.encode(M, N, V, mask=mask)
        nnz = int(rp[-1])
        o1 = torch.full((max(nnz, 1) * V,), 7.0, dtype=torch.float16, device="cuda")
        o2 = torch.full_like(o1, 3.0)
        drp, dci, dA, dBt = dev(rp), dev(ci), dev(A), dev(Bt)
        vs.vs_sddmm(M, N, K, V, drp, dci, dA, dBt, o1)
        single.append((o1, nnz * V))
        batch.append((M, N, K, V, drp, dci, dA, dBt, o2))
        ref.append(oracle.sddmm(M, N, K, V, rp, ci, A, Bt))
    vs.vs_sddmm_batched(batch)
    torch.cuda.synchronize()
    for (o1, n), b, (o64, s64), c in zip(single, batch, ref, cases):
        assert torch.equal(o1[:n].view(torch.int16), b[8][:n].view(torch.int16)), c
        assert_within(host(o1[:n]), o64, s64, f"batched dense {c}")


def test_sddmm_dense_batched_many_problems(vs):
    """More dense-eligible problems than one dense launch takes (32): several dense launches in one
    batched call, then the gather launch; every output vs the oracle, batch == single bitwise."""
    rng = gen.make_rng("gdense_many")
    single, batch, ref = [], [], []
    for i in range(40):
        M, N, K, V = int(rng.integers(64, 300)), int(rng.integers(64, 400)), 256, int(rng.choice([2, 4, 8]))
        mask = gen.colvec_mask(rng, M, N, V, 0.5)
        A = gen.dense_operand(rng, M, K)
        Bt = gen.dense_operand(rng, N, K)
        rp, ci, _ = oracle.encode(M, N, V, mask=mask)
        nnz = int(rp[-1])
        o1 = torch.full((max(nnz, 1) * V,), 7.0, dtype=torch.float16, device="cuda")
        o2 = torch.full_like(o1, 3.0)
        drp, dci, dA, dBt = dev(rp), dev(ci), dev(A), dev(Bt)
        vs.vs_sddmm(M, N, K, V, drp, dci, dA, dBt, o1)
        single.append((o1, nnz * V))
        batch.append((M, N, K, V, drp, dci, dA, dBt, o2))
        ref.append(oracle.sddmm(M, N, K, V, rp, ci, A, Bt))
    vs.vs_sddmm_batched(batch)
    torch.cuda.synchronize()
    for (o1, n), b, (o64, s64) in zip(single, batch, ref):
        assert torch.equal(o1[:n].view(torch.int16), b[8][:n].view(torch.int16))
        assert_within(host(b[8][:n]), o64, s64, "many")


def test_sddmm_dense_deterministic(vs):
    rng = gen.make_rng("gdense_det")
    M, N, K, V = 512, 512, 256, 4
    mask = gen.colvec_mask(rng, M, N, V, 0.5)
    A = gen.dense_operand(rng, M, K)
    Bt = gen.dense_operand(rng, N, K)
    o1, _, _ = run_sddmm(vs, mask, A, Bt, V)
    o2, _, _ = run_sddmm(vs, mask, A, Bt, V)
    assert np.array_equal(o1.view(np.uint16), o2.view(np.uint16))


# ------------------------------------------------------------------------------ SpMM

def run_spmm(vs, A, B, V, rp=None, ci=None, va=None):
    M, K = A.shape
    N = B.shape[1]
    if rp is None:
        orp, oci, ova = oracle.encode(M, K, V, dense=A)
    else:
        orp, oci, ova = rp, ci, va
    C = host(vs.spmm(dev(orp), dev(oci), dev(ova), dev(B), M, V))
    C64, S64 = oracle.spmm(M, K, N, V, orp, oci, ova, B)
    return C, C64, S64


@pytest.mark.parametrize("V", [2, 4, 8])
@pytest.mark.parametrize("M,K,N", [(256, 256, 64), (300, 200, 136), (128, 640, 256), (200, 2048, 128),
                                   (130, 129, 72), (512, 1024, 512)])
def test_spmm_dense_blocks(vs, V, M, K, N):
    rng = gen.make_rng(f"gdense_sp_{V}_{M}_{K}_{N}")
    A = gen.colvec_dense(rng, M, K, V, 0.6)
    B = gen.dense_operand(rng, K, N)
    C, C64, S64 = run_spmm(vs, A, B, V)
    assert_within(C, C64, S64, f"dense spmm V{V} {M}x{K}x{N}")


@pytest.mark.parametrize("V", [2, 4, 8])
@pytest.mark.parametrize("K", [64, 512, 1500])
def test_spmm_mixed_blocks(vs, V, K):
    rng = gen.make_rng(f"gdense_spmix_{V}_{K}")
    M, N = 640, 200
    A = np.zeros((M, K), np.float16)
    for i0 in range(0, M, 128):
        rows = min(128, M - i0)
        A[i0:i0 + rows] = gen.colvec_dense(rng, rows, K, V, 0.7 if (i0 // 128) % 2 == 0 else 0.01)
    B = gen.dense_operand(rng, K, N)
    C, C64, S64 = run_spmm(vs, A, B, V)
    assert_within(C, C64, S64, f"mixed spmm V{V} K{K}")


@pytest.mark.parametrize("V", [2, 8])
def test_spmm_dense_integer_exact_bitwise(vs, V):
    rng = gen.make_rng(f"gdense_spint_{V}")
    M, K, N = 200, 300, 128
    A = gen.colvec_dense(rng, M, K, V, 0.8, exact=True)
    B = gen.dense_operand(rng, K, N, exact=True)
    C, C64, _ = run_spmm(vs, A, B, V)
    assert np.array_equal(C.astype(np.float64), C64.astype(np.float16).astype(np.float64))


@pytest.mark.parametrize("V", [2, 4, 8])
def test_spmm_dense_unsorted_windows_stay_exact(vs, V):
    """Dense row blocks whose windows are shuffled / duplicated: those windows go to the gather
    kernel, the sorted ones to the dense tile; all within the tolerance of the oracle on the
    same arrays (duplicates sum)."""
    rng = gen.make_rng(f"gdense_spunsorted_{V}")
    M, K, N = 384, 512, 136
    A = gen.colvec_dense(rng, M, K, V, 0.7)
    B = gen.dense_operand(rng, K, N)
    rp, ci, va = oracle.encode(M, K, V, dense=A)
    ci = ci.copy()
    va2 = va.reshape(-1, V).copy()
    W = len(rp) - 1
    for w in range(0, W, 3):                      # every third window shuffled
        lo, hi = rp[w], rp[w + 1]
        perm = rng.permutation(hi - lo)
        ci[lo:hi] = ci[lo:hi][perm]
        va2[lo:hi] = va2[lo:hi][perm]
    for w in range(1, W, 7):                      # some windows with a duplicated column
        lo, hi = rp[w], rp[w + 1]
        if hi - lo >= 2:
            ci[lo + 1] = ci[lo]
    C, C64, S64 = run_spmm(vs, A, B, V, rp, ci, va2.reshape(-1))
    assert_within(C, C64, S64, f"unsorted dense spmm V{V}")


def test_spmm_dense_scatter(vs):
    from paper_conf_sc_chenqldx21_b200 import dist as vsd
    V, M, K, N = 4, 256, 512, 512
    rng = gen.make_rng("gdense_spscat")
    A = gen.colvec_dense(rng, M, K, V, 0.6)
    B = dev(gen.dense_operand(rng, K, N))
    rp, ci, va = vs.encode(V, dense=dev(A))
    full = vs.spmm(rp, ci, va, B, M, V)
    reps = [torch.full((M, N), -1.0, dtype=torch.float16, device="cuda") for _ in range(2)]
    b = vsd.panel_bounds(N, 2)
    for r in range(2):
        Bp = B[:, b[r]:b[r + 1]].contiguous()
        vs.vs_spmm_scatter(M, K, b[r + 1] - b[r], V, rp, ci, va, Bp,
                           vsd.scatter_dst_ptrs([x.data_ptr() for x in reps], b[r]), N)
    torch.cuda.synchronize()
    for rep in reps:
        assert torch.equal(rep.view(torch.int16), full.view(torch.int16))

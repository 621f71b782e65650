"""GPU parity: the CUDA path (through the C ABI) against the fp64 oracle on the same seeded
inputs.  Encoder outputs bit-exact; SpMM / SDDMM within |gpu - oracle| <= 2e-3*S + 2^-24
(S = sum |a*b|, the north star's bound with fp32 accumulation);
integer-exact and identity inputs bitwise."""
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


@pytest.fixture(params=["shipped"])
def sddmm_path(request):
    """The SDDMM kernel of the loaded library.  (The tcgen05 SDDMM of round 1 is an opt-in
    build, -DVS_WITH_SDDMM_TC=1; the shipped libvs.so has one SDDMM path.  Running this file
    with VS_LIB_PATH pointing at such a build checks it with the same suite.)"""
    return request.param


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


def gpu_encode(vs, V, dense=None, mask=None, capacity=None):
    rp, ci, va = vs.encode(V, dense=None if dense is None else dev(dense),
                           mask=None if mask is None else dev(mask), capacity=capacity)
    torch.cuda.synchronize()
    n = int(rp[-1].item())
    return host(rp), host(ci)[:n], (None if va is None else host(va)[:n * V])


# ------------------------------------------------------------------------- encoder

ENC_SHAPES = [(1, 1), (3, 5), (8, 8), (13, 17), (64, 256), (67, 300), (200, 1000), (31, 8)]


@pytest.mark.parametrize("V", [1, 2, 4, 8])
@pytest.mark.parametrize("M,K", ENC_SHAPES)
def test_encode_dense_bitexact(vs, V, M, K):
    rng = gen.make_rng(f"genc_{V}_{M}_{K}")
    X = gen.colvec_dense(rng, M, K, V, 0.3, inner_zero_frac=0.2, neg_zero_frac=0.03)
    orp, oci, ova = oracle.encode(M, K, V, dense=X)
    rp, ci, va = gpu_encode(vs, V, dense=X)
    assert np.array_equal(rp, orp)
    assert np.array_equal(ci, oci)
    assert np.array_equal(va.view(np.uint16), ova.view(np.uint16))


@pytest.mark.parametrize("V", [1, 2, 4, 8])
@pytest.mark.parametrize("M,K", [(5, 7), (64, 256), (67, 301), (256, 64)])
def test_encode_mask_and_capacity_modes(vs, V, M, K):
    rng = gen.make_rng(f"gencm_{V}_{M}_{K}")
    X = gen.colvec_dense(rng, M, K, V, 0.25)
    mask = gen.colvec_mask(rng, M, K, V, 0.2)
    # mask only
    orp, oci, _ = oracle.encode(M, K, V, mask=mask)
    rp, ci, va = gpu_encode(vs, V, mask=mask)
    assert va is None and np.array_equal(rp, orp) and np.array_equal(ci, oci)
    # mask decides, vals copied from dense
    orp, oci, ova = oracle.encode(M, K, V, dense=X, mask=mask)
    W = -(-M // V)
    rp, ci, va = gpu_encode(vs, V, dense=X, mask=mask, capacity=W * K)
    assert np.array_equal(rp, orp) and np.array_equal(ci, oci)
    assert np.array_equal(va.view(np.uint16), ova.view(np.uint16))


def test_encode_fig8_example(vs):
    X = np.zeros((6, 7), np.float16)
    X[1, 0], X[0, 2], X[1, 2], X[0, 6], X[1, 6] = 1, 2, 3, 4, 5
    X[2, 3], X[3, 3], X[4, 1], X[5, 1], X[4, 6], X[5, 6] = 6, 7, 8, 9, 10, 11
    rp, ci, va = gpu_encode(vs, 2, dense=X)
    assert rp.tolist() == [0, 3, 4, 6]
    assert ci.tolist() == [0, 2, 6, 3, 1, 6]
    assert va.astype(np.float32).tolist() == list(range(12))


def test_encode_unaligned_dense(vs):
    """A dense pointer that is not 16-byte aligned takes the scalar path; same result."""
    rng = gen.make_rng("genc_unal")
    M, K, V = 40, 64, 4
    X = gen.colvec_dense(rng, M, K, V, 0.3)
    flat = torch.zeros(M * K + 1, dtype=torch.float16, device="cuda")
    flat[1:] = dev(X).reshape(-1)
    Xd = flat[1:].view(M, K)
    rp, ci, va = vs.encode(V, dense=Xd)
    orp, oci, ova = oracle.encode(M, K, V, dense=X)
    assert np.array_equal(host(rp), orp) and np.array_equal(host(ci), oci)
    assert np.array_equal(host(va).view(np.uint16), ova.view(np.uint16))


# ---------------------------------------------------------------------------- SpMM

def run_spmm(vs, A, B, V):
    M, K = A.shape
    N = B.shape[1]
    rp, ci, va = vs.encode(V, dense=dev(A))
    C = vs.spmm(rp, ci, va, dev(B), M, V)
    torch.cuda.synchronize()
    orp, oci, ova = oracle.encode(M, K, V, dense=A)
    C64, S64 = oracle.spmm(M, K, N, V, orp, oci, ova, B)
    return host(C), C64, S64


@pytest.mark.parametrize("V", [1, 2, 4, 8])
@pytest.mark.parametrize("density", [0.0, 0.3, 1.0])
def test_spmm_tiny_sweep(vs, V, density):
    for M, K, N in itertools.product([1, 3, 8, 9, 16], [1, 5, 16], [1, 7, 8, 16, 24]):
        rng = gen.make_rng(f"gspmm_{V}_{density}_{M}_{K}_{N}")
        A = gen.colvec_dense(rng, M, K, V, density)
        B = gen.dense_operand(rng, K, N)
        C, C64, S64 = run_spmm(vs, A, B, V)
        assert_within(C, C64, S64, f"spmm M{M} K{K} N{N} V{V} d{density}")


@pytest.mark.parametrize("V", [1, 2, 4, 8])
@pytest.mark.parametrize("M,K,N", [(256, 256, 64), (300, 257, 200), (129, 1000, 136),
                                   (64, 64, 130), (512, 512, 256), (100, 300, 1000),
                                   (64, 2100, 72), (33, 4200, 64)])  # SPLIT = 8, 16
@pytest.mark.parametrize("density", [0.1, 0.5])
def test_spmm_multitile(vs, V, M, K, N, density):
    rng = gen.make_rng(f"gspmm_mt_{V}_{M}_{K}_{N}_{density}")
    A = gen.colvec_dense(rng, M, K, V, density)
    B = gen.dense_operand(rng, K, N)
    C, C64, S64 = run_spmm(vs, A, B, V)
    assert_within(C, C64, S64, f"spmm {M}x{K}x{N} V{V}")


@pytest.mark.parametrize("V", [1, 2, 4, 8])
@pytest.mark.parametrize("N", [24, 64, 128, 200, 13])
def test_spmm_integer_exact_bitwise(vs, V, N):
    rng = gen.make_rng(f"gspmm_int_{V}_{N}")
    M, K = 77, 200  # |sum| <= 4*200 < 2048: exact in fp32 and in the fp16 output
    A = gen.colvec_dense(rng, M, K, V, 0.5, exact=True)
    B = gen.dense_operand(rng, K, N, exact=True)
    C, C64, _ = run_spmm(vs, A, B, V)
    assert np.array_equal(C.astype(np.float64), C64)


@pytest.mark.parametrize("V", [1, 4, 8])
def test_spmm_identity_B_bitwise(vs, V):
    rng = gen.make_rng(f"gspmm_eye_{V}")
    M, K = 70, 96
    A = gen.colvec_dense(rng, M, K, V, 0.3)
    C, _, _ = run_spmm(vs, A, np.eye(K, dtype=np.float16), V)
    assert np.array_equal(C.astype(np.float64), A.astype(np.float64))


def test_spmm_unaligned_B_and_C(vs):
    rng = gen.make_rng("gspmm_unal")
    M, K, N, V = 64, 80, 64, 8
    A = gen.colvec_dense(rng, M, K, V, 0.3)
    B = gen.dense_operand(rng, K, N)
    rp, ci, va = vs.encode(V, dense=dev(A))
    fb = torch.zeros(K * N + 1, dtype=torch.float16, device="cuda")
    fb[1:] = dev(B).reshape(-1)
    fc = torch.empty(M * N + 1, dtype=torch.float16, device="cuda")
    vs.vs_spmm(M, K, N, V, rp, ci, va, fb[1:], fc[1:])
    C_unal = host(fc[1:]).reshape(M, N)
    C = host(vs.spmm(rp, ci, va, dev(B), M, V))
    assert np.array_equal(C_unal.view(np.uint16), C.view(np.uint16))


def test_spmm_skewed_rows_and_determinism(vs):
    """One full window, many empty ones, and two runs bitwise equal (no atomics)."""
    rng = gen.make_rng("gspmm_skew")
    M, K, N, V = 256, 2048, 128, 8
    A = np.zeros((M, K), np.float16)
    A[8:16] = gen.fp16_values(rng, (8, K))                      # window 1 full
    A[100:104, ::7] = gen.fp16_values(rng, (4, len(range(0, K, 7))))
    B = gen.dense_operand(rng, K, N)
    C, C64, S64 = run_spmm(vs, A, B, V)
    assert_within(C, C64, S64, "skewed")
    C2, _, _ = run_spmm(vs, A, B, V)
    assert np.array_equal(C.view(np.uint16), C2.view(np.uint16))


def test_spmm_degenerate(vs):
    B = dev(gen.dense_operand(gen.make_rng("d"), 16, 8))
    A0 = torch.zeros((12, 16), dtype=torch.float16, device="cuda")
    rp, ci, va = vs.encode(4, dense=A0)
    C = torch.full((12, 8), 7.0, dtype=torch.float16, device="cuda")
    vs.vs_spmm(12, 16, 8, 4, rp, ci, va, B, C)          # nnz_v == 0 -> zeros
    assert torch.count_nonzero(C).item() == 0
    C.fill_(7.0)
    vs.vs_spmm(12, 0, 8, 4, rp, ci, va, None, C)       # K == 0 -> zeros
    assert torch.count_nonzero(C).item() == 0
    vs.vs_spmm(0, 16, 8, 4, rp, ci, va, B, C)          # M == 0 -> no-op


# --------------------------------------------------------------------------- SDDMM

def run_sddmm(vs, mask, A, Bt, V):
    M, N = mask.shape
    K = A.shape[1]
    rp, ci, _ = vs.encode(V, mask=dev(mask))
    out = vs.sddmm(rp, ci, dev(A), dev(Bt), V)
    torch.cuda.synchronize()
    orp, oci, _ = oracle.encode(M, N, V, mask=mask)
    o64, s64 = oracle.sddmm(M, N, K, V, orp, oci, A, Bt)
    return host(out), o64, s64


@pytest.mark.parametrize("V", [1, 2, 4, 8])
@pytest.mark.parametrize("density", [0.0, 0.3, 1.0])
def test_sddmm_tiny_sweep(vs, sddmm_path, V, density):
    for M, N, K in itertools.product([1, 3, 8, 9, 16], [1, 5, 16, 17], [1, 8, 16, 24, 72]):
        rng = gen.make_rng(f"gsddmm_{V}_{density}_{M}_{N}_{K}")
        mask = gen.colvec_mask(rng, M, N, V, density)
        A = gen.dense_operand(rng, M, K)
        Bt = gen.dense_operand(rng, N, K)
        out, o64, s64 = run_sddmm(vs, mask, A, Bt, V)
        assert_within(out, o64, s64, f"sddmm M{M} N{N} K{K} V{V} d{density}")


@pytest.mark.parametrize("V", [1, 2, 4, 8])
@pytest.mark.parametrize("M,N,K", [(256, 64, 256), (300, 257, 200), (129, 1000, 64),
                                   (64, 64, 1000), (512, 512, 128), (100, 300, 13)])
@pytest.mark.parametrize("density", [0.1, 0.5])
def test_sddmm_multitile(vs, sddmm_path, V, M, N, K, density):
    rng = gen.make_rng(f"gsddmm_mt_{V}_{M}_{N}_{K}_{density}")
    mask = gen.colvec_mask(rng, M, N, V, density)
    A = gen.dense_operand(rng, M, K)
    Bt = gen.dense_operand(rng, N, K)
    out, o64, s64 = run_sddmm(vs, mask, A, Bt, V)
    assert_within(out, o64, s64, f"sddmm {M}x{N}x{K} V{V}")


@pytest.mark.parametrize("V", [1, 2, 4, 8])
@pytest.mark.parametrize("K", [64, 200, 384])
def test_sddmm_integer_exact_bitwise(vs, sddmm_path, V, K):
    rng = gen.make_rng(f"gsddmm_int_{V}_{K}")
    M, N = 61, 90
    mask = gen.colvec_mask(rng, M, N, V, 0.4)
    A = gen.dense_operand(rng, M, K, exact=True)
    Bt = gen.dense_operand(rng, N, K, exact=True)
    out, o64, _ = run_sddmm(vs, mask, A, Bt, V)
    assert np.array_equal(out.astype(np.float64), o64)


@pytest.mark.parametrize("V", [1, 2, 4, 8])
def test_sddmm_all_ones_mask_equals_gemm(vs, sddmm_path, V):
    rng = gen.make_rng(f"gsddmm_ones_{V}")
    M, N, K = 64, 96, 128
    mask = np.ones((M, N), np.uint8)
    A = gen.dense_operand(rng, M, K)
    Bt = gen.dense_operand(rng, N, K)
    out, o64, s64 = run_sddmm(vs, mask, A, Bt, V)
    assert_within(out, o64, s64, "ones")
    Gd = o64.reshape(M // V, N, V).transpose(0, 2, 1).reshape(M, N)
    np.testing.assert_allclose(Gd, A.astype(np.float64) @ Bt.astype(np.float64).T, rtol=1e-12, atol=1e-12)


@pytest.mark.parametrize("V", [1, 4, 8])
def test_sddmm_identity_A_bitwise(vs, sddmm_path, V):
    rng = gen.make_rng(f"gsddmm_eye_{V}")
    M = K = 64
    N = 77
    mask = gen.colvec_mask(rng, M, N, V, 0.4)
    Bt = gen.dense_operand(rng, N, K)
    out, o64, _ = run_sddmm(vs, mask, np.eye(M, dtype=np.float16), Bt, V)
    assert np.array_equal(out.astype(np.float64), o64)


def test_sddmm_degenerate(vs, sddmm_path):
    mask = np.zeros((16, 10), np.uint8)
    rp, ci, _ = vs.encode(4, mask=dev(mask))
    vs.vs_sddmm(16, 10, 32, 4, rp, ci, dev(np.zeros((16, 32), np.float16)),
                dev(np.zeros((10, 32), np.float16)), None)  # nnz_v == 0
    mask[3, 4] = 1
    rp, ci, _ = vs.encode(4, mask=dev(mask))
    out = torch.full((4,), 3.0, dtype=torch.float16, device="cuda")
    vs.vs_sddmm(16, 10, 0, 4, rp, ci, None, None, out)  # K == 0 -> zeros
    torch.cuda.synchronize()
    assert torch.count_nonzero(out).item() == 0


def test_sddmm_padded_rows_are_zero(vs, sddmm_path):
    rng = gen.make_rng("gsddmm_pad")
    M, N, K, V = 13, 40, 64, 8   # last window has 5 padded rows
    mask = gen.colvec_mask(rng, M, N, V, 0.5)
    A = gen.dense_operand(rng, M, K)
    Bt = gen.dense_operand(rng, N, K)
    out, o64, s64 = run_sddmm(vs, mask, A, Bt, V)
    assert_within(out, o64, s64, "pad")
    rp, _, _ = oracle.encode(M, N, V, mask=mask)
    last = out.reshape(-1, V)[rp[-2]:rp[-1], M % V:]
    assert np.all(last.view(np.uint16) == 0)


# ----------------------------------------------------- SpMM <-> SDDMM adjoint on GPU

@pytest.mark.parametrize("V", [2, 4, 8])
def test_adjoint_identity_gpu(vs, V):
    """<SpMM(W,X), G> = <vals_W, SDDMM(pattern W; G, X)>, both kernels."""
    rng = gen.make_rng(f"gadj_{V}")
    M, K, N = 512, 512, 256
    Wd = gen.colvec_dense(rng, M, K, V, 0.3)
    X = gen.dense_operand(rng, K, N)
    G = gen.dense_operand(rng, M, N)
    rp, ci, va = vs.encode(V, dense=dev(Wd))
    Y = vs.spmm(rp, ci, va, dev(X), M, V).double()
    dW = vs.sddmm(rp, ci, dev(G), dev(X), V).double()
    lhs = float((Y * dev(G).double()).sum())
    rhs = float((va.double() * dW).sum())
    scale = float((dev(np.abs(Wd.astype(np.float64))) @ dev(np.abs(X.astype(np.float64)))
                   * dev(np.abs(G.astype(np.float64)))).sum())
    assert abs(lhs - rhs) <= 2e-3 * scale


# ------------------------------------------------ sharding invariants with the kernels

@pytest.mark.parametrize("V", [2, 8])
def test_sharded_equals_unsharded_spmm(vs, V):
    """N-panel shards (dist.panel_bounds) computed separately == the full SpMM, bitwise."""
    from paper_conf_sc_chenqldx21_b200 import dist as vsd
    rng = gen.make_rng(f"gshard_spmm_{V}")
    M, K, N = 512, 1024, 1000
    A = gen.colvec_dense(rng, M, K, V, 0.1)
    B = dev(gen.dense_operand(rng, K, N))
    rp, ci, va = vs.encode(V, dense=dev(A))
    full = vs.spmm(rp, ci, va, B, M, V)
    for P in (2, 3, 8):
        b = vsd.panel_bounds(N, P)
        parts = [vs.spmm(rp, ci, va, B[:, b[i]:b[i + 1]].contiguous(), M, V) for i in range(P)]
        assert torch.equal(torch.cat(parts, dim=1).view(torch.int16), full.view(torch.int16))


@pytest.mark.parametrize("V", [2, 8])
def test_sharded_equals_unsharded_sddmm(vs, V):
    """Row-window shards (dist.window_bounds) computed separately == the full SDDMM, bitwise."""
    from paper_conf_sc_chenqldx21_b200 import dist as vsd
    rng = gen.make_rng(f"gshard_sddmm_{V}")
    M, N, K = 600, 700, 256
    mask = gen.colvec_mask(rng, M, N, V, 0.1)
    A = dev(gen.dense_operand(rng, M, K))
    Bt = dev(gen.dense_operand(rng, N, K))
    rp, ci, _ = vs.encode(V, mask=dev(mask))
    full = vs.sddmm(rp, ci, A, Bt, V)
    rph = host(rp)
    for P in (2, 3, 8):
        # shards start on 128-row blocks (the unit of the gather / dense-tile choice)
        wb = vsd.window_bounds(rph, P, align=128 // V)
        segs = []
        for r in range(P):
            sh = vsd.sddmm_shard(rph, M, V, wb, r)
            segs.append(vs.sddmm(dev(sh.row_ptr), ci[sh.p0:sh.p1].contiguous(),
                                 A[sh.row0:sh.row1].contiguous(), Bt, V, nnz=sh.p1 - sh.p0))
        assert torch.equal(torch.cat(segs).view(torch.int16), full.view(torch.int16))


# ------------------------------------------------- full-size (C5) sampled parity

def test_c5_spmm_sampled(vs):
    """C5 SpMM at full size (M=K=16384, N=65536, V=8, S=0.9), the launch the sharded bench
    runs per panel; 4096 sampled outputs against the oracle, plus the adjoint check."""
    M = K = 16384
    N, V, S = 65536, 8, 0.9
    A = gen.torch_colvec_dense(M, K, V, 1 - S, seed=501)
    B = gen.torch_dense_operand(K, N, seed=502)
    rp, ci, va = vs.encode(V, dense=A)
    C = vs.spmm(rp, ci, va, B, M, V)
    torch.cuda.synchronize()
    nnz = int(rp[-1].item())
    assert abs(nnz - (M // V) * K * (1 - S)) < 0.01 * nnz
    rng = np.random.default_rng(7)
    rows = rng.integers(0, M, 4096)
    cols = rng.integers(0, N, 4096)
    o, s = oracle.spmm_sample(M, K, N, V, host(rp), host(ci)[:nnz], host(va)[:nnz * V],
                              host(B), rows, cols)
    g = host(C[torch.from_numpy(rows).cuda(), torch.from_numpy(cols).cuda()])
    assert_within(g, o, s, "C5 spmm sample")
    # oracle-free encode check on a slice: GPU encode of the first 64 rows vs oracle encode
    orp, oci, ova = oracle.encode(64, K, V, dense=host(A[:64]))
    assert np.array_equal(host(rp[:9]), orp)
    assert np.array_equal(host(ci[:orp[-1]]), oci)


def test_c5_sddmm_sampled(vs):
    """C5 SDDMM (mask 16384 x 65536, inner K=16384, V=8, S=0.9): 512 sampled vectors."""
    M, N, K, V, S = 16384, 65536, 16384, 8, 0.9
    g = torch.Generator(device="cuda")
    g.manual_seed(503)
    keep = (torch.rand((M // V, N), generator=g, device="cuda") < (1 - S))
    mask = keep.repeat_interleave(V, dim=0).to(torch.uint8)
    del keep
    rp, ci, _ = vs.encode(V, mask=mask)
    del mask
    A = gen.torch_dense_operand(M, K, seed=504)
    Bt = gen.torch_dense_operand(N, K, seed=505)
    nnz = int(rp[-1].item())
    out = vs.sddmm(rp, ci, A, Bt, V, nnz=nnz)
    torch.cuda.synchronize()
    ps = np.random.default_rng(8).integers(0, nnz, 512)
    o, s = oracle.sddmm_sample(M, N, K, V, host(rp), host(ci)[:nnz], host(A), host(Bt), ps)
    gv = host(out.view(-1, V)[torch.from_numpy(ps).cuda()])
    assert_within(gv, o, s, "C5 sddmm sample")

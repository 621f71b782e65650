"""Batched entry points (vs_*_batched) against the single calls: bitwise identical results
for a heterogeneous mix of problems (every V, ragged and aligned shapes, the scalar tail
path, empty patterns, K == 0 and M == 0 entries) — the single calls are themselves checked
against the oracle in test_gpu_parity.py; here one mixed batch is also checked against it."""
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


def problem_mix():
    rng = np.random.default_rng(11)
    out = []
    for i in range(40):
        V = int(rng.choice([1, 2, 4, 8]))
        M = int(rng.integers(1, 300))
        K = int(rng.choice([7, 64, 100, 256, 512, 1024, 2100]))
        N = int(rng.choice([1, 13, 64, 96, 128, 256, 300]))
        d = float(rng.choice([0.0, 0.02, 0.1, 0.5]))
        out.append((M, K, N, V, d))
    out += [(0, 64, 64, 4, 0.3), (16, 0, 32, 2, 0.3), (40, 64, 0, 8, 0.3)]
    return out


def make(p, i):
    M, K, N, V, d = p
    rng = gen.make_rng(f"batch_{i}")
    A = gen.colvec_dense(rng, M, K, V, d) if M * K else np.zeros((M, K), np.float16)
    B = gen.dense_operand(rng, K, N) if K * N else np.zeros((K, N), np.float16)
    G = gen.dense_operand(rng, M, N) if M * N else np.zeros((M, N), np.float16)
    return A, B, G


def test_batched_matches_single_calls(vs):
    """Batched == single calls bit for bit (encode, SpMM, SDDMM)."""
    probs = problem_mix()
    data = [make(p, i) for i, p in enumerate(probs)]
    enc_single, enc_batch, sp_b, sd_b = [], [], [], []
    for (M, K, N, V, _), (A, B, G) in zip(probs, data):
        W = -(-M // V) if M else 0
        cap = max(W * K, 1)
        Ad = dev(A)
        rp1, ci1, va1 = (torch.zeros(W + 1, dtype=torch.int32, device="cuda"),
                         torch.zeros(cap, dtype=torch.int32, device="cuda"),
                         torch.zeros(cap * V, dtype=torch.float16, device="cuda"))
        rp2, ci2, va2 = rp1.clone(), ci1.clone(), va1.clone()
        vs.vs_encode_colvec(M, K, V, Ad, None, rp1, ci1, va1)
        enc_single.append((rp1, ci1, va1))
        enc_batch.append((M, K, V, Ad, None, rp2, ci2, va2))
    vs.vs_encode_colvec_batched(enc_batch)
    torch.cuda.synchronize()
    for (rp1, ci1, va1), e in zip(enc_single, enc_batch):
        rp2, ci2, va2 = e[5], e[6], e[7]
        n = int(rp1[-1].item())
        assert torch.equal(rp1, rp2)
        assert torch.equal(ci1[:n], ci2[:n])
        assert torch.equal(va1[:n * e[2]].view(torch.int16), va2[:n * e[2]].view(torch.int16))

    singles_c, singles_o, spmm_list, sddmm_list = [], [], [], []
    for (M, K, N, V, _), (A, B, G), (rp, ci, va) in zip(probs, data, enc_single):
        Bd, Gd = dev(B), dev(G)
        # unaligned B / C for every 5th problem (scalar tail path)
        C1 = torch.zeros((M, N), dtype=torch.float16, device="cuda")
        C2 = torch.full((M * N + 1,), 7.0, dtype=torch.float16, device="cuda")[1:].view(M, N) \
            if len(spmm_list) % 5 == 0 and M * N else torch.full((M, N), 7.0, dtype=torch.float16, device="cuda")
        vs.vs_spmm(M, K, N, V, rp, ci, va, Bd, C1)
        spmm_list.append((M, K, N, V, rp, ci, va, Bd, C2))
        singles_c.append(C1)
        n = int(rp[-1].item()) if M else 0
        o1 = torch.zeros(max(n, 1) * V, dtype=torch.float16, device="cuda")
        o2 = torch.full_like(o1, 3.0)
        # SDDMM at the same pattern, inner dimension N (A = G [M x N], Bt = B [K x N])
        vs.vs_sddmm(M, K, N, V, rp, ci, Gd, Bd, o1)
        sddmm_list.append((M, K, N, V, rp, ci, Gd, Bd, o2))
        singles_o.append((o1, n * V))
    vs.vs_spmm_batched(spmm_list)
    vs.vs_sddmm_batched(sddmm_list)
    torch.cuda.synchronize()
    for C1, p in zip(singles_c, spmm_list):
        assert torch.equal(C1.view(torch.int16), p[8].view(torch.int16))
    for (o1, n), p in zip(singles_o, sddmm_list):
        assert torch.equal(o1[:n].view(torch.int16), p[8][:n].view(torch.int16))

    # and one batch entry against the oracle directly
    j = 3
    M, K, N, V, _ = probs[j]
    A, B, G = data[j]
    orp, oci, ova = oracle.encode(M, K, V, dense=A)
    C64, S64 = oracle.spmm(M, K, N, V, orp, oci, ova, B)
    err = np.abs(spmm_list[j][8].float().cpu().numpy().astype(np.float64) - C64)
    assert np.all(err <= oracle.tolerance(S64))


def test_batched_rejects_bad_entry_before_launch(vs):
    x = torch.zeros(8, dtype=torch.int32, device="cuda")
    with pytest.raises(vs.VSError):
        vs.vs_spmm_batched([(8, 8, 8, 3, x, x, None, None, None)])


def test_batched_spmm_stream_order_across_configs(vs):
    """One batched SpMM call spanning six kernel configurations (V, panel width, SPLIT):
    the launches after the first use programmatic dependent launch (DESIGN 7.2), so a copy
    enqueued right after the call on the same stream — no synchronisation in between — must
    still see every problem's final C, equal bit for bit to the single calls."""
    probs = []
    for i, (K, N) in enumerate([(4096, 256), (1024, 256), (256, 256), (4096, 64), (1024, 64), (256, 64)]):
        M, V = 2048 - 8 * i, 4
        rng = gen.make_rng(f"pdl_{i}")
        probs.append((M, K, N, V, gen.colvec_dense(rng, M, K, V, 0.3), gen.dense_operand(rng, K, N)))
    singles, batch = [], []
    for M, K, N, V, A, B in probs:
        rp, ci, va = vs.encode(V, dense=dev(A))
        Bd = dev(B)
        C1 = torch.empty((M, N), dtype=torch.float16, device="cuda")
        vs.vs_spmm(M, K, N, V, rp, ci, va, Bd, C1)
        singles.append(C1)
        batch.append((M, K, N, V, rp, ci, va, Bd, torch.full((M, N), 5.0, dtype=torch.float16, device="cuda")))
    torch.cuda.synchronize()
    for _ in range(3):
        for p in batch:
            p[8].fill_(5.0)
        vs.vs_spmm_batched(batch)
        snap = torch.cat([p[8].flatten() for p in batch])  # same stream, no sync
        torch.cuda.synchronize()
        assert torch.equal(snap.view(torch.int16), torch.cat([c.flatten() for c in singles]).view(torch.int16))

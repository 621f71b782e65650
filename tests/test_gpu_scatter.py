"""the fused replicated-output SpMM epilogue (vs_spmm_scatter).

Every destination must receive exactly vs_spmm's bits in its column window and nothing
elsewhere (the invariant of §8(c) "sharded == unsharded bitwise": the N-panel of rank r,
scattered into every replica, reassembles the full C).  On one GPU the destinations are
distinct local buffers standing in for the peers' symmetric-memory buffers; the last test
runs the real symmetric-memory path (rendezvous, peer pointers, stream barrier) on a
one-rank NCCL group."""
import os
import socket

import numpy as np
import pytest

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


@pytest.mark.parametrize("V", [1, 2, 4, 8])
@pytest.mark.parametrize("M,K,N,P", [(256, 512, 1024, 4), (300, 257, 200, 3), (64, 2100, 520, 2),
                                     (129, 1000, 64, 1)])
def test_scatter_panels_reassemble_unsharded(vs, V, M, K, N, P):
    from paper_conf_sc_chenqldx21_b200 import dist as vsd
    rng = gen.make_rng(f"gscat_{V}_{M}_{K}_{N}_{P}")
    A = gen.colvec_dense(rng, M, K, V, 0.2)
    B = dev(gen.dense_operand(rng, K, N))
    rp, ci, va = vs.encode(V, dense=dev(A))
    full = vs.spmm(rp, ci, va, B, M, V)
    reps = [torch.full((M, N), -7.0, dtype=torch.float16, device="cuda") for _ in range(3)]
    ptrs = [r.data_ptr() for r in reps]
    b = vsd.panel_bounds(N, P)
    for r in range(P):
        Bp = B[:, b[r]:b[r + 1]].contiguous()
        vs.vs_spmm_scatter(M, K, b[r + 1] - b[r], V, rp, ci, va, Bp,
                           vsd.scatter_dst_ptrs(ptrs, b[r]), N)
    torch.cuda.synchronize()
    for rep in reps:
        assert torch.equal(rep.view(torch.int16), full.view(torch.int16))


@pytest.mark.parametrize("ldc_pad", [0, 3, 8])
def test_scatter_leaves_other_columns(vs, ldc_pad):
    """Columns outside [n0, n0 + N) and the ldc padding are not written; unaligned
    destinations (ldc_pad = 3) take the guarded path with the same bits."""
    V, M, K, N = 4, 96, 300, 136
    rng = gen.make_rng(f"gscat_cols_{ldc_pad}")
    A = gen.colvec_dense(rng, M, K, V, 0.3)
    B = dev(gen.dense_operand(rng, K, N))
    rp, ci, va = vs.encode(V, dense=dev(A))
    full = vs.spmm(rp, ci, va, B, M, V)
    ldc = 64 + N + 64 + ldc_pad
    dst = torch.full((M, ldc), 3.0, dtype=torch.float16, device="cuda")
    vs.vs_spmm_scatter(M, K, N, V, rp, ci, va, B, [dst.data_ptr() + 2 * 64], ldc)
    torch.cuda.synchronize()
    assert torch.equal(dst[:, 64:64 + N].view(torch.int16), full.view(torch.int16))
    assert torch.all(dst[:, :64] == 3.0) and torch.all(dst[:, 64 + N:] == 3.0)


def test_scatter_k0_zero_fills_window(vs):
    M, N, V = 16, 24, 4
    rp = torch.zeros(5, dtype=torch.int32, device="cuda")
    dst = torch.full((M, 40), 5.0, dtype=torch.float16, device="cuda")
    vs.vs_spmm_scatter(M, 0, N, V, rp, None, None, None, [dst.data_ptr() + 2 * 8], 40)
    torch.cuda.synchronize()
    assert torch.all(dst[:, 8:8 + N] == 0) and torch.all(dst[:, :8] == 5) and torch.all(dst[:, 8 + N:] == 5)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def test_symmetric_memory_replicated_path(vs):
    """dist.spmm_npanel_replicated on a one-rank NCCL group: symmetric-memory C, peer
    pointers from the rendezvous, scatter epilogue, stream barrier -> C == vs_spmm bitwise."""
    import torch.distributed as dist
    from paper_conf_sc_chenqldx21_b200 import dist as vsd
    try:
        import torch.distributed._symmetric_memory  # noqa: F401
    except ImportError:
        pytest.skip("torch symmetric memory unavailable")
    own = not dist.is_initialized()
    if own:
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        os.environ["MASTER_PORT"] = str(_free_port())
        dist.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", 0))
    try:
        V, M, K, N = 8, 512, 1024, 512
        rng = gen.make_rng("gscat_symm")
        A = gen.colvec_dense(rng, M, K, V, 0.1)
        B = dev(gen.dense_operand(rng, K, N))
        rp, ci, va = vs.encode(V, dense=dev(A))
        full = vs.spmm(rp, ci, va, B, M, V)
        rep = vsd.ReplicatedC(M, N, torch.device("cuda", 0))
        C = vsd.spmm_npanel_replicated(rp, ci, va, B, M, V, [0, N], 0, rep)
        torch.cuda.synchronize()
        assert torch.equal(C.view(torch.int16), full.view(torch.int16))
    finally:
        if own:
            dist.destroy_process_group()

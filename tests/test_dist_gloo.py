"""Multi-process (world_size 2, gloo, CPU) tests of the partitioner in dist.py.

The per-shard compute is injected: here a CPU stand-in built on the oracle (rounded to
fp16), since there is no GPU; on the GPU box the same partition is checked with the CUDA
kernels in test_gpu_parity.py::test_sharded_equals_unsharded_*.  The invariant is the one
of SURVEY §8(c): sharded results == unsharded results, bit for bit."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
from paper_conf_sc_chenqldx21_b200 import dist as vsd
from synth import gen


def test_panel_bounds():
    assert vsd.panel_bounds(256, 2) == [0, 128, 256]
    assert vsd.panel_bounds(65536, 8) == [8192 * i for i in range(9)]
    b = vsd.panel_bounds(200, 3)
    assert b[0] == 0 and b[-1] == 200 and all(x % 64 == 0 for x in b[:-1])
    assert all(b[i] <= b[i + 1] for i in range(3))
    assert vsd.panel_bounds(10, 4)[-1] == 10


def test_window_bounds_balanced():
    rng = gen.make_rng("wb")
    counts = rng.integers(0, 50, size=300)
    rp = np.concatenate([[0], np.cumsum(counts)])
    for P in (1, 2, 3, 8):
        b = vsd.window_bounds(rp, P)
        assert b[0] == 0 and b[-1] == 300 and all(b[i] <= b[i + 1] for i in range(P))
        loads = [rp[b[i + 1]] - rp[b[i]] for i in range(P)]
        assert max(loads) - rp[-1] / P <= counts.max() + 1


def test_sddmm_shard_rebases():
    rp = np.array([0, 3, 3, 7, 9, 12])
    sh = vsd.sddmm_shard(rp, M=10, V=2, bounds=[0, 2, 5], rank=1)
    assert (sh.w0, sh.w1, sh.p0, sh.p1, sh.row0, sh.row1) == (2, 5, 3, 12, 4, 10)
    assert sh.row_ptr.tolist() == [0, 4, 6, 9]


# --------------------------------------------------------------- 2-process gloo runs

def cpu_spmm(row_ptr, col_idx, vals, B, M, V, out=None):
    K, N = B.shape
    C64, _ = oracle.spmm(M, K, N, V, row_ptr.numpy(), col_idx.numpy(), vals.numpy(), B.numpy())
    return torch.from_numpy(C64.astype(np.float16))


def cpu_sddmm(row_ptr, col_idx, A, Bt, V, nnz=None, out=None):
    M, K = A.shape
    N = Bt.shape[0]
    o64, _ = oracle.sddmm(M, N, K, V, row_ptr.numpy(), col_idx.numpy(), A.numpy(), Bt.numpy())
    return torch.from_numpy(o64.astype(np.float16))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _worker(rank, world, port, results):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        # ---- SpMM: N-panels, A replicated
        M, K, N, V = 52, 70, 200, 4
        rng = gen.make_rng("dist_spmm")
        Ad = gen.colvec_dense(rng, M, K, V, 0.3)
        B = gen.dense_operand(rng, K, N)
        rp, ci, va = oracle.encode(M, K, V, dense=Ad)
        bounds = vsd.panel_bounds(N, world)
        n0, n1 = bounds[rank], bounds[rank + 1]
        Bp = torch.from_numpy(np.ascontiguousarray(B[:, n0:n1]))
        Cp = vsd.spmm_npanel(torch.from_numpy(rp), torch.from_numpy(ci), torch.from_numpy(va),
                             Bp, M, V, compute=cpu_spmm)
        C = vsd.gather_panels(Cp, bounds)
        full = cpu_spmm(torch.from_numpy(rp), torch.from_numpy(ci), torch.from_numpy(va),
                        torch.from_numpy(B), M, V)
        ok_spmm = torch.equal(C.view(torch.int16), full.view(torch.int16))

        # ---- SDDMM: row windows, Bt replicated
        M2, N2, K2 = 61, 90, 48
        rng = gen.make_rng("dist_sddmm")
        mask = gen.colvec_mask(rng, M2, N2, V, 0.3)
        A = gen.dense_operand(rng, M2, K2)
        Bt = gen.dense_operand(rng, N2, K2)
        rp2, ci2, _ = oracle.encode(M2, N2, V, mask=mask)
        wb = vsd.window_bounds(rp2, world)
        sh = vsd.sddmm_shard(rp2, M2, V, wb, rank)
        seg = vsd.sddmm_rowwin(sh, torch.from_numpy(sh.row_ptr),
                               torch.from_numpy(ci2[sh.p0:sh.p1].copy()),
                               torch.from_numpy(np.ascontiguousarray(A[sh.row0:sh.row1])),
                               torch.from_numpy(Bt), V, compute=cpu_sddmm)
        counts = [(int(rp2[wb[i + 1]]) - int(rp2[wb[i]])) * V for i in range(world)]
        allv = vsd.gather_segments(seg, counts)
        full2 = cpu_sddmm(torch.from_numpy(rp2), torch.from_numpy(ci2), torch.from_numpy(A),
                          torch.from_numpy(Bt), V)
        ok_sddmm = torch.equal(allv.view(torch.int16), full2.view(torch.int16))
        results[rank] = (bool(ok_spmm), bool(ok_sddmm), sh.p1 - sh.p0)
    finally:
        dist.destroy_process_group()


def test_two_rank_gloo_sharding_matches_unsharded():
    world = 2
    mgr = mp.Manager()
    results = mgr.dict()
    mp.spawn(_worker, args=(world, _free_port(), results), nprocs=world, join=True)
    assert len(results) == world
    for r in range(world):
        ok_spmm, ok_sddmm, nloc = results[r]
        assert ok_spmm, f"rank {r}: gathered SpMM panels differ from the unsharded result"
        assert ok_sddmm, f"rank {r}: gathered SDDMM segments differ from the unsharded result"
        assert nloc > 0


# ------------------------------------------- bench.py multi-GPU launcher and C5 plan

def test_bench_launch_command_and_world_check(monkeypatch):
    """`bench.py --gpus N` outside torchrun re-launches itself as N ranks (one node,
    127.0.0.1); under torchrun a WORLD_SIZE that disagrees with --gpus is an error, never a
    silent 1-GPU run."""
    import bench
    cmd = bench.launch_command(4, ["--gpus", "4", "--steps", "2"], port=12345)
    assert cmd[1:3] == ["-m", "torch.distributed.run"]
    assert "--nproc-per-node=4" in cmd and "--master-addr=127.0.0.1" in cmd
    assert "--master-port=12345" in cmd and cmd[-3:] == ["--gpus", "4", "--steps", "2"][-3:]
    assert cmd[cmd.index("--master-port=12345") + 1].endswith("bench.py")
    monkeypatch.delenv("WORLD_SIZE", raising=False)
    assert bench.check_world(bench.parse_args(["--gpus", "8"])) == "spawn"
    assert bench.check_world(bench.parse_args(["--gpus", "1"])) == "run"
    monkeypatch.setenv("WORLD_SIZE", "8")
    assert bench.check_world(bench.parse_args(["--gpus", "8"])) == "run"
    with pytest.raises(SystemExit):
        bench.check_world(bench.parse_args(["--gpus", "4"]))
    monkeypatch.setenv("WORLD_SIZE", "1")
    with pytest.raises(SystemExit):
        bench.check_world(bench.parse_args(["--gpus", "2"]))


def _plan_worker(rank, world, port, results):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import bench
        # the global C5 mask's row_ptr (same seed on every rank, as in bench.run_c5)
        rng = gen.make_rng("c5_plan_rowptr")
        counts = rng.binomial(65536, 0.1, size=2048)
        rp = np.concatenate([[0], np.cumsum(counts)]).astype(np.int64)
        plan = bench.c5_plan(world, rank, rp)
        mine = (plan["n0"], plan["n1"], plan["shard"].w0, plan["shard"].w1,
                plan["shard"].p1 - plan["shard"].p0)
        allp = [None] * world
        dist.all_gather_object(allp, mine)
        results[rank] = (allp, plan["panel_bounds"], plan["window_bounds"], int(rp[-1]))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_c5_plan_partitions_cover_once(world):
    mgr = mp.Manager()
    results = mgr.dict()
    mp.spawn(_plan_worker, args=(world, _free_port(), results), nprocs=world, join=True)
    allp, pb, wb, nnz = results[0]
    for r in range(world):
        assert results[r][0] == allp and results[r][1] == pb and results[r][2] == wb
    # panels tile [0, N) in whole 4096-column generator blocks; windows tile [0, W)
    assert allp[0][0] == 0 and allp[-1][1] == 65536
    assert all(allp[r][1] == allp[r + 1][0] for r in range(world - 1))
    assert all(a[0] % 4096 == 0 for a in allp)
    assert allp[0][2] == 0 and allp[-1][3] == 2048
    assert all(allp[r][3] == allp[r + 1][2] for r in range(world - 1))
    loads = [a[4] for a in allp]
    assert sum(loads) == nnz and max(loads) - nnz / world <= 0.01 * nnz
    assert all(a[2] % 16 == 0 for a in allp)  # 128-row blocks of V = 8 windows


def test_scatter_dst_ptrs():
    assert vsd.scatter_dst_ptrs([1000, 5000], 64) == [1128, 5128]
    assert vsd.scatter_dst_ptrs([0], 0, elem_bytes=4) == [0]

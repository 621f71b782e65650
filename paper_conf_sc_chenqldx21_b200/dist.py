"""Multi-GPU partitioning of the hot path (one process per GPU, torch.distributed).

The paper is single-GPU; the sharding follows the north star: the two ops
split into independent units, so ranks compute with NO data-path collective, and an NCCL
all-gather runs only when the caller asks for a replicated output.

  SpMM  (C = A B):  N-panels.  Rank p owns the columns [n_p, n_{p+1}) of B and C (panel
        widths multiples of 64, the paper's TileN); A (column-vector CSR) is
        replicated.  Per-element accumulation order does not depend on the panel, so the
        sharded result equals the 1-GPU result bit for bit.
  SDDMM (out = (A B^T) o D): row windows.  Rank p owns windows [w_p, w_{p+1}) chosen by a
        binary search of row_ptr so that each rank gets ~nnz_v/P stored vectors; its A rows,
        a rebased row_ptr slice, and the contiguous col_idx / out_vals slices.  Bt is
        replicated.  The concatenated out_vals equal the unsharded ones bit for bit.

Only host-side bookkeeping lives here; the per-shard compute is an ordinary vs_spmm /
vs_sddmm call on the shard's buffers (``compute=`` hooks exist so the partition logic can
be tested on CPU with a stand-in).
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np

__all__ = ["panel_bounds", "window_bounds", "SddmmShard", "sddmm_shard", "spmm_npanel",
           "sddmm_rowwin", "gather_panels", "gather_segments", "scatter_dst_ptrs",
           "ReplicatedC", "spmm_npanel_replicated"]


def panel_bounds(N: int, world: int, align: int = 64) -> list:
    """Column boundaries [n_0 = 0, ..., n_P = N] of P panels whose widths are multiples of
    ``align`` (except possibly the last), as equal as possible."""
    units = -(-N // align) if N > 0 else 0
    out = [0]
    for p in range(1, world + 1):
        out.append(min(N, (units * p // world) * align))
    out[-1] = N
    return out


def window_bounds(row_ptr: np.ndarray, world: int, align: int = 1) -> list:
    """Window boundaries [w_0 = 0, ..., w_P = W] with row_ptr[w_p] ~ p * nnz_v / P
    (balanced to within `align` windows' vectors).  With align = 128 / V every shard starts on
    a 128-row block boundary, so the per-row-block choice between the gather and the dense-tile
    SDDMM kernels (dense_select.cuh) is the same in a shard as in the unsharded problem."""
    row_ptr = np.asarray(row_ptr, dtype=np.int64)
    W = row_ptr.size - 1
    nnz = int(row_ptr[-1])
    out = [0]
    for p in range(1, world):
        target = (nnz * p) // world
        w = int(np.searchsorted(row_ptr, target, side="left"))
        if align > 1:
            w = int(round(w / align)) * align
        out.append(min(max(w, out[-1]), W))
    out.append(W)
    return out


@dataclass
class SddmmShard:
    w0: int           # first window
    w1: int           # one past the last window
    p0: int           # first stored vector (global index)
    p1: int           # one past the last stored vector
    row0: int         # first scalar row of A = w0 * V
    row1: int         # one past the last scalar row (clipped to M)
    row_ptr: np.ndarray  # rebased row_ptr slice, int32 [w1 - w0 + 1]


def sddmm_shard(row_ptr: np.ndarray, M: int, V: int, bounds: list, rank: int) -> SddmmShard:
    row_ptr = np.asarray(row_ptr, dtype=np.int64)
    w0, w1 = bounds[rank], bounds[rank + 1]
    p0, p1 = int(row_ptr[w0]), int(row_ptr[w1])
    local = (row_ptr[w0:w1 + 1] - p0).astype(np.int32)
    return SddmmShard(w0, w1, p0, p1, w0 * V, min(M, w1 * V), local)


def spmm_npanel(row_ptr, col_idx, vals, B_panel, M: int, V: int, compute=None, out=None):
    """This rank's panel of C = A B: an ordinary SpMM on the local [K x Np] panel of B.
    ``compute(row_ptr, col_idx, vals, B_panel, M, V, out)`` defaults to the CUDA kernel."""
    if compute is None:
        from . import spmm as compute
    return compute(row_ptr, col_idx, vals, B_panel, M, V, out=out)


def sddmm_rowwin(shard: SddmmShard, row_ptr_local, col_idx_local, A_rows, Bt, V: int,
                 compute=None, out=None):
    """This rank's out_vals segment (vectors [p0, p1)) of the sampled product."""
    if compute is None:
        from . import sddmm as compute
    return compute(row_ptr_local, col_idx_local, A_rows, Bt, V, nnz=shard.p1 - shard.p0, out=out)


def gather_panels(C_panel, bounds: list, group=None, row_major: bool = True):
    """All-gather of the C panels (optional replicated output).  Panels are padded to the
    widest one, gathered with all_gather_into_tensor ([P, M, Np_max], panel-major) and, if
    ``row_major``, permuted into the row-major [M, N] matrix."""
    import torch
    import torch.distributed as dist
    world = len(bounds) - 1
    widths = [bounds[i + 1] - bounds[i] for i in range(world)]
    wmax = max(widths)
    M = C_panel.shape[0]
    send = C_panel
    if C_panel.shape[1] != wmax:
        send = torch.zeros((M, wmax), dtype=C_panel.dtype, device=C_panel.device)
        send[:, :C_panel.shape[1]] = C_panel
    recv = torch.empty((world * M, wmax), dtype=C_panel.dtype, device=C_panel.device)
    dist.all_gather_into_tensor(recv, send.contiguous(), group=group)
    recv = recv.view(world, M, wmax)
    if not row_major:
        return recv
    return torch.cat([recv[i, :, :widths[i]] for i in range(world)], dim=1)


def gather_segments(segment, counts: list, group=None):
    """All-gather-v of contiguous out_vals segments (rank i contributes counts[i] values) into
    the global array, via a padded all_gather_into_tensor."""
    import torch
    import torch.distributed as dist
    world = len(counts)
    cmax = max(counts) if counts else 0
    send = torch.zeros(cmax, dtype=segment.dtype, device=segment.device)
    send[:segment.numel()] = segment.reshape(-1)
    recv = torch.empty(world * cmax, dtype=segment.dtype, device=segment.device)
    dist.all_gather_into_tensor(recv, send, group=group)
    recv = recv.view(world, cmax)
    return torch.cat([recv[i, :counts[i]] for i in range(world)])


# ------------------------------------------- fused replicated-output epilogue (§8(f)-4)
#
# Instead of computing the panel into a local buffer and all-gathering + permuting it
# (gather_panels), every rank's SpMM epilogue stores its C tiles straight into EVERY rank's
# row-major C [M x N] (vs_spmm_scatter): the C buffers are symmetric memory
# (torch.distributed._symmetric_memory), so each rank holds device pointers to all peers'
# buffers (NVLink / NVSwitch peer stores).  One barrier on the stream afterwards orders the
# peers' reads after every rank's stores.  Same bits as gather_panels (same kernel body and
# accumulation order; only the store addresses differ).

def scatter_dst_ptrs(buffer_ptrs, n0: int, elem_bytes: int = 2) -> list:
    """Destination pointers of this rank's panel [*, n0:...] in every rank's row-major C:
    each peer buffer's base address + n0 elements."""
    return [int(p) + int(n0) * elem_bytes for p in buffer_ptrs]


class ReplicatedC:
    """Symmetric-memory C [M x N] fp16 on this rank, rendezvoused over ``group``; holds the
    peer pointers the scatter epilogue writes to."""

    def __init__(self, M: int, N: int, device, group=None):
        import torch
        import torch.distributed as dist
        import torch.distributed._symmetric_memory as symm_mem
        self.M, self.N = M, N
        self.group = group if group is not None else dist.group.WORLD
        self.C = symm_mem.empty((M, N), dtype=torch.float16, device=device)
        self.hdl = symm_mem.rendezvous(self.C, self.group)
        self.world = self.hdl.world_size
        self.buffer_ptrs = list(self.hdl.buffer_ptrs)

    def barrier(self):
        """Stream-ordered barrier across the ranks: after it, every rank's stores into every
        replica are visible to this rank."""
        self.hdl.barrier(channel=0)


def spmm_npanel_replicated(row_ptr, col_idx, vals, B_panel, M: int, V: int, bounds: list,
                           rank: int, rep: "ReplicatedC", barrier: bool = True):
    """This rank's panel of C = A B, stored by the kernel epilogue into every rank's
    replicated row-major C (rep.C holds the full C on every rank after the barrier)."""
    from . import vs_spmm_scatter
    K, Np = B_panel.shape
    n0 = bounds[rank]
    assert bounds[rank + 1] - n0 == Np and rep.N == bounds[-1]
    vs_spmm_scatter(M, K, Np, V, row_ptr, col_idx, vals, B_panel,
                    scatter_dst_ptrs(rep.buffer_ptrs, n0), rep.N)
    if barrier:
        rep.barrier()
    return rep.C

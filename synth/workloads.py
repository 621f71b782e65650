"""Workload definitions (shapes only, no arithmetic) for bench.py and the GPU tests.

BASELINE.json configs:
  C1  SpMM + SDDMM M=K=256, N=64, V=4, S=0.9 (oracle in seconds)
  C2  DLMC-transformer-shaped SpMM (M=2048, K=512 etc.), V=2/4/8, S=50/70/90/98%, N=64/128/256
  C3  SDDMM at the same masks and shapes, inner K=64/128/256
  C4  ResNet-50 1x1-conv-shaped SpMM, batch-folded N=3136, V=8, S=70-95%
  C5  M=K=16384, N=65536, V=8, S=0.9 SpMM (N-panels) and SDDMM (row windows), sharded

The bench "layer" problem couples C2 and C3 the way the paper's training equations do
(P:1625-1633): a sparse weight W [M x K] (column-vector pattern, grain V, sparsity S) is
encoded, Y = W X (SpMM, X [K x N]) and dW = (G X^T) o pattern(W) (SDDMM with inner
dimension N, G [M x N]).  The SDDMM mask is the SpMM pattern, and its inner K is the SpMM N
(so C3's K in {64,128,256} is C2's N set).
"""
from __future__ import annotations

from dataclasses import dataclass, asdict


@dataclass(frozen=True)
class Problem:
    M: int
    K: int
    N: int
    V: int
    S: float
    kind: str = "bern"

    @property
    def id(self) -> str:
        return f"layer_M{self.M}_K{self.K}_N{self.N}_V{self.V}_S{self.S:.2f}_{self.kind}"

    def asdict(self):
        return asdict(self)


# (M, K) shapes of DLMC-transformer layers (d_model=512, d_ff=2048) plus the paper's
# profiling shape A 2048x1024.
DLMC_MK = [(512, 512), (2048, 512), (512, 2048), (2048, 1024)]
DLMC_V = [2, 4, 8]
DLMC_S = [0.5, 0.7, 0.9, 0.98]
DLMC_N = [64, 128, 256]

# ResNet-50 1x1 convolutions as GEMM (Cout, Cin), batch-folded N = 3136.
RN50_MK = [(64, 64), (64, 256), (256, 64), (128, 256), (128, 512), (512, 128), (512, 256),
           (256, 512), (256, 1024), (1024, 256), (1024, 512), (512, 1024), (512, 2048),
           (2048, 512), (2048, 1024)]
RN50_S = [0.7, 0.8, 0.9, 0.95]


# the paper's full sparsity grid (Fig. 17/19 captions)
DLMC_S_GRID = [0.5, 0.7, 0.8, 0.9, 0.95, 0.98]


def dlmc_grid_workload():
    """configs[1] x configs[2] on the paper's full sparsity grid {.5,.7,.8,.9,.95,.98}: the
    per-V crossover with cuBLAS."""
    return [Problem(M, K, N, V, S) for (M, K) in DLMC_MK for V in DLMC_V for S in DLMC_S_GRID
            for N in DLMC_N]


def dlmc_layer_workload():
    """configs[1] x configs[2]: 4 shapes x V{2,4,8} x S{.5,.7,.9,.98} x N{64,128,256}."""
    return [Problem(M, K, N, V, S) for (M, K) in DLMC_MK for V in DLMC_V for S in DLMC_S
            for N in DLMC_N]


def rn50_workload():
    return [Problem(M, K, 3136, 8, S) for (M, K) in RN50_MK for S in RN50_S]


def c1_problem():
    return Problem(256, 256, 64, 4, 0.9)


def c5_problem():
    return Problem(16384, 16384, 65536, 8, 0.9)


def custom_workload():
    """Problems from the environment: VS_PROBLEMS="M,K,N,V,S;M,K,N,V,S" (tuning/profiling)."""
    import os
    out = []
    for item in filter(None, os.environ.get("VS_PROBLEMS", "").split(";")):
        M, K, N, V, S = item.split(",")
        out.append(Problem(int(M), int(K), int(N), int(V), float(S)))
    return out


WORKLOADS = {
    "custom": custom_workload,
    "dlmc_layer": dlmc_layer_workload,
    "dlmc_grid": dlmc_grid_workload,
    "rn50_layer": rn50_workload,
    "c1": lambda: [c1_problem()],
    # the paper's profiling case: A 2048x1024 x B 1024x256, 90% (Tables 2/3)
    "profile": lambda: [Problem(2048, 1024, 256, 4, 0.9), Problem(2048, 1024, 256, 8, 0.9)],
    "c5": lambda: [c5_problem()],
}

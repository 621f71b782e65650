"""Seeded synthetic inputs shared by the oracle tests, the GPU parity tests and bench.py.

This module holds NO arithmetic of the method (no encoding, no SpMM/SDDMM): it only draws
random dense matrices whose nonzeros form V x 1 column vectors, random masks, and dense
operands.  Both sides of every parity check (``oracle/`` and the CUDA path) receive the
same arrays from here and do their own work on them.

Recipe:
  * Pattern.  The paper builds its benchmarks from DLMC CSR patterns "and randomly generate
    a nonzero vector with length V for each indexed position".  Offline we
    draw the pattern directly at W = ceil(M/V) row windows (reading R14):
      - "bern": each (window, column) vector is kept independently with probability 1-S
        (row lengths Binomial(K, 1-S), a proxy for DLMC's uneven rows);
      - "unif": exactly round((1-S)*K) distinct uniform columns per window (the paper's
        Blocked-ELL construction).
  * Values.  Uniform in [-1, 1), rounded to fp16; exact zeros are resampled so stored
    vectors are nonzero (reading R15).  ``exact=True`` draws from {-2,-1,1,2} instead so that
    every fp32 partial sum is an exactly representable integer.
  * Seeds.  numpy ``Generator(PCG64(seed))`` with ``seed = zlib.crc32(config_id)``.
"""
from __future__ import annotations

import math
import zlib

import numpy as np

__all__ = [
    "config_seed", "make_rng", "fp16_values", "vector_keep", "colvec_dense", "colvec_mask",
    "attention_mask",
    "dense_operand", "torch_colvec_dense", "torch_dense_operand",
]


def config_seed(config_id: str) -> int:
    """Deterministic 32-bit seed of a config id string."""
    return zlib.crc32(config_id.encode("utf-8")) & 0xFFFFFFFF


def make_rng(seed_or_id) -> np.random.Generator:
    seed = config_seed(seed_or_id) if isinstance(seed_or_id, str) else int(seed_or_id)
    return np.random.Generator(np.random.PCG64(seed))


def fp16_values(rng: np.random.Generator, shape, exact: bool = False) -> np.ndarray:
    """fp16 array of nonzero values: U[-1,1) rounded to fp16 (zeros resampled), or, with
    ``exact``, uniform over {-2,-1,1,2}."""
    shape = tuple(int(s) for s in np.atleast_1d(shape)) if not isinstance(shape, tuple) else shape
    if exact:
        return rng.choice(np.array([-2.0, -1.0, 1.0, 2.0], dtype=np.float16), size=shape)
    out = (rng.random(shape) * 2.0 - 1.0).astype(np.float16)
    bad = out == 0
    while bad.any():
        out[bad] = (rng.random(int(bad.sum())) * 2.0 - 1.0).astype(np.float16)
        bad = out == 0
    return out


def vector_keep(rng: np.random.Generator, W: int, K: int, density: float,
                kind: str = "bern") -> np.ndarray:
    """bool [W, K]: which (row window, column) vectors are nonzero."""
    if kind == "bern":
        return rng.random((W, K)) < density
    if kind == "unif":
        n = int(round(density * K))
        keep = np.zeros((W, K), dtype=bool)
        for w in range(W):
            keep[w, rng.choice(K, size=n, replace=False)] = True
        return keep
    raise ValueError(f"unknown pattern kind {kind!r}")


def colvec_dense(rng: np.random.Generator, M: int, K: int, V: int, density: float,
                 kind: str = "bern", exact: bool = False, inner_zero_frac: float = 0.0,
                 neg_zero_frac: float = 0.0) -> np.ndarray:
    """fp16 [M, K] whose nonzeros are V x 1 column vectors (rows grouped by windows of V).

    ``inner_zero_frac`` replaces that fraction of elements inside kept vectors with +0.0
    (a kept vector may hold zeros, as (0,1) in Fig. 8); ``neg_zero_frac`` puts -0.0
    at that fraction of ALL positions (bit pattern 0x8000, kept by the encoder).
    """
    W = -(-M // V) if M > 0 else 0
    keep = vector_keep(rng, W, K, density, kind)
    vals = fp16_values(rng, (W * V, K), exact=exact)
    full = np.where(np.repeat(keep, V, axis=0), vals, np.float16(0.0))[:M]
    if inner_zero_frac > 0:
        z = rng.random(full.shape) < inner_zero_frac
        full = np.where(z, np.float16(0.0), full)
    if neg_zero_frac > 0:
        z = rng.random(full.shape) < neg_zero_frac
        full = np.where(z, np.float16(-0.0), full)
    return np.ascontiguousarray(full.astype(np.float16))


def block_dense(rng: np.random.Generator, M: int, K: int, V: int, density: float,
                exact: bool = False) -> np.ndarray:
    """fp16 [M, K] made of square V x V nonzero blocks (each kept with probability
    ``density``): the pattern under which both W and W^T are column-vector encodings
    (§8 Case 1)."""
    W = -(-M // V) if M > 0 else 0
    KB = -(-K // V) if K > 0 else 0
    keep = rng.random((W, KB)) < density
    full = np.repeat(np.repeat(keep, V, axis=0), V, axis=1)[:M, :K]
    vals = fp16_values(rng, (M, K), exact=exact)
    return np.ascontiguousarray(np.where(full, vals, np.float16(0.0)).astype(np.float16))


def colvec_mask(rng: np.random.Generator, M: int, N: int, V: int, density: float,
                kind: str = "bern") -> np.ndarray:
    """uint8 [M, N] binary mask made of V x 1 column vectors (the SDDMM mask D)."""
    W = -(-M // V) if M > 0 else 0
    keep = vector_keep(rng, W, N, density, kind)
    return np.ascontiguousarray(np.repeat(keep, V, axis=0)[:M].astype(np.uint8))


def attention_mask(rng: np.random.Generator, l: int, V: int, sparsity: float,
                   band: int = 256) -> np.ndarray:
    """uint8 [l, l] attention mask of V x 1 vectors: a dense band of width
    `band` along the diagonal plus uniformly random off-band vectors, with the off-band
    probability chosen so that the overall density is 1 - sparsity (when the band alone is
    sparser than that)."""
    W = -(-l // V)
    wi = np.arange(W)[:, None] * V + V // 2
    cj = np.arange(l)[None, :]
    in_band = np.abs(cj - wi) < band // 2
    band_frac = in_band.mean()
    target = 1.0 - sparsity
    p_off = max(0.0, (target - band_frac) / max(1e-12, 1.0 - band_frac))
    keep = in_band | (rng.random((W, l)) < p_off)
    return np.ascontiguousarray(np.repeat(keep, V, axis=0)[:l].astype(np.uint8))


def dense_operand(rng: np.random.Generator, rows: int, cols: int, exact: bool = False) -> np.ndarray:
    """fp16 [rows, cols] dense operand (B of SpMM, A / Bt of SDDMM)."""
    return np.ascontiguousarray(fp16_values(rng, (rows, cols), exact=exact))


# ---- device-side generation for operands too large to build on the host (C5) ----------

def _torch_gen(seed: int, device):
    import torch
    g = torch.Generator(device=device)
    g.manual_seed(int(seed))
    return g


def torch_dense_operand(rows: int, cols: int, seed: int, device="cuda"):
    """fp16 [rows, cols] U[-1,1) on ``device``; exact zeros replaced by 0.5 (no resampling
    on device, same effect: stored values are nonzero)."""
    import torch
    g = _torch_gen(seed, device)
    x = (torch.rand((rows, cols), generator=g, device=device) * 2.0 - 1.0).to(torch.float16)
    return torch.where(x == 0, torch.full_like(x, 0.5), x)


def torch_colvec_dense(M: int, K: int, V: int, density: float, seed: int, device="cuda"):
    """fp16 [M, K] column-vector-sparse matrix (Bernoulli pattern) built on ``device``."""
    import torch
    W = -(-M // V)
    g = _torch_gen(seed, device)
    keep = torch.rand((W, K), generator=g, device=device) < density
    x = (torch.rand((W * V, K), generator=g, device=device) * 2.0 - 1.0).to(torch.float16)
    x = torch.where(x == 0, torch.full_like(x, 0.5), x)
    x = torch.where(keep.repeat_interleave(V, dim=0), x, torch.zeros_like(x))
    return x[:M].contiguous()


def expected_nnz_vec(M: int, K: int, V: int, density: float) -> float:
    """Expected number of stored vectors of a Bernoulli pattern (for sizing only)."""
    return math.ceil(M / V) * K * density

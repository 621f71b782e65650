#!/usr/bin/env python
"""Phase timing of the dense-tile SDDMM CTAs (tuning aid; needs a -DVS_SD_TIMING=1 build loaded
with VS_LIB_PATH).  Prints the median clock64 span of each phase over the CTAs of one launch:

  VS_LIB_PATH=build/variants/libvs_sdt.so python tools/sd_timing.py M N K V S   (one vs_sddmm call)
  VS_LIB_PATH=build/variants/libvs_sdt.so python tools/sd_timing.py batch      (DLMC K=256 batch, V=2)
"""
import ctypes
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

PHASES = ["rowptr RT + decode", "barrier init + TMEM alloc", "search (thread 64)", "TMA+MMA wait (from alloc)",
          "drain", "store pass"]


def main():
    import torch
    import paper_conf_sc_chenqldx21_b200 as vs
    from synth import gen
    lib = vs.load()
    fn = lib.vs_debug_sd_timing
    fn.argtypes = [ctypes.c_void_p, ctypes.c_int]
    if sys.argv[1] == "batch":
        probs = [(M, K, 256, 2, S) for (M, K) in [(512, 512), (2048, 512), (512, 2048), (2048, 1024)]
                 for S in (0.5, 0.7)]
    else:
        M, N, K, V, S = sys.argv[1:6]
        probs = [(int(M), int(N), int(K), int(V), float(S))]
    batch = []
    for (M, N, K, V, S) in probs:
        rng = gen.make_rng(f"sdt_{M}_{N}_{K}_{V}_{S}")
        W = torch.from_numpy(gen.colvec_dense(rng, M, N, V, 1 - S)).cuda()
        A = torch.from_numpy(gen.dense_operand(rng, M, K)).cuda()
        Bt = torch.from_numpy(gen.dense_operand(rng, N, K)).cuda()
        rp, ci, _ = vs.encode(V, dense=W)
        out = torch.empty(int(rp[-1].item()) * V, dtype=torch.float16, device="cuda")
        batch.append((M, N, K, V, rp, ci, A, Bt, out))
    for _ in range(3):
        if len(batch) == 1:
            vs.vs_sddmm(*batch[0])
        else:
            vs.vs_sddmm_batched(batch)
    torch.cuda.synchronize()
    n = 8192
    buf = np.zeros((n, 8), np.uint64)
    fn(buf.ctypes.data, n)
    t = buf.astype(np.int64)
    ok = (t[:, 6] > t[:, 0]) & (t[:, 1] >= t[:, 0]) & (t[:, 5] >= t[:, 4]) & (t[:, 6] - t[:, 0] < 10 ** 8)
    t = t[ok]
    print("dense CTAs timed:", len(t))
    spans = [t[:, 1] - t[:, 0], t[:, 2] - t[:, 1], t[:, 3] - t[:, 2], t[:, 4] - t[:, 2], t[:, 5] - t[:, 4],
             t[:, 6] - t[:, 5]]
    for name, sp in zip(PHASES, spans):
        print("%-28s median %7d  p90 %7d cycles" % (name, int(np.median(sp)), int(np.percentile(sp, 90))))
    tot = t[:, 6] - t[:, 0]
    print("%-28s median %7d  p90 %7d cycles" % ("total", int(np.median(tot)), int(np.percentile(tot, 90))))


if __name__ == "__main__":
    main()

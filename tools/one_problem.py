#!/usr/bin/env python
"""Runs one SpMM / SDDMM problem a few times (for ncu captures of a single kernel).

  python tools/one_problem.py --op spmm --M 2048 --K 1024 --N 256 --V 2 --S 0.5 [--reps 3]
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--op", default="spmm")
    ap.add_argument("--M", type=int, default=2048)
    ap.add_argument("--K", type=int, default=1024)
    ap.add_argument("--N", type=int, default=256)
    ap.add_argument("--V", type=int, default=2)
    ap.add_argument("--S", type=float, default=0.5)
    ap.add_argument("--reps", type=int, default=3)
    a = ap.parse_args()
    import torch
    import paper_conf_sc_chenqldx21_b200 as vs
    from synth import gen
    rng = gen.make_rng(f"one_{a.op}_{a.M}_{a.K}_{a.N}_{a.V}_{a.S}")
    W = torch.from_numpy(gen.colvec_dense(rng, a.M, a.K, a.V, 1 - a.S)).cuda()
    X = torch.from_numpy(gen.dense_operand(rng, a.K, a.N)).cuda()
    G = torch.from_numpy(gen.dense_operand(rng, a.M, a.N)).cuda()
    rp, ci, va = vs.encode(a.V, dense=W)
    for _ in range(a.reps):
        if a.op == "spmm":
            vs.spmm(rp, ci, va, X, a.M, a.V)
        else:
            vs.sddmm(rp, ci, G, X, a.V)
    torch.cuda.synchronize()


if __name__ == "__main__":
    main()

#!/usr/bin/env python
"""Kernel-configuration sweep on the GPU (tuning aid, not part of the product).

For every configuration (a set of VS_* environment knobs read by libvs at first launch),
spawns a process that times every problem of a workload per op (CUDA graph of `reps`
launches, L2 warm), and prints a per-config geomean / sum table.

  python tools/tune.py --op spmm --workload dlmc_layer \
      --cfg "VS_SPMM_UNROLL=1,VS_SPMM_NC=0" --cfg "VS_SPMM_UNROLL=2,VS_SPMM_NC=1"
"""
from __future__ import annotations

import argparse
import json
import math
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def child_batched(op, workload, reps):
    """Times one batched call over the whole workload (CUDA graph of `reps` calls)."""
    import torch
    import paper_conf_sc_chenqldx21_b200 as vs
    from synth.workloads import WORKLOADS
    from bench import layer_inputs
    torch.cuda.set_device(0)
    st = torch.cuda.Stream()
    enc, sp, sd = [], [], []
    for p in WORKLOADS[workload]():
        Wd, X, G = layer_inputs(p)
        Wd, X, G = (torch.from_numpy(a).cuda() for a in (Wd, X, G))
        rp, ci, va = vs.encode(p.V, dense=Wd)
        nnz = int(rp[-1].item())
        Y = torch.empty((p.M, p.N), dtype=torch.float16, device="cuda")
        dW = torch.empty(max(nnz, 1) * p.V, dtype=torch.float16, device="cuda")
        enc.append((p.M, p.K, p.V, Wd, None, rp, ci, va))
        sp.append((p.M, p.K, p.N, p.V, rp, ci, va, X, Y))
        sd.append((p.M, p.K, p.N, p.V, rp, ci, G, X, dW))
    arr = {"encode": vs.make_encode_batch(enc), "spmm": vs.make_spmm_batch(sp),
           "sddmm": vs.make_sddmm_batch(sd)}[op]
    call = {"encode": vs.vs_encode_colvec_batched, "spmm": vs.vs_spmm_batched,
            "sddmm": vs.vs_sddmm_batched}[op]
    with torch.cuda.stream(st):
        call(arr)
    st.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=st):
        for _ in range(reps):
            call(arr)
    with torch.cuda.stream(st):
        g.replay()
    best = 1e30
    for _ in range(3):
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        with torch.cuda.stream(st):
            s.record()
            g.replay()
            e.record()
        e.synchronize()
        best = min(best, s.elapsed_time(e) * 1e3 / reps)
    print("JSON" + json.dumps([{"id": f"{workload}:{op}_batched", "us": best, "nnz_v": 0}]))


def child(op, workload, reps):
    if op.endswith("_batched"):
        return child_batched(op[:-8], workload, reps)
    import torch
    import paper_conf_sc_chenqldx21_b200 as vs
    from synth.workloads import WORKLOADS
    from bench import layer_inputs
    torch.cuda.set_device(0)
    st = torch.cuda.Stream()
    out = []
    for p in WORKLOADS[workload]():
        Wd, X, G = layer_inputs(p)
        Wd, X, G = (torch.from_numpy(a).cuda() for a in (Wd, X, G))
        rp, ci, va = vs.encode(p.V, dense=Wd)
        nnz = int(rp[-1].item())
        Y = torch.empty((p.M, p.N), dtype=torch.float16, device="cuda")
        dW = torch.empty(max(nnz, 1) * p.V, dtype=torch.float16, device="cuda")
        if op == "spmm":
            fn = lambda: vs.vs_spmm(p.M, p.K, p.N, p.V, rp, ci, va, X, Y)
        elif op == "sddmm":
            fn = lambda: vs.vs_sddmm(p.M, p.K, p.N, p.V, rp, ci, G, X, dW)
        else:
            cap = ci.numel()
            fn = lambda: vs.vs_encode_colvec(p.M, p.K, p.V, Wd, None, rp, ci, va)
        with torch.cuda.stream(st):
            fn()
        st.synchronize()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=st):
            for _ in range(reps):
                fn()
        with torch.cuda.stream(st):
            g.replay()
        best = 1e30
        for _ in range(3):
            s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            with torch.cuda.stream(st):
                s.record()
                g.replay()
                e.record()
            e.synchronize()
            best = min(best, s.elapsed_time(e) * 1e3 / reps)
        out.append({"id": p.id, "us": best, "nnz_v": nnz})
    print("JSON" + json.dumps(out))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--op", default="spmm")
    ap.add_argument("--workload", default="dlmc_layer")
    ap.add_argument("--reps", type=int, default=20)
    ap.add_argument("--cfg", action="append", default=[])
    ap.add_argument("--child", action="store_true")
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "tune.json"))
    a = ap.parse_args()
    if a.child:
        child(a.op, a.workload, a.reps)
        return
    results = {}
    for cfg in a.cfg or [""]:
        env = dict(os.environ)
        for kv in filter(None, cfg.split(",")):
            k, v = kv.split("=")
            env[k] = v
        r = subprocess.run([sys.executable, __file__, "--child", "--op", a.op, "--workload",
                            a.workload, "--reps", str(a.reps)], env=env, capture_output=True,
                           text=True)
        line = [l for l in r.stdout.splitlines() if l.startswith("JSON")]
        if not line:
            print(cfg, "FAILED", r.stderr[-2000:])
            continue
        results[cfg] = json.loads(line[0][4:])
    base = None
    for cfg, rows in results.items():
        us = [x["us"] for x in rows]
        gm = math.exp(sum(math.log(x) for x in us) / len(us))
        if base is None:
            base = us
        rel = math.exp(sum(math.log(x / b) for x, b in zip(us, base)) / len(us))
        print(f"{cfg or 'default':50s} sum={sum(us):9.1f}us geomean={gm:7.2f}us rel={rel:.3f}")
    os.makedirs(os.path.dirname(a.out), exist_ok=True)
    json.dump(results, open(a.out, "w"), indent=1)


if __name__ == "__main__":
    main()

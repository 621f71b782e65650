#!/usr/bin/env python
"""bench.py — throughput of the column-vector-sparse hot path on B200.

One STEP = one pass of the whole hot path (encode -> SpMM -> SDDMM) over the
workload's batch of synthetic layer problems (synth/workloads.py).  Per problem:
  vs_encode_colvec(W dense)                         -> (row_ptr, col_idx, vals)   [a1]
  vs_spmm(W, X)            Y  [M x N] = W X          (§5)            [a2-a6]
  vs_sddmm(pattern W; G, X) dW = (G X^T) o pattern   (§6)           [a7-a10]
(the forward / weight-gradient pair of P:1625-1633; SDDMM inner dimension = N).

metric = effective TFLOP/s = (2*nnz*N [SpMM] + 2*nnz*N [SDDMM]) / step time, nnz = stored
scalars (nnz_v * V), summed over all problems and all ranks, divided by the max over ranks
of the step time (device time, CUDA events).  The step is replayed as one CUDA graph; the
L2 is flushed (512 MiB write) between timed steps and the flush is not timed.

Also reported: per-kernel-class device time (events inside an instrumented graph), the
roofline of the dominant kernel, end-to-end throughput with host buffers (H2D + D2H inside
the timed region), the fp64 oracle on the host cores (cpu_baseline), same-box cuBLAS Hgemm /
GemmEx and cuSPARSE speedups per cell, and SM clocks sampled during the timed region.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
                  [--workload dlmc_layer|rn50_layer|c1] [--no-baselines] [--no-cpu]
"""
from __future__ import annotations

import argparse
import json
import math
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

METRIC = "SpMM/SDDMM effective TFLOP/s & speedup vs cuBLAS Hgemm, V=2/4/8, 50–98% sparse"
UNIT = "TFLOP/s"
DEFAULT_WORKLOAD = "dlmc_layer"


def parse_args(argv=None):
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--workload", default=None,
                    help="default: dlmc_layer at --gpus 1 (configs[1] x configs[2]); c5 at --gpus N > 1 "
                         "(configs[4], the case that shards)")
    ap.add_argument("--priority", choices=["none", "first", "sddmm", "encode"], default="first",
                    help="high stream priority for part of the chain schedule (see step_chains)")
    ap.add_argument("--schedule", choices=["chains", "phases"], default="chains",
                    help="batched step as one chain per V group on concurrent branches, or as "
                         "three phases (encode, then SpMM || SDDMM)")
    ap.add_argument("--no-baselines", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--e2e-chunks", type=int, default=12,
                    help="chunks of the pipelined end-to-end step (copies overlap compute)")
    ap.add_argument("--reps", type=int, default=20, help="launches per per-cell micro timing")
    ap.add_argument("--detail", default=os.path.join(ROOT, "gpurun_out", "bench_detail.json"))
    ap.add_argument("--cpu-seconds", type=float, default=8.0,
                    help="CPU work per thread setting of the cpu_baseline leg (x3 runs)")
    ap.add_argument("--streams", type=int, default=8,
                    help="concurrent graph branches across independent problems")
    return ap.parse_args(argv)


# ----------------------------------------------------------------------- helpers

def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return {"hbm_gbs": d["hbm_gbs"], "bf16_tflops": d["bf16_tflops"],
                "bf16_tflops_sustained": d.get("bf16_tflops_sustained", d["bf16_tflops"]),
                "source": "measured (MEASURED_PEAKS.json)"}
    return {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "bf16_tflops_sustained": 1400.0,
            "source": "fallback (B200_PROFILING.md)"}


class ClockSampler:
    """SM clock and throttle reasons sampled every 10 ms (NVML) while the timed region runs;
    falls back to `nvidia-smi -lms 200` if NVML is unavailable."""
    REASONS = {0x4: "sw_power_cap", 0x8: "hw_slowdown", 0x20: "sw_thermal_slowdown",
               0x40: "hw_thermal_slowdown", 0x80: "hw_power_brake_slowdown"}

    def __init__(self, device_index: int, pci_bus_id: str = None):
        self.dev = device_index
        self.bus = pci_bus_id
        self.sm = []
        self.mask = 0
        self.max_mhz = None
        self._stop = threading.Event()
        self.thread = None
        self.proc = None

    def start(self):
        try:
            import pynvml
            pynvml.nvmlInit()
            h = None
            if self.bus:
                try:
                    h = pynvml.nvmlDeviceGetHandleByPciBusId(self.bus)
                except Exception:
                    h = None
            if h is None:
                h = pynvml.nvmlDeviceGetHandleByIndex(self.dev)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(h, pynvml.NVML_CLOCK_SM)
            get_reasons = getattr(pynvml, "nvmlDeviceGetCurrentClocksEventReasons", None) or \
                pynvml.nvmlDeviceGetCurrentClocksThrottleReasons

            def loop():
                while not self._stop.is_set():
                    self.sm.append(pynvml.nvmlDeviceGetClockInfo(h, pynvml.NVML_CLOCK_SM))
                    self.mask |= int(get_reasons(h))
                    time.sleep(0.01)
            self.thread = threading.Thread(target=loop, daemon=True)
            self.thread.start()
        except Exception:
            self._start_smi()
        return self

    def _start_smi(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "--query-gpu=clocks.sm,clocks.max.sm,clocks_event_reasons.active",
                 "--format=csv,noheader,nounits", "-lms", "200", "-i", str(self.dev)],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except OSError:
            return

        def read():
            for line in self.proc.stdout:
                parts = [x.strip() for x in line.split(",")]
                try:
                    self.sm.append(float(parts[0]))
                    self.max_mhz = float(parts[1])
                    self.mask |= int(parts[2], 16)
                except (ValueError, IndexError):
                    pass
        self.thread = threading.Thread(target=read, daemon=True)
        self.thread.start()

    def stop(self):
        self._stop.set()
        if self.proc is not None:
            self.proc.terminate()
        if self.thread is not None:
            self.thread.join(timeout=2)
        reasons = sorted(n for b, n in self.REASONS.items() if self.mask & b)
        return {"sm_mhz": statistics.median(self.sm) if self.sm else None,
                "sm_max_mhz": self.max_mhz, "reasons": reasons, "samples": len(self.sm)}


def dist_env():
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return ws, rank, local


def init_dist(torch, local):
    """One process per GPU over NCCL.  VS_BENCH_HARNESS_TEST=1 (harness validation only: several
    ranks sharing the GPUs of a smaller box, over gloo) maps rank -> GPU modulo the device count;
    its timings are not measurements."""
    import torch.distributed as dist
    if os.environ.get("VS_BENCH_HARNESS_TEST") == "1":
        torch.cuda.set_device(local % torch.cuda.device_count())
        dist.init_process_group("gloo")
        return
    torch.cuda.set_device(local)
    dist.init_process_group("nccl", device_id=torch.device("cuda", local))


def problem_flops(nnz_v, p):
    nnz = nnz_v * p.V
    return 2.0 * nnz * p.N, 2.0 * nnz * p.N  # SpMM, SDDMM (inner dimension N)


def alg_bytes(p, nnz_v, k_ref):
    """Algorithmic HBM bytes per launch."""
    W = -(-p.M // p.V)
    spmm = 4 * (W + 1) + nnz_v * (4 + 2 * p.V) + 2 * k_ref * p.N + 2 * p.M * p.N
    sddmm = 4 * (W + 1) + 4 * nnz_v + 2 * p.M * p.N + 2 * k_ref * p.N + 2 * nnz_v * p.V
    encode = 2 * p.M * p.K + 4 * (W + 1) + nnz_v * (4 + 2 * p.V)
    return {"encode": encode, "spmm": spmm, "sddmm": sddmm}


def count_launches(bufs):
    """Kernel launches of one batched step, by the library's grouping rules: encode groups by
    V (3 kernels per group of <= 128 problems: count, scan, compact); SpMM (cp.async path,
    spmm.cu spmm_config) by (V, panel width NC = 1 for N <= 64 else 2, SPLIT from K); SDDMM
    (sddmm.cu sddmm_variant) by V (one kernel serves both K-block variants), plus the dense-tile
    SDDMM kernel (dense_tile.cu: problems with inner dimension >= VS_SDDMM_DENSE_KMIN = 256,
    32 problems per launch) before each V group's gather launch."""
    import math as _m
    from collections import Counter
    def split(K):
        q = K >> 8
        return 16 if q >= 16 else 8 if q >= 8 else 4 if q >= 4 else 2 if q >= 2 else 1
    enc = Counter(b.p.V for b in bufs)
    sp = Counter((b.p.V, 1 if b.p.N <= 64 else 2, split(b.p.K)) for b in bufs)
    sd = Counter(b.p.V for b in bufs)  # one mixed-K kernel per V (sddmm_window_any)
    sd_dense = Counter(b.p.V for b in bufs if b.p.N >= 256 and b.p.N % 8 == 0)  # SDDMM inner = N
    per = {"encode": sum(3 * _m.ceil(n / 128) for n in enc.values()),
           "spmm": sum(_m.ceil(n / 128) for n in sp.values()),
           "sddmm": sum(_m.ceil(n / 128) for n in sd.values()) + sum(_m.ceil(n / 32) for n in sd_dense.values())}
    return {"per_class": per, "total": sum(per.values())}


# Measured on-chip ceiling of the gather both kernels are made of (tools/gather_bench.cu,
# profiles/r01e_gather.md): random 128-byte rows, LDG.128 with 8 lanes per line, 64 warps/SM.
GATHER_PEAK_GBS = 20674.0


def gathered_bytes(p, nnz_v):
    """Bytes of the gathered dense operand that reach the SMs (rows of B panels in SpMM,
    rows of Bt in SDDMM): 2 * nnz_v * N per op (V flop per gathered byte)."""
    return {"encode": 0.0, "spmm": 2.0 * nnz_v * p.N, "sddmm": 2.0 * nnz_v * p.N}


# --------------------------------------------------------------- reference (oracle) arm

_INPUT_CACHE = {}


def layer_inputs(p):
    """Seeded host inputs of one layer problem (W dense, X, G), memoised."""
    from synth import gen
    if p.id not in _INPUT_CACHE:
        rng = gen.make_rng(p.id)
        Wd = gen.colvec_dense(rng, p.M, p.K, p.V, 1.0 - p.S, kind=p.kind)
        X = gen.dense_operand(rng, p.K, p.N)
        G = gen.dense_operand(rng, p.M, p.N)
        _INPUT_CACHE[p.id] = (Wd, X, G)
    return _INPUT_CACHE[p.id]


def oracle_sample_run(problems, seconds, threads=0, reps=1):
    """Runs the fp64 oracle (encode + SpMM + SDDMM of each layer problem, timed inside
    oracle.c with the monotonic clock, oracle.time_layer) over problems in order until
    ~seconds of CPU work; per problem the median of `reps` runs counts.
    Returns (flops, elapsed, n_problems)."""
    import oracle
    flops, t_used, n = 0.0, 0.0, 0
    for p in problems:
        Wd, X, G = layer_inputs(p)
        secs, nnz = oracle.time_layer(p.M, p.K, p.N, p.V, Wd, X, G, threads=threads, reps=reps)
        t_used += statistics.median(secs)
        f1, f2 = problem_flops(nnz, p)
        flops += f1 + f2
        n += 1
        if t_used * reps >= seconds:
            break
    return flops, t_used, n


def cpu_baseline_protocol(problems, seconds):
    """the oracle as it stands, all cores and one thread, median of 3 runs
    per problem (monotonic clock inside oracle.c), over a bounded interleaved sample of the
    workload (about `seconds` of CPU work per thread setting)."""
    import oracle
    cores = oracle.use_all_cores()
    f_all, t_all, n_all = oracle_sample_run(problems, seconds, threads=0, reps=3)
    # one thread on the same first problems (it takes ~cores x longer: fewer problems fit)
    f_one, t_one, n_one = oracle_sample_run(problems, seconds, threads=1, reps=3)
    return {"value": f_all / t_all / 1e12, "unit": UNIT, "cores": cores, "kind": "oracle",
            "sample": f"first {n_all} problems of the interleaved workload order (encode+SpMM+SDDMM, "
                      f"fp64 C oracle, median of 3 runs each, {t_all:.1f} s per run set)",
            "one_thread": {"value": f_one / t_one / 1e12, "unit": UNIT, "cores": 1,
                           "sample": f"first {n_one} problems, median of 3 runs each"},
            "timer": "clock_gettime(CLOCK_MONOTONIC) inside oracle.c (oracle_time_layer)"}


def sample_order(problems):
    """Deterministic interleaving so a bounded sample spans shapes, V and S."""
    return problems[::7] + [p for i, p in enumerate(problems) if i % 7]


def parity_gate(bufs, every=7, n_spmm=512, n_sddmm=256, replay=None):
    """Oracle gate on the outputs of the TIMED launch configuration:
    for every `every`-th problem of the batch, the GPU encoding (row_ptr, col_idx, vals) must
    equal the oracle encoder bit for bit, and sampled SpMM outputs Y[i][j] / SDDMM vectors dW[p]
    must be within 2e-3*sum|ab| + 2^-24 of the fp64 oracle.  Raises on any failure, so bench.py
    never prints a value for a step whose results are wrong."""
    import numpy as np
    import oracle
    worst, checked, ns, nd = 0.0, 0, 0, 0
    for j, b in enumerate(bufs):
        if j % every:
            continue
        p = b.p
        Wd, X, G = layer_inputs(p)
        rp = b.row_ptr.cpu().numpy()
        nnz = int(rp[-1])
        ci = b.col_idx[:nnz].cpu().numpy()
        va = b.vals[:nnz * p.V].cpu().numpy()
        orp, oci, ova = oracle.encode(p.M, p.K, p.V, dense=Wd)
        if not (np.array_equal(rp, orp) and np.array_equal(ci, oci)
                and np.array_equal(va.view(np.uint16), ova.view(np.uint16))):
            raise AssertionError(f"parity gate: encoding of {p.id} differs from the oracle")
        rng = np.random.default_rng(j)
        rows = rng.integers(0, p.M, n_spmm)
        cols = rng.integers(0, p.N, n_spmm)
        o, sc = oracle.spmm_sample(p.M, p.K, p.N, p.V, orp, oci, ova, X, rows, cols)
        Y = b.Y.cpu().numpy()
        e = np.abs(Y[rows, cols].astype(np.float64) - o) / oracle.tolerance(sc)
        if nnz:
            ps = rng.integers(0, nnz, n_sddmm)
            od, sd = oracle.sddmm_sample(p.M, p.K, p.N, p.V, orp, oci, G, X, ps)
            dW = b.dW[:nnz * p.V].cpu().numpy().reshape(-1, p.V)
            e2 = np.abs(dW[ps].astype(np.float64) - od) / oracle.tolerance(sd)
            e = np.concatenate([e.ravel(), e2.ravel()])
            nd += ps.size
        ns += rows.size
        worst = max(worst, float(e.max()) if e.size else 0.0)
        if worst > 1.0:
            raise AssertionError(f"parity gate: {p.id} outside the tolerance (ratio {worst:.3g})")
        checked += 1
    return {"problems_checked": checked, "of": len(bufs), "every": every,
            "encode": "bit-exact vs oracle.encode", "spmm_samples": ns, "sddmm_vectors": nd,
            "worst_err_over_tol": worst, "tolerance": "2e-3*sum|ab| + 2^-24",
            "outputs_of": "the timed graph (one extra replay after the timed region)"}


def run_reference(args):
    ws, rank, _ = dist_env()
    if rank != 0:
        return 0
    import oracle
    from synth.workloads import WORKLOADS
    oracle.use_all_cores()
    if args.workload == "c5":
        return run_reference_c5(args)
    problems = sample_order(WORKLOADS[args.workload]())
    per_step = max(2.0, min(20.0, 150.0 / max(1, args.steps + args.warmup)))
    for _ in range(args.warmup):
        oracle_sample_run(problems, per_step)
    vals, tot_t, tot_f, nprob = [], 0.0, 0.0, 0
    for _ in range(args.steps):
        f, t, n = oracle_sample_run(problems, per_step)
        vals.append(f / t / 1e12)
        tot_t += t
        tot_f += f
        nprob = n
    value = tot_f / tot_t / 1e12
    cores = oracle.num_threads()
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": UNIT,
        "n_gpus": ws, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": 1e3 * tot_t / max(1, args.steps), "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": args.workload, "sample": f"first {nprob} problems of the "
                   "interleaved workload order per step"},
        "cpu_baseline": {"value": value, "unit": UNIT, "cores": cores, "kind": "oracle",
                         "sample": f"{nprob} problems (~{per_step:.0f} s of fp64 oracle work) per step"},
        "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)
    return 0


def run_reference_c5(args):
    """Reference arm for configs[4]: the fp64 oracle on the deterministic C5 sample
    (c5_oracle_sample), one sample per step, throughput extrapolated in flops."""
    import oracle
    ws, _, _ = dist_env()
    for _ in range(args.warmup):
        c5_oracle_sample()
    tot_f, tot_t = 0.0, 0.0
    for _ in range(args.steps):
        f, t, desc = c5_oracle_sample()
        tot_f += f
        tot_t += t
    value = tot_f / tot_t / 1e12
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": ws,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * tot_t / max(1, args.steps),
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic", "config": {"workload": "c5", "sample": desc},
            "cpu_baseline": {"value": value, "unit": UNIT, "cores": oracle.num_threads(),
                             "kind": "oracle", "sample": desc},
            "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


# ------------------------------------------------------------------------ our arm

class LayerBuffers:
    """Device (and pinned host) buffers of one layer problem."""

    def __init__(self, p, torch, dev, with_host: bool):
        self.p = p
        Wd, X, G = layer_inputs(p)
        self.W = -(-p.M // p.V)
        self.cap = self.W * p.K
        self.Wd = torch.from_numpy(Wd).to(dev)
        self.X = torch.from_numpy(X).to(dev)
        self.G = torch.from_numpy(G).to(dev)
        self.row_ptr = torch.zeros(self.W + 1, dtype=torch.int32, device=dev)
        self.col_idx = torch.zeros(self.cap, dtype=torch.int32, device=dev)
        self.vals = torch.zeros(self.cap * p.V, dtype=torch.float16, device=dev)
        self.Y = torch.zeros((p.M, p.N), dtype=torch.float16, device=dev)
        self.dW = torch.zeros(self.cap * p.V, dtype=torch.float16, device=dev)
        if with_host:
            self.h_Wd = torch.from_numpy(Wd).pin_memory()
            self.h_X = torch.from_numpy(X).pin_memory()
            self.h_G = torch.from_numpy(G).pin_memory()
            self.h_Y = torch.empty((p.M, p.N), dtype=torch.float16).pin_memory()
            self.h_dW = None  # sized after the first encode
        self.nnz_v = None
        self.k_ref = None

    # the three ABI calls of one problem
    def encode(self, vs):
        p = self.p
        vs.vs_encode_colvec(p.M, p.K, p.V, self.Wd, None, self.row_ptr, self.col_idx, self.vals)

    def spmm(self, vs):
        p = self.p
        vs.vs_spmm(p.M, p.K, p.N, p.V, self.row_ptr, self.col_idx, self.vals, self.X, self.Y)

    def sddmm(self, vs):
        p = self.p
        vs.vs_sddmm(p.M, p.K, p.N, p.V, self.row_ptr, self.col_idx, self.G, self.X, self.dW)


def capture(torch, fn, stream):
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=stream):
        fn()
    return g


def time_graph(torch, g, stream, reps=1):
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with torch.cuda.stream(stream):
        s.record()
        for _ in range(reps):
            g.replay()
        e.record()
    e.synchronize()
    return s.elapsed_time(e) / reps


def run_ours(args):
    import numpy as np
    import torch
    import paper_conf_sc_chenqldx21_b200 as vs
    from synth.workloads import WORKLOADS

    ws, rank, local = dist_env()
    assert ws == args.gpus or ws == 1, f"--gpus {args.gpus} but WORLD_SIZE={ws}"
    if ws > 1:
        init_dist(torch, local)
    else:
        torch.cuda.set_device(0)
    dev = torch.device("cuda", torch.cuda.current_device())
    vs.load()
    peaks = load_peaks()
    problems = WORKLOADS[args.workload]()
    stream = torch.cuda.Stream()
    bufs = [LayerBuffers(p, torch, dev, with_host=not args.no_e2e) for p in problems]

    # eager pass: sizes (nnz_v, referenced columns) and a sanity check of the launch path
    with torch.cuda.stream(stream):
        for b in bufs:
            b.encode(vs)
            b.spmm(vs)
            b.sddmm(vs)
    stream.synchronize()
    for b in bufs:
        b.nnz_v = int(b.row_ptr[-1].item())
        ci = b.col_idx[:b.nnz_v].cpu().numpy()
        b.k_ref = int(np.unique(ci).size)
        if not args.no_e2e:
            b.h_dW = torch.empty(b.nnz_v * b.p.V, dtype=torch.float16).pin_memory()

    flops_spmm = sum(problem_flops(b.nnz_v, b.p)[0] for b in bufs)
    flops_sddmm = sum(problem_flops(b.nnz_v, b.p)[1] for b in bufs)
    flops_step = flops_spmm + flops_sddmm
    launches_per_step = count_launches(bufs)

    # the step through the batched C ABI: one encode batch, then the SpMM batch and (on a
    # forked graph branch, it only needs the encoding) the SDDMM batch
    enc_arr = vs.make_encode_batch([(b.p.M, b.p.K, b.p.V, b.Wd, None, b.row_ptr, b.col_idx, b.vals)
                                    for b in bufs])
    spmm_arr = vs.make_spmm_batch([(b.p.M, b.p.K, b.p.N, b.p.V, b.row_ptr, b.col_idx, b.vals, b.X, b.Y)
                                   for b in bufs])
    sddmm_arr = vs.make_sddmm_batch([(b.p.M, b.p.K, b.p.N, b.p.V, b.row_ptr, b.col_idx, b.G, b.X, b.dW)
                                     for b in bufs])
    side = torch.cuda.Stream()

    def step_batched(pre=None, post=None):
        cur = torch.cuda.current_stream()
        if pre:
            pre()
        vs.vs_encode_colvec_batched(enc_arr)
        side.wait_stream(cur)
        vs.vs_spmm_batched(spmm_arr)
        with torch.cuda.stream(side):
            vs.vs_sddmm_batched(sddmm_arr)
        cur.wait_stream(side)
        if post:
            post()

    # the same batched calls scheduled as one chain per V group (encode -> SpMM || SDDMM of
    # that group), the chains on concurrent graph branches: a group's SpMM/SDDMM overlap the
    # other groups' encode and fill each other's tails.  Same kernels, same work, same bits.
    groups = {}
    for b in bufs:
        groups.setdefault(b.p.V, []).append(b)
    chain_arrs = []
    for V in sorted(groups):
        gb = groups[V]
        chain_arrs.append((
            vs.make_encode_batch([(b.p.M, b.p.K, b.p.V, b.Wd, None, b.row_ptr, b.col_idx, b.vals) for b in gb]),
            vs.make_spmm_batch([(b.p.M, b.p.K, b.p.N, b.p.V, b.row_ptr, b.col_idx, b.vals, b.X, b.Y) for b in gb]),
            vs.make_sddmm_batch([(b.p.M, b.p.K, b.p.N, b.p.V, b.row_ptr, b.col_idx, b.G, b.X, b.dW) for b in gb])))
    # --priority: which chain streams get the high stream priority (captured into the graph's
    # kernel nodes): "first" = the V = 2 chain (its SDDMM and SpMM are the longest; default since
    # the dense-tile SDDMM: 0.829 -> 0.819 ms per step, profiles/r03_dense_sddmm.md), "sddmm" =
    # every SDDMM branch (round 1's default: 0.916 -> 0.902 ms, profiles/r01g_priority.md),
    # "encode" = every encode -> SpMM branch, "none" = all default.
    def _prio(i, side):
        hi = {"first": i == 0, "sddmm": side, "encode": not side}.get(args.priority, False)
        return torch.cuda.Stream(priority=-1) if hi else torch.cuda.Stream()
    chain_streams = [(_prio(i, False), _prio(i, True)) for i in range(len(chain_arrs))]

    def step_chains(pre=None, post=None):
        cur = torch.cuda.current_stream()
        if pre:
            pre()
        for (enc_a, sp_a, sd_a), (s_main, s_side) in zip(chain_arrs, chain_streams):
            s_main.wait_stream(cur)
            with torch.cuda.stream(s_main):
                vs.vs_encode_colvec_batched(enc_a)
                s_side.wait_stream(s_main)
                vs.vs_spmm_batched(sp_a)
            with torch.cuda.stream(s_side):
                vs.vs_sddmm_batched(sd_a)
        for s_main, s_side in chain_streams:
            cur.wait_stream(s_main)
            cur.wait_stream(s_side)
        if post:
            post()

    step_main, step_alt = ((step_chains, step_batched) if args.schedule == "chains"
                           else (step_batched, step_chains))

    # per-problem calls (single entry points) on 8 concurrent graph branches: comparison only
    branches = [torch.cuda.Stream() for _ in range(max(1, args.streams))]

    def step_per_problem():
        cur = torch.cuda.current_stream()
        for st in branches:
            st.wait_stream(cur)
        for i, b in enumerate(bufs):
            with torch.cuda.stream(branches[i % len(branches)]):
                b.encode(vs)
                b.spmm(vs)
                b.sddmm(vs)
        for st in branches:
            cur.wait_stream(st)

    # instrumented serial copy of the batched step: external events around each batched call
    ev = []

    def step_instr():
        for name, fn in (("encode", lambda: vs.vs_encode_colvec_batched(enc_arr)),
                         ("spmm", lambda: vs.vs_spmm_batched(spmm_arr)),
                         ("sddmm", lambda: vs.vs_sddmm_batched(sddmm_arr))):
            s0 = torch.cuda.Event(enable_timing=True, external=True)
            e0 = torch.cuda.Event(enable_timing=True, external=True)
            s0.record()
            fn()
            e0.record()
            ev.append((name, s0, e0))

    g_step = capture(torch, step_main, stream)
    g_alt = capture(torch, step_alt, stream)
    g_pp = capture(torch, step_per_problem, stream)
    g_instr = capture(torch, step_instr, stream)
    flush = torch.empty(512 * 1024 * 1024 // 4, dtype=torch.int32, device=dev)

    for i in range(args.warmup):
        with torch.cuda.stream(stream):
            flush.fill_(i)
            g_step.replay()
            g_alt.replay()
            g_pp.replay()
            g_instr.replay()
    stream.synchronize()

    # ---------------- timed region (max over ranks) ----------------
    if ws > 1:
        torch.distributed.barrier()
    torch.cuda.synchronize()
    props = torch.cuda.get_device_properties(dev)
    bus = None
    if hasattr(props, "pci_bus_id"):
        bus = "%08X:%02X:%02X.0" % (getattr(props, "pci_domain_id", 0), props.pci_bus_id,
                                   getattr(props, "pci_device_id", 0))
    clocks = ClockSampler(dev.index, bus).start()
    starts = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps)]
    ends = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps)]
    with torch.cuda.stream(stream):
        for i in range(args.steps):
            flush.fill_(i + 1)           # L2 flush, not timed
            starts[i].record()
            g_step.replay()
            ends[i].record()
    torch.cuda.synchronize()
    step_ms = [s0.elapsed_time(e0) for s0, e0 in zip(starts, ends)]
    alt_ms = []
    for i in range(args.steps):
        with torch.cuda.stream(stream):
            flush.fill_(i + 3)
        alt_ms.append(time_graph(torch, g_alt, stream))
    pp_ms = []
    for i in range(args.steps):
        with torch.cuda.stream(stream):
            flush.fill_(i + 5)
        pp_ms.append(time_graph(torch, g_pp, stream))
    # instrumented replays (same inputs) for the per-kernel attribution
    per_class = {"encode": [], "spmm": [], "sddmm": []}
    for i in range(args.steps):
        with torch.cuda.stream(stream):
            flush.fill_(i + 7)
            g_instr.replay()
        stream.synchronize()
        for name, s0, e0 in ev:
            per_class[name].append(s0.elapsed_time(e0))
    if ws > 1:
        torch.distributed.barrier()
    torch.cuda.synchronize()
    clk = clocks.stop()

    # per-class device times on stderr before the gate (kernel variants under study keep their
    # timings even when the gate rejects their outputs)
    print("classes_ms " + json.dumps({k: round(sum(v) / args.steps, 4) for k, v in per_class.items()}) +
          " step_ms %.4f" % (sum(step_ms) / args.steps), file=sys.stderr)
    # oracle gate on the timed launch configuration's outputs (raises on failure)
    with torch.cuda.stream(stream):
        g_step.replay()
    stream.synchronize()
    gate = parity_gate(bufs)

    total_ms = sum(step_ms)
    if ws > 1:
        t = torch.tensor([total_ms], device=dev, dtype=torch.float64)
        torch.distributed.all_reduce(t, op=torch.distributed.ReduceOp.MAX)
        total_ms = float(t.item())
    ms_per_step = total_ms / args.steps
    value = ws * flops_step / (ms_per_step * 1e-3) / 1e12
    ms_pp = sum(pp_ms) / args.steps

    # ---------------- kernel attribution + roofline ----------------
    nb = len(bufs)
    cls_ms = {k: sum(v) / args.steps for k, v in per_class.items()}
    instr_total = sum(cls_ms.values())
    dominant = max(("spmm", "sddmm", "encode"), key=lambda k: cls_ms[k])
    bytes_cls = {"encode": 0.0, "spmm": 0.0, "sddmm": 0.0}
    for b in bufs:
        for k, v in alg_bytes(b.p, b.nnz_v, b.k_ref).items():
            bytes_cls[k] += v
    flops_cls = {"encode": 0.0, "spmm": flops_spmm, "sddmm": flops_sddmm}
    n_launch = launches_per_step["per_class"][dominant]
    dom_avg_ms = cls_ms[dominant] / n_launch
    achieved_gbs = (bytes_cls[dominant] / n_launch) / (dom_avg_ms * 1e-3) / 1e9
    traffic = None
    tp = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if os.path.exists(tp):
        tr = json.load(open(tp)).get(f"{args.workload}:{dominant}")
        if tr is not None:
            traffic = tr / n_launch
    roofline = {"bound": "hbm", "achieved": achieved_gbs, "peak": peaks["hbm_gbs"],
                "unit": "GB/s", "frac": achieved_gbs / peaks["hbm_gbs"], "traffic": traffic,
                "kernel": dominant, "peak_source": peaks["source"],
                "launches_per_step": n_launch,
                "algorithmic_bytes_per_launch": bytes_cls[dominant] / n_launch,
                "avg_launch_us": dom_avg_ms * 1e3}
    tensor_tf = flops_cls[dominant] / (cls_ms[dominant] * 1e-3) / 1e12 if flops_cls[dominant] else 0.0
    roofline_tensor = {"bound": "tensor", "achieved": tensor_tf, "peak": peaks["bf16_tflops"],
                       "unit": "TFLOP/s", "frac": tensor_tf / peaks["bf16_tflops"],
                       "kernel": dominant}
    gath = sum(gathered_bytes(b.p, b.nnz_v)[dominant] for b in bufs)
    gath_gbs = gath / (cls_ms[dominant] * 1e-3) / 1e9 if cls_ms[dominant] else 0.0
    roofline_gather = {"bound": "l2_gather", "achieved": gath_gbs, "peak": GATHER_PEAK_GBS,
                       "unit": "GB/s", "frac": gath_gbs / GATHER_PEAK_GBS, "kernel": dominant,
                       "peak_source": "measured: tools/gather_bench.cu ldg_line (profiles/r01e_gather.md)",
                       "note": "the working set of the DLMC problems is L2-resident after the first "
                               "touch; the kernels are bound by the random-row gather into the SMs, "
                               "not by HBM (DESIGN.md 9)"}

    line = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": ws, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms_per_step, "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "f16", "data": "synthetic",
        "config": {"workload": args.workload, "problems": nb,
                   "shapes": ("(M,K) in {(512,512),(2048,512),(512,2048),(2048,1024)} x V{2,4,8} "
                              "x S{.5,.7,.9,.98} x N{64,128,256}") if args.workload == "dlmc_layer" else
                             ("same shapes x S{.5,.7,.8,.9,.95,.98}" if args.workload == "dlmc_grid"
                              else args.workload),
                   "step": "per problem: encode W -> SpMM Y=WX -> SDDMM dW=(G X^T) o pattern(W)",
                   "flops_per_step": flops_step, "l2": "flushed between timed steps (512 MiB write, untimed)",
                   "launch": "batched C ABI (vs_*_batched), step replayed as one CUDA graph; " + (
                             "one chain per V group (encode -> SpMM || SDDMM), chains on concurrent "
                             "graph branches" + (f", high stream priority: {args.priority}"
                                                 if args.priority != "none" else "")
                             if args.schedule == "chains" else
                             "encode batch, then SpMM batch || SDDMM batch"),
                   "accumulate": "fp32"},
        "alt_schedule": {"schedule": "phases" if args.schedule == "chains" else "chains",
                         "ms_per_step": sum(alt_ms) / args.steps,
                         "value": ws * flops_step / (sum(alt_ms) / args.steps * 1e-3) / 1e12},
        "per_problem_calls": {"ms_per_step": ms_pp, "value": ws * flops_step / (ms_pp * 1e-3) / 1e12,
                              "note": "same step through the single-problem entry points, "
                                      f"{len(branches)} concurrent graph branches"},
        "roofline": roofline,
        "roofline_tensor": roofline_tensor,
        "roofline_gather": roofline_gather,
        "kernels": {k: {"ms_per_step": v, "share": (v / instr_total if instr_total else None),
                        "launches_per_step": launches_per_step["per_class"][k],
                        "tflops": (flops_cls[k] / (v * 1e-3) / 1e12 if v and flops_cls[k] else None),
                        "alg_GBps": bytes_cls[k] / (v * 1e-3) / 1e9 if v else None}
                    for k, v in cls_ms.items()},
        "gpu_launches": launches_per_step["total"] * args.steps,
        "clocks": clk,
        "parity_gate": gate,
    }

    detail = {"problems": [], "step_ms": step_ms}
    for b in bufs:
        detail["problems"].append({**b.p.asdict(), "nnz_v": b.nnz_v, "k_ref": b.k_ref})

    # ---------------- end to end with host buffers ----------------
    if not args.no_e2e:
        def h2d():
            for b in bufs:
                b.Wd.copy_(b.h_Wd, non_blocking=True)
                b.X.copy_(b.h_X, non_blocking=True)
                b.G.copy_(b.h_G, non_blocking=True)

        def d2h():
            for b in bufs:
                b.h_Y.copy_(b.Y, non_blocking=True)
                b.h_dW.copy_(b.dW[:b.nnz_v * b.p.V], non_blocking=True)
        # serialized reference: every H2D copy, then the step, then every D2H copy
        g_e2e_serial = capture(torch, lambda: step_main(h2d, d2h), stream)

        # pipelined: the batch in `e2e_chunks` interleaved chunks, each chunk's chain (H2D of its
        # inputs -> encode batch -> SpMM batch || SDDMM batch -> D2H of its outputs) on its own
        # graph branch, so the copies of one chunk overlap the compute of another and the two
        # PCIe directions overlap each other.  Same calls, same bytes, same results.
        # Each chunk's inputs (W, X, G of its problems) live in ONE pinned host arena and ONE device
        # arena, its outputs (Y, then dW) in one device / host arena each: one H2D copy and two
        # D2H copies per chunk instead of 3 + 2 per problem.
        nch = max(1, min(args.e2e_chunks, len(bufs)))
        chunks = [bufs[i::nch] for i in range(nch)]
        arenas = []
        for c in chunks:
            n_in = sum(b.p.M * b.p.K + b.p.K * b.p.N + b.p.M * b.p.N for b in c)
            n_y = sum(b.p.M * b.p.N for b in c)
            n_dw = sum(b.nnz_v * b.p.V for b in c)
            a = {"h_in": torch.empty(n_in, dtype=torch.float16).pin_memory(),
                 "d_in": torch.empty(n_in, dtype=torch.float16, device=dev),
                 "d_y": torch.empty(n_y, dtype=torch.float16, device=dev),
                 "h_y": torch.empty(n_y, dtype=torch.float16).pin_memory(),
                 "d_dw": torch.empty(max(n_dw, 1), dtype=torch.float16, device=dev),
                 "h_dw": torch.empty(max(n_dw, 1), dtype=torch.float16).pin_memory(), "views": []}
            o_in = o_y = o_dw = 0
            for b in c:
                p = b.p
                views = {}
                for name, shape, src in (("Wd", (p.M, p.K), b.Wd), ("X", (p.K, p.N), b.X), ("G", (p.M, p.N), b.G)):
                    n = shape[0] * shape[1]
                    a["h_in"][o_in:o_in + n].copy_(src.reshape(-1).cpu())
                    views[name] = a["d_in"][o_in:o_in + n].view(shape)
                    o_in += n
                views["Y"] = a["d_y"][o_y:o_y + p.M * p.N].view(p.M, p.N)
                o_y += p.M * p.N
                views["dW"] = a["d_dw"][o_dw:o_dw + b.nnz_v * p.V]
                o_dw += b.nnz_v * p.V
                a["views"].append(views)
            a["n_dw"] = n_dw
            arenas.append(a)
        ch_arrs = [(vs.make_encode_batch([(b.p.M, b.p.K, b.p.V, v["Wd"], None, b.row_ptr, b.col_idx, b.vals)
                                          for b, v in zip(c, a["views"])]),
                    vs.make_spmm_batch([(b.p.M, b.p.K, b.p.N, b.p.V, b.row_ptr, b.col_idx, b.vals, v["X"], v["Y"])
                                        for b, v in zip(c, a["views"])]),
                    vs.make_sddmm_batch([(b.p.M, b.p.K, b.p.N, b.p.V, b.row_ptr, b.col_idx, v["G"], v["X"],
                                          v["dW"] if b.nnz_v else None) for b, v in zip(c, a["views"])]))
                   for c, a in zip(chunks, arenas)]
        nst = min(nch, 4)
        e2e_streams = [(torch.cuda.Stream(), torch.cuda.Stream(priority=-1)) for _ in range(nst)]

        def step_e2e_pipelined():
            cur = torch.cuda.current_stream()
            for i, (a, (ea, sa, da)) in enumerate(zip(arenas, ch_arrs)):
                s_main, s_side = e2e_streams[i % nst]
                s_main.wait_stream(cur)
                with torch.cuda.stream(s_main):
                    a["d_in"].copy_(a["h_in"], non_blocking=True)
                    vs.vs_encode_colvec_batched(ea)
                    s_side.wait_stream(s_main)
                    vs.vs_spmm_batched(sa)
                    a["h_y"].copy_(a["d_y"], non_blocking=True)
                with torch.cuda.stream(s_side):
                    vs.vs_sddmm_batched(da)
                    if a["n_dw"]:
                        a["h_dw"][:a["n_dw"]].copy_(a["d_dw"][:a["n_dw"]], non_blocking=True)
            for s_main, s_side in e2e_streams:
                cur.wait_stream(s_main)
                cur.wait_stream(s_side)
        g_e2e = capture(torch, step_e2e_pipelined, stream)
        with torch.cuda.stream(stream):
            g_e2e.replay()
            g_e2e_serial.replay()
        stream.synchronize()
        e2e_ms, e2e_serial_ms = [], []
        for i in range(args.steps):
            with torch.cuda.stream(stream):
                flush.fill_(i + 3)
            e2e_ms.append(time_graph(torch, g_e2e, stream))
            with torch.cuda.stream(stream):
                flush.fill_(i + 4)
            e2e_serial_ms.append(time_graph(torch, g_e2e_serial, stream))
        e2e_total = sum(e2e_ms)
        if ws > 1:
            t = torch.tensor([e2e_total], device=dev, dtype=torch.float64)
            torch.distributed.all_reduce(t, op=torch.distributed.ReduceOp.MAX)
            e2e_total = float(t.item())
        h2d_b = sum(2 * (b.p.M * b.p.K + b.p.K * b.p.N + b.p.M * b.p.N) for b in bufs)
        d2h_b = sum(2 * (b.p.M * b.p.N + b.nnz_v * b.p.V) for b in bufs)
        line["e2e"] = {"value": ws * flops_step / (e2e_total / args.steps * 1e-3) / 1e12,
                       "unit": UNIT, "h2d_bytes_per_step": h2d_b, "d2h_bytes_per_step": d2h_b,
                       "ms_per_step": e2e_total / args.steps,
                       "path": f"pinned host -> device copies, batched C-ABI calls, device -> pinned "
                               f"host, one CUDA graph; pipelined in {nch} interleaved chunks on "
                               f"{nst} branch pairs (copies of one chunk overlap compute of another); "
                               f"per chunk one H2D copy of its packed inputs and one D2H copy each "
                               f"of its packed Y and dW",
                       "serialized_ms_per_step": sum(e2e_serial_ms) / args.steps,
                       "serialized_note": "all H2D, then the step, then all D2H (round 1's e2e)"}

    # ---------------- same-box library baselines, per cell ----------------
    if not args.no_baselines and rank == 0:
        try:
            line.update(library_baselines(args, torch, vs, bufs, stream, detail))
        except Exception as exc:  # baselines are context; never fail the bench on them
            line["baselines_error"] = repr(exc)[:300]

    # ---------------- CPU oracle baseline ----------------
    if not args.no_cpu and rank == 0 and ws == 1:
        line["cpu_baseline"] = cpu_baseline_protocol(sample_order(problems), args.cpu_seconds)
    if rank == 0:
        os.makedirs(os.path.dirname(args.detail), exist_ok=True)
        json.dump(detail, open(args.detail, "w"), indent=1)
        print(json.dumps(line), flush=True)
    if ws > 1:
        torch.distributed.destroy_process_group()
    return 0


def geomean(xs):
    xs = [x for x in xs if x and x > 0 and math.isfinite(x)]
    return math.exp(sum(math.log(x) for x in xs) / len(xs)) if xs else None


def library_baselines(args, torch, vs, bufs, stream, detail):
    """Per-cell micro timings (each implementation captured as a graph of `reps` launches,
    L2 warm, same protocol for all): ours SpMM / SDDMM vs cublasHgemm / GemmEx on the dense
    M x K x N problem, cusparseSpMM (Blocked-ELL, CSR) and cusparseSDDMM (CSR)."""
    import numpy as np
    import baselines
    from synth import gen
    L = baselines.lib()
    h = L.bl_create()
    reps = args.reps
    sptr = stream.cuda_stream
    cells = {}
    for j, b in enumerate(bufs):
        p = b.p
        d = detail["problems"][j]
        Cd = torch.empty((p.M, p.N), dtype=torch.float16, device=b.X.device)

        def rep(fn):
            with torch.cuda.stream(stream):
                fn()  # eager warm-up (library workspaces are set up outside capture)
            stream.synchronize()

            def run():
                for _ in range(reps):
                    fn()
            g = capture(torch, run, stream)
            with torch.cuda.stream(stream):
                g.replay()
            return 1e3 * time_graph(torch, g, stream, reps=3) / reps  # us per launch

        t_spmm = rep(lambda: b.spmm(vs))
        t_sddmm = rep(lambda: b.sddmm(vs))
        ptr = lambda t: t.data_ptr()
        t_h = rep(lambda: L.bl_hgemm(h, p.M, p.N, p.K, ptr(b.Wd), ptr(b.X), ptr(Cd),
                                     torch.cuda.current_stream().cuda_stream))
        t_gx = rep(lambda: L.bl_gemmex(h, p.M, p.N, p.K, ptr(b.Wd), ptr(b.X), ptr(Cd),
                                       torch.cuda.current_stream().cuda_stream))
        d.update({"spmm_us_warm": t_spmm, "sddmm_us_warm": t_sddmm, "hgemm_us": t_h, "gemmex_us": t_gx})
        # cuSPARSE Blocked-ELL with block = V (reading R12)
        try:
            rng = gen.make_rng("bell_" + p.id)
            nb = max(1, int(round(p.K / p.V * (1.0 - p.S))))
            nbr = p.M // p.V
            ci = np.stack([np.sort(rng.choice(p.K // p.V, size=nb, replace=False)) for _ in range(nbr)]).astype(np.int32)
            ev = gen.fp16_values(rng, (p.M, nb * p.V))
            d_ci, d_ev = torch.from_numpy(ci).cuda(), torch.from_numpy(ev).cuda()
            st = ctypes_int()
            plan = L.bl_spmm_bell_plan(h, p.M, p.K, p.N, p.V, nb * p.V, ptr(d_ci), ptr(d_ev),
                                       ptr(b.X), ptr(Cd), sptr, st)
            if plan:
                t_bell = rep(lambda: L.bl_plan_run(plan))
                d["cusparse_bell_us"] = t_bell
                L.bl_plan_free(plan)
            else:
                d["cusparse_bell_status"] = st.value
        except Exception as exc:
            d["cusparse_bell_error"] = repr(exc)[:200]
        # scalar CSR (V-expanded) for cusparseSpMM / SDDMM
        try:
            rp = b.row_ptr.cpu().numpy().astype(np.int64)
            ci = b.col_idx[:b.nnz_v].cpu().numpy()
            W = len(rp) - 1
            rows_rp = [0]
            cols = []
            for w in range(W):
                seg = ci[rp[w]:rp[w + 1]]
                for r in range(p.V):
                    if w * p.V + r < p.M:
                        cols.append(seg)
                        rows_rp.append(rows_rp[-1] + seg.size)
            s_rp = torch.from_numpy(np.asarray(rows_rp, np.int32)).cuda()
            s_ci = torch.from_numpy(np.concatenate(cols).astype(np.int32) if cols else np.zeros(0, np.int32)).cuda()
            nnz_s = int(rows_rp[-1])
            s_v = torch.ones(max(nnz_s, 1), dtype=torch.float16, device=b.X.device)
            st = ctypes_int()
            plan = L.bl_spmm_csr_plan(h, p.M, p.K, p.N, nnz_s, ptr(s_rp), ptr(s_ci), ptr(s_v),
                                      ptr(b.X), ptr(Cd), sptr, st)
            if plan:
                d["cusparse_csr_spmm_us"] = rep(lambda: L.bl_plan_run(plan))
                L.bl_plan_free(plan)
            else:
                d["cusparse_csr_spmm_status"] = st.value
            Xt = b.X.t().contiguous()  # cuSPARSE SDDMM B operand [N x K] row-major
            for vt, tag, A_, B_ in ((0, "fp16", b.G, Xt), (1, "fp32", b.G.float(), Xt.float())):
                out = torch.empty(max(nnz_s, 1), dtype=A_.dtype, device=b.X.device)
                st = ctypes_int()
                plan = L.bl_sddmm_csr_plan(h, p.M, p.K, p.N, nnz_s, ptr(s_rp), ptr(s_ci), ptr(out),
                                           ptr(A_), ptr(B_), vt, sptr, st)
                if plan:
                    d[f"cusparse_sddmm_{tag}_us"] = rep(lambda: L.bl_plan_run(plan))
                    L.bl_plan_free(plan)
                    break
                d[f"cusparse_sddmm_{tag}_status"] = st.value
        except Exception as exc:
            d["cusparse_csr_error"] = repr(exc)[:200]
        key = (p.V, p.S)
        c = cells.setdefault(key, {"spmm_vs_h": [], "sddmm_vs_h": [], "spmm_vs_bell": [],
                                   "spmm_vs_best_cublas": [], "sddmm_vs_cusparse": []})
        c["spmm_vs_h"].append(t_h / t_spmm)
        c["sddmm_vs_h"].append(t_h / t_sddmm)
        c["spmm_vs_best_cublas"].append(min(t_h, t_gx) / t_spmm)
        if "cusparse_bell_us" in d:
            c["spmm_vs_bell"].append(d["cusparse_bell_us"] / t_spmm)
        sd = d.get("cusparse_sddmm_fp16_us") or d.get("cusparse_sddmm_fp32_us")
        if sd:
            c["sddmm_vs_cusparse"].append(sd / t_sddmm)
    L.bl_destroy(h)
    summary = {}
    for (V, S), c in sorted(cells.items()):
        summary[f"V{V}_S{S:.2f}"] = {k: (round(geomean(v), 3) if geomean(v) else None) for k, v in c.items()}
    # per-V crossover: the smallest sparsity from which every cell's geomean speedup >= 1
    crossover = {}
    for V in sorted({k[0] for k in cells}):
        Ss = sorted(S for (v, S) in cells if v == V)
        ent = {}
        for op, key in (("spmm_vs_hgemm", "spmm_vs_h"), ("spmm_vs_best_cublas", "spmm_vs_best_cublas"),
                        ("sddmm_vs_hgemm", "sddmm_vs_h")):
            wins = [S for S in Ss if (geomean(cells[(V, S)][key]) or 0) >= 1.0]
            # smallest S such that all S' >= S win
            cross = None
            for S in Ss:
                if all(S2 in wins for S2 in Ss if S2 >= S):
                    cross = S
                    break
            ent[op] = cross
        crossover[f"V{V}"] = ent
    all_spmm = [x for c in cells.values() for x in c["spmm_vs_h"]]
    all_sddmm = [x for c in cells.values() for x in c["sddmm_vs_h"]]
    return {"speedup_vs_cublas_hgemm": {
        "geomean_spmm": geomean(all_spmm), "geomean_sddmm": geomean(all_sddmm),
        "per_cell_geomean": summary,
        "crossover_sparsity": crossover,
        "protocol": f"{args.reps} launches per CUDA graph, L2 warm, per-launch mean; dense "
                    "counterpart = cublasHgemm M x K x N (both ops)"}}


def ctypes_int():
    import ctypes
    return ctypes.c_int(0)


C5_BLOCK = 4096  # B is generated in 4096-column blocks: the same global B for every world size


def c5_plan(ws: int, rank: int, mask_row_ptr=None):
    """Host-side partition of configs[4]: SpMM N-panels of B / C (widths whole
    generator blocks, dist.panel_bounds) and SDDMM row windows balanced by stored vectors
    (dist.window_bounds on the global mask's row_ptr).  Pure bookkeeping (gloo-tested)."""
    from paper_conf_sc_chenqldx21_b200 import dist as vsd
    M = K = 16384
    N, V, S = 65536, 8, 0.9
    W = M // V
    pb = vsd.panel_bounds(N, ws, align=C5_BLOCK)
    plan = {"M": M, "K": K, "N": N, "V": V, "S": S, "W": W, "panel_bounds": pb,
            "n0": pb[rank], "n1": pb[rank + 1]}
    if mask_row_ptr is not None:
        wb = vsd.window_bounds(mask_row_ptr, ws, align=128 // V)
        sh = vsd.sddmm_shard(mask_row_ptr, M, V, wb, rank)
        plan.update({"window_bounds": wb, "shard": sh})
    return plan


def run_c5(args):
    """configs[4]: M=K=16384, N=65536, V=8, S=0.9.  SpMM sharded over N-panels of B/C (A
    replicated) and SDDMM (mask 16384 x 65536, inner K=16384) sharded over row windows balanced
    by stored vectors (dist.window_bounds; Bt replicated), no collective on the data path
    (SURVEY §8(e)).  Strong scaling: the total problem is fixed; every rank generates the same
    global operands (seeded) and computes its shard.  Timed separately: the optional replicated
    output, through NCCL (gather_panels / gather_segments) and through the fused SpMM scatter
    epilogue into symmetric memory (dist.spmm_npanel_replicated).  Same-box dense cuBLAS
    (Hgemm, GemmEx) on this rank's dense counterpart.  Inputs are far larger than L2."""
    import numpy as np
    import torch
    import paper_conf_sc_chenqldx21_b200 as vs
    from paper_conf_sc_chenqldx21_b200 import dist as vsd
    from synth import gen

    ws, rank, local = dist_env()
    if ws > 1:
        init_dist(torch, local)
    else:
        torch.cuda.set_device(0)
    dev = torch.device("cuda", torch.cuda.current_device())
    vs.load()
    peaks = load_peaks()
    plan = c5_plan(ws, rank)
    M, K, N, V, S, W = (plan[k] for k in ("M", "K", "N", "V", "S", "W"))
    n0, n1 = plan["n0"], plan["n1"]
    Np = n1 - n0
    # ---- SpMM shard: A replicated, this rank's N-panel of the global B (4096-column blocks)
    Ad = gen.torch_colvec_dense(M, K, V, 1 - S, seed=gen.config_seed("c5_A"), device=dev)
    Bp = torch.empty((K, Np), dtype=torch.float16, device=dev)
    for blk in range(n0 // C5_BLOCK, -(-n1 // C5_BLOCK)):
        c0, c1 = blk * C5_BLOCK, min(N, (blk + 1) * C5_BLOCK)
        Bp[:, c0 - n0:c1 - n0] = gen.torch_dense_operand(K, c1 - c0, seed=gen.config_seed(f"c5_Bblk_{blk}"),
                                                         device=dev)
    Cp = torch.empty((M, Np), dtype=torch.float16, device=dev)
    capA = W * K
    rpA = torch.empty(W + 1, dtype=torch.int32, device=dev)
    ciA = torch.empty(capA, dtype=torch.int32, device=dev)
    vaA = torch.empty(capA * V, dtype=torch.float16, device=dev)
    # ---- SDDMM: the global mask (same seed on every rank) -> its row_ptr -> balanced windows
    g = torch.Generator(device=dev)
    g.manual_seed(gen.config_seed("c5_mask"))
    keep = torch.rand((W, N), generator=g, device=dev) < (1 - S)
    mask = keep.repeat_interleave(V, dim=0).to(torch.uint8).contiguous()
    del keep
    rp_glob = torch.empty(W + 1, dtype=torch.int32, device=dev)
    vs.vs_encode_colvec(M, N, V, None, mask, rp_glob)              # count mode (setup)
    plan = c5_plan(ws, rank, rp_glob.cpu().numpy())
    sh = plan["shard"]
    Ml = sh.row1 - sh.row0
    maskl = mask[sh.row0:sh.row1]                                  # contiguous row slice
    A_sd = gen.torch_dense_operand(M, K, seed=gen.config_seed("c5_Asd"), device=dev)
    Al = A_sd[sh.row0:sh.row1]
    Bt = gen.torch_dense_operand(N, K, seed=gen.config_seed("c5_Bt"), device=dev)
    nnzM = sh.p1 - sh.p0
    rpM = torch.empty(sh.w1 - sh.w0 + 1, dtype=torch.int32, device=dev)
    ciM = torch.empty(max(nnzM, 1), dtype=torch.int32, device=dev)
    outM = torch.empty(max(nnzM, 1) * V, dtype=torch.float16, device=dev)

    def step():
        vs.vs_encode_colvec(M, K, V, Ad, None, rpA, ciA, vaA)
        vs.vs_spmm(M, K, Np, V, rpA, ciA, vaA, Bp, Cp)
        vs.vs_encode_colvec(Ml, N, V, None, maskl, rpM, ciM, None)
        vs.vs_sddmm(Ml, N, K, V, rpM, ciM, Al, Bt, outM)

    stream = torch.cuda.Stream()
    with torch.cuda.stream(stream):
        step()
    stream.synchronize()
    nnzA = int(rpA[-1].item())
    assert int(rpM[-1].item()) == nnzM, "local mask encoding disagrees with the global row_ptr"
    assert torch.equal(rpM.cpu(), torch.from_numpy(sh.row_ptr.astype(np.int32))), "shard row_ptr"
    flops = 2.0 * nnzA * V * Np + 2.0 * nnzM * V * K
    ev = {k: (torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
          for k in ("encA", "spmm", "encM", "sddmm")}

    def step_instr():
        for k, fn in (("encA", lambda: vs.vs_encode_colvec(M, K, V, Ad, None, rpA, ciA, vaA)),
                      ("spmm", lambda: vs.vs_spmm(M, K, Np, V, rpA, ciA, vaA, Bp, Cp)),
                      ("encM", lambda: vs.vs_encode_colvec(Ml, N, V, None, maskl, rpM, ciM, None)),
                      ("sddmm", lambda: vs.vs_sddmm(Ml, N, K, V, rpM, ciM, Al, Bt, outM))):
            ev[k][0].record()
            fn()
            ev[k][1].record()

    for _ in range(args.warmup):
        with torch.cuda.stream(stream):
            step()
    stream.synchronize()
    if ws > 1:
        torch.distributed.barrier()
    torch.cuda.synchronize()
    clocks = ClockSampler(dev.index).start()
    s0, e0 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with torch.cuda.stream(stream):
        s0.record()
        for _ in range(args.steps):
            step()
        e0.record()
    e0.synchronize()
    ms = s0.elapsed_time(e0) / args.steps
    cls = {k: 0.0 for k in ev}
    for _ in range(2):
        with torch.cuda.stream(stream):
            step_instr()
        stream.synchronize()
        for k, (a, b) in ev.items():
            cls[k] += a.elapsed_time(b) / 2
    if ws > 1:
        torch.distributed.barrier()
    clk = clocks.stop()
    tot_flops = flops
    if ws > 1:
        t = torch.tensor([ms], device=dev, dtype=torch.float64)
        torch.distributed.all_reduce(t, op=torch.distributed.ReduceOp.MAX)
        ms = float(t.item())
        f = torch.tensor([flops], device=dev, dtype=torch.float64)
        torch.distributed.all_reduce(f)
        tot_flops = float(f.item())
    value = tot_flops / (ms * 1e-3) / 1e12

    # ---- parity: sampled outputs of this rank's shard against the fp64 oracle
    gate = c5_parity_gate(rank, M, K, N, V, n0, Np, rpA, ciA, vaA, Bp, Cp, sh, ciM, Al, Bt, outM)

    # ---- replicated output (optional for callers; timed apart from the step)
    rep_out = None
    if ws > 1:
        rep_out = c5_replicated_output(args, torch, vs, vsd, plan, rpA, ciA, vaA, Bp, Cp, outM, nnzM,
                                       stream, dev)

    # ---- same-box dense cuBLAS on this rank's dense counterpart (M x K x Np)
    dense = c5_dense_cublas(torch, Ad, Bp, Cp, stream) if not args.no_baselines else None

    kref = K  # every column of B is referenced at 10% density over 2048 windows
    bytes_spmm = 4 * (W + 1) + nnzA * (4 + 2 * V) + 2 * kref * Np + 2 * M * Np
    bytes_sddmm = 4 * (sh.w1 - sh.w0 + 1) + 4 * nnzM + 2 * Ml * K + 2 * N * K + 2 * nnzM * V
    dom = "spmm" if cls["spmm"] >= cls["sddmm"] else "sddmm"
    db = bytes_spmm if dom == "spmm" else bytes_sddmm
    ach = db / (cls[dom] * 1e-3) / 1e9
    flops_dom = 2.0 * nnzA * V * Np if dom == "spmm" else 2.0 * nnzM * V * K
    gb = 2.0 * nnzA * Np if dom == "spmm" else 2.0 * nnzM * K
    line = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": ws, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True, "scaling": "strong",
        "vs_baseline": None, "dtype": "f16", "data": "synthetic",
        "config": {"workload": "c5", "M": M, "K": K, "N": N, "V": V, "S": S,
                   "step": "encode A, SpMM on this rank's N-panel (A replicated); encode this "
                           "rank's mask rows, SDDMM (mask 16384x65536, inner 16384, Bt replicated)",
                   "l2": "inputs far larger than L2 (no flush)", "nnz_v_spmm": nnzA,
                   "nnz_v_sddmm_this_rank": nnzM, "panel": [n0, n1],
                   "windows": [sh.w0, sh.w1],
                   "parallelism": f"spmm N-panels x{ws} (dist.panel_bounds), sddmm row windows x{ws} "
                                  "(dist.window_bounds, balanced by stored vectors)"},
        "roofline": {"bound": "hbm", "achieved": ach, "peak": peaks["hbm_gbs"], "unit": "GB/s",
                     "frac": ach / peaks["hbm_gbs"], "traffic": None, "kernel": dom,
                     "algorithmic_bytes_per_launch": db, "avg_launch_us": cls[dom] * 1e3,
                     "peak_source": peaks["source"]},
        "roofline_tensor": {"bound": "tensor", "achieved": flops_dom / (cls[dom] * 1e-3) / 1e12,
                            "peak": peaks["bf16_tflops_sustained"], "unit": "TFLOP/s",
                            "frac": flops_dom / (cls[dom] * 1e-3) / 1e12 / peaks["bf16_tflops_sustained"],
                            "kernel": dom, "peak_source": "sustained dense bf16 (MEASURED_PEAKS.json)"},
        "roofline_gather": {"bound": "l2_gather", "achieved": gb / (cls[dom] * 1e-3) / 1e9,
                            "peak": GATHER_PEAK_GBS, "unit": "GB/s",
                            "frac": gb / (cls[dom] * 1e-3) / 1e9 / GATHER_PEAK_GBS, "kernel": dom,
                            "peak_source": "measured: tools/gather_bench.cu ldg_line (profiles/r01e_gather.md)"},
        "kernels": {k: {"ms": v} for k, v in cls.items()},
        # per step: encode A (count, scan, compact), SpMM, encode the mask rows (count, scan, compact
        # without values), the dense-tile SDDMM launch (inner K >= 256: its CTAs find no dense block
        # at 10 % density / V = 8 and exit) and the gather SDDMM
        "gpu_launches": 9 * args.steps,
        "clocks": clk,
        "parity_gate": gate,
        "replicated_output": rep_out,
        "dense_cublas_this_rank": dense,
        "e2e": None,
    }
    if dense:
        line["speedup_vs_cublas_hgemm"] = {
            "spmm": dense["hgemm_ms"] / cls["spmm"], "sddmm": dense["hgemm_ms"] * (Ml / M) / cls["sddmm"],
            "spmm_vs_best_cublas": min(dense["hgemm_ms"], dense["gemmex_ms"]) / cls["spmm"],
            "step_vs_dense_pair": 2 * min(dense["hgemm_ms"], dense["gemmex_ms"]) / ms,
            "note": "dense counterpart of this rank's SpMM = M x K x Np GEMM; of its SDDMM = the "
                    "same GEMM restricted to its rows (Ml/M of it); step_vs_dense_pair compares "
                    "the step with two dense GEMMs (forward + weight gradient)"}
    if not args.no_e2e:
        line["e2e"] = c5_e2e(torch, step, stream, [Ad, Bp, maskl, Al, Bt], [Cp, outM[:nnzM * V]],
                             tot_flops, ws, dev)
    if not args.no_cpu and rank == 0 and ws == 1:
        line["cpu_baseline"] = c5_cpu_baseline(args.cpu_seconds)
    if rank == 0:
        print(json.dumps(line), flush=True)
    if ws > 1:
        torch.distributed.destroy_process_group()
    return 0


def c5_parity_gate(rank, M, K, N, V, n0, Np, rpA, ciA, vaA, Bp, Cp, sh, ciM, Al, Bt, outM,
                   n_spmm=2048, n_sddmm=256):
    """Sampled oracle check of the timed C5 launch on this rank (the full problem is too large
    for the host): SpMM outputs C[i][n0 + j] and SDDMM stored vectors of this rank's windows,
    against oracle.spmm_sample / sddmm_sample (2e-3*sum|ab| + 2^-24).  Raises on failure."""
    import numpy as np
    import torch
    import oracle
    nnzA = int(rpA[-1].item())
    rng = np.random.default_rng(11 + rank)
    rows = rng.integers(0, M, n_spmm)
    cols = rng.integers(0, Np, n_spmm)
    ucols = np.unique(cols)
    Bsub = Bp[:, torch.from_numpy(ucols).to(Bp.device)].cpu().numpy()
    o, s = oracle.spmm_sample(M, K, ucols.size, V, rpA.cpu().numpy(), ciA[:nnzA].cpu().numpy(),
                              vaA[:nnzA * V].cpu().numpy(), Bsub, rows, np.searchsorted(ucols, cols))
    g = Cp[torch.from_numpy(rows).to(Cp.device), torch.from_numpy(cols).to(Cp.device)].cpu().numpy()
    e1 = np.abs(g.astype(np.float64) - o) / oracle.tolerance(s)
    nnzM = sh.p1 - sh.p0
    worst = float(e1.max())
    if nnzM:
        ps = rng.integers(0, nnzM, n_sddmm)
        ci = ciM[:nnzM].cpu().numpy()
        used = np.unique(ci[ps])
        Btsub = Bt[torch.from_numpy(used).to(Bt.device)].cpu().numpy()
        remap = np.zeros(N, np.int32)
        remap[used] = np.arange(used.size, dtype=np.int32)
        od, sd = oracle.sddmm_sample(sh.row1 - sh.row0, used.size, K, V, sh.row_ptr, remap[ci],
                                     Al.cpu().numpy(), Btsub, ps)
        gd = outM.view(-1, V)[torch.from_numpy(ps).to(outM.device)].cpu().numpy()
        worst = max(worst, float((np.abs(gd.astype(np.float64) - od) / oracle.tolerance(sd)).max()))
    if worst > 1.0:
        raise AssertionError(f"C5 parity gate failed on rank {rank}: err/tol {worst:.3g}")
    return {"spmm_samples": n_spmm, "sddmm_vectors": n_sddmm if nnzM else 0,
            "worst_err_over_tol": worst, "tolerance": "2e-3*sum|ab| + 2^-24",
            "oracle": "oracle.spmm_sample / sddmm_sample on this rank's shard"}


def c5_replicated_output(args, torch, vs, vsd, plan, rpA, ciA, vaA, Bp, Cp, outM, nnzM, stream, dev):
    """Replicated outputs of the sharded C5 (caller option), each timed
    with CUDA events over `reps` rounds, max over ranks:
      nccl_allgather_ms : gather_panels (all_gather_into_tensor + permute into row-major C)
      scatter_spmm_ms   : the SpMM whose epilogue stores into every rank's symmetric-memory C
                          (vs_spmm_scatter) + the stream barrier -- compare with spmm_ms +
                          nccl_allgather_ms, the unfused pair
      sddmm_allgather_ms: gather_segments of the out_vals segments."""
    import torch.distributed as dist
    M, K, V = plan["M"], plan["K"], plan["V"]
    pb, n0, n1 = plan["panel_bounds"], plan["n0"], plan["n1"]
    Np = n1 - n0
    counts = [int(plan["shard"].p1 - plan["shard"].p0)]
    allc = [None] * dist.get_world_size()
    dist.all_gather_object(allc, counts[0])  # (host objects: any backend)
    counts = [c * V for c in allc]
    reps = 3
    out = {"world": dist.get_world_size(), "reps": reps}

    def timed(fn):
        torch.cuda.synchronize()
        dist.barrier()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        with torch.cuda.stream(stream):
            fn()  # warm
            a.record()
            for _ in range(reps):
                fn()
            b.record()
        b.synchronize()
        t = torch.tensor([a.elapsed_time(b) / reps], device=dev, dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    out["spmm_ms"] = timed(lambda: vs.vs_spmm(M, K, Np, V, rpA, ciA, vaA, Bp, Cp))
    try:
        out["nccl_allgather_ms"] = timed(lambda: vsd.gather_panels(Cp, pb))
        out["sddmm_allgather_ms"] = timed(lambda: vsd.gather_segments(outM[:nnzM * V], counts))
    except Exception as exc:  # (a backend without all_gather_into_tensor: report, do not fail)
        out["allgather_error"] = repr(exc)[:300]
    try:
        rep = vsd.ReplicatedC(M, plan["N"], dev)
        out["scatter_spmm_ms"] = timed(lambda: vsd.spmm_npanel_replicated(rpA, ciA, vaA, Bp, M, V, pb,
                                                                          dist.get_rank(), rep))
        # parity: the fused replica equals the NCCL-gathered one bit for bit
        full = vsd.gather_panels(Cp, pb)
        torch.cuda.synchronize()
        out["scatter_equals_allgather"] = bool(torch.equal(full.view(torch.int16), rep.C.view(torch.int16)))
        out["unfused_pair_ms"] = out["spmm_ms"] + out.get("nccl_allgather_ms", float("nan"))
    except Exception as exc:  # symmetric memory needs a capable NCCL / driver; report, do not fail
        out["scatter_error"] = repr(exc)[:300]
    return out


def c5_dense_cublas(torch, Ad, Bp, Cp, stream, reps=3):
    """cublasHgemm / cublasGemmEx (fp32 compute) of the dense M x K x Np product on this rank,
    CUDA events, mean of `reps` after one warm-up (paper's comparison point)."""
    import baselines
    L = baselines.lib()
    h = L.bl_create()
    M, K = Ad.shape
    Np = Bp.shape[1]
    out = {}
    try:
        for name, fn in (("hgemm_ms", L.bl_hgemm), ("gemmex_ms", L.bl_gemmex)):
            with torch.cuda.stream(stream):
                fn(h, M, Np, K, Ad.data_ptr(), Bp.data_ptr(), Cp.data_ptr(), stream.cuda_stream)
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record()
                for _ in range(reps):
                    fn(h, M, Np, K, Ad.data_ptr(), Bp.data_ptr(), Cp.data_ptr(), stream.cuda_stream)
                b.record()
            b.synchronize()
            out[name] = a.elapsed_time(b) / reps
        out["dense_tflops_hgemm"] = 2.0 * M * K * Np / (out["hgemm_ms"] * 1e-3) / 1e12
        out["dense_tflops_gemmex"] = 2.0 * M * K * Np / (out["gemmex_ms"] * 1e-3) / 1e12
        out["shape"] = [M, K, Np]
    finally:
        L.bl_destroy(h)
    return out


def c5_e2e(torch, step, stream, inputs, outputs, tot_flops, ws, dev, reps=2):
    """End to end through the public API: pinned host -> device copies of this rank's inputs,
    the step, device -> pinned host copies of its outputs, all inside the timed region."""
    try:
        h_in = [t.cpu().pin_memory() for t in inputs]
        h_out = [torch.empty(t.shape, dtype=t.dtype).pin_memory() for t in outputs]
    except Exception as exc:
        return {"value": None, "error": f"pinned host buffers: {exc!r}"[:200]}

    def run():
        for d, h in zip(inputs, h_in):
            d.copy_(h, non_blocking=True)
        step()
        for d, h in zip(outputs, h_out):
            h.copy_(d, non_blocking=True)
    with torch.cuda.stream(stream):
        run()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        for _ in range(reps):
            run()
        b.record()
    b.synchronize()
    ms = a.elapsed_time(b) / reps
    if ws > 1:
        t = torch.tensor([ms], device=dev, dtype=torch.float64)
        torch.distributed.all_reduce(t, op=torch.distributed.ReduceOp.MAX)
        ms = float(t.item())
    return {"value": tot_flops / (ms * 1e-3) / 1e12, "unit": UNIT, "ms_per_step": ms,
            "h2d_bytes_per_step": int(sum(t.numel() * t.element_size() for t in inputs)),
            "d2h_bytes_per_step": int(sum(t.numel() * t.element_size() for t in outputs)),
            "path": "pinned host -> device, step (vs_encode_colvec, vs_spmm, vs_sddmm), device -> pinned host"}


def c5_oracle_sample(seconds_hint=None):
    """The fp64 oracle on a deterministic sample of configs[4]: SpMM of
    4 windows x 2048 output columns and SDDMM of 4 windows x all their stored vectors, with
    host-generated inputs of the C5 distribution (V = 8, density 0.1, K = 16384).  Returns
    (flops, seconds, description); throughput extrapolates linearly in flops."""
    import numpy as np
    import oracle
    from synth import gen
    K, V, d, Ns = 16384, 8, 0.1, 2048
    rng = gen.make_rng("c5_cpu_sample")
    Ms = 4 * V
    A = gen.colvec_dense(rng, Ms, K, V, d)
    B = gen.dense_operand(rng, K, Ns)
    t0 = time.perf_counter()
    rp, ci, va = oracle.encode(Ms, K, V, dense=A)
    oracle.spmm(Ms, K, Ns, V, rp, ci, va, B)
    t_spmm = time.perf_counter() - t0
    f_spmm = 2.0 * int(rp[-1]) * V * Ns
    # SDDMM: 8 windows of the 16384 x 65536 mask, all their vectors; Bt rows restricted to the
    # columns they reference (the oracle reads only those)
    Nm = 65536
    mask = gen.colvec_mask(rng, Ms, Nm, V, d)
    mrp, mci, _ = oracle.encode(Ms, Nm, V, mask=mask)
    used = np.unique(mci)
    remap = np.zeros(Nm, np.int32)
    remap[used] = np.arange(used.size, dtype=np.int32)
    Al = gen.dense_operand(rng, Ms, K)
    Bt = gen.dense_operand(rng, used.size, K)
    t0 = time.perf_counter()
    oracle.sddmm(Ms, used.size, K, V, mrp, remap[mci], Al, Bt)
    t_sd = time.perf_counter() - t0
    f_sd = 2.0 * int(mrp[-1]) * V * K
    return (f_spmm + f_sd, t_spmm + t_sd,
            "C5 sample: SpMM 4 windows x 2048 columns + SDDMM 4 windows x all stored vectors "
            "(host-generated inputs of the C5 distribution), extrapolated linearly in flops")


def c5_cpu_baseline(seconds):
    import oracle
    oracle.use_all_cores()
    f, t, desc = c5_oracle_sample()
    return {"value": f / t / 1e12, "unit": UNIT, "cores": oracle.num_threads(), "kind": "oracle",
            "sample": desc + f" ({t:.1f} s, all cores, time.perf_counter)", "extrapolated": True}


def run_attention(args):
    """NEXT item, the Fig. 20 analogue: sparse multi-head attention of Eq. 1
     on band-256 + random V x 1 masks, batch 8 x 4 heads.
    Workload name: attention_l<l>_k<k>_s<S>[_v<V>] (default l=4096, k=64, S=0.9, V=8).
    Step = SDDMM batch (scores) -> softmax batch -> SpMM batch, one CUDA graph.  Compared
    with dense fp16 attention (torch: cuBLAS matmul, masked softmax, matmul) on the same box."""
    import math
    import re
    import torch
    import paper_conf_sc_chenqldx21_b200 as vs
    from synth import gen

    m = re.match(r"attention(?:_l(\d+))?(?:_k(\d+))?(?:_s([0-9.]+))?(?:_v(\d+))?$", args.workload)
    l = int(m.group(1) or 4096)
    k = int(m.group(2) or 64)
    S = float(m.group(3) or 0.9)
    V = int(m.group(4) or 8)
    heads = 32
    torch.cuda.set_device(0)
    dev = torch.device("cuda", 0)
    vs.load()
    rng = gen.make_rng(f"attn_l{l}_s{S}_v{V}")
    mask = torch.from_numpy(gen.attention_mask(rng, l, V, S)).to(dev)  # one mask for all heads
    rp, ci, _ = vs.encode(V, mask=mask)
    nnz = int(rp[-1].item())
    Qs = [gen.torch_dense_operand(l, k, seed=gen.config_seed(f"q{h}"), device=dev) for h in range(heads)]
    Ks = [gen.torch_dense_operand(l, k, seed=gen.config_seed(f"k{h}"), device=dev) for h in range(heads)]
    Vs = [gen.torch_dense_operand(l, k, seed=gen.config_seed(f"v{h}"), device=dev) for h in range(heads)]
    Ss = [torch.empty(nnz * V, dtype=torch.float16, device=dev) for _ in range(heads)]
    Os = [torch.empty((l, k), dtype=torch.float16, device=dev) for _ in range(heads)]
    scale = 1.0 / math.sqrt(k)
    sd = vs.make_sddmm_batch([(l, l, k, V, rp, ci, Qs[h], Ks[h], Ss[h]) for h in range(heads)])
    sm = vs.make_softmax_batch([(l, V, scale, rp, Ss[h], Ss[h]) for h in range(heads)])
    sp = vs.make_spmm_batch([(l, l, k, V, rp, ci, Ss[h], Vs[h], Os[h]) for h in range(heads)])

    def step():
        vs.vs_sddmm_batched(sd)
        vs.vs_softmax_colvec_batched(sm)
        vs.vs_spmm_batched(sp)

    Qd = torch.stack(Qs)
    Kd = torch.stack(Ks)
    Vd = torch.stack(Vs)
    neg = torch.zeros((l, l), dtype=torch.float16, device=dev).masked_fill(mask == 0, float("-inf"))

    def dense():
        a = torch.matmul(Qd, Kd.transpose(1, 2)) * scale + neg
        return torch.matmul(torch.softmax(a, dim=-1), Vd)

    stream = torch.cuda.Stream()
    g = capture(torch, step, stream)
    with torch.cuda.stream(stream):
        for _ in range(args.warmup):
            g.replay()
        dense()
    stream.synchronize()
    gd = capture(torch, dense, stream)
    clocks = ClockSampler(0).start()
    t_sparse = min(time_graph(torch, g, stream) for _ in range(max(1, args.steps)))
    t_dense = min(time_graph(torch, gd, stream) for _ in range(max(1, args.steps)))
    clk = clocks.stop()
    flops = heads * (2.0 * nnz * V * k) * 2  # SDDMM + SpMM (softmax not counted)
    line = {"metric": METRIC, "value": flops / (t_sparse * 1e-3) / 1e12, "unit": UNIT, "n_gpus": 1,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": t_sparse,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f16",
            "data": "synthetic",
            "config": {"workload": args.workload, "l": l, "k": k, "sparsity": S, "V": V,
                       "heads_x_batch": heads, "mask": "band 256 + random (P:1560-1566)",
                       "nnz_v": nnz, "l2": "warm (per-step graph timing, min of steps)"},
            "dense_attention_ms": t_dense, "speedup_vs_dense": t_dense / t_sparse,
            "gpu_launches": 3 * args.steps, "clocks": clk, "e2e": None}
    print(json.dumps(line), flush=True)
    return 0


def run_train(args):
    """NEXT items: one training step of sparse layers with square V x V block
    patterns (§8 Case 1): per layer, W^T's values refreshed from W's on the
    device (vs_transpose_colvec_values; the pattern of W^T is built once by
    vs_transpose_colvec, W's values change every step), Y = W X (vs_spmm), dX = W^T dY
    (vs_spmm on the transposed encoding), dW = (dY X^T) o pattern(W) (vs_sddmm).  Workload
    name: train[_s<S>] (default S = 0.9); layers = the DLMC (M, K) shapes x V in {2, 4, 8},
    batch N = 256.  Compared with the dense fp16 step (torch.matmul: W X, W^T dY, dY X^T)."""
    import re
    import torch
    import paper_conf_sc_chenqldx21_b200 as vs
    from synth import gen
    from synth.workloads import DLMC_MK

    m = re.match(r"train(?:_s([0-9.]+))?$", args.workload)
    S = float(m.group(1) or 0.9)
    N = 256
    torch.cuda.set_device(0)
    dev = torch.device("cuda", 0)
    vs.load()
    layers = []
    for (M, K) in DLMC_MK:
        for V in (2, 4, 8):
            rng = gen.make_rng(f"train_{M}_{K}_{V}_{S}")
            Wd = torch.from_numpy(gen.block_dense(rng, M, K, V, 1 - S)).to(dev)
            X = torch.from_numpy(gen.dense_operand(rng, K, N)).to(dev)
            dY = torch.from_numpy(gen.dense_operand(rng, M, N)).to(dev)
            rp, ci, va = vs.encode(V, dense=Wd)
            nnz = int(rp[-1].item())
            # W^T's pattern from W's STORED pattern (pattern-only transpose), so the per-step
            # value refresh places every stored element of W, zero now or not (vs.h)
            rT, cT, vT, ws = vs.transpose_pattern(rp, ci[:nnz], M, K, V)
            nT = int(rT[-1].item())
            layers.append(dict(M=M, K=K, V=V, Wd=Wd, X=X, dY=dY, rp=rp, ci=ci[:nnz], va=va[:nnz * V],
                               rT=rT, cT=cT, vT=vT, ws=ws, nnz=nnz, nT=nT,
                               Y=torch.empty((M, N), dtype=torch.float16, device=dev),
                               dX=torch.empty((K, N), dtype=torch.float16, device=dev),
                               dW=torch.empty(max(nnz, 1) * V, dtype=torch.float16, device=dev)))
    sp_f = vs.make_spmm_batch([(L["M"], L["K"], N, L["V"], L["rp"], L["ci"], L["va"], L["X"], L["Y"])
                               for L in layers])
    sp_b = vs.make_spmm_batch([(L["K"], L["M"], N, L["V"], L["rT"], L["cT"], L["vT"], L["dY"], L["dX"])
                               for L in layers])
    sd = vs.make_sddmm_batch([(L["M"], L["K"], N, L["V"], L["rp"], L["ci"], L["dY"], L["X"], L["dW"])
                              for L in layers])

    # graph branches: the per-layer transposes (small, launch-bound kernels) spread over 4
    # branches, then dX = W^T dY; Y = W X and dW on a parallel branch (they do not need W^T)
    tr_streams = [torch.cuda.Stream() for _ in range(4)]
    fw = torch.cuda.Stream()

    def step():
        cur = torch.cuda.current_stream()
        fw.wait_stream(cur)
        with torch.cuda.stream(fw):
            vs.vs_spmm_batched(sp_f)
            vs.vs_sddmm_batched(sd)
        for i, L in enumerate(layers):
            st = tr_streams[i % len(tr_streams)]
            if i < len(tr_streams):
                st.wait_stream(cur)
            with torch.cuda.stream(st):
                vs.vs_transpose_colvec_values(L["M"], L["K"], L["V"], L["rp"], L["ci"], L["va"],
                                              L["rT"], L["vT"], L["ws"])
        for st in tr_streams:
            cur.wait_stream(st)
        vs.vs_spmm_batched(sp_b)
        cur.wait_stream(fw)

    def dense():
        for L in layers:
            torch.matmul(L["Wd"], L["X"])
            torch.matmul(L["Wd"].t(), L["dY"])
            torch.matmul(L["dY"], L["X"].t())

    # the pattern of W^T is fixed (pruned weights): built once per layer before the steps
    # (transpose_pattern); every step refreshes W^T's values from W's (vs_transpose_colvec_values)
    # parity spot check of the step's transposed operand against a dense transpose product
    stream = torch.cuda.Stream()
    with torch.cuda.stream(stream):
        step()
    stream.synchronize()
    L0 = layers[-1]
    ref = torch.matmul(L0["Wd"].t().float(), L0["dY"].float())
    assert torch.allclose(L0["dX"].float(), ref, rtol=2e-2, atol=2e-2), "train: dX mismatch"
    g = capture(torch, step, stream)
    gd = capture(torch, dense, stream)
    with torch.cuda.stream(stream):
        for _ in range(max(3, args.warmup)):
            g.replay()
            gd.replay()
    stream.synchronize()
    clocks = ClockSampler(0).start()
    t_sparse = min(time_graph(torch, g, stream) for _ in range(max(1, args.steps)))
    t_dense = min(time_graph(torch, gd, stream) for _ in range(max(1, args.steps)))
    clk = clocks.stop()
    # transpose kernels per layer: rowT memset + P memset + mark + colscan + scan + zero + place
    flops = sum(3 * 2.0 * L["nnz"] * L["V"] * N for L in layers)
    line = {"metric": METRIC, "value": flops / (t_sparse * 1e-3) / 1e12, "unit": UNIT, "n_gpus": 1,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": t_sparse,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f16",
            "data": "synthetic",
            "config": {"workload": args.workload, "layers": len(layers), "batch_N": N, "sparsity": S,
                       "pattern": "square V x V blocks (P:1633-1636)",
                       "step": "per layer: W^T values refreshed from W's (vs_transpose_colvec_values; "
                               "the W^T pattern is built once by vs_transpose_colvec), Y = W X, "
                               "dX = W^T dY (vs_spmm), dW = (dY X^T) o pattern(W) (vs_sddmm)",
                       "schedule": "transposes on 4 graph branches -> dX batch; Y and dW batches on "
                                   "a parallel branch",
                       "l2": "warm (per-step graph timing, min of steps)"},
            "dense_step_ms": t_dense, "speedup_vs_dense": t_dense / t_sparse,
            # + 1: the dense-tile SDDMM launch ahead of the dW gather launch (inner N = 256 >= 256)
            "gpu_launches": len(layers) * 2 + 3 * 3 + 1, "clocks": clk, "e2e": None}
    print(json.dumps(line), flush=True)
    return 0


def free_port() -> int:
    import socket
    sk = socket.socket()
    sk.bind(("127.0.0.1", 0))
    port = sk.getsockname()[1]
    sk.close()
    return port


def launch_command(gpus: int, argv, port: int = None):
    """torchrun command that runs this file on `gpus` ranks of one node (one process per GPU),
    rendezvous on 127.0.0.1."""
    return [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={gpus}",
            "--master-addr=127.0.0.1", f"--master-port={port or free_port()}",
            os.path.abspath(__file__), *argv]


def check_world(args) -> str:
    """'spawn' when --gpus N > 1 was asked for outside torchrun, 'run' when the rank count
    matches; raises SystemExit when WORLD_SIZE disagrees with --gpus (never falls back to a
    1-GPU run under a multi-GPU flag)."""
    ws = os.environ.get("WORLD_SIZE")
    if ws is None:
        return "spawn" if args.gpus > 1 else "run"
    if int(ws) != args.gpus:
        raise SystemExit(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={ws}")
    return "run"


def main(argv=None):
    argv = list(sys.argv[1:] if argv is None else argv)
    args = parse_args(argv)
    if check_world(args) == "spawn":
        env = dict(os.environ)
        # NCCL init lines (communicator size, transport) go to per-rank files, not stdout
        env.setdefault("NCCL_DEBUG", "INFO")
        env.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
        os.makedirs(os.path.join(ROOT, "gpurun_out"), exist_ok=True)
        env.setdefault("NCCL_DEBUG_FILE", os.path.join(ROOT, "gpurun_out", "nccl_init.%h.%p.log"))
        return subprocess.call(launch_command(args.gpus, argv), env=env)
    if args.workload is None:
        args.workload = "c5" if args.gpus > 1 else DEFAULT_WORKLOAD
    if args.impl == "reference":
        return run_reference(args)
    if args.workload == "c5":
        return run_c5(args)
    if args.workload.startswith("attention"):
        return run_attention(args)
    if args.workload.startswith("train"):
        return run_train(args)
    return run_ours(args)


if __name__ == "__main__":
    sys.exit(main())

#!/usr/bin/env python
"""bench.py -- V:N:M SpMM on B200 sparse tensor cores (BASELINE.json metric).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--workload NAME] [--impl ours|reference]

One step = one pass of the hot path over the workload: the X-row permutation, the
tcgen05.mma.sp SpMM, the residual CSR SpMM and the Y-row unpermutation (SURVEY §8(a)
a5-a8), with the permutations folded into the SpMM's gather/scatter indices
(NM_PACK_ORIGINAL_ORDER): Y = A X in the original vertex order.  Reordering (a1-a2) and
packing (a4) are offline preprocessing -- run and reported, not timed.

Multi-GPU (torchrun, N > 1): the rows of B = P A P^T are split into contiguous,
panel-aligned blocks of balanced cost (stored entries + Y rows), one per rank, X replicated
(SURVEY §8(e)); the SpMM needs no exchange
(the GCN driver in paper_conf_ppopp_chensz0s25_b200/dist.py all-gathers).  Total work is
fixed: "scaling": "strong".  Time = max over ranks of the device-timed region.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

_GNN_RO = dict(max_outer=0, max_stage1=10, max_stage2=0)
WORKLOADS = {
    # configs[0]: ER n = 2048, m = 16384, F = 32, 2:4, fp16 (oracle-sized correctness case)
    "c1-er-n2048-f32-1:2:4": dict(kind="er", n=2048, m=16384, F=32, V=1, M=4, dtype="f16", tau=0),
    # configs[2]: Reddit-shaped (n 232,965, ~114.8M directed edges + I), GCN aggregation of
    # the 602 -> 128 layer at F = 128, bf16, Ahat sym-normalised (the N = 1 headline)
    # (reorder: one Alg. 1 iteration -- Stage-1 sorts + one Stage-2 pass; the full MAXITER = 10
    # schedule takes tens of minutes at 115M entries with the host Stage-2)
    "c3-reddit-f128-1:2:4": dict(kind="gnn", graph="reddit", F=128, V=1, M=4, dtype="bf16", tau=None, **_GNN_RO),
    "c3-reddit-f128-128:2:16": dict(kind="gnn", graph="reddit", F=128, V=128, M=16, dtype="bf16", tau=None,
                                    **_GNN_RO),
    # configs[3]: ogbn-proteins-shaped (132,534 / 79.12M directed + I), F = 256, 128:2:16
    "c4-proteins-f256-128:2:16": dict(kind="gnn", graph="proteins", F=256, V=128, M=16, dtype="bf16",
                                      tau=None, **_GNN_RO),
    # configs[4]: ogbn-products-shaped (2,449,029 / 123.72M directed + I), aggregation at
    # F = 100 (aggregate-first 100 -> 256), 128:2:8
    "c5-products-f100-128:2:8": dict(kind="gnn", graph="products", F=100, V=128, M=8, dtype="bf16",
                                     tau=None, **_GNN_RO),
}
# configs[1] (SuiteSparse-shaped sweep): any point named
#   c2-{banded|powerlaw}-n{65k|262k|1m}-d{8|16|32|64}-f{F}-{V}:2:{M}[-tau{T}]
# (tau omitted = nm_pack_auto: the threshold minimising the library's time model; tau0 = plain pack).
DEFAULT = "c3-reddit-f128-1:2:4"  # configs[2], the N = 1 headline
SWEEP = ["c2-banded-n1m-d16-f128-1:2:4", "c2-banded-n1m-d32-f128-1:2:4", "c2-banded-n262k-d16-f128-64:2:8",
         "c2-powerlaw-n262k-d16-f128-1:2:4", "c2-powerlaw-n262k-d16-f128-128:2:16"]
_SIZES = {"65k": 1 << 16, "262k": 1 << 18, "1m": 1 << 20}


def parse_workload(name):
    if name in WORKLOADS:
        return dict(WORKLOADS[name])
    import re
    m = re.fullmatch(r"c2-(banded|powerlaw)-n(65k|262k|1m)-d(\d+)-f(\d+)-(\d+):2:(\d+)(?:-tau(\d+))?", name)
    if not m:
        raise SystemExit("unknown workload %r (see bench.py WORKLOADS / c2 grammar)" % name)
    kind, ns, d, F, V, M, tau = m.groups()
    return dict(kind="band" if kind == "banded" else "pl", n=_SIZES[ns], d=int(d), F=int(F), V=int(V),
                M=int(M), dtype="f16", tau=None if tau is None else int(tau))


METRIC = "V:N:M SpMM GFLOP/s & % sparse-MMA/HBM roofline vs cuSPARSE, 1/2/4/8 B200"


def default_reorder_opts(w):
    """The reorder options bench.py uses for workload w (nm_reorder defaults: MAXITER = 10 for
    Alg. 1-3; the GNN-shaped graphs take the workload's own caps)."""
    return dict(max_outer=w.get("max_outer", 10), max_stage1=w.get("max_stage1", 10),
                max_stage2=w.get("max_stage2", 10), gain_rule=0)


def make_graph(w):
    from paper_conf_ppopp_chensz0s25_b200 import graphs
    if w["kind"] == "band":
        seed = graphs.seed_of("banded", w["n"], w["d"])
        ip, ic = graphs.banded_graph(w["n"], w["d"], seed)
    elif w["kind"] == "pl":
        seed = graphs.seed_of("powerlaw", w["n"], w["d"])
        ip, ic = graphs.lmcl_graph(w["n"], w["n"] * w["d"] // 2, 2.1, 1, 0.0, seed, scramble=True)
    elif w["kind"] == "er":
        seed = 1
        ip, ic = graphs.er_graph(w["n"], w["m"], seed)
    elif w["kind"] == "gnn":
        ip, ic = graphs.gnn_graph(w["graph"])
        w["n"] = len(ip) - 1
        # Ahat values (GCN normalisation) and an N(0,1) operand of the aggregation's width
        return ip, ic, graphs.gcn_norm_values(ip, ic), graphs.features(w["n"], w["F"], 7, "normal")
    else:
        raise ValueError(w["kind"])
    vals = graphs.symmetric_values(ip, ic, seed + 1)
    X32 = graphs.features(w["n"], w["F"], seed + 2)
    return ip, ic, vals, X32


def l2_gather_peak():
    """Random 256-byte X-row gathers served by L2, GB/s: tools/probes/probe_gather_rate.cu's best
    figure on B200 (cp.async.cg 16 B + commit/wait_group, 148 CTAs, L2-resident X), read from its
    committed output; the fallback is the same measurement's value."""
    p = os.path.join(ROOT, "tools", "probes", "probe_gather_rate.b200.txt")
    best = 0.0
    if os.path.exists(p):
        import re
        for ln in open(p):
            m = re.search(r"X=(\d+)MB\s*:.*?([\d.]+) GB/s", ln)
            if m and int(m.group(1)) <= 128:  # L2-resident sizes only
                best = max(best, float(m.group(2)))
    return (best, "measured (tools/probes/probe_gather_rate.b200.txt)") if best else (18944.0, "fallback")


def sparse_peak(bf16_tf, BN, sm_mhz):
    """Sparse (2:4) tensor peak for the kernel's MMA shape (M = 128, N = BN, K = 32 logical), logical
    TFLOP/s at the SM clock the bench ran at: the cycles per tcgen05.mma.sp that
    tools/probes/probe_mma_issue.cu measured on B200 with the tensor pipe saturated (96 cycles at
    N = 128, 160 at N = 256, 64 at N = 64) x 148 SMs.  Fallback: 2x the measured dense
    bf16 rate (NVIDIA's 2:4 ratio), labelled so."""
    import re
    p = os.path.join(ROOT, "tools", "probes", "probe_mma_issue.b200.txt")
    if os.path.exists(p) and sm_mhz:
        for ln in open(p):
            m = re.match(r"sparse N=\s*(\d+) unroll=1 A=noswzK B=sw128MN:\s*([\d.]+) cycles/MMA", ln)
            if m and int(m.group(1)) == BN:
                cyc = float(m.group(2))
                tf = 2.0 * 128 * BN * 32 * 148 * sm_mhz * 1e6 / cyc / 1e12
                return tf, "measured (tools/probes/probe_mma_issue.b200.txt: %.0f cycles per M128xN%dxK32 " \
                           "MMA, at %.0f MHz)" % (cyc, BN, sm_mhz)
    return 2.0 * bf16_tf, "assumed 2x measured dense bf16"


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return d.get("hbm_gbs", 6650.0), d.get("bf16_tflops", 1590.0), "measured"
    return 6650.0, 1590.0, "fallback"


class ClockSampler:
    """SM clock and throttle-reason sampling DURING the timed region (B200_PROFILING.md's
    clocks line), through NVML in a background thread every ~2 ms (the timed region of one
    SpMM step is well under nvidia-smi's 100 ms sampling period).  Falls back to a single
    nvidia-smi query before/after if NVML is unavailable."""

    REASONS = {  # nvmlClocksEventReason bits
        0x8: "hw_slowdown", 0x40: "hw_thermal_slowdown", 0x20: "sw_thermal_slowdown",
        0x4: "sw_power_cap", 0x80: "hw_power_brake_slowdown",
    }

    def __init__(self, index):
        self.index = index
        self.samples = []
        self.reasons = set()
        self.max_mhz = None
        self._stop = threading.Event()
        self._nvml = None

    def __enter__(self):
        try:
            import pynvml
            pynvml.nvmlInit()
            self._nvml = pynvml
            self._h = pynvml.nvmlDeviceGetHandleByIndex(self.index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self._h, pynvml.NVML_CLOCK_SM)
            self._t = threading.Thread(target=self._run, daemon=True)
            self._t.start()
        except Exception:
            self._nvml = None
        return self

    def _run(self):
        nv = self._nvml
        while not self._stop.is_set():
            try:
                self.samples.append(nv.nvmlDeviceGetClockInfo(self._h, nv.NVML_CLOCK_SM))
                r = nv.nvmlDeviceGetCurrentClocksEventReasons(self._h)
                for bit, name in self.REASONS.items():
                    if r & bit:
                        self.reasons.add(name)
            except Exception:
                pass
            time.sleep(0.002)

    def __exit__(self, *a):
        self._stop.set()
        if self._nvml:
            self._t.join(timeout=2)

    def summary(self):
        return {"sm_mhz": statistics.median(self.samples) if self.samples else None,
                "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons),
                "samples": len(self.samples), "source": "nvml" if self._nvml else "unavailable"}


class OracleSample:
    """The oracle (fp64 CSR SpMM, all host cores) on a bounded row block of the workload:
    the same 16-bit-rounded A and X the GPU consumes, rows [0, rows) with rows sized so one
    pass takes ~budget_s seconds (never more than the whole matrix)."""

    def __init__(self, ip, ic, vals, X32, dtype, budget_s, threads=None):
        import oracle
        from paper_conf_ppopp_chensz0s25_b200 import graphs
        self.oracle = oracle
        self.ip, self.ic = ip, ic
        _, self.v64 = graphs.round16(vals, dtype)
        _, self.x64 = graphs.round16(X32, dtype)
        self.cores = threads or len(os.sched_getaffinity(0))
        n = len(ip) - 1
        rows = max(1, n // 256)
        dt = self._run(rows)[0]
        self.rows = int(min(n, max(rows, rows * budget_s / max(dt, 1e-4))))

    def _run(self, rows):
        ip, ic = self.ip, self.ic
        t0 = time.perf_counter()
        _, _, used = self.oracle.spmm(ip[:rows + 1], ic[:ip[rows]], self.v64[:ip[rows]], self.x64,
                                      nthreads=self.cores)
        return time.perf_counter() - t0, used

    def __call__(self):
        dt, used = self._run(self.rows)
        F = self.x64.shape[1]
        nnz = int(self.ip[self.rows])
        n = len(self.ip) - 1
        return {"value": 2.0 * nnz * F / dt / 1e9, "unit": "GFLOP/s", "cores": used, "kind": "oracle",
                "sample": "fp64 CSR SpMM over the first %d of %d rows (%d nnz), F=%d, %.2f s per pass" %
                          (self.rows, n, nnz, F, dt)}


def cpu_oracle_sample(ip, ic, vals, X32, dtype, budget_s=12.0, passes=3):
    s = OracleSample(ip, ic, vals, X32, dtype, budget_s / passes)
    runs = [s() for _ in range(passes)]
    best = sorted(runs, key=lambda r: r["value"])[len(runs) // 2]
    best["sample"] += " (median of %d passes)" % passes
    # the same oracle on one thread, a smaller row block of ~3 s
    one = OracleSample(ip, ic, vals, X32, dtype, 3.0, threads=1)()
    best["single_thread"] = {"value": one["value"], "unit": one["unit"], "cores": one["cores"],
                             "sample": one["sample"]}
    return best


def run_reference(args, w):
    """--impl reference: the oracle as it stands, timed on the host cores (rank 0 only)."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    ip, ic, vals, X32 = make_graph(w)
    budget = min(5.0, max(0.05, 90.0 / max(1, args.steps + args.warmup)))
    s = OracleSample(ip, ic, vals, X32, w["dtype"], budget)
    for _ in range(args.warmup):
        s()
    samples = [s() for _ in range(args.steps)]
    val = statistics.median(r["value"] for r in samples)
    F = w["F"]
    nnz = int(ip[-1])
    step_ms = 2.0 * nnz * F / (val * 1e9) * 1e3
    line = {"metric": METRIC, "value": val, "unit": "GFLOP/s", "n_gpus": args.gpus, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": step_ms, "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": "f64", "data": "synthetic", "impl": "reference",
            "config": {"workload": args.workload, "n": w["n"], "nnz": nnz, "F": F,
                       "pattern": "%d:2:%d" % (w["V"], w["M"]), "parallelism": "cpu"},
            "cpu_baseline": dict(samples[-1], value=val),
            "e2e": {"value": val, "unit": "GFLOP/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=100)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--workload", default=DEFAULT, help="c1-er-n2048-f32-1:2:4 or a c2 sweep point (see top)")
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--no-cusparse", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--order", default="original", choices=["original", "permuted"])
    ap.add_argument("--layout", default="auto", choices=["auto", "reordered", "natural"],
                    help="timed layout: the reorder's, the natural order, or the faster of the two (auto)")
    ap.add_argument("--no-reorder", action="store_true", help="profiling: skip nm_reorder (natural order)")
    ap.add_argument("--xpad", type=int, default=32, help="X / Y rows padded to a multiple of this many elements "
                    "(>= 8; e.g. 32 aligns C5's 100-feature rows to 256 B)")
    ap.add_argument("--tau", type=int, default=None, help="hybrid threshold (default: the workload's / nm_pack_auto)")
    ap.add_argument("--max-outer", type=int, default=None, help="Alg. 1 cap (default: the workload's, else 10, L496)")
    ap.add_argument("--max-stage1", type=int, default=None)
    ap.add_argument("--max-stage2", type=int, default=None)
    ap.add_argument("--gain-rule", type=int, default=0, help="0 = paper (footnote L440), 1 = positive only")
    ap.add_argument("--sptc-format", type=int, default=0, help="tensor-core kernel: 0 = the pack's choice, 1 = full "
                    "records, 2 = compressed records, 3 = compressed records with A in tensor memory "
                    "(nm_spmm_sptc_format)")
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)
    w = parse_workload(args.workload)
    if args.tau is not None:
        w["tau"] = args.tau
    ropts = default_reorder_opts(w)
    for k in ("max_outer", "max_stage1", "max_stage2"):
        if getattr(args, k) is not None:
            ropts[k] = getattr(args, k)
    ropts["gain_rule"] = args.gain_rule
    if args.impl == "reference":
        return run_reference(args, w)

    if int(os.environ.get("WORLD_SIZE", "1")) > 1 and os.environ.get("OMP_NUM_THREADS", "1") == "1":
        # the ranks of one node share the host cores for the (untimed) reorder's OpenMP Stage-2
        # and the packer's host steps: split them (torchrun's default of 1 thread per rank would
        # make the C3 reorder ~16x slower) -- set before torch, libnm and the oracle load their
        # OpenMP runtimes
        os.environ["OMP_NUM_THREADS"] = str(max(1, len(os.sched_getaffinity(0)) // int(os.environ["WORLD_SIZE"])))
    import torch
    import torch.distributed as dist
    from paper_conf_ppopp_chensz0s25_b200 import api, graphs

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    # NM_DIST_BACKEND=gloo runs the multi-rank logic with CPU collectives (lets several ranks
    # share one GPU for testing); the product setting is NCCL over NVLink, one rank per GPU
    backend = os.environ.get("NM_DIST_BACKEND", "nccl")
    local_dev = local % max(1, torch.cuda.device_count()) if backend == "gloo" else local
    torch.cuda.set_device(local_dev)
    dev = torch.device("cuda", local_dev)
    cdev = dev if backend == "nccl" else torch.device("cpu")  # where collective buffers live
    if world > 1:
        import datetime
        tmo = datetime.timedelta(hours=2)  # graph generation + reorder run before the first collective
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=dev, timeout=tmo)
        else:
            dist.init_process_group("gloo", timeout=tmo)

    # ---------------- inputs (seeded, synthetic) and offline preprocessing ----------------
    t0 = time.perf_counter()
    ip, ic, vals, X32 = make_graph(w)
    gen_s = time.perf_counter() - t0
    n, F, V, M, dt = w["n"], w["F"], w["V"], w["M"], w["dtype"]
    nnz = int(ip[-1])
    # nm_reorder_gpu (untimed preprocessing).  Deterministic: every rank computes the same
    # permutation itself, so no rank waits in a collective while another reorders
    if args.no_reorder:  # profiling runs: natural order, no reorder kernels in the launch list
        perm = np.arange(n, dtype=np.int32)
        rst = {"omega_init": 0, "omega_final": 0, "mb_init": 0, "mb_final": 0, "seconds": 0.0}
        args.layout = "reordered"
    else:
        perm, rst = api.reorder(ip, ic, V, 2, M, device=True, **ropts)
    # contiguous panel-aligned row blocks balanced by stored entries + Y rows
    from paper_conf_ppopp_chensz0s25_b200.dist import balanced_bounds, panel_costs
    rb, re = balanced_bounds(panel_costs(ip, perm), n, world)[rank]
    t0 = time.perf_counter()
    # hybrid threshold: the workload's / --tau, else nm_pack_auto (the tau minimising the
    # library's time model for this F)
    tau = w["tau"] if w["tau"] is not None else "auto"
    P = api.pack(ip, ic, perm, V, 2, M, dtype=dt, val=vals, row_begin=rb, row_end=re, order=args.order, tau=tau, F=F)
    torch.cuda.synchronize()
    pack_s = time.perf_counter() - t0
    xbits, _ = graphs.round16(X32, dt)
    tdt = torch.float16 if dt == "f16" else torch.bfloat16
    xa = max(8, args.xpad)  # 32: 64-byte rows, the gathers' DRAM sectors aligned (C5: 100 -> 128)
    Fp = (F + xa - 1) // xa * xa  # X / Y row pitch (ldx % 8 == 0)
    Xpad = torch.zeros((n, Fp), dtype=torch.int16, device=dev)
    Xpad[:, :F] = torch.from_numpy(xbits.view(np.int16)).to(dev)
    X = Xpad.view(tdt)[:, :F]
    Y = torch.empty((n, Fp), dtype=torch.float32, device=dev)[:, :F]
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)  # > 126 MB L2
    # layout choice (offline, like picking a cuSPARSE algorithm): the reorder's layout vs the
    # natural order, each packed and timed for a few L2-flushed steps; the faster one is timed
    layout_trial = None
    if args.layout == "auto" and args.order == "original":
        P_nat = api.pack(ip, ic, None, V, 2, M, dtype=dt, val=vals, row_begin=rb, row_end=re, order="original", tau=tau,
                         F=F)
        trial = {}
        # (layout, tensor-core kernel) pairs: full records (format 1) or compressed records with
        # A in TMEM (format 3) -- the faster depends on the graph
        fmts = (args.sptc_format,) if args.sptc_format else (1, 3)
        for name, Pk in (("reordered", P), ("natural", P_nat)):
            for fmt in fmts:
                def run():
                    api.spmm(Pk, X, Y, part="sptc", format=fmt)
                    if Pk.info()["residual_nnz"]:
                        api.spmm(Pk, X, Y, part="residual")
                for _ in range(3):
                    run()
                ts = []
                for _ in range(8):
                    flush.zero_()
                    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    a.record()
                    run()
                    b.record()
                    ts.append((a, b))
                torch.cuda.synchronize()
                t = torch.tensor([statistics.median(x.elapsed_time(y) for x, y in ts)], dtype=torch.float64,
                                 device=cdev)
                if world > 1:
                    dist.all_reduce(t, op=dist.ReduceOp.MAX)
                trial["%s/format%d" % (name, fmt)] = float(t.item())
        best = min(trial, key=trial.get)
        layout_trial = dict(trial_ms=trial, chosen=best.split("/")[0])
        args.sptc_format = int(best.split("format")[1])
        if layout_trial["chosen"] == "natural":
            P, perm = P_nat, np.arange(n, dtype=np.int32)
        else:
            del P_nat
    elif args.layout == "natural":
        P = api.pack(ip, ic, None, V, 2, M, dtype=dt, val=vals, row_begin=rb, row_end=re, order=args.order, tau=tau,
                     F=F)
        perm = np.arange(n, dtype=np.int32)
    tau = P.tau  # the threshold actually packed with
    info = P.info()
    perm_d = torch.from_numpy(perm).to(dev)
    PX = padded_like(X) if args.order == "permuted" else None
    Yp = torch.empty((re - rb, F), dtype=torch.float32, device=dev) if args.order == "permuted" else None
    stream = torch.cuda.current_stream()
    has_res = info["residual_nnz"] > 0

    # nm_spmm = the tensor-core kernel, then the residual kernel (stream-ordered); the two are
    # timed separately here (a residual fused into the tensor-core kernel was measured slower,
    # DESIGN.md §6)
    def step(ev=None):
        if args.order == "original":
            if ev: ev[0].record(stream)
            api.spmm(P, X, Y, part="sptc", format=args.sptc_format)
            if ev: ev[1].record(stream)
            if has_res:
                api.spmm(P, X, Y, part="residual")
            if ev: ev[2].record(stream)
        else:
            if ev: ev[0].record(stream)
            api.permute_rows(X, PX, perm_d, dt)
            api.spmm(P, PX, Yp, part="sptc", format=args.sptc_format)
            if ev: ev[1].record(stream)
            if has_res:
                api.spmm(P, PX, Yp, part="residual")
            api.unpermute_rows(Yp, Y, perm_d[rb:re], "f32")
            if ev: ev[2].record(stream)

    launches_per_step = 1 + int(has_res) + (2 if args.order == "permuted" else 0)
    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()

    # ---------------- timed region (device events; L2 flushed between steps) ----------------
    evs = [[torch.cuda.Event(enable_timing=True) for _ in range(3)] for _ in range(args.steps)]
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    with ClockSampler(local) as clk:
        for k in range(args.steps):
            flush.zero_()
            step(evs[k])
        torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    step_ms = [e[0].elapsed_time(e[2]) for e in evs]
    sptc_ms = [e[0].elapsed_time(e[1]) for e in evs]
    total_ms = torch.tensor([sum(step_ms)], dtype=torch.float64, device=cdev)
    if world > 1:
        dist.all_reduce(total_ms, op=dist.ReduceOp.MAX)
    total_ms = float(total_ms.item())
    ms_per_step = total_ms / args.steps
    useful_flop = 2.0 * nnz * F  # all ranks together (strong scaling: fixed total work)
    value = useful_flop / (ms_per_step * 1e-3) / 1e9

    # ---------------- roofline of the dominant kernel (this rank) ----------------
    hbm_gbs, bf16_tf, peak_src = peaks()
    chunks = info["n_chunks"]
    rows_b = re - rb
    # X rows each kernel must read at least once: distinct columns of B (permuted labels) with a
    # packed entry (k_spmm_sptc gathers exactly those: zero-count selected columns are skipped)
    # or a residual entry (k_residual); counted on the host from the shard's rows of B
    iperm = np.empty(n, np.int64)
    iperm[perm] = np.arange(n)
    shard_vertices = perm[rb:re].astype(np.int64)
    starts, ends = ip[shard_vertices], ip[shard_vertices + 1]
    lens = ends - starts
    idx = np.repeat(starts - np.concatenate([[0], np.cumsum(lens)[:-1]]), lens) + np.arange(lens.sum())
    col_all = np.bincount(iperm[ic[idx]], minlength=n)
    res = P.export_canonical(residual_only=True)
    col_res = np.bincount(res["res_col"], minlength=n) if res["res_nnz"] else np.zeros(n, np.int64)
    x_rows_sptc = int(np.count_nonzero(col_all > col_res))
    x_rows_res = int(np.count_nonzero(col_res))
    res_rows = int(np.count_nonzero(np.diff(res["res_rowptr"])))
    x_rows = int(np.count_nonzero(col_all))
    # Roofline terms per kernel, algorithmic bytes / flops per launch:
    #   k_spmm_sptc: HBM = the chunk records it streams (full records: 4736 B per K = 32 chunk =
    #                SURVEY §8(d)'s #mb * (Vp * 4.5 + 4) slot formula; compressed: image_bytes)
    #                + X read once + Y written once (rows * F * 4 B);  L2 = the gathered X rows
    #                (gather_rows * F * 2 B, served from L2 when X fits) + the records per F tile;
    #                tensor = one sparse M128 x BN x K32 MMA per chunk and F tile at the sparse peak
    #   k_residual : HBM = (col, value) 6 B per residual nonzero + row pointers + the Y rows it
    #                read-modify-writes (8 F B each);  L2 = one gathered X row per nonzero (F * 2 B)
    # bound = the largest of the terms' times; frac = that time / the measured kernel time.
    pst = P.stats()
    fmt = args.sptc_format or 1
    BN = 64 if F <= 64 else (128 if F <= 128 else 256)
    nft = (F + BN - 1) // BN
    rec_bytes = pst["full_image_bytes"] if fmt == 1 else pst["image_bytes"]
    l2_gbs, l2_src = l2_gather_peak()
    clocks = clk.summary()
    sp_tf, sp_src = sparse_peak(bf16_tf, BN, clocks.get("sm_mhz") or clocks.get("sm_max_mhz") or 1965.0)
    sptc_terms = {"hbm_bytes": rec_bytes + x_rows_sptc * F * 2 + rows_b * F * 4,
                  "l2_bytes": pst["gather_rows"] * F * 2 + rec_bytes * nft,
                  "mma_flop": 2.0 * chunks * nft * 128 * BN * 32}
    res_terms = {"hbm_bytes": res["res_nnz"] * 6 + (rows_b + 1) * 8 + res_rows * F * 8,
                 "l2_bytes": res["res_nnz"] * F * 2, "mma_flop": 0.0} if has_res else None
    kern = {"k_spmm_sptc": dict(sptc_terms, ms=statistics.mean(sptc_ms),
                                format={1: "full", 2: "compressed", 3: "compressed-tmem"}[fmt])}
    if has_res:
        kern["k_residual"] = dict(res_terms, ms=statistics.mean(b - a for a, b in zip(sptc_ms, step_ms)))
    for k in kern.values():
        t = {"hbm": k["hbm_bytes"] / (hbm_gbs * 1e9) * 1e3, "l2": k["l2_bytes"] / (l2_gbs * 1e9) * 1e3,
             "tensor": k["mma_flop"] / (sp_tf * 1e12) * 1e3}
        k["t_roof_ms"] = t
        k["bound"] = max(t, key=t.get)
        k["frac"] = t[k["bound"]] / k["ms"]
        k["hbm_frac"] = t["hbm"] / k["ms"]
    dom = max(kern, key=lambda k: kern[k]["ms"])
    kd = kern[dom]
    k_ms = kd["ms"]
    if kd["bound"] == "tensor":
        achieved, peak, unit = kd["mma_flop"] / (k_ms * 1e-3) / 1e12, sp_tf, "TFLOP/s"
    elif kd["bound"] == "l2":
        achieved, peak, unit = kd["l2_bytes"] / (k_ms * 1e-3) / 1e9, l2_gbs, "GB/s"
    else:
        achieved, peak, unit = kd["hbm_bytes"] / (k_ms * 1e-3) / 1e9, hbm_gbs, "GB/s"
    roofline = {"bound": kd["bound"], "achieved": achieved, "peak": peak, "unit": unit, "frac": achieved / peak,
                "traffic": None, "kernel": dom, "kernel_ms": k_ms,
                "peaks": {"hbm_gbs": hbm_gbs, "hbm_source": peak_src, "l2_gather_gbs": l2_gbs, "l2_source": l2_src,
                          "sparse_tflops": sp_tf, "sparse_source": sp_src},
                "kernels": kern,
                "step_frac": sum(max(k["t_roof_ms"].values()) for k in kern.values()) / ms_per_step}
    prof = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if os.path.exists(prof) and world == 1:  # the committed capture is of the 1-GPU launch
        try:
            tr = json.load(open(prof)).get(args.workload)
            if tr and tr.get("kernel", "").startswith(dom) and tr.get("tau", tau) == tau:
                roofline["traffic"] = tr["dram_bytes_per_launch"]
                roofline["traffic_source"] = "profiles/ncu_traffic.json (%s)" % tr.get("round", "")
            if tr and tr.get("tau", tau) == tau and "k_spmm_sptc" in tr:  # tensor-pipe evidence (ncu)
                ks = tr["k_spmm_sptc"]
                kern["k_spmm_sptc"]["ncu"] = {"dram_bytes_per_launch": ks.get("dram_bytes_per_launch"),
                                              "tensor_pipe": ks.get("tensor_pipe"),
                                              "source": ks.get("source")}
        except Exception:
            pass

    # ---------------- end-to-end through the public API with host buffers ----------------
    e2e = None
    if world == 1 and args.order == "original":
        e2e = e2e_pipelined(P, X, Y, F, max(4, args.steps // 4), useful_flop, fmt=args.sptc_format)

    # ---------------- cuSPARSE on the same box (original order, same rounded inputs) ----------
    cus = None
    if not args.no_cusparse and world == 1:
        try:
            cus = cusparse_baseline(ip, ic, vals, X, dt, F, dev, args.steps, flush)
            # the Table 4 lesson: cuSPARSE on the reordered matrix too
            Bp, Bc, Bv = permuted_csr(ip, ic, vals, perm)
            PXc = X[torch.from_numpy(perm.astype(np.int64)).to(dev)].contiguous()
            rco = cusparse_baseline(Bp, Bc, Bv, PXc, dt, F, dev, args.steps, flush)
            del PXc
            cus["reordered"] = {k: v for k, v in rco.items() if k != "note"}
            if "ms" in rco and rco["ms"] < cus.get("ms", float("inf")):
                cus["ms"], cus["gflops"], cus["best_order"] = rco["ms"], rco["gflops"], "reordered"
            else:
                cus["best_order"] = "original"
        except Exception as ex:  # report, never fake
            cus = {"error": str(ex)[:200]}

    # ---------------- CPU oracle baseline (rank 0, N = 1) ----------------
    cpu = None
    if world == 1 and not args.no_cpu:
        cpu = cpu_oracle_sample(ip, ic, vals, X32, dt)

    clocks = clk.summary()
    if rank == 0:
        line = {"metric": METRIC, "value": value, "unit": "GFLOP/s", "n_gpus": world, "steps": args.steps,
                "warmup": args.warmup, "ms_per_step": ms_per_step, "higher_is_better": True,
                "scaling": "strong", "vs_baseline": None, "dtype": dt, "data": "synthetic",
                "config": {"workload": args.workload, "graph": w.get("graph", w["kind"]), "n": n, "nnz": nnz, "F": F,
                           "layout": (layout_trial or {}).get("chosen", args.layout),
                           "pattern": "%d:2:%d" % (V, M), "order": args.order, "tau": tau,
                           "sptc_format": args.sptc_format or 1,
                           "parallelism": "row-shard x%d" % world,
                           "l2": "flushed between steps (256 MiB write outside the event-timed intervals)"},
                "gpu_launches": launches_per_step * args.steps,
                "roofline": roofline, "cpu_baseline": cpu, "e2e": e2e, "clocks": clocks,
                "cusparse": cus,
                "preprocess": {"gen_s": gen_s, "reorder": "nm_reorder_gpu", "reorder_opts": ropts, "layout": layout_trial, "reorder_s": rst["seconds"], "pack_s": pack_s,
                               "omega_init": rst["omega_init"], "omega_final": rst["omega_final"],
                               "mb_init": rst["mb_init"], "mb_final": rst["mb_final"],
                               "violation_removal": (None if rst["omega_init"] == 0 else
                                                     1.0 - rst["omega_final"] / rst["omega_init"]),
                               "n_mb": info["n_mb"], "n_chunks": chunks,
                               "slots_per_nnz": chunks * 8 * 128 * 2 /
                               max(1, info["packed_nnz"] + info["residual_nnz"]),
                               "x_rows_read": x_rows,
                               "residual_nnz": info["residual_nnz"],
                               "residual_rows": res_rows, "x_rows_sptc": x_rows_sptc,
                               "x_rows_residual": x_rows_res,
                               "sptc_share_of_nnz": info["packed_nnz"] / max(1, nnz),
                               "packed_bytes": info["device_bytes"], "image_bytes": pst["image_bytes"],
                               "image_bytes_per_packed_nnz": pst["image_bytes"] / max(1, info["packed_nnz"]),
                               "residual_items": pst["residual_items"],
                               "residual_split_rows": pst["residual_split_rows"]},
                "step_ms_median": statistics.median(step_ms), "sptc_ms_median": statistics.median(sptc_ms)}
        if cus and "ms" in cus:
            line["speedup_vs_cusparse"] = cus["ms"] / ms_per_step
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


def padded_like(t):
    """Uninitialised tensor of t's shape and dtype whose rows keep t's (16-byte padded) stride."""
    import torch
    base = torch.empty((t.shape[0], t.stride(0)), dtype=t.dtype, device=t.device)
    return base[:, :t.shape[1]]


def e2e_pipelined(P, X, Y, F, steps, useful_flop, fmt=0):
    """End to end through the public API with host buffers: every step copies its X from
    pinned host memory, runs nm_spmm and reads Y back to pinned host memory.  Serving-style
    pipelining: device X/Y are double-buffered and H2D, SpMM and D2H run on three streams, so
    step k's D2H overlaps step k+1's H2D (PCIe is full duplex).  Time = first H2D to last D2H
    (CUDA events, device clock), divided by the number of steps."""
    import torch
    from paper_conf_ppopp_chensz0s25_b200 import api
    Xh = torch.empty(X.shape, dtype=X.dtype).pin_memory()
    Xh.copy_(X.cpu())
    Yh = [torch.empty((Y.shape[0], F), dtype=torch.float32).pin_memory() for _ in range(2)]
    Xd = [X, padded_like(X)]
    Yd = [Y, padded_like(Y)]
    s_h2d, s_cmp, s_d2h = torch.cuda.Stream(), torch.cuda.Stream(), torch.cuda.Stream()
    ev = lambda: torch.cuda.Event(enable_timing=True)

    def run(k_steps):
        h2d_done = [None, None]
        cmp_done = [None, None]
        d2h_done = [None, None]
        start, end = ev(), ev()
        start.record(s_h2d)
        for k in range(k_steps):
            b = k & 1
            if cmp_done[b] is not None:
                s_h2d.wait_event(cmp_done[b])          # step k-2 finished reading Xd[b]
            with torch.cuda.stream(s_h2d):
                Xd[b].copy_(Xh, non_blocking=True)
            h2d_done[b] = ev()
            h2d_done[b].record(s_h2d)
            s_cmp.wait_event(h2d_done[b])
            if d2h_done[b] is not None:
                s_cmp.wait_event(d2h_done[b])          # step k-2's Y read back
            if fmt:  # the tensor-core kernel the layout trial chose, then the residual (nm.h calls)
                api.spmm(P, Xd[b], Yd[b], stream=s_cmp, part="sptc", format=fmt)
                api.spmm(P, Xd[b], Yd[b], stream=s_cmp, part="residual")
            else:
                api.spmm(P, Xd[b], Yd[b], stream=s_cmp)
            cmp_done[b] = ev()
            cmp_done[b].record(s_cmp)
            s_d2h.wait_event(cmp_done[b])
            with torch.cuda.stream(s_d2h):
                Yh[b].copy_(Yd[b], non_blocking=True)
            d2h_done[b] = ev()
            d2h_done[b].record(s_d2h)
        end.record(s_d2h)
        torch.cuda.synchronize()
        return start.elapsed_time(end) / k_steps

    run(2)
    ms = run(steps)
    return {"value": useful_flop / (ms * 1e-3) / 1e9, "unit": "GFLOP/s", "ms_per_step": ms,
            "h2d_bytes_per_step": int(Xh.numel() * Xh.element_size()),
            "d2h_bytes_per_step": int(Yh[0].numel() * Yh[0].element_size()),
            "pipeline": "double-buffered X/Y; H2D, nm_spmm, D2H on 3 streams (pinned host buffers)"}


def permuted_csr(ip, ic, vals, perm):
    """B = P A P^T as a CSR (rows perm order, columns relabelled and sorted) -- host numpy, for
    the cuSPARSE baseline on the reordered matrix."""
    n = len(ip) - 1
    iperm = np.empty(n, np.int64)
    iperm[perm] = np.arange(n)
    pv = perm.astype(np.int64)
    lens = ip[pv + 1] - ip[pv]
    Bp = np.concatenate([[0], np.cumsum(lens)]).astype(np.int64)
    idx = np.repeat(ip[pv] - Bp[:-1], lens) + np.arange(Bp[-1])
    rows = np.repeat(np.arange(n, dtype=np.int64), lens)
    cols = iperm[ic[idx]]
    o = np.argsort(rows * n + cols)
    return Bp, cols[o].astype(np.int32), vals[idx][o]


def cusparse_baseline(ip, ic, vals, X, dt, F, dev, steps, flush):
    import ctypes

    import torch
    from paper_conf_ppopp_chensz0s25_b200 import build, graphs
    lib = ctypes.CDLL(build.build_baseline())
    lib.cs_create.restype = ctypes.c_int
    n = len(ip) - 1
    rp = torch.from_numpy(ip.astype(np.int32)).to(dev)
    ci = torch.from_numpy(ic).to(dev)
    vb, _ = graphs.round16(vals, dt)
    va = torch.from_numpy(vb.view(np.int16)).to(dev)
    Yc = torch.empty((n, F), dtype=torch.float32, device=dev)
    res = {}
    for name, alg in (("csr_alg2", 2), ("default", 0)):
        h = ctypes.c_void_p()
        yf = ctypes.c_int()
        rc = lib.cs_create(ctypes.c_int64(n), ctypes.c_int64(len(ic)), ctypes.c_void_p(rp.data_ptr()),
                           ctypes.c_void_p(ci.data_ptr()), ctypes.c_void_p(va.data_ptr()), int(dt == "bf16"),
                           F, ctypes.c_void_p(X.data_ptr()), ctypes.c_int64(X.stride(0)),
                           ctypes.c_void_p(Yc.data_ptr()), ctypes.c_int64(F), alg, ctypes.byref(h),
                           ctypes.byref(yf))
        if rc != 0:
            res[name] = {"error": "cs_create rc=%d" % rc}
            continue
        s = ctypes.c_void_p(torch.cuda.current_stream().cuda_stream)
        for _ in range(3):
            lib.cs_run(h, s)
        ts = []
        for _ in range(steps):
            flush.zero_()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record()
            rc = lib.cs_run(h, s)
            b.record()
            ts.append((a, b))
        torch.cuda.synchronize()
        ms = statistics.mean(a.elapsed_time(b) for a, b in ts)
        res[name] = {"ms": ms, "gflops": 2.0 * len(ic) * F / (ms * 1e-3) / 1e9, "y_fp32": bool(yf.value),
                     "rc": rc}
        lib.cs_destroy(h)
    best = min((v for v in res.values() if "ms" in v), key=lambda v: v["ms"], default=None)
    if best:
        res["ms"] = best["ms"]
        res["gflops"] = best["gflops"]
    res["note"] = "cusparseSpMM CSR, 16-bit A/X, fp32 compute; original order (top level) and reordered"
    return res


if __name__ == "__main__":
    main()

#!/usr/bin/env python
"""bench.py -- HPCCG CG hot path on B200 (BASELINE.json metric).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
                    [--workload hpccg256|hpccg128|hpccg20|hpccg512s|blas1|tridiag|lbm]

One STEP = one whole HPCCG solve on the synthetic on-device-generated problem:
x0 = 0 (our waxpby kernel), init (p = x, Ap = A p, r = b - Ap, r.r), the CG
iterations (SpMV with fused p.Ap, fused x/r update + r.r, p update; device-side
scalars; one CUDA graph with a device-driven WHILE node) and the max|x - 1|
verification -- rows a.2-a.9 of DESIGN.md.  The problem (a.1) is generated once
per workload (HPCCG times only the solve): config.gen_ms.

Default workload, at EVERY N: hpccg256 = BASELINE configs[2] (256^3 per GPU,
weak scaling, 200 iterations, tol 0), the configuration north_star's targets
are set on; so a scaling run's N = 1 point is this line.  Before timing, every
workload runs a tol 1e-12 correctness solve of the GLOBAL problem and checks
niters against SURVEY's independent counts (`correctness`).  The same line
carries `sub_configs`: configs[1] (128^3, 500 iterations), configs[0]
(20x30x10 at tol 1e-12 / 150, as BASELINE states it) at N = 1, configs[3]
(512^3 global, strong) at every N -- each with t_iter, GFLOP/s and e2e -- and
configs[4] (the JACC BLAS-1 AXPY/DOT sweep 1e3..1e9, DOT sharded at N > 1).

value = CG GFLOP/s of the whole job = sum over ranks of niters (2 nnz + 10 n)
        / max-over-ranks device time of the K timed steps (exact nnz, A15).
e2e   = the same metric through the public C-ABI with HOST buffers: every
        step copies x0 from pinned host memory in and the solution x back out.
roofline = the SpMV kernel (dominant), algorithmic bytes 12 nnz + 16 n per
        launch / its CUDA-event launch duration (events pass); the fused vector
        kernels (48n, 24n B) against 8 TB/s beside it (north_star's 75 % target).
Multi-GPU (torchrun): z-slab, one rank per GPU; the halo exchange and the
        allreduces run inside the library (peer memory fused into the CG kernels
        by default, NCCL as the agreed fallback); torch.distributed only
        bootstraps and aggregates.  `ranks` records, per rank, the transport,
        exchange mode, NCCL's rank count and the correctness solve.
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

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "HPCCG CG GFLOP/s and SpMV HBM GB/s (fp64) at 1/2/4/8 B200 vs HBM roofline"
WORKLOADS = {
    # weak: nz planes per GPU; strong: nz global planes split over the GPUs.
    # tol 0 runs exactly max_iter - 1 iterations (HPCCG loop, A4); configs[0]
    # is quoted at tol 1e-12 / 150 (50 iterations).  sub_steps: timed steps when
    # the workload is a sub-record of another workload's line.
    "hpccg256": dict(nx=256, ny=256, nz=256, max_iter=201, tol=0.0, cfg=2, scaling="weak", sub_steps=5,
                     ref_iters=6),
    "hpccg128": dict(nx=128, ny=128, nz=128, max_iter=501, tol=0.0, cfg=1, scaling="weak", sub_steps=10,
                     ref_iters=20),
    "hpccg20": dict(nx=20, ny=30, nz=10, max_iter=150, tol=1e-12, cfg=0, scaling="weak", sub_steps=20),
    "hpccg512s": dict(nx=512, ny=512, nz=512, max_iter=101, tol=0.0, cfg=3, scaling="strong", sub_steps=3,
                      ref_iters=6),
}
BLAS1_METRIC = "JACC BLAS-1 AXPY+DOT fp64 HBM GB/s (host-synchronous calls)"
TRI_METRIC = "Fig. 12 CG time per iteration, tridiagonal SIZE = 1e8 (fp64)"
LBM_METRIC = "D2Q9 pull LBM (Fig. 10) time per step, 1000^2 (fp64)"
FALLBACK_HBM_GBS = 6650.0  # B200_PROFILING.md fallback, used only without MEASURED_PEAKS.json


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return FALLBACK_HBM_GBS, "fallback (B200_PROFILING.md)"


class ClockSampler:
    """SM clock + throttle reasons sampled DURING the timed region: NVML polled
    every 5 ms from a thread (short regions still get samples), else
    `nvidia-smi -lms 100` filtered to samples with the GPU busy."""

    def __new__(cls, index: int):
        if cls is ClockSampler:
            try:
                import pynvml
                pynvml.nvmlInit()
                return super().__new__(NvmlClockSampler)
            except Exception:
                pass
        return super().__new__(cls)
    Q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap,utilization.gpu")

    def __init__(self, index: int):
        self.index, self.proc, self.lines = index, None, []

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), "--query-gpu=" + self.Q,
                 "--format=csv,noheader,nounits", "-lms", "100"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def __exit__(self, *a):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()

    def summary(self):
        sm, mx, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            f = [x.strip() for x in ln.split(",")]
            if len(f) < 8:
                continue
            try:
                s, m, util = float(f[0]), float(f[1]), float(f[7])
            except ValueError:
                continue
            mx = m
            if util > 0:
                sm.append(s)
                for nm, v in zip(names, f[3:7]):
                    if v.lower().startswith("active"):
                        reasons.add(nm)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": mx,
                "reasons": sorted(reasons), "samples": len(sm)}


class NvmlClockSampler(ClockSampler):
    REASONS = {"hw_slowdown": 0x8, "sw_thermal_slowdown": 0x20, "hw_thermal_slowdown": 0x40,
               "sw_power_cap": 0x4}

    def __init__(self, index: int):
        self.index, self.samples, self.stop = index, [], None

    def __enter__(self):
        import pynvml
        self.nv = pynvml
        self.h = pynvml.nvmlDeviceGetHandleByIndex(self.index)
        self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
        self.stop = threading.Event()

        def poll():
            while not self.stop.is_set():
                try:
                    mhz = self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_SM)
                    rs = self.nv.nvmlDeviceGetCurrentClocksThrottleReasons(self.h)
                    self.samples.append((mhz, rs))
                except Exception:
                    pass
                time.sleep(0.005)
        self.t = threading.Thread(target=poll, daemon=True)
        self.t.start()
        return self

    def __exit__(self, *a):
        self.stop.set()
        self.t.join(timeout=2)

    def summary(self):
        reasons = sorted({nm for _, rs in self.samples for nm, bit in self.REASONS.items() if rs & bit})
        mhz = [m for m, _ in self.samples]
        return {"sm_mhz": statistics.median(mhz) if mhz else None, "sm_max_mhz": self.max_mhz,
                "reasons": reasons, "samples": len(mhz), "source": "nvml 5 ms"}


def cg_flops(niters, nnz, n):
    return float(niters) * (2.0 * nnz + 10.0 * n)


# ------------------------------------------------------------ oracle (CPU)

def oracle_cg_timed(prob, max_iter, sr=False):
    """One oracle CG solve (HPCCG's, or f2's single-reduction) -> (result, seconds)."""
    import oracle
    t0 = time.perf_counter()
    r = oracle.cg_sr(prob, max_iter, 0.0) if sr else oracle.cg(prob, max_iter, 0.0)
    return r, time.perf_counter() - t0


def oracle_sample(nx, ny, nz, iters_cap, budget_s, sr=False):
    """Time the CPU oracle (as it stands) on a bounded sample of the
    workload: the same generated problem, m CG iterations, all host cores."""
    import oracle
    t0 = time.perf_counter()
    prob = oracle.generate(nx, ny, nz)
    gen_s = time.perf_counter() - t0
    _, per_it = oracle_cg_timed(prob, 2, sr)   # calibrate: 1 iteration
    per_it = max(per_it, 1e-6)
    m = int(max(1, min(iters_cap, budget_s / per_it)))
    r, t = oracle_cg_timed(prob, m + 1, sr)
    gflops = cg_flops(r["niters"], prob.nnz, prob.n) / t * 1e-9
    return {"value": gflops, "iters": r["niters"], "seconds": t, "gen_s": gen_s,
            "cores": oracle.get_threads(), "prob": prob}


def run_reference(args, w):
    """The reference arm for the CG workloads: the oracle as it stands, on the
    host cores, in our arm's metric / unit.  A tol > 0 workload (configs[0])
    runs its whole solve per step; a fixed-iteration one a bounded number of
    its iterations per step (the same problem, `sample` says how many)."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    import oracle
    oracle.build()
    nx, ny, nz = w["nx"], w["ny"], w["nz"]
    if w["scaling"] == "strong":
        nz = nz // args.gpus
    if nx * ny * nz > (1 << 25):          # host RAM of the oracle's CSR: time the 256^3 problem
        nx, ny, nz = 256, 256, 256
    prob = oracle.generate(nx, ny, nz)
    sr = args.cg_variant == "sr"
    if w["tol"] > 0:
        max_iter, tol = w["max_iter"], w["tol"]
        what = f"the whole solve (tol {tol:g}, max_iter {max_iter}) per step"
    else:
        m = max(1, min(w["max_iter"] - 1, args.ref_iters or w.get("ref_iters", 20)))
        max_iter, tol = m + 1, 0.0
        what = f"{m} iterations per step (bounded sample of the {w['max_iter'] - 1}-iteration step)"

    def one():
        t0 = time.perf_counter()
        r = oracle.cg_sr(prob, max_iter, tol) if sr else oracle.cg(prob, max_iter, tol)
        return r, time.perf_counter() - t0

    for _ in range(args.warmup):
        one()
    tot, flops = 0.0, 0.0
    for _ in range(args.steps):
        r, t = one()
        tot += t
        flops += cg_flops(r["niters"], prob.nnz, prob.n)
    val = flops / tot * 1e-9
    sample = (f"oracle CG (C, OpenMP, all host cores) on the {nx}x{ny}x{nz} problem, {what}"
              + ("; one GPU's slab of the global problem" if args.gpus > 1 else ""))
    line = {
        "metric": METRIC, "value": round(val, 4), "unit": "GFLOP/s", "impl": "reference",
        "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": round(tot / args.steps * 1e3, 3), "higher_is_better": True,
        "scaling": w["scaling"], "vs_baseline": None, "dtype": "f64",
        "data": "synthetic (HPCCG generation, deterministic)",
        "config": {"workload": args.workload, "baseline_config": w["cfg"], "nx": nx, "ny": ny,
                   "nz": nz, "iters_per_step": r["niters"], "tol": tol},
        "cpu_baseline": {"value": round(val, 4), "unit": "GFLOP/s", "cores": oracle.get_threads(),
                         "kind": "oracle", "sample": sample},
        "e2e": {"value": round(val, 4), "unit": "GFLOP/s", "h2d_bytes_per_step": 0,
                "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)
    return 0


def _reference_line(args, metric, value, unit, hib, ms_per_step, config, sample, scaling="none"):
    """The reference arm's JSON line for the f1 / f4 / BLAS-1 workloads: the
    oracle as it stands, on the host cores, in our arm's metric / unit / config."""
    import oracle
    line = {"metric": metric, "value": round(value, 5), "unit": unit, "impl": "reference",
            "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": round(ms_per_step, 4), "higher_is_better": hib,
            "scaling": scaling, "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": config,
            "cpu_baseline": {"value": round(value, 5), "unit": unit, "cores": oracle.get_threads(),
                             "kind": "oracle", "sample": sample},
            "e2e": {"value": round(value, 5), "unit": unit, "h2d_bytes_per_step": 0,
                    "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


def run_reference_tridiag(args):
    """Fig. 12 CG per-iteration time of the oracle at SIZE: each step
    times a 1- and a 3-iteration oracle solve; per iteration = the difference / 2."""
    if int(os.environ.get("RANK", "0")) != 0:
        return 0
    import oracle
    oracle.build()
    n = args.tri_n
    tr = oracle.Tri(n)

    def one():
        o1 = oracle.tri_cg(tr, 1, 0.0)["seconds"]
        o3 = oracle.tri_cg(tr, 3, 0.0)["seconds"]
        return max((o3 - o1) / 2, o1 / 2) * 1e3

    for _ in range(args.warmup):
        one()
    ms = sum(one() for _ in range(args.steps)) / args.steps
    return _reference_line(args, TRI_METRIC, ms, "ms/iteration", False, ms,
                           {"workload": "tridiag", "n": n},
                           f"oracle Fig. 12 CG (C, OpenMP, compensated dots) at n = {n}: "
                           f"(3-iteration - 1-iteration solve) / 2 per step")


def run_reference_lbm(args):
    """Fig. 10 D2Q9 pull step of the oracle at SIZE^2, one step per bench step."""
    if int(os.environ.get("RANK", "0")) != 0:
        return 0
    import numpy as np
    import oracle
    import synth
    oracle.build()
    S = args.lbm_size
    f0 = synth.lbm_state(S, 21)
    a, b, f = f0.copy(), f0.copy(), np.zeros_like(f0)
    for _ in range(args.warmup):
        oracle.lbm_step(S, a, f, b, 0.8)
        a, b = b, a
    t0 = time.perf_counter()
    for _ in range(args.steps):
        oracle.lbm_step(S, a, f, b, 0.8)
        a, b = b, a
    ms = (time.perf_counter() - t0) / args.steps * 1e3
    return _reference_line(args, LBM_METRIC, ms, "ms/step", False, ms,
                           {"workload": "lbm", "size": S},
                           f"oracle Fig. 10 step (C, OpenMP) at {S}^2, one step per bench step")


def run_reference_blas1(args):
    """JACC AXPY + DOT of the oracle (Fig. 2 inputs) at a bounded n (the GPU arm's
    headline is n = 1e9 per GPU; the host sample stops at 1e8 = 2.4 GB of vectors)."""
    if int(os.environ.get("RANK", "0")) != 0:
        return 0
    import numpy as np
    import oracle
    import synth
    oracle.build()
    n = min(args.blas1_max or 10 ** 9, 10 ** 8)
    gen = min(n, 1 << 24)
    x = np.resize(synth.jacc_vector(gen, 42), n)
    y = np.resize(synth.jacc_vector(gen, 43), n)
    w = np.empty(n)

    def one():
        t0 = time.perf_counter()
        oracle.waxpby(1.0, x, 2.5, y, w)
        t1 = time.perf_counter()
        oracle.ddot(x, y)
        return t1 - t0, time.perf_counter() - t1

    for _ in range(args.warmup):
        one()
    ta = td = 0.0
    for _ in range(args.steps):
        a, d = one()
        ta, td = ta + a, td + d
    ta, td = ta / args.steps, td / args.steps
    gbs = (24.0 + 16.0) * n / (ta + td) / 1e9
    return _reference_line(args, BLAS1_METRIC, gbs, "GB/s", True, (ta + td) * 1e3,
                           {"workload": "blas1", "baseline_config": 4, "n": n},
                           f"oracle waxpby (w = x + 2.5 y) + compensated ddot (C, OpenMP) at "
                           f"n = {n} (bounded sample of the 1e9 headline)", scaling="weak")


# -------------------------------------------------------------------- ours

# tol = 1e-12 / max_iter 150 iteration counts of the GLOBAL problem (SURVEY 8(c)
# pins: two independent numpy implementations, HPCCG loop semantics A4),
# keyed by (nx, ny, nz_global): the N-rank correctness solve is checked against them
EXPECTED_NITERS = {(20, 30, 10): 50, (32, 32, 32): 60, (64, 64, 64): 89, (128, 128, 128): 106,
                   (256, 256, 256): 112, (256, 256, 512): 113, (256, 256, 1024): 114,
                   (256, 256, 2048): 115, (512, 512, 512): 115}


def _stats_add(acc, prob, r):
    st = prob.stats()
    acc["spmv_ms"] += st["spmv_ms"]
    acc["spmv_n"] += st["spmv_launches"]
    acc["update_ms"] += st["update_ms"]
    acc["pupdate_ms"] += st["pupdate_ms"]
    acc["niters"] += r["niters"]
    acc["graph_mode"] = st["graph_mode"]
    acc["x_deferred"] = int(st["x_deferred"])  # deferral depth m (0 off; m >= 2: ring of m + 1 p buffers)


class CgRunner:
    """One generated problem and the bench's timing protocol around it: a step
    is x0 = 0 (our waxpby kernel), one hpccg_solve(max_iter, tol), max|x - 1|.
    Times are CUDA events on the library stream, max over ranks; L2 is flushed
    between timed steps (outside the events) when the working set fits in L2."""

    def __init__(self, H, D, ctx, prob, stream, world, coll_dev, max_iter, tol, local):
        import torch
        self.H, self.D, self.ctx, self.prob, self.stream = H, D, ctx, prob, stream
        self.world, self.coll_dev, self.max_iter, self.tol = world, coll_dev, max_iter, tol
        self.n = prob.n
        self.nnz_local = prob.info["nnz_local"]
        self.xptr = prob.vec_ptr(H.HPCCG_VEC_X)
        l2_bytes = torch.cuda.get_device_properties(local).L2_cache_size
        work_bytes = (324 + 6 * 8) * self.n
        self.flush_buf = None
        if work_bytes < l2_bytes:
            self.flush_buf = torch.empty(2 * l2_bytes // 8, dtype=torch.float64, device="cuda")
        self.l2_note = ("L2 flushed between timed steps (a %d MB write; working set %.1f MB < L2 %.0f MB); "
                        "per-step events" % (2 * l2_bytes >> 20, work_bytes / 1e6, l2_bytes / 1e6)
                        if self.flush_buf is not None else
                        "inputs larger than L2 (ELL %.0f MB/GPU > %.0f MB)" % (324e-6 * self.n, l2_bytes / 1e6))

    def flush(self):
        import torch
        with torch.cuda.stream(self.stream):
            self.flush_buf.zero_()

    def barrier(self):
        import torch
        import torch.distributed as dist
        if self.world > 1:
            dist.barrier()
        torch.cuda.synchronize()

    def step(self):
        self.ctx.waxpby(self.n, 0.0, self.xptr, 0.0, self.xptr, self.xptr)   # x0 = 0 (A5)
        r = self.prob.solve(self.max_iter, self.tol)
        return r, self.prob.maxabsdiff()

    def timed(self, k_steps, step=None):
        """K steps between barriers; one event pair around all of them (inputs
        larger than L2) or around each step (L2 flushed outside the events)."""
        import torch
        step = step or self.step
        t0, t1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        acc = {"spmv_ms": 0.0, "spmv_n": 0, "niters": 0, "update_ms": 0.0, "pupdate_ms": 0.0, "ms": 0.0}
        self.barrier()
        if self.flush_buf is not None:
            for _ in range(k_steps):
                self.flush()
                t0.record(self.stream)
                r, err = step()
                t1.record(self.stream)
                t1.synchronize()
                acc["ms"] += t0.elapsed_time(t1)
                _stats_add(acc, self.prob, r)
            self.barrier()
        else:
            t0.record(self.stream)
            for _ in range(k_steps):
                r, err = step()
                _stats_add(acc, self.prob, r)
            t1.record(self.stream)
            self.barrier()
            acc["ms"] = t0.elapsed_time(t1)
        acc["r"], acc["err"] = r, err
        return acc

    def value(self, acc):
        """(whole-job GFLOP/s, max-over-ranks ms) of a timed region."""
        ms, flops = self.D.max_time_sum_work(acc["ms"], cg_flops(acc["niters"], self.nnz_local, self.n),
                                             self.coll_dev)
        return flops / (ms * 1e-3) * 1e-9, ms

    def e2e(self, k_steps):
        """The same metric through the public C-ABI with HOST buffers: every
        step copies x0 in from pinned memory and x back out (+ max|x-1|)."""
        import numpy as np
        import torch
        H, prob = self.H, self.prob
        h_x0 = torch.zeros(self.n, dtype=torch.float64).pin_memory()
        h_x = torch.empty(self.n, dtype=torch.float64).pin_memory()

        def step_e2e():
            prob.set_vec_ptr(H.HPCCG_VEC_X, h_x0.data_ptr())   # H2D 8n
            r = prob.solve(self.max_iter, self.tol)
            prob.get_vec_ptr(H.HPCCG_VEC_X, h_x.data_ptr())    # D2H 8n
            return r, prob.maxabsdiff()                         # D2H 8 B

        step_e2e()
        acc = self.timed(k_steps, step_e2e)
        val, _ = self.value(acc)
        return {"value": round(val, 3), "unit": "GFLOP/s", "h2d_bytes_per_step": 8 * self.n,
                "d2h_bytes_per_step": 8 * self.n + 8,
                "max_abs_x_minus_1_host": float(np.max(np.abs(h_x.numpy() - 1.0)))}

    def correctness(self, nx, ny, nz_global):
        """tol 1e-12 / max_iter 150 solve of the global problem before any timing:
        niters against SURVEY's independent counts, max|x-1| < 1e-13 (every rank
        reports the same values: the loop decisions come from the allreduces)."""
        self.ctx.waxpby(self.n, 0.0, self.xptr, 0.0, self.xptr, self.xptr)
        r = self.prob.solve(150, 1e-12)
        err = self.prob.maxabsdiff()
        want = EXPECTED_NITERS.get((nx, ny, nz_global))
        ok = err < 1e-13 and r["normr"] <= 1e-12 and (want is None or abs(r["niters"] - want) <= 1)
        return {"tol": 1e-12, "max_iter": 150, "niters": r["niters"], "expected_niters": want,
                "normr": r["normr"], "max_abs_x_minus_1": err, "ok": bool(ok),
                "expected_from": "SURVEY 8(c) pins (independent numpy CG), niters +-1"}


def measure_workload(H, D, ctx, stream, world, rank, local, coll_dev, name, steps, warmup,
                     events=False, trace=False, clocks=False, opts=(), setup=None):
    """Generate `name`'s problem, self-check it, time it; a dict of results."""
    import numpy as np
    import torch
    w = WORKLOADS[name]
    slab = D.slab_for(w["nx"], w["ny"], w["nz"], rank, world, w["scaling"])
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    prob = H.Problem(ctx, slab.nx, slab.ny, slab.nz)
    e1.record(stream)
    torch.cuda.synchronize()
    gen_ms = e0.elapsed_time(e1)
    prob.set_option(H.HPCCG_OPT_GRAPH, 1)
    for k, v in opts:
        prob.set_option(k, v)
    out = {"workload": name, "baseline_config": w["cfg"], "nx": slab.nx, "ny": slab.ny,
           "nz_per_gpu": slab.nz, "global_rows": prob.n * world, "global_nnz": prob.info["nnz_global"],
           "scaling": w["scaling"], "gen_ms": round(gen_ms, 3)}
    if setup is not None:
        out.update(setup(prob))
    max_iter = w["max_iter"]
    tol = w["tol"]
    run = CgRunner(H, D, ctx, prob, stream, world, coll_dev, max_iter, tol, local)
    out["tol"], out["max_iter"] = tol, max_iter
    out["correctness"] = run.correctness(slab.nx, slab.ny, slab.nz_global)
    for _ in range(warmup):
        run.step()
    l0 = ctx.launch_count
    clk = ClockSampler(local) if clocks else None
    if clk:
        clk.__enter__()
    main = run.timed(steps)
    out["gpu_launches"] = ctx.launch_count - l0
    ev = tr = None
    if events:
        # the same K steps with CUDA events around every phase (plain launches)
        prob.set_option(H.HPCCG_OPT_TIMING, 1)
        run.step()
        ev = run.timed(steps)
        prob.set_option(H.HPCCG_OPT_TIMING, 0)
    if trace and world == 1 and main.get("graph_mode") == 2:
        # one step of the product configuration with the device-side trace
        # (%globaltimer, first-block start -> last-block end of each CG kernel)
        k_tr = min(main["niters"] // max(steps, 1), 200)
        prob.set_option(H.HPCCG_OPT_TRACE, k_tr)
        run.step()
        t = prob.trace(k_tr).astype("float64")[5:]
        prob.set_option(H.HPCCG_OPT_TRACE, 0)
        if len(t):
            # means over the traced iterations: with the ring-deferred x update
            # every m-th p update also flushes x (a periodic pattern, not noise)
            dur = np.mean((t[:, :, 1] - t[:, :, 0]) / 1e3, axis=0)   # us
            period = float(np.mean(np.diff(t[:, 0, 0])) / 1e3) if len(t) > 1 else None
            tr = {"period_us": round(period, 2) if period else None,
                  "pupdate_us": round(float(dur[0]), 2), "spmv_us": round(float(dur[1]), 2),
                  "update_us": round(float(dur[2]), 2)}
    if clk:
        clk.__exit__(None, None, None)
        out["clocks"] = clk.summary()
    val, ms_max = run.value(main)
    out.update({"value": round(val, 3), "unit": "GFLOP/s", "steps": steps, "warmup": warmup,
                "ms_per_step": round(ms_max / steps, 4),
                "t_iter_us": round(ms_max * 1e3 / max(main["niters"], 1), 3),
                "niters_per_step": main["niters"] // steps, "x_deferred": main.get("x_deferred"),
                "max_abs_x_minus_1": main["err"], "normr": main["r"]["normr"],
                "solve_graph": {5: "on-chip cluster kernel", 4: "one-cluster persistent kernel",
                                3: "cooperative persistent kernel", 2: "while-graph",
                                1: "per-iteration graph", 0: "plain"}.get(main.get("graph_mode"), "?"),
                "l2": run.l2_note})
    out["e2e"] = run.e2e(steps)
    out["_ev"], out["_trace"], out["_n"], out["_nnz_local"] = ev, tr, prob.n, run.nnz_local
    out["_prob"] = prob
    return out


def read_peak_gbs(ctx, stream, nbytes=4 << 30, reps=6):
    """Live pure-read ceiling: our dot kernel (2 reads, no writes) over two
    nbytes vectors, best of `reps` event-timed calls -- the SpMV reads 97 % of
    its bytes, so this is its ceiling; the contract's `peak` (a copy) stays."""
    import torch
    n = nbytes // 8
    x = torch.ones(n, dtype=torch.float64, device="cuda")
    y = torch.ones(n, dtype=torch.float64, device="cuda")
    torch.cuda.synchronize()
    t0, t1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    best = None
    for _ in range(reps + 2):
        t0.record(stream)
        ctx.ddot(n, x.data_ptr(), y.data_ptr())
        t1.record(stream)
        t1.synchronize()
        ms = t0.elapsed_time(t1)
        best = ms if best is None else min(best, ms)
    del x, y
    torch.cuda.empty_cache()
    return 16.0 * n / (best * 1e-3) * 1e-9


def _strip(d):
    return {k: v for k, v in d.items() if not k.startswith("_")}


def run_ours(args):
    import torch
    import torch.distributed as dist

    from paper_conf_sc_valero_laragmtv24_b200 import dist as D
    from paper_conf_sc_valero_laragmtv24_b200 import hpccg as H

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world != args.gpus:
        raise SystemExit(f"--gpus {args.gpus} but WORLD_SIZE={world}")
    if not torch.cuda.is_available():
        raise SystemExit("bench.py needs a CUDA device (no CPU fallback)")
    # --share-device (a test of the N > 1 code path on a one-GPU box): every rank on
    # cuda:0, torch.distributed over gloo, peer-only library contexts (NCCL refuses
    # two ranks on one GPU); the ranks' kernels time-slice, so its numbers are not
    # a scaling measurement
    share = args.share_device and world > 1
    if share:
        local = 0
    transport = "peer" if share else args.transport
    if world > 1 and transport == "peer" and args.halo == "nccl":
        raise SystemExit("--transport peer has no NCCL halo (use --halo fused or peer)")
    if world > 1 and transport == "nccl" and "NCCL_DEBUG" not in os.environ:
        # keep NCCL's communicator-init lines (nRanks per comm) on stderr, off stdout
        os.environ.update({"NCCL_DEBUG": "INFO", "NCCL_DEBUG_SUBSYS": "INIT",
                           "NCCL_DEBUG_FILE": "/dev/stderr"})
    coll_dev = "cpu" if share else "cuda"
    torch.cuda.set_device(local)
    uid = None
    if world > 1:
        if share:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        if transport == "nccl":
            uid = D.broadcast_unique_id(H.hpccg_unique_id)

    stream = torch.cuda.Stream()
    ctx = H.Context(local, stream=stream.cuda_stream, rank=rank, nranks=world, unique_id=uid,
                    peer=(world > 1 and transport == "peer"))
    sr = args.cg_variant == "sr"
    dia = args.spmv_format == "dia"
    opts = [(H.HPCCG_OPT_CG_VARIANT, 1 if sr else 0), (H.HPCCG_OPT_SPMV_FORMAT, 1 if dia else 0)]
    if args.no_defer_x:
        opts.append((H.HPCCG_OPT_DEFER_X, 0))
    elif args.defer_x is not None:
        opts.append((H.HPCCG_OPT_DEFER_X, args.defer_x))
    if args.spmv_cluster is not None:
        opts.append((H.HPCCG_OPT_SPMV_CLUSTER, args.spmv_cluster))
    for kv in args.opt:  # experiments: any library option, e.g. --opt SMEM_HALO=0
        k, v = kv.split("=")
        opts.append((getattr(H, "HPCCG_OPT_" + k), int(v)))
    mode_want = 1 if args.halo == "peer" else 2

    def setup_multirank(prob):
        """The exchange path every rank agrees on (recorded per rank)."""
        if world == 1:
            return {"halo": "none (1 slab)"}
        if transport == "peer":
            # peer-only context: no NCCL anywhere; every rank maps its neighbours'
            # buffers from the exported CUDA-IPC blobs (gathered over torch.distributed)
            prob.peer_attach(D.allgather_peer_blobs(prob.peer_export()))
            prob.set_option(H.HPCCG_OPT_HALO_PEER, mode_want)
            return {"halo": ("peer memory fused into the CG kernels (HALO_PEER 2, while-graph), "
                             "peer-only context" if mode_want == 2 else
                             "peer-memory push + post/collect allreduce kernels (while-graph), "
                             "peer-only context"), "halo_mode": mode_want, "fallback": None}
        if args.halo == "nccl":
            return {"halo": "NCCL send/recv + ncclAllReduce", "halo_mode": 0, "fallback": None}
        # NCCL context: every rank maps its neighbours' buffers (CUDA IPC over NVLink),
        # then a short collective solve proves the mapping end to end; every rank takes
        # the same path (auto falls back to NCCL if any rank fails either stage)
        dec = D.decide_peer_path(
            try_map=lambda: prob.set_option(H.HPCCG_OPT_HALO_PEER, mode_want),
            try_proof=lambda: prob.solve(4, 0.0),
            reset=lambda: prob.set_option(H.HPCCG_OPT_HALO_PEER, 0))
        if not dec["peer"]:
            if args.halo != "auto":
                raise RuntimeError("peer-memory path failed: %s" % dec)
            return {"halo": "NCCL send/recv + ncclAllReduce (peer path refused: %s)" % dec["why"],
                    "halo_mode": 0, "fallback": dec}
        return {"halo": ("peer memory fused into the CG kernels (HALO_PEER 2, while-graph)" if mode_want == 2
                         else "peer-memory push + post/collect allreduce kernels (while-graph)"),
                "halo_mode": mode_want, "fallback": None}

    main = measure_workload(H, D, ctx, stream, world, rank, local, coll_dev, args.workload,
                            args.steps, args.warmup, events=True, trace=not sr, clocks=True,
                            opts=opts, setup=setup_multirank)
    n, nnz_local = main["_n"], main["_nnz_local"]
    defer = int(main.get("x_deferred") or 0)
    ev, trace = main["_ev"], main["_trace"]
    # per-rank record of what actually ran (transport, exchange mode, NCCL view)
    cinfo = ctx.info()
    me = {"rank": rank, "local_rank": local, "device": torch.cuda.get_device_name(local),
          "pci_bus": torch.cuda.get_device_properties(local).pci_bus_id
          if hasattr(torch.cuda.get_device_properties(local), "pci_bus_id") else None,
          "transport": transport if world > 1 else None, "halo_mode": main.get("halo_mode", 0),
          "lib_nranks": cinfo["nranks"], "lib_rank": cinfo["rank"],
          "correct": main["correctness"]["ok"], "niters_tol": main["correctness"]["niters"]}
    ranks = [me]
    if world > 1:
        ranks = [None] * world
        dist.all_gather_object(ranks, me)
    main["_prob"].free()

    # sub-records: the other BASELINE configs of the same metric on this job
    # (1-GPU configs at N = 1; the strong-scaling config at every N)
    subs = {}
    if not args.no_sub_configs:
        names = (["hpccg128", "hpccg20", "hpccg512s"] if world == 1 else ["hpccg512s"])
        for nm in names:
            if nm == args.workload:
                continue
            k = max(1, min(args.steps, WORKLOADS[nm]["sub_steps"]))
            sub = measure_workload(H, D, ctx, stream, world, rank, local, coll_dev, nm, k, 3,
                                   opts=opts, setup=setup_multirank)
            sub["_prob"].free()
            subs[nm] = _strip(sub)
            torch.cuda.empty_cache()
    # configs[4]: the JACC BLAS-1 sweep (AXPY + DOT, 1e3..1e9 per GPU; at N > 1 the
    # DOT is sharded with the allreduce inside hpccg_ddot) -- needs a NCCL or single context
    if not args.no_sub_configs and not (world > 1 and transport == "peer"):
        rows = blas1_sweep(ctx, world, rank, [10 ** k for k in range(3, 10)], 3, reps_cap=50)
        big = rows[-1]
        subs["blas1"] = {
            "workload": "blas1", "baseline_config": 4, "metric": BLAS1_METRIC, "unit": "GB/s",
            "value": round((24.0 + 16.0) * big["n_per_gpu"] * world /
                           ((big["axpy_us"] + big["dot_us"]) * 1e-6) / 1e9, 1),
            "how": "AXPY x += 2.5 y then DOT x.y at n = 1e9 per GPU, host-synchronous calls (launch + "
                   "sync included); inputs round(rand*100) (Fig. 2); max over ranks",
            "all_dot_exact": all(r["dot_exact"] for r in rows) if world == 1 else None,
            "sweep": rows}
    peak_read = read_peak_gbs(ctx, stream) if world == 1 else None

    if rank == 0:
        peak, peak_src = peaks()
        # ELL-27: 8 B value + 4 B column per stored entry, x read + y written once;
        # DIA-27 (--spmv-format dia, "effective"): all 27 value slots, no columns
        spmv_bytes = (216.0 * n if dia else 12.0 * nnz_local) + 16.0 * n
        roof = None
        if ev and ev["spmv_n"] > 0 and ev["spmv_ms"] > 0:
            avg_ms = ev["spmv_ms"] / ev["spmv_n"]
            ach = spmv_bytes / (avg_ms * 1e-3) * 1e-9
            roof = {"bound": "hbm",
                    "kernel": ("spmv27x2_kernel<2> (w = A r with the r.r, w.r epilogue, f2)" if sr else
                               "spmv27x2_kernel<1> (p.Ap epilogue)") +
                              " -- 2 rows/thread; spmv27_kernel if n or the plane is odd" +
                              ("; DIA-27 reading: EFFECTIVE, a different method (SURVEY 8(d): OUT), "
                               "216n + 16n B per launch" if dia else ""),
                    "achieved": round(ach, 1),
                    "peak": peak, "unit": "GB/s", "frac": round(ach / peak, 4),
                    "peak_source": peak_src,
                    "frac_of_8TBs_nominal": round(ach / 8000.0, 4),
                    "traffic": traffic_from_profiles(args.workload + ("_dia" if dia else "")),
                    "algorithmic_bytes_per_launch": spmv_bytes, "avg_launch_us": round(avg_ms * 1e3, 2),
                    "spmv_share_of_step": round(ev["spmv_ms"] / ev["ms"], 4) if ev["ms"] > 0 else None,
                    "measured_in": "events pass: the same K steps re-run with a CUDA event pair "
                                   "around every phase launch on the library stream (plain launches)",
                    "events_pass_ms_per_step": round(ev["ms"] / args.steps, 4)}
            if peak_read:
                roof["peak_read_GBs"] = round(peak_read, 1)
                roof["frac_of_read_peak"] = round(ach / peak_read, 4)
                roof["frac_note"] = ("peak is MEASURED_PEAKS' copy stream (half writes); the SpMV is "
                                     "97 % reads, so frac > 1 is expected -- frac_of_read_peak divides "
                                     "by a pure-read stream measured live here (our dot kernel, 2 x 4 GiB, best of 6)")
            # the fused vector kernels (north_star: >= 75 % of the 8 TB/s HBM peak on
            # "SpMV and fused waxpby/ddot"): x/r update + r.r 48n B, p update 24n B;
            # with the deferred x update (default) r update + r.r 24n, x and p update 40n;
            # deferred over a ring of m + 1 p buffers (m >= 2): per m iterations the p
            # update reads r, p m times, x once and m - 1 old p's, writes p m times and
            # x once: (32 + 8/m) n per iteration on average
            vec = {}
            u_bytes, p_bytes = ((72.0 * n, None) if sr else
                                (24.0 * n, (32.0 + 8.0 / defer) * n) if defer >= 2 else
                                (24.0 * n, 40.0 * n) if defer else (48.0 * n, 24.0 * n))
            u_us = ev["update_ms"] * 1e3 / max(ev["niters"], 1)
            p_us = ev["pupdate_ms"] * 1e3 / max(ev["niters"], 1)
            for nm_k, by, us_ev, us_tr in (("update", u_bytes, u_us, trace and trace["update_us"]),
                                           ("pupdate", p_bytes, p_us, trace and trace["pupdate_us"])):
                if not by or us_ev <= 0:
                    continue
                g_ev = by / (us_ev * 1e-6) * 1e-9
                rec = {"algorithmic_bytes": by, "events_us": round(us_ev, 2), "events_GBs": round(g_ev, 1),
                       "events_frac_of_8TBs": round(g_ev / 8000.0, 4)}
                if us_tr:
                    g_tr = by / (us_tr * 1e-6) * 1e-9
                    rec.update({"in_graph_us": us_tr, "in_graph_GBs": round(g_tr, 1),
                                "in_graph_frac_of_8TBs": round(g_tr / 8000.0, 4),
                                "in_graph_frac_of_measured": round(g_tr / peak, 4)})
                vec[nm_k] = rec
            roof["update_GBs"] = vec.get("update", {}).get("in_graph_GBs") or \
                vec.get("update", {}).get("events_GBs")
            roof["pupdate_GBs"] = vec.get("pupdate", {}).get("in_graph_GBs") or \
                vec.get("pupdate", {}).get("events_GBs")
            roof["vector_kernels"] = dict(vec, target_frac_of_8TBs=0.75,
                                          how="in_graph = device trace (%globaltimer) of the product "
                                              "while-graph; events = the events pass (plain launches)")
            if trace:
                trace["spmv_GBs"] = round(spmv_bytes / (trace["spmv_us"] * 1e-6) * 1e-9, 1)
                trace["how"] = ("device trace (%globaltimer) of one step of the product while-graph: "
                                "median first-block-start -> last-block-end per kernel, iterations 6..")
                roof["in_graph_trace"] = trace
            if main["l2"].startswith("L2 flushed"):
                roof["note"] = ("latency-bound configuration (the problem fits in L2): the fraction is "
                                "not a meaningful target here")
        cpu = None
        if world == 1 and not args.no_cpu_baseline:
            # the oracle's CSR needs ~430 B/row of host RAM: above 2^25 rows it
            # is timed on the 256^3 problem instead (said in `sample`)
            w = WORKLOADS[args.workload]
            ox, oy, oz = (w["nx"], w["ny"], w["nz"]) if n <= (1 << 25) else (256, 256, 256)
            it = main["niters_per_step"]
            cs = oracle_sample(ox, oy, oz, it, args.cpu_budget, sr)
            cpu = {"value": round(cs["value"], 4), "unit": "GFLOP/s", "cores": cs["cores"],
                   "kind": "oracle",
                   "sample": f"oracle CG (C, OpenMP) on the {ox}x{oy}x{oz} problem, "
                             f"{cs['iters']} iterations ({cs['seconds']:.1f} s) of the "
                             f"{it}-iteration step"}
        wl = WORKLOADS[args.workload]
        cfg = {k: main[k] for k in ("workload", "baseline_config", "nx", "ny", "nz_per_gpu", "global_rows",
                                    "global_nnz", "tol", "max_iter", "solve_graph", "l2", "gen_ms")}
        cfg.update({"iters": main["niters_per_step"], "parallelism": f"zslab{world}",
                    "cg_variant": "single-reduction (Chronopoulos-Gear, f2)" if sr else "HPCCG",
                    "x_update": (f"deferred over a ring of {defer + 1} p buffers (HPCCG_OPT_DEFER_X = {defer}, "
                                 f"auto when the CG vectors exceed L2): x += alpha_j p_j applied every "
                                 f"{defer} iterations, 12 nnz + {72 + 8 / defer:g}n B per iteration"
                                 if defer >= 2 else
                                 "deferred into the next p update (HPCCG_OPT_DEFER_X 1): 12 nnz + 80n B "
                                 "per iteration" if defer
                                 else "in the x/r update: 12 nnz + 88n B per iteration"),
                    "spmv_format": ("DIA-27 (columns from stencil offsets) -- EFFECTIVE, a different "
                                    "method (SURVEY 8(d): OUT)") if dia
                    else "ELL-27 (val[27][n] + col[27][n])",
                    "halo": main.get("halo"), "transport": transport if world > 1 else None,
                    "shared_device": bool(share)})
        line = {
            "metric": METRIC, "value": main["value"], "unit": "GFLOP/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": main["ms_per_step"],
            "higher_is_better": True, "scaling": wl["scaling"], "vs_baseline": None, "dtype": "f64",
            "data": "synthetic (HPCCG 27-point problem generated on device, b = A.1)",
            "config": cfg,
            "t_iter_us": main["t_iter_us"],
            "niters_per_step": main["niters_per_step"],
            "max_abs_x_minus_1": main["max_abs_x_minus_1"], "normr": main["normr"],
            "correctness": main["correctness"],
            "ranks": ranks,
            "multi_gpu_ok": (all(r["correct"] and r["lib_nranks"] == world for r in ranks)
                             and len({r["halo_mode"] for r in ranks}) == 1),
            "gpu_launches": main["gpu_launches"],
            "clocks": main.get("clocks"),
            "e2e": main["e2e"],
            "roofline": roof,
            "cpu_baseline": cpu,
            "sub_configs": subs,
        }
        if main.get("fallback"):
            line["peer_fallback"] = main["fallback"]
        print(json.dumps(line), flush=True)
    ctx.close()
    if world > 1:
        dist.destroy_process_group()
    return 0


def f1f4_traffic(key, field):
    """DRAM bytes of the f1 / f4 hot path from the committed ncu summary
    (profiles/r1_ncu_f1f4.json, tools/summarize_f1f4.py)."""
    p = os.path.join(ROOT, "profiles", "r1_ncu_f1f4.json")
    try:
        return json.load(open(p)).get(key, {}).get(field)
    except Exception:
        return None


def traffic_from_profiles(workload):
    """dram bytes per SpMV launch from the committed ncu --set full summary."""
    p = os.path.join(ROOT, "profiles", "spmv_traffic.json")
    if not os.path.exists(p):
        return None
    try:
        return json.load(open(p)).get(workload, {}).get("dram_bytes_per_launch")
    except Exception:
        return None


def blas1_sweep(ctx, world, rank, sizes, warmup, reps_cap=200):
    """The configs[4] sweep: per size, host-synchronous AXPY x += 2.5 y and DOT x.y
    calls (JACC's synchronous constructs) on the paper's inputs
    round(rand*100) (Fig. 2), each rank its own shard of n; the
    seeded 2^24-element pattern is generated on the host and tiled ON THE DEVICE
    (so n = 1e9 costs no 8 GB host copy).  Times: max over ranks.  DOT checked
    against the exact integer (int64 closed form over the tiles) at every n."""
    import numpy as np
    import torch
    import torch.distributed as dist

    import synth
    P = 1 << 24
    xb, yb = synth.jacc_vector(P, 42 + rank), synth.jacc_vector(P, 43 + rank)
    xi, yi = xb.astype(np.int64), yb.astype(np.int64)
    xb_d, yb_d = torch.from_numpy(xb).cuda(), torch.from_numpy(yb).cuda()
    rows = []
    for n in sizes:
        reps_t, rem = divmod(n, P)
        x = xb_d.repeat(reps_t + 1)[:n].contiguous()
        y = yb_d.repeat(reps_t + 1)[:n].contiguous()
        exact_dot = float(reps_t * int(np.dot(xi, yi)) + int(np.dot(xi[:rem], yi[:rem])))
        torch.cuda.synchronize()
        xp, yp = x.data_ptr(), y.data_ptr()   # raw pointers: no per-call torch sync
        res0 = ctx.ddot(n, xp, yp)            # before any AXPY: the exact integer
        reps = max(3, min(reps_cap, int(2e9 / (24 * n))))
        for _ in range(warmup):
            ctx.waxpby(n, 1.0, xp, 2.5, yp, xp)
            ctx.ddot(n, xp, yp)
        if world > 1:
            dist.barrier()
        t0 = time.perf_counter()
        for _ in range(reps):
            ctx.waxpby(n, 1.0, xp, 2.5, yp, xp)
        t_axpy = (time.perf_counter() - t0) / reps
        if world > 1:
            dist.barrier()
        t0 = time.perf_counter()
        for _ in range(reps):
            ctx.ddot(n, xp, yp)
        t_dot = (time.perf_counter() - t0) / reps
        tt = torch.tensor([t_axpy, t_dot], dtype=torch.float64, device="cuda")
        if world > 1:
            dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        t_axpy, t_dot = float(tt[0]), float(tt[1])
        rows.append({"n_per_gpu": n, "axpy_us": round(t_axpy * 1e6, 2),
                     "axpy_GBs": round(world * 24.0 * n / t_axpy / 1e9, 1),
                     "dot_us": round(t_dot * 1e6, 2),
                     "dot_GBs": round(world * 16.0 * n / t_dot / 1e9, 1),
                     "dot_exact": (res0 == exact_dot) if world == 1 else None})
        del x, y
        torch.cuda.empty_cache()
    del xb_d, yb_d
    torch.cuda.empty_cache()
    return rows


def run_blas1(args):
    """BASELINE configs[4]: JACC BLAS-1 sweep, AXPY x += alpha y (hpccg_waxpby(n, 1, x,
    alpha, y, x)) and DOT (hpccg_ddot, host-synchronous like JACC's constructs)
    on the paper's inputs round(rand*100), alpha = 2.5 (Fig. 2), n = 1e3..1e9
    per GPU; multi-GPU: DOT sharded n per rank + NCCL allreduce inside hpccg_ddot."""
    import numpy as np
    import torch
    import torch.distributed as dist

    import synth
    from paper_conf_sc_valero_laragmtv24_b200 import dist as D
    from paper_conf_sc_valero_laragmtv24_b200 import hpccg as H

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    uid = None
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        uid = D.broadcast_unique_id(H.hpccg_unique_id)
    stream = torch.cuda.Stream()
    ctx = H.Context(local, stream=stream.cuda_stream, rank=rank, nranks=world, unique_id=uid)
    sizes = [10 ** k for k in range(3, 10)]
    if args.blas1_max:
        sizes = [s for s in sizes if s <= args.blas1_max]
    clk = ClockSampler(local)
    clk.__enter__()
    rows = blas1_sweep(ctx, world, rank, sizes, args.warmup)
    clk.__exit__(None, None, None)
    # f3: the 2-D constructs (Fig. 2) at SIZE x SIZE, SIZE = 1000 in the paper
    rows2d = []
    for size in [100, 1000, 10000, 31623]:
        if args.blas1_max and size * size > args.blas1_max:
            continue
        n = size * size
        gen = min(n, 1 << 24)
        xh, yh = synth.jacc_vector(gen, 42 + rank), synth.jacc_vector(gen, 43 + rank)
        x = torch.from_numpy(np.resize(xh, n)).cuda()
        y = torch.from_numpy(np.resize(yh, n)).cuda()
        torch.cuda.synchronize()
        xp, yp = x.data_ptr(), y.data_ptr()
        reps = max(3, min(200, int(2e9 / (24 * n))))
        for _ in range(args.warmup):
            ctx.waxpby2d(size, size, size, 1.0, xp, 2.5, yp, xp)
            ctx.ddot2d(size, size, size, xp, yp)
        t0 = time.perf_counter()
        for _ in range(reps):
            ctx.waxpby2d(size, size, size, 1.0, xp, 2.5, yp, xp)
        ta = (time.perf_counter() - t0) / reps
        t0 = time.perf_counter()
        for _ in range(reps):
            ctx.ddot2d(size, size, size, xp, yp)
        td = (time.perf_counter() - t0) / reps
        rows2d.append({"size": size, "axpy2d_us": round(ta * 1e6, 2),
                       "axpy2d_GBs": round(world * 24.0 * n / ta / 1e9, 1),
                       "dot2d_us": round(td * 1e6, 2), "dot2d_GBs": round(world * 16.0 * n / td / 1e9, 1)})
        del x, y
        torch.cuda.empty_cache()
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        # the oracle (as it stands) on a bounded sample: n = 1e8, one AXPY + one DOT
        import oracle
        nb = min(sizes[-1], 10 ** 8)
        xb = np.resize(synth.jacc_vector(min(nb, 1 << 24), 42), nb)
        yb = np.resize(synth.jacc_vector(min(nb, 1 << 24), 43), nb)
        wb = np.empty(nb)
        t0 = time.perf_counter()
        oracle.waxpby(1.0, xb, 2.5, yb, wb)
        t1 = time.perf_counter()
        oracle.ddot(xb, yb)
        t2 = time.perf_counter()
        cpu = {"value": round(40.0 * nb / (t2 - t0) / 1e9, 2), "unit": "GB/s",
               "cores": oracle.get_threads(), "kind": "oracle",
               "sample": f"oracle waxpby + compensated ddot (C, OpenMP) at n = {nb}: "
                         f"AXPY {round((t1 - t0) * 1e3, 2)} ms, DOT {round((t2 - t1) * 1e3, 2)} ms"}
        del xb, yb, wb
    if rank == 0:
        peak, src = peaks()
        big = rows[-1]
        ach = (24.0 + 16.0) * big["n_per_gpu"] / ((big["axpy_us"] + big["dot_us"]) * 1e-6) / 1e9
        roof = {"bound": "hbm", "kernel": "waxpby_kernel + dot_kernel at n = %d per GPU (host-synchronous "
                "calls, launch + sync included)" % big["n_per_gpu"],
                "achieved": round(ach, 1), "peak": peak, "unit": "GB/s", "frac": round(ach / peak, 4),
                "peak_source": src, "axpy_GBs": big["axpy_GBs"], "dot_GBs": big["dot_GBs"],
                "traffic": None}
        line = {"metric": BLAS1_METRIC,
                "value": round((24.0 + 16.0) * big["n_per_gpu"] * world /
                               ((big["axpy_us"] + big["dot_us"]) * 1e-6) / 1e9, 1),
                "unit": "GB/s", "n_gpus": world, "steps": None, "warmup": args.warmup,
                "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64",
                "data": "synthetic round(rand*100), alpha 2.5 (Fig. 2, P:L70-L73)",
                "config": {"workload": "blas1", "baseline_config": 4, "sizes": sizes,
                           "parallelism": f"shard{world}"},
                "sweep": rows, "sweep_2d": rows2d, "peak_hbm_GBs": peak, "peak_source": src,
                "roofline": roof, "clocks": clk.summary(), "cpu_baseline": cpu,
                "gpu_launches_per_call": {"axpy": 1, "dot": 1}}
        print(json.dumps(line), flush=True)
    ctx.close()
    if world > 1:
        dist.destroy_process_group()
    return 0


def run_tridiag(args):
    """the paper's own CG measurement: one iteration of Fig. 12's CG
    on the tridiagonal matrix of SIZE = 1e8.  Reports the
    time per iteration of Fig. 12 as written (variant 0: 3 copies, 1 matvec,
    5 dots, 3 axpys; 208n bytes), fused (variant 1: 112n bytes) and fused with
    x deferred over 8 iterations through a ring of p buffers (variant 2, the
    headline: 97n bytes, bitwise variant 1's results), with the
    CPU oracle's time per iteration beside it (the paper quotes GPU/CPU ratios:
    68x A100, 17x MI100, 4x Max 1550 vs a 64-core EPYC 7742)."""
    import torch

    from paper_conf_sc_valero_laragmtv24_b200 import hpccg as H

    if int(os.environ.get("WORLD_SIZE", "1")) > 1 and int(os.environ.get("RANK", "0")) != 0:
        return 0          # single-device workload: other ranks idle
    n = args.tri_n
    torch.cuda.set_device(int(os.environ.get("LOCAL_RANK", "0")))
    ctx = H.Context(int(os.environ.get("LOCAL_RANK", "0")))
    t = H.Tri(ctx, n)
    K = 20
    res = {}
    with ClockSampler(int(os.environ.get("LOCAL_RANK", "0"))) as clk:
        for v in (0, 1, 2):
            for _ in range(args.warmup):
                t.solve(K + 1, 0.0, v)
            one = min(t.solve(1, 0.0, v)["ms"] for _ in range(args.steps))
            many = min(t.solve(K + 1, 0.0, v)["ms"] for _ in range(args.steps))
            res[v] = (many - one) / K
    l0 = ctx.launch_count
    t.solve(K + 1, 0.0, 2)
    launches = ctx.launch_count - l0
    t.free()
    peak, src = peaks()
    cpu = None
    if not args.no_cpu_baseline:
        import oracle
        tr = oracle.Tri(n)
        o1 = oracle.tri_cg(tr, 1, 0.0)["seconds"]
        o3 = oracle.tri_cg(tr, 3, 0.0)["seconds"]
        cpu_ms = max((o3 - o1) / 2, o1 / 2) * 1e3
        cpu = {"value": round(cpu_ms, 3), "unit": "ms/iteration", "cores": oracle.get_threads(),
               "kind": "oracle", "sample": f"oracle Fig. 12 CG (C, OpenMP, compensated dots) at "
                                           f"n = {n}, 3 iterations"}
    fused_ms = res[2]
    B2 = 97 * n  # variant 2: matvec 40n, r update 24n, p update (32 + 8/8)n
    line = {"metric": TRI_METRIC,
            "value": round(fused_ms, 4), "unit": "ms/iteration", "higher_is_better": False,
            "n_gpus": 1, "steps": args.steps, "warmup": args.warmup, "scaling": "none",
            "vs_baseline": None, "dtype": "f64",
            "data": "synthetic tridiag(1,4,1), r = p = 0.5 (Fig. 12, P:L475-L484; A18)",
            "config": {"workload": "tridiag", "n": n, "variant": "fused (1 matvec+dot, "
                       "1 r update+dot, 1 p update) with x deferred over 8 iterations (variant 2)"},
            "fig12_as_written_ms": round(res[0], 4),
            "fused_x_every_iteration_ms": round(res[1], 4),
            "bytes_per_iteration": {"fused_ring": B2, "fused": 112 * n, "fig12": 208 * n},
            "GBs": {"fused_ring": round(B2 / (fused_ms * 1e-3) / 1e9, 1),
                    "fused": round(112 * n / (res[1] * 1e-3) / 1e9, 1),
                    "fig12": round(208 * n / (res[0] * 1e-3) / 1e9, 1)},
            "roofline": {"bound": "hbm", "achieved": round(B2 / (fused_ms * 1e-3) / 1e9, 1),
                         "peak": peak, "unit": "GB/s",
                         "frac": round(B2 / (fused_ms * 1e-3) / 1e9 / peak, 4),
                         "peak_source": src,
                         "kernel": "the fused iteration (tri_spmv<true> + tri_update<true> + "
                                   "tri_pupdate_ring), averaged over the 8-iteration flush cycle",
                         "traffic": None,
                         "traffic_unit": "DRAM bytes per iteration (ncu of variant 1, SIZE 1e8: "
                                         "see fused_traffic)",
                         "algorithmic_bytes_per_iteration": B2},
            "fused_traffic": (f1f4_traffic("tridiag", "dram_bytes_per_iteration")
                              if n == 100_000_000 else None),
            "gpu_launches_per_iteration": launches / (K + 1),
            "clocks": clk.summary(), "cpu_baseline": cpu,
            "speedup_vs_cpu_oracle": (round(cpu["value"] / fused_ms, 1) if cpu else None)}
    print(json.dumps(line), flush=True)
    ctx.close()
    return 0


def run_lbm(args):
    """the paper's LBM measurement (Fig. 11): the D2Q9 pull step of
    Fig. 10 on SIZE x SIZE = 1000^2, 2 lattices.  Reports ms/step,
    MLUPS and HBM GB/s (144 B per interior site: 9 pulled loads + 9 stores),
    with the CPU oracle's step time beside it (the paper: 20x A100, 14x MI100,
    6.5x Max 1550 vs a 64-core EPYC 7742)."""
    import torch

    import synth
    from paper_conf_sc_valero_laragmtv24_b200 import hpccg as H

    if int(os.environ.get("WORLD_SIZE", "1")) > 1 and int(os.environ.get("RANK", "0")) != 0:
        return 0
    S = args.lbm_size
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    ctx = H.Context(local)
    l = H.Lbm(ctx, S)
    f0 = synth.lbm_state(S, 21)
    l.set(0, f0)
    l.set(1, f0)
    K = 200
    with ClockSampler(local) as clk:
        for _ in range(args.warmup):
            l.run(10, 0.8)
        ms = min(l.run(K, 0.8) for _ in range(args.steps)) / K
    l.free()
    sites = (S - 2) ** 2
    gbs = 144.0 * sites / (ms * 1e-3) / 1e9
    peak, src = peaks()
    cpu = None
    if not args.no_cpu_baseline:
        import numpy as np
        import oracle
        a, b, f = f0.copy(), f0.copy(), np.zeros_like(f0)
        t0 = time.perf_counter()
        for _ in range(5):
            oracle.lbm_step(S, a, f, b, 0.8)
            a, b = b, a
        cms = (time.perf_counter() - t0) / 5 * 1e3
        cpu = {"value": round(cms, 3), "unit": "ms/step", "cores": oracle.get_threads(),
               "kind": "oracle", "sample": f"oracle Fig. 10 step (C, OpenMP) at {S}^2, 5 steps"}
    line = {"metric": LBM_METRIC,
            "value": round(ms, 5), "unit": "ms/step", "higher_is_better": False, "n_gpus": 1,
            "steps": args.steps, "warmup": args.warmup, "scaling": "none", "vs_baseline": None,
            "dtype": "f64", "data": "synthetic positive D2Q9 state (seeded), tau 0.8",
            "config": {"workload": "lbm", "size": S, "steps_per_sample": K},
            "MLUPS": round(sites / (ms * 1e-3) / 1e6, 1),
            "roofline": {"bound": "hbm", "achieved": round(gbs, 1), "peak": peak, "unit": "GB/s",
                         "frac": round(gbs / peak, 4), "peak_source": src,
                         "algorithmic_bytes_per_step": 144 * sites,
                         "kernel": "lbm_pull_kernel<0, 1>",
                         "traffic": f1f4_traffic("lbm", "dram_bytes_per_launch") if S == 1000 else None,
                         "traffic_note": "cold-cache ncu replay: the step's writes mostly stay in L2 "
                                         "(read 72.0 MB = the pulled lattice once)"},
            "clocks": clk.summary(), "cpu_baseline": cpu,
            "speedup_vs_cpu_oracle": round(cpu["value"] / ms, 1) if cpu else None}
    print(json.dumps(line), flush=True)
    ctx.close()
    return 0


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--workload", choices=sorted(WORKLOADS) + ["blas1", "tridiag", "lbm"],
                    default="hpccg256",
                    help="hpccg256 (default, every N: configs[2], 256^3 per GPU, weak) -- its line "
                         "carries configs[1] / [0] / [3] as sub_configs")
    ap.add_argument("--blas1-max", type=int, default=None, help="largest BLAS-1 n")
    ap.add_argument("--tri-n", type=int, default=100_000_000, help="tridiag SIZE (P:L475)")
    ap.add_argument("--lbm-size", type=int, default=1000, help="LBM SIZE (P:L411)")
    ap.add_argument("--iters", type=int, default=None, help="override CG iterations per step")
    ap.add_argument("--halo", choices=["auto", "nccl", "peer", "fused"], default="auto",
                    help="multi-GPU exchange: peer memory fused into the CG kernels (HALO_PEER 2, "
                         "auto, both CG variants), our separate peer-memory kernels (HALO_PEER 1), "
                         "or NCCL; auto falls back to NCCL if CUDA IPC is refused")
    ap.add_argument("--transport", choices=["nccl", "peer"], default="nccl",
                    help="N > 1 library context: NCCL communicator (bootstrap + fallback), or "
                         "peer-only (CUDA IPC blobs over torch.distributed, no NCCL)")
    ap.add_argument("--share-device", action="store_true",
                    help="test of the N > 1 code path on one GPU: all ranks on cuda:0, gloo, "
                         "peer-only contexts (time-sliced kernels: not a scaling number)")
    ap.add_argument("--cg-variant", choices=["hpccg", "sr"], default="hpccg",
                    help="hpccg: HPCCG's CG (default); sr: single-reduction CG (SURVEY f2)")
    ap.add_argument("--spmv-format", choices=["ell", "dia"], default="ell",
                    help="HPCCG_OPT_SPMV_FORMAT: ELL-27 (default) or the DIA-27 reading (no col[]) -- "
                         "EFFECTIVE numbers of a different method (SURVEY 8(d): OUT), never the headline")
    ap.add_argument("--no-defer-x", action="store_true",
                    help="HPCCG_OPT_DEFER_X 0: update x in the x/r update (88n instead of 80n B/iteration)")
    ap.add_argument("--opt", action="append", default=[], metavar="NAME=VALUE",
                    help="set HPCCG_OPT_<NAME> on every CG problem (experiments; repeatable)")
    ap.add_argument("--spmv-cluster", type=int, default=None, choices=[-1, 0, 1],
                    help="HPCCG_OPT_SPMV_CLUSTER: the CG SpMV in 8-CTA clusters, one p.Ap partial "
                         "per cluster (default: the library's)")
    ap.add_argument("--defer-x", type=int, default=None,
                    help="HPCCG_OPT_DEFER_X: 1 = x deferred by one iteration, m = 2..8 over a ring of "
                         "m + 1 p buffers (default: the library's auto)")
    ap.add_argument("--no-sub-configs", action="store_true",
                    help="skip the configs[1] / [0] / [3] sub-records of the CG line")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-budget", type=float, default=12.0, help="seconds of oracle CG")
    ap.add_argument("--ref-iters", type=int, default=None,
                    help="oracle iterations per reference step (default per workload)")
    args = ap.parse_args()
    if args.warmup < 3:
        raise SystemExit("--warmup must be >= 3")
    if args.workload == "lbm":
        if args.impl == "reference":
            return run_reference_lbm(args)
        return run_lbm(args)
    if args.workload == "tridiag":
        if args.impl == "reference":
            return run_reference_tridiag(args)
        return run_tridiag(args)
    if args.workload == "blas1":
        if args.impl == "reference":
            return run_reference_blas1(args)
        return run_blas1(args)
    w = dict(WORKLOADS[args.workload])
    if args.iters:                       # fixed iteration count (tol 0), e.g. for tests
        w.update(max_iter=args.iters + 1, tol=0.0)
        WORKLOADS[args.workload] = w
    if args.impl == "reference":
        return run_reference(args, w)
    return run_ours(args)


if __name__ == "__main__":
    sys.exit(main())

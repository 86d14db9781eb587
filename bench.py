#!/usr/bin/env python
"""bench.py -- HPCCG CG hot path on B200 (BASELINE.json metric).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
                    [--workload hpccg128|hpccg20|hpccg256|hpccg512s]

One STEP = one whole HPCCG solve on the synthetic on-device-generated problem:
init (p = x, Ap = A p, r = b - Ap, r.r) + `iters` CG iterations (SpMV with
fused p.Ap, fused x/r update + r.r, p update; device-side scalars; CUDA-graph
replay) + the max|x - 1| verification -- rows a.2-a.9 of DESIGN.md.  The
problem (a.1) is generated once per run (HPCCG times only the solve); its
time is reported as config.gen_ms.  x is reset to 0 (x0, A5) before every
step by our waxpby kernel.

value = CG GFLOP/s of the whole job = sum over ranks of niters (2 nnz + 10 n)
        / max-over-ranks device time of the K timed steps (exact nnz, A15).
e2e   = the same metric through the public C-ABI with HOST buffers: every
        step copies x0 from pinned host memory in and the solution x back out.
roofline = the SpMV kernel (dominant), algorithmic bytes 12 nnz + 16 n per
        launch / its CUDA-event launch duration inside the timed region.
Multi-GPU (torchrun): z-slab weak scaling, one rank per GPU, NCCL halo +
        allreduce inside the library; torch.distributed only bootstraps.
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
    # name: (nx, ny, nz, CG iterations, BASELINE config index, scaling)
    # weak: nz planes per GPU; strong: nz global planes split over the GPUs
    "hpccg128": (128, 128, 128, 500, 1, "weak"),
    "hpccg20": (20, 30, 10, 149, 0, "weak"),
    "hpccg256": (256, 256, 256, 200, 2, "weak"),
    "hpccg512s": (512, 512, 512, 200, 3, "strong"),
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


def run_reference(args, nx, ny, nz, iters, cfg_index):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    import oracle
    oracle.build()
    prob = oracle.generate(nx, ny, nz)
    m = max(1, min(iters, args.ref_iters))
    sr = args.cg_variant == "sr"
    for _ in range(args.warmup):
        oracle_cg_timed(prob, m + 1, sr)
    tot, flops = 0.0, 0.0
    for _ in range(args.steps):
        r, t = oracle_cg_timed(prob, m + 1, sr)
        tot += t
        flops += cg_flops(r["niters"], prob.nnz, prob.n)
    val = flops / tot * 1e-9
    sample = (f"oracle CG on the {nx}x{ny}x{nz} problem, {m} iterations per step "
              f"(bounded sample of the {iters}-iteration workload), OpenMP all host cores")
    line = {
        "metric": METRIC, "value": round(val, 4), "unit": "GFLOP/s", "impl": "reference",
        "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": round(tot / args.steps * 1e3, 3), "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "f64",
        "data": "synthetic (HPCCG generation, deterministic)",
        "config": {"workload": args.workload, "baseline_config": cfg_index, "nx": nx, "ny": ny,
                   "nz": nz, "iters_per_step": m},
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

def run_ours(args, nx, ny, nz, iters, cfg_index, scaling):
    import numpy as np
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
    coll_dev = "cpu" if share else "cuda"
    torch.cuda.set_device(local)
    slab = D.slab_for(nx, ny, nz, rank, world, scaling)
    nz = slab.nz
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
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    prob = H.Problem(ctx, nx, ny, nz)
    e1.record(stream)
    torch.cuda.synchronize()
    gen_ms = e0.elapsed_time(e1)
    n, nnz_local = prob.n, prob.info["nnz_local"]
    nnz_global = prob.info["nnz_global"]
    prob.set_option(H.HPCCG_OPT_GRAPH, 1)
    sr = args.cg_variant == "sr"
    prob.set_option(H.HPCCG_OPT_CG_VARIANT, 1 if sr else 0)
    dia = args.spmv_format == "dia"
    prob.set_option(H.HPCCG_OPT_SPMV_FORMAT, 1 if dia else 0)
    halo = "none (1 slab)"
    if world > 1 and transport == "peer":
        # peer-only context: no NCCL anywhere; every rank maps its neighbours' buffers
        # from the exported CUDA-IPC blobs (gathered over torch.distributed)
        prob.peer_attach(D.allgather_peer_blobs(prob.peer_export()))
        mode = 1 if args.halo == "peer" else 2
        prob.set_option(H.HPCCG_OPT_HALO_PEER, mode)
        halo = ("peer memory fused into the CG kernels (HALO_PEER 2, while-graph), peer-only context"
                if mode == 2 else
                "peer-memory push + post/collect allreduce kernels (while-graph), peer-only context")
    elif world > 1:
        halo = "NCCL send/recv + ncclAllReduce"
        if args.halo in ("peer", "fused", "auto"):
            # collective: every rank maps its neighbours' buffers (CUDA IPC over NVLink);
            # auto = fused (the exchange and the allreduce(s) inside the CG kernels,
            # either CG variant); peer = the separate peer kernels; auto falls back to
            # NCCL if the mapping is refused
            mode = 1 if args.halo == "peer" else 2
            err = None
            try:
                prob.set_option(H.HPCCG_OPT_HALO_PEER, mode)
                # a short collective solve proves the peer mapping end to end (a wait
                # that times out returns an error instead of hanging)
                prob.solve(4, 0.0)
            except H.HpccgError as e:
                err = str(e)
            ok = torch.tensor([0.0 if err else 1.0], device=torch.device("cuda", local))
            dist.all_reduce(ok, op=dist.ReduceOp.MIN)   # every rank takes the same path
            if ok.item() == 1.0:
                halo = ("peer memory fused into the CG kernels (HALO_PEER 2, while-graph)" if mode == 2
                        else "peer-memory push + post/collect allreduce kernels (while-graph)")
            else:
                if args.halo != "auto":
                    raise RuntimeError("peer-memory path failed: %s" % err)
                prob.set_option(H.HPCCG_OPT_HALO_PEER, 0)
                halo = "NCCL (peer path failed on some rank: %s)" % err
    xptr = prob.vec_ptr(H.HPCCG_VEC_X)
    # working set (ELL 324 B/row + 6 vectors): when it fits in L2, flush L2
    # between timed steps (outside the timed events) so no step starts warm
    l2_bytes = torch.cuda.get_device_properties(local).L2_cache_size
    work_bytes = (324 + 6 * 8) * n
    flush_buf = None
    if work_bytes < l2_bytes:
        flush_buf = torch.empty(2 * l2_bytes // 8, dtype=torch.float64, device="cuda")
    l2_note = ("L2 flushed between timed steps (a %d MB write; working set %.1f MB < L2 %.0f MB); "
               "per-step events" % (2 * l2_bytes >> 20, work_bytes / 1e6, l2_bytes / 1e6)
               if flush_buf is not None else
               "inputs larger than L2 (ELL %.0f MB/GPU > %.0f MB)" % (324e-6 * n, l2_bytes / 1e6))

    def flush():
        with torch.cuda.stream(stream):
            flush_buf.zero_()

    def barrier():
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()

    def step():
        ctx.waxpby(n, 0.0, xptr, 0.0, xptr, xptr)        # x0 = 0 (A5)
        r = prob.solve(iters + 1, 0.0)                     # `iters` iterations (A4)
        err = prob.maxabsdiff()
        return r, err

    def timed(k_steps):
        """K steps between barriers; CUDA events on the library stream (one
        pair per step, L2 flushed outside them, when the problem fits in L2)."""
        t0, t1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        acc = {"spmv_ms": 0.0, "spmv_n": 0, "niters": 0, "update_ms": 0.0, "pupdate_ms": 0.0}
        barrier()
        if flush_buf is not None:
            ms = 0.0
            for _ in range(k_steps):
                flush()
                t0.record(stream)
                r, err = step()
                t1.record(stream)
                t1.synchronize()
                ms += t0.elapsed_time(t1)
                st = prob.stats()
                acc["spmv_ms"] += st["spmv_ms"]
                acc["spmv_n"] += st["spmv_launches"]
                acc["update_ms"] += st["update_ms"]
                acc["pupdate_ms"] += st["pupdate_ms"]
                acc["niters"] += r["niters"]
                acc["graph_mode"] = st["graph_mode"]
            barrier()
            acc["ms"], acc["r"], acc["err"] = ms, r, err
            return acc
        t0.record(stream)
        for _ in range(k_steps):
            r, err = step()
            st = prob.stats()
            acc["spmv_ms"] += st["spmv_ms"]
            acc["spmv_n"] += st["spmv_launches"]
            acc["update_ms"] += st["update_ms"]
            acc["pupdate_ms"] += st["pupdate_ms"]
            acc["niters"] += r["niters"]
            acc["graph_mode"] = st["graph_mode"]
        t1.record(stream)
        barrier()
        acc["ms"] = t0.elapsed_time(t1)
        acc["r"], acc["err"] = r, err
        return acc

    for _ in range(args.warmup):
        step()
    l0 = ctx.launch_count
    with ClockSampler(local) as clk:
        # (1) the product configuration: whole solve = one graph with a
        #     device-driven while node; this region gives `value`
        main = timed(args.steps)
        launches = ctx.launch_count - l0
        # (2) the same K steps with CUDA events around every phase (plain
        #     launches): the SpMV roofline and the phase split come from here
        prob.set_option(H.HPCCG_OPT_TIMING, 1)
        step()
        ev = timed(args.steps)
        prob.set_option(H.HPCCG_OPT_TIMING, 0)
        # (3) one step of the product configuration with the device-side
        #     trace (%globaltimer, first-block start -> last-block end of each
        #     CG kernel inside the while-graph): per-kernel times with no events
        trace = None
        if world == 1 and not sr and main.get("graph_mode") == 2:
            k_tr = min(iters, 200)
            prob.set_option(H.HPCCG_OPT_TRACE, k_tr)
            step()
            tr = prob.trace(k_tr).astype("float64")[5:]
            prob.set_option(H.HPCCG_OPT_TRACE, 0)
            if len(tr):
                dur = np.median((tr[:, :, 1] - tr[:, :, 0]) / 1e3, axis=0)   # us
                period = float(np.median(np.diff(tr[:, 0, 0])) / 1e3) if len(tr) > 1 else None
                trace = {"period_us": round(period, 2) if period else None,
                         "pupdate_us": round(float(dur[0]), 2), "spmv_us": round(float(dur[1]), 2),
                         "update_us": round(float(dur[2]), 2)}
        # (4) the other SpMV reading of the same matrix (ELL-27 <-> DIA-27,
        #     HPCCG_OPT_SPMV_FORMAT), same K steps in the product configuration:
        #     reported beside the line, never as `value`
        prob.set_option(H.HPCCG_OPT_SPMV_FORMAT, 0 if dia else 1)
        step()
        alt = timed(args.steps)
        prob.set_option(H.HPCCG_OPT_SPMV_FORMAT, 1 if dia else 0)
    ms = main["ms"]
    niters_tot = main["niters"]
    r, err = main["r"], main["err"]
    spmv_ms, spmv_n = ev["spmv_ms"], ev["spmv_n"]
    ms_max, flops = D.max_time_sum_work(ms, cg_flops(niters_tot, nnz_local, n), coll_dev)
    value = flops / (ms_max * 1e-3) * 1e-9
    alt_ms, alt_flops = D.max_time_sum_work(alt["ms"], cg_flops(alt["niters"], nnz_local, n), coll_dev)
    alt_line = {"spmv_format": "ELL-27" if dia else "DIA-27 (HPCCG_OPT_SPMV_FORMAT 1)",
                "value": round(alt_flops / (alt_ms * 1e-3) * 1e-9, 3), "unit": "GFLOP/s",
                "t_iter_us": round(alt_ms * 1e3 / max(alt["niters"], 1), 3),
                "same_normr_bits": alt["r"]["normr"] == r["normr"] and alt["niters"] == niters_tot,
                "how": "the same K steps, same timing rules, the other reading of the same "
                       "slot-major matrix (bench.py region 4); not the headline" +
                       ("; this size runs the persistent / on-chip solve, which reads col[] in "
                        "both readings" if main.get("graph_mode") in (3, 4, 5) else "")}

    # ---- e2e: public API with host buffers (pinned) each step
    h_x0 = torch.zeros(n, dtype=torch.float64).pin_memory()
    h_x = torch.empty(n, dtype=torch.float64).pin_memory()

    def step_e2e():
        prob.set_vec_ptr(H.HPCCG_VEC_X, h_x0.data_ptr())   # H2D 8n
        r = prob.solve(iters + 1, 0.0)
        prob.get_vec_ptr(H.HPCCG_VEC_X, h_x.data_ptr())    # D2H 8n
        err = prob.maxabsdiff()                             # D2H 8 B
        return r, err

    step_e2e()
    barrier()
    t0, t1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ni_e2e, te_local = 0, 0.0
    if flush_buf is not None:          # same L2 rule as the device-timed region
        for _ in range(args.steps):
            flush()
            t0.record(stream)
            r_e, _ = step_e2e()
            t1.record(stream)
            t1.synchronize()
            te_local += t0.elapsed_time(t1)
            ni_e2e += r_e["niters"]
        barrier()
    else:
        t0.record(stream)
        for _ in range(args.steps):
            r_e, _ = step_e2e()
            ni_e2e += r_e["niters"]
        t1.record(stream)
        barrier()
        te_local = t0.elapsed_time(t1)
    te, fe = D.max_time_sum_work(te_local, cg_flops(ni_e2e, nnz_local, n), coll_dev)
    e2e_value = fe / (te * 1e-3) * 1e-9
    x_host_err = float(np.max(np.abs(h_x.numpy() - 1.0)))

    if rank == 0:
        peak, peak_src = peaks()
        # ELL-27: 8 B value + 4 B column per stored entry, x read + y written once;
        # DIA-27 (--spmv-format dia): all 27 value slots (padding included), no columns
        spmv_bytes = (216.0 * n if dia else 12.0 * nnz_local) + 16.0 * n
        roof = None
        if spmv_n > 0 and spmv_ms > 0:
            avg_ms = spmv_ms / spmv_n
            ach = spmv_bytes / (avg_ms * 1e-3) * 1e-9
            roof = {"bound": "hbm",
                    "kernel": ("spmv27x2_kernel<2> (w = A r with the r.r, w.r epilogue, f2)" if sr else
                               "spmv27x2_kernel<1> (p.Ap epilogue)") +
                              " -- 2 rows/thread; spmv27_kernel if n or the plane is odd" +
                              ("; DIA-27 reading (columns formed from the stencil offsets, "
                               "216n + 16n B per launch)" if dia else ""),
                    "achieved": round(ach, 1),
                    "peak": peak, "unit": "GB/s", "frac": round(ach / peak, 4),
                    "frac_of_8TBs_nominal": round(ach / 8000.0, 4),
                    "traffic": traffic_from_profiles(args.workload + ("_dia" if dia else "")),
                    "algorithmic_bytes_per_launch": spmv_bytes, "avg_launch_us": round(avg_ms * 1e3, 2),
                    "peak_source": peak_src,
                    "spmv_share_of_step": round(spmv_ms / ev["ms"], 4) if ev["ms"] > 0 else None,
                    "measured_in": "events pass: the same K steps re-run with a CUDA event pair "
                                   "around every phase launch (plain launches, bench.py region 2)",
                    "events_pass_ms_per_step": round(ev["ms"] / args.steps, 4),
                    "update_avg_us": round(ev["update_ms"] * 1e3 / max(ev["niters"], 1), 2),
                    "pupdate_avg_us": round(ev["pupdate_ms"] * 1e3 / max(ev["niters"], 1), 2)}
            # the fused vector kernels against the same peak (north_star: >= 75 % of HBM peak
            # on "SpMV and fused waxpby/ddot"): x/r update + r.r 48n B, p update 24n B
            if trace:
                trace["spmv_GBs"] = round(spmv_bytes / (trace["spmv_us"] * 1e-6) * 1e-9, 1)
                trace["update_GBs"] = round(48.0 * n / (trace["update_us"] * 1e-6) * 1e-9, 1)
                trace["pupdate_GBs"] = round(24.0 * n / (trace["pupdate_us"] * 1e-6) * 1e-9, 1)
                trace["how"] = ("device trace (%globaltimer) of one step of the product while-graph: "
                                "median first-block-start -> last-block-end per kernel, iterations 6..")
                roof["in_graph_trace"] = trace
            if ev["update_ms"] > 0 and not sr:
                u_us = ev["update_ms"] * 1e3 / max(ev["niters"], 1)
                p_us = ev["pupdate_ms"] * 1e3 / max(ev["niters"], 1)
                roof["update_GBs"] = round(48.0 * n / (u_us * 1e-6) * 1e-9, 1)
                roof["pupdate_GBs"] = round(24.0 * n / (p_us * 1e-6) * 1e-9, 1) if p_us > 0 else None
            elif ev["update_ms"] > 0:
                u_us = ev["update_ms"] * 1e3 / max(ev["niters"], 1)
                roof["update_GBs"] = round(72.0 * n / (u_us * 1e-6) * 1e-9, 1)
            if flush_buf is not None:
                roof["note"] = ("latency-bound configuration (the problem fits in L2; the product path is "
                                "one on-chip kernel): the fraction is not a meaningful target here")
        cpu = None
        if world == 1 and not args.no_cpu_baseline:
            # the oracle's CSR needs ~430 B/row of host RAM: above 2^25 rows it
            # is timed on the 256^3 problem instead (said in `sample`)
            ox, oy, oz = (nx, ny, nz) if n <= (1 << 25) else (256, 256, 256)
            cs = oracle_sample(ox, oy, oz, iters, args.cpu_budget, sr)
            nx_s = f"{ox}x{oy}x{oz}"
            cpu = {"value": round(cs["value"], 4), "unit": "GFLOP/s", "cores": cs["cores"],
                   "kind": "oracle",
                   "sample": f"oracle CG (C, OpenMP) on the {nx_s} problem, "
                             f"{cs['iters']} iterations ({cs['seconds']:.1f} s) of the "
                             f"{iters}-iteration step"}
        t_iter_us = ms_max * 1e3 / max(niters_tot, 1)
        line = {
            "metric": METRIC, "value": round(value, 3), "unit": "GFLOP/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(ms_max / args.steps, 4),
            "higher_is_better": True, "scaling": scaling, "vs_baseline": None, "dtype": "f64",
            "data": "synthetic (HPCCG 27-point problem generated on device, b = A.1)",
            "config": {"workload": args.workload, "baseline_config": cfg_index,
                       "nx": nx, "ny": ny, "nz_per_gpu": nz, "iters": iters,
                       "global_rows": n * world, "global_nnz": nnz_global,
                       "parallelism": f"zslab{world}",
                       "cg_variant": "single-reduction (Chronopoulos-Gear, f2)" if sr else "HPCCG",
                       "spmv_format": "DIA-27 (val[27][n], columns from stencil offsets)" if dia
                                      else "ELL-27 (val[27][n] + col[27][n])",
                       "halo": halo, "transport": transport if world > 1 else None,
                       "shared_device": bool(share),
                       "solve_graph": {5: "on-chip cluster kernel", 4: "one-cluster persistent kernel",
                                       3: "cooperative persistent kernel", 2: "while-graph",
                                       1: "per-iteration graph", 0: "plain"}.get(
                           main.get("graph_mode"), "?"),
                       "l2": l2_note,
                       "gen_ms": round(gen_ms, 3)},
            "t_iter_us": round(t_iter_us, 3),
            "alt_spmv_format": alt_line,
            "niters_per_step": niters_tot // args.steps,
            "max_abs_x_minus_1": err, "normr": r["normr"],
            "gpu_launches": launches,
            "clocks": clk.summary(),
            "e2e": {"value": round(e2e_value, 3), "unit": "GFLOP/s", "h2d_bytes_per_step": 8 * n,
                    "d2h_bytes_per_step": 8 * n + 8, "max_abs_x_minus_1_host": x_host_err},
            "roofline": roof,
            "cpu_baseline": cpu,
        }
        print(json.dumps(line), flush=True)
    prob.free()
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
    rows = []
    clk = ClockSampler(local)
    clk.__enter__()
    for n in sizes:
        # seeded inputs generated once on the host (splitmix64), per-rank shard
        gen = min(n, 1 << 24)
        xh = synth.jacc_vector(gen, 42 + rank)
        yh = synth.jacc_vector(gen, 43 + rank)
        x = torch.from_numpy(np.resize(xh, n)).cuda() if n > gen else torch.from_numpy(xh).cuda()
        y = torch.from_numpy(np.resize(yh, n)).cuda() if n > gen else torch.from_numpy(yh).cuda()
        torch.cuda.synchronize()
        xp, yp = x.data_ptr(), y.data_ptr()   # raw pointers: no per-call torch sync
        reps = max(3, min(200, int(2e9 / (24 * n))))
        for _ in range(args.warmup):
            ctx.waxpby(n, 1.0, xp, 2.5, yp, xp)
            ctx.ddot(n, xp, yp)
        # AXPY, host-synchronous per call
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
            res = ctx.ddot(n, xp, yp)
        t_dot = (time.perf_counter() - t0) / reps
        tt = torch.tensor([t_axpy, t_dot], dtype=torch.float64, device="cuda")
        if world > 1:
            dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        t_axpy, t_dot = float(tt[0]), float(tt[1])
        # exactness: x stays integer-valued (multiples of 0.5 scaled) -> dot exact
        xc = x.cpu().numpy()
        exact = None
        if world == 1 and n <= 10 ** 8:
            exact = float(np.dot((2 * xc).astype(np.int64), y.cpu().numpy().astype(np.int64))) / 2
        rows.append({"n_per_gpu": n, "axpy_us": round(t_axpy * 1e6, 2),
                     "axpy_GBs": round(world * 24.0 * n / t_axpy / 1e9, 1),
                     "dot_us": round(t_dot * 1e6, 2),
                     "dot_GBs": round(world * 16.0 * n / t_dot / 1e9, 1),
                     "dot_exact": (res == exact) if exact is not None else None})
        del x, y
        torch.cuda.empty_cache()
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
    5 dots, 3 axpys; 208n bytes) and fused (variant 1: 112n bytes), with the
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
        for v in (0, 1):
            for _ in range(args.warmup):
                t.solve(K + 1, 0.0, v)
            one = min(t.solve(1, 0.0, v)["ms"] for _ in range(args.steps))
            many = min(t.solve(K + 1, 0.0, v)["ms"] for _ in range(args.steps))
            res[v] = (many - one) / K
    l0 = ctx.launch_count
    t.solve(K + 1, 0.0, 1)
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
    fused_ms = res[1]
    line = {"metric": TRI_METRIC,
            "value": round(fused_ms, 4), "unit": "ms/iteration", "higher_is_better": False,
            "n_gpus": 1, "steps": args.steps, "warmup": args.warmup, "scaling": "none",
            "vs_baseline": None, "dtype": "f64",
            "data": "synthetic tridiag(1,4,1), r = p = 0.5 (Fig. 12, P:L475-L484; A18)",
            "config": {"workload": "tridiag", "n": n, "variant": "fused (1 matvec+dot, "
                       "1 update+dot, 1 p update)"},
            "fig12_as_written_ms": round(res[0], 4),
            "bytes_per_iteration": {"fused": 112 * n, "fig12": 208 * n},
            "GBs": {"fused": round(112 * n / (fused_ms * 1e-3) / 1e9, 1),
                    "fig12": round(208 * n / (res[0] * 1e-3) / 1e9, 1)},
            "roofline": {"bound": "hbm", "achieved": round(112 * n / (fused_ms * 1e-3) / 1e9, 1),
                         "peak": peak, "unit": "GB/s",
                         "frac": round(112 * n / (fused_ms * 1e-3) / 1e9 / peak, 4),
                         "peak_source": src,
                         "kernel": "the fused iteration (tri_spmv<true> + tri_update + tri_pupdate)",
                         "traffic": (f1f4_traffic("tridiag", "dram_bytes_per_iteration")
                                     if n == 100_000_000 else None),
                         "traffic_unit": "DRAM bytes per iteration (ncu, SIZE 1e8)",
                         "algorithmic_bytes_per_iteration": 112 * n},
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
                    default="hpccg128")
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
                    help="HPCCG_OPT_SPMV_FORMAT: ELL-27 (default) or the DIA-27 reading (no col[])")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-budget", type=float, default=12.0, help="seconds of oracle CG")
    ap.add_argument("--ref-iters", type=int, default=20, help="oracle iterations per reference step")
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
    nx, ny, nz, iters, cfg, scaling = WORKLOADS[args.workload]
    if args.iters:
        iters = args.iters
    if args.impl == "reference":
        if scaling == "strong":
            nz = nz // args.gpus
        return run_reference(args, nx, ny, nz, iters, cfg)
    return run_ours(args, nx, ny, nz, iters, cfg, scaling)


if __name__ == "__main__":
    sys.exit(main())

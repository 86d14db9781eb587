"""bench.py's N > 1 code path on a one-GPU box: torchrun with 2 / 3 ranks and
--share-device (every rank on cuda:0, torch.distributed over gloo, peer-only
library contexts: the fused exchange and allreduces over CUDA IPC between the
rank processes).  Checks the one JSON line rank 0 prints -- whole-job work,
weak / strong slab split, the solution error of the global problem -- not the
speed (the ranks' kernels time-slice on the one GPU)."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _torchrun(n, *argv, port):
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={n}",
           "--master-addr", "127.0.0.1", "--master-port", str(port),
           os.path.join(ROOT, "bench.py"), "--gpus", str(n), "--share-device", *argv]
    return subprocess.run(cmd, cwd=ROOT, capture_output=True, text=True, timeout=600)


@pytest.mark.gpu
@pytest.mark.parametrize("n,variant,halo,port", [(2, "hpccg", "auto", 29611), (3, "hpccg", "peer", 29612),
                                                 (2, "sr", "auto", 29613)])
def test_bench_multirank_shared_device(n, variant, halo, port):
    r = _torchrun(n, "--workload", "hpccg20", "--iters", "30", "--steps", "3", "--warmup", "3",
                  "--cg-variant", variant, "--halo", halo, "--no-sub-configs", port=port)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, r.stdout[-2000:]
    d = json.loads(lines[0])
    assert d["n_gpus"] == n and d["scaling"] == "weak" and d["value"] > 0
    c = d["config"]
    assert c["parallelism"] == f"zslab{n}" and c["shared_device"] is True
    assert c["transport"] == "peer" and "peer-only" in c["halo"]
    assert c["global_rows"] == 20 * 30 * 10 * n
    assert d["niters_per_step"] == 30
    assert d["max_abs_x_minus_1"] < 1.0          # 30 iterations: on the way to x = 1
    assert d["e2e"]["value"] > 0 and d["gpu_launches"] > 0
    # the N > 1 line verifies itself: the tol 1e-12 solve of the global problem,
    # and per rank the transport / exchange mode / library rank count
    cor = d["correctness"]
    assert cor["ok"] and cor["max_abs_x_minus_1"] < 1e-13 and cor["normr"] <= 1e-12
    ranks = d["ranks"]
    assert [q["rank"] for q in ranks] == list(range(n))
    assert all(q["transport"] == "peer" and q["lib_nranks"] == n and q["correct"] for q in ranks)
    assert {q["halo_mode"] for q in ranks} == {1 if halo == "peer" else 2}
    assert d["multi_gpu_ok"] is True


@pytest.mark.gpu
def test_bench_multirank_strong_split():
    """Strong scaling (hpccg512s's split rule) on a reduced iteration count: the
    global 512 planes are split over the ranks (config nz_per_gpu = 512 / n)."""
    r = _torchrun(2, "--workload", "hpccg512s", "--iters", "3", "--steps", "1", "--warmup", "3",
                  "--no-sub-configs", port=29614)
    assert r.returncode == 0, r.stderr[-3000:]
    d = json.loads([l for l in r.stdout.splitlines() if l.startswith("{")][0])
    assert d["scaling"] == "strong" and d["config"]["nz_per_gpu"] == 256
    assert d["config"]["global_rows"] == 512 ** 3
    cor = d["correctness"]              # 512^3 global at tol 1e-12: SURVEY's 115 (+-1)
    assert cor["expected_niters"] == 115 and cor["ok"], cor


@pytest.mark.gpu
def test_bench_multirank_weak_256_correctness_and_subconfig():
    """The default workload on 2 ranks (256^2 x 512 global): the correctness solve
    must hit SURVEY's independent count (113 +- 1), and the strong-scaling
    sub-record (512^3 split over the 2 ranks, its own 100 iterations; --iters
    shortens only the main workload) is carried in sub_configs."""
    r = _torchrun(2, "--steps", "1", "--warmup", "3", "--iters", "5", port=29615)
    assert r.returncode == 0, r.stderr[-3000:]
    d = json.loads([l for l in r.stdout.splitlines() if l.startswith("{")][0])
    assert d["config"]["workload"] == "hpccg256" and d["scaling"] == "weak"
    cor = d["correctness"]
    assert cor["expected_niters"] == 113 and cor["ok"], cor
    sub = d["sub_configs"]["hpccg512s"]
    assert sub["scaling"] == "strong" and sub["nz_per_gpu"] == 256 and sub["correctness"]["ok"]
    assert sub["value"] > 0 and sub["e2e"]["value"] > 0

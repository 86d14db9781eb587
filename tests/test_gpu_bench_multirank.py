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
                  "--cg-variant", variant, "--halo", halo, port=port)
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


@pytest.mark.gpu
def test_bench_multirank_strong_split():
    """Strong scaling (hpccg512s's split rule) on a reduced iteration count: the
    global 512 planes are split over the ranks (config nz_per_gpu = 512 / n)."""
    r = _torchrun(2, "--workload", "hpccg512s", "--iters", "3", "--steps", "1", "--warmup", "3",
                  port=29614)
    assert r.returncode == 0, r.stderr[-3000:]
    d = json.loads([l for l in r.stdout.splitlines() if l.startswith("{")][0])
    assert d["scaling"] == "strong" and d["config"]["nz_per_gpu"] == 256
    assert d["config"]["global_rows"] == 512 ** 3

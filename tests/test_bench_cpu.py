"""bench.py contract on the CPU host: the reference arm (the oracle, as it
stands -- the one other place bench.py runs oracle/) prints one JSON line per
workload in our arm's metric / unit, only rank 0 prints under torchrun, and
our arm refuses to run without a CUDA device (no CPU fallback)."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
KEYS = {"metric", "value", "unit", "impl", "n_gpus", "steps", "warmup", "ms_per_step",
        "higher_is_better", "scaling", "vs_baseline", "dtype", "config", "cpu_baseline", "e2e"}


def _bench(*argv, env=None):
    e = dict(os.environ)
    e.update(env or {})
    return subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), *argv], cwd=ROOT,
                          env=e, capture_output=True, text=True, timeout=300)


@pytest.mark.parametrize("argv,unit,hib", [
    (["--workload", "hpccg20"], "GFLOP/s", True),
    (["--workload", "lbm", "--lbm-size", "64"], "ms/step", False),
    (["--workload", "tridiag", "--tri-n", "100000"], "ms/iteration", False),
    (["--workload", "blas1", "--blas1-max", "100000"], "GB/s", True),
])
def test_reference_arm_line(argv, unit, hib):
    r = _bench("--impl", "reference", "--steps", "2", "--warmup", "3", *argv)
    assert r.returncode == 0, r.stderr
    lines = [l for l in r.stdout.splitlines() if l.strip()]
    assert len(lines) == 1
    d = json.loads(lines[0])
    assert KEYS <= set(d), KEYS - set(d)
    assert d["impl"] == "reference" and "unavailable" not in d
    assert d["unit"] == unit and d["higher_is_better"] is hib and d["value"] > 0
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["value"] == d["value"]
    assert d["cpu_baseline"]["cores"] >= 1
    assert d["e2e"] == {"value": d["value"], "unit": unit, "h2d_bytes_per_step": 0,
                        "d2h_bytes_per_step": 0}
    assert d["config"]["workload"] == argv[1]


def test_reference_arm_other_ranks_silent():
    r = _bench("--impl", "reference", "--workload", "hpccg20", "--gpus", "2",
               env={"RANK": "1", "WORLD_SIZE": "2"})
    assert r.returncode == 0 and r.stdout.strip() == ""


def test_reference_arm_warmup_floor():
    r = _bench("--impl", "reference", "--workload", "hpccg20", "--warmup", "2")
    assert r.returncode != 0


def test_our_arm_fails_loudly_without_cuda():
    r = _bench("--workload", "hpccg20", "--steps", "1", "--warmup", "3",
               env={"CUDA_VISIBLE_DEVICES": ""})
    assert r.returncode != 0
    assert r.stdout.strip() == ""

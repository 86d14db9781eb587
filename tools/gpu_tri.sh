#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "tri" > gpurun_out/tri_tests.log 2>&1; echo "rc=$?" >> gpurun_out/tri_tests.log
timeout 600 python bench.py --workload tridiag > gpurun_out/tri_bench.log 2>&1
timeout 600 python bench.py --workload tridiag --no-cpu-baseline > gpurun_out/tri_bench2.log 2>&1
tail -3 gpurun_out/tri_tests.log
grep '^{' gpurun_out/tri_bench*.log | cut -c1-600

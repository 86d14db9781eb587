#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "defer_x or scaling_configs or fused" > gpurun_out/zr_tests.log 2>&1; echo "rc=$?" >> gpurun_out/zr_tests.log
timeout 900 python -m pytest tests/test_gpu_peer_ipc.py tests/test_gpu_bench_multirank.py -x -q >> gpurun_out/zr_tests.log 2>&1; echo "rc=$?" >> gpurun_out/zr_tests.log
grep -E "passed|failed|rc=" gpurun_out/zr_tests.log

#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "smem_halo or persistent or cg_vs_oracle or sr" > gpurun_out/smem_tests.log 2>&1; echo "rc=$?" >> gpurun_out/smem_tests.log
timeout 900 python -m pytest tests/test_gpu_sr.py -x -q >> gpurun_out/smem_tests.log 2>&1; echo "rc=$?" >> gpurun_out/smem_tests.log
timeout 600 python tools/smem_halo_probe.py > gpurun_out/smem_probe.log 2>&1
tail -3 gpurun_out/smem_tests.log; cat gpurun_out/smem_probe.log

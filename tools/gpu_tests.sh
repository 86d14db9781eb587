#!/bin/bash
# GPU check of a selection (run under gpurun): SEL="-k expr" (default: all -m gpu
# tests), then smoke().  Logs in gpurun_out/.
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -x -q -m gpu ${SEL} > gpurun_out/pytest_gpu.log 2>&1; echo "pytest_gpu rc=$?" >> gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
tail -n 2 gpurun_out/pytest_gpu.log gpurun_out/smoke.log

#!/bin/bash
# Full check after a product change (run under gpurun): GPU tests, smoke, the
# default bench line, then the round's ncu captures (profile_round.sh).
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -x -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo "pytest_gpu rc=$?" >> gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 600 python bench.py > gpurun_out/bench.log 2>&1; echo "bench rc=$?" >> gpurun_out/bench.log
[ -n "${NCU}" ] && bash tools/profile_round.sh
tail -n 2 gpurun_out/pytest_gpu.log gpurun_out/smoke.log gpurun_out/bench.log

#!/bin/bash
# One batched GPU call: box info, GPU tests, smoke, bench, ncu launch list and
# one full capture of the SpMV.  Everything lands in gpurun_out/.
set -x
mkdir -p gpurun_out
python tools/box_info.py > gpurun_out/box.log 2>&1
timeout 900 python -m pytest tests -x -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo "pytest_gpu rc=$?" >> gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 600 python bench.py ${BENCH_ARGS} > gpurun_out/bench.log 2>&1; echo "bench rc=$?" >> gpurun_out/bench.log
if [ -n "${NCU}" ]; then
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
     --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_launch.log 2>&1
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:spmv27 -s 4 -c 2 \
     -o gpurun_out/prof_spmv -f python bench.py --steps 1 --warmup 3 --iters 5 --no-cpu-baseline > gpurun_out/ncu_full.log 2>&1
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:"cg_update|cg_pupdate" -s 4 -c 2 \
     -o gpurun_out/prof_upd -f python bench.py --steps 1 --warmup 3 --iters 5 --no-cpu-baseline > gpurun_out/ncu_full_upd.log 2>&1
fi
tail -n 3 gpurun_out/*.log

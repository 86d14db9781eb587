#!/bin/bash
# DIA-27 SpMV reading (HPCCG_OPT_SPMV_FORMAT 1): full GPU tests + smoke, bench
# lines (DIA at 128^3 / 256^3 / 512^3, f2), ncu full captures and launch list.
mkdir -p gpurun_out
timeout 900 python -m pytest tests -x -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 600 python bench.py --spmv-format dia > gpurun_out/bench_dia128.json 2> gpurun_out/bench_dia128.err
timeout 900 python bench.py --workload hpccg256 --spmv-format dia > gpurun_out/bench_dia256.json 2> gpurun_out/bench_dia256.err
timeout 900 python bench.py --workload hpccg512s --steps 3 --spmv-format dia > gpurun_out/bench_dia512s.json 2> gpurun_out/bench_dia512s.err
timeout 600 python bench.py --cg-variant sr --spmv-format dia > gpurun_out/bench_dia128_sr.json 2> gpurun_out/bench_dia128_sr.err
timeout 600 python bench.py > gpurun_out/bench_ell128.json 2> gpurun_out/bench_ell128.err
timeout 900 ncu --set full --clock-control none --import-source on -k regex:spmv27 -s 4 -c 2 \
   -o gpurun_out/prof_spmv_dia -f python bench.py --steps 1 --warmup 3 --iters 5 --no-cpu-baseline --spmv-format dia > gpurun_out/ncu_dia.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:spmv27 -s 4 -c 2 \
   -o gpurun_out/prof_spmv_dia256 -f python bench.py --workload hpccg256 --steps 1 --warmup 3 --iters 5 --no-cpu-baseline --spmv-format dia > gpurun_out/ncu_dia256.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
   --log-file gpurun_out/launches_dia.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --spmv-format dia > gpurun_out/ncu_launch_dia.log 2>&1
tail -n 2 gpurun_out/pytest_gpu.log gpurun_out/smoke.log

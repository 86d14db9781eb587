#!/bin/bash
# Every bench line of the round (run under gpurun): the default line (configs[2]
# with configs[1]/[0]/[3]/[4] sub-records), the f2 line, the f1 tridiagonal CG,
# the f4 LBM; JSON lines land in gpurun_out/bench_*.json.
mkdir -p gpurun_out
timeout 900 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
timeout 600 python bench.py --cg-variant sr > gpurun_out/bench_hpccg128_sr.json 2> gpurun_out/bench_sr.err
timeout 600 python bench.py --workload tridiag > gpurun_out/bench_tridiag.json 2> gpurun_out/bench_tridiag.err
timeout 600 python bench.py --workload lbm > gpurun_out/bench_lbm.json 2> gpurun_out/bench_lbm.err
for f in gpurun_out/bench_*.json; do echo "$f: $(head -c 300 $f)"; done

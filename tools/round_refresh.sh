#!/bin/bash
# Full round refresh (run under gpurun): round_evidence.sh (default bench line,
# ncu launch list + full captures, 256^3 / 512^3 / 20x30x10 lines, multi-slab
# probes) plus the f2, BLAS-1, tridiag (f1) and LBM (f4) bench lines.
mkdir -p gpurun_out
bash tools/round_evidence.sh
timeout 600 python bench.py --cg-variant sr > gpurun_out/bench_hpccg128_sr.json 2> gpurun_out/bench_hpccg128_sr.err
timeout 600 python bench.py --workload blas1 > gpurun_out/bench_blas1.json 2> gpurun_out/bench_blas1.err
timeout 600 python bench.py --workload tridiag > gpurun_out/bench_tridiag.json 2> gpurun_out/bench_tridiag.err
timeout 600 python bench.py --workload lbm > gpurun_out/bench_lbm.json 2> gpurun_out/bench_lbm.err

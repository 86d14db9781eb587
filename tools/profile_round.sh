#!/bin/bash
# Round profile capture (run under gpurun): bench line, ncu launch list of the
# same bench command, one `ncu --set full` capture of each hot kernel.
# Outputs land in gpurun_out/; tools/summarize_profiles.py turns them into
# the committed profiles/ summaries.
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,clocks.mem,power.draw --format=csv > gpurun_out/smi.txt 2>&1
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
    --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline \
    > gpurun_out/ncu_launch.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:spmv27 -s 6 -c 2 \
    -o gpurun_out/prof_spmv -f python bench.py --steps 1 --warmup 3 --iters 5 --no-cpu-baseline \
    > gpurun_out/ncu_spmv.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"cg_update|cg_pupdate" -s 6 -c 2 \
    -o gpurun_out/prof_vec -f python bench.py --steps 1 --warmup 3 --iters 5 --no-cpu-baseline \
    > gpurun_out/ncu_vec.log 2>&1
tail -n 2 gpurun_out/*.log

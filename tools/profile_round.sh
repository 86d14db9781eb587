#!/bin/bash
# Round profile capture (run under gpurun, one GPU): the ncu launch list of the
# default bench command and `ncu --set full` captures of the three CG kernels
# at the default workload (256^3), cold cache (ncu's default flush before every
# replayed launch) and warm cache (--cache-control none: L2 as the previous
# kernel left it, i.e. as inside the product loop).  Outputs land in
# gpurun_out/; tools/summarize_profiles.py turns them into profiles/ summaries.
#   usage: bash tools/profile_round.sh [WORKLOAD]   (default hpccg256)
W=${1:-hpccg256}
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,clocks.mem,power.draw --format=csv > gpurun_out/smi.txt 2>&1
B="python bench.py --workload $W --no-cpu-baseline --no-sub-configs"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 800 --csv \
    --log-file gpurun_out/launches.csv $B --steps 2 --warmup 3 > gpurun_out/ncu_launch.log 2>&1
for cc in all none; do
  tag=$([ $cc = all ] && echo cold || echo warm)
  timeout 900 ncu --set full --clock-control none --cache-control $cc --import-source on \
      -k regex:"spmv27x2_kernel|cg_update1_kernel|cg_pupdate1_kernel" -s 0 -c 9 \
      -o gpurun_out/prof_${W}_$tag -f $B --steps 1 --warmup 3 --iters 5 > gpurun_out/ncu_$tag.log 2>&1
  # the ring-deferred p update (HPCCG_OPT_DEFER_X auto = 8 beyond L2): p updates 1..10
  # of the first solve -- 1 (p = r), 2..8 (2R:1W), 9 (the flush: x and 8 directions)
  timeout 900 ncu --set full --clock-control none --cache-control $cc --import-source on \
      -k regex:"cg_pupdate_ring_kernel" -s 0 -c 10 \
      -o gpurun_out/prof_${W}_ring_$tag -f $B --steps 1 --warmup 3 --iters 12 > gpurun_out/ncu_ring_$tag.log 2>&1
done
tail -n 2 gpurun_out/ncu_*.log

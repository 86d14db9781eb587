#!/bin/bash
# A/B of bench.py flag sets on one box, alternating runs (run under gpurun).
#   usage: bash tools/ab_bench.sh WORKLOAD ROUNDS "flags A" "flags B" ...
W=$1; R=$2; shift 2
mkdir -p gpurun_out/ab
for r in $(seq 1 $R); do
  i=0
  for f in "$@"; do
    python bench.py --workload $W --steps 20 --warmup 5 --no-cpu-baseline --no-sub-configs $f \
      > gpurun_out/ab/$W.$i.$r.json 2>/dev/null
    python -c "import json,sys;d=json.load(open('gpurun_out/ab/$W.$i.$r.json'));t=d['roofline'].get('in_graph_trace') or {};print('$W', r'$f' or 'default', 'run $r', d['t_iter_us'], d['value'], t.get('period_us'), t.get('pupdate_us'), t.get('spmv_us'), t.get('update_us'))"
    i=$((i+1))
  done
done

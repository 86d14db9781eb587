#!/bin/bash
# ring-deferred x update: parity tests, then a bench A/B of the deferral depth
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "defer_x or fused_pspmv_bitwise or maxabsdiff" > gpurun_out/ring_tests.log 2>&1; echo "rc=$?" >> gpurun_out/ring_tests.log
for d in 1 8 4 6 1 8; do
  timeout 300 python bench.py --no-sub-configs --no-cpu-baseline --steps 10 --warmup 3 --defer-x $d > gpurun_out/ring_b$d.log 2>&1
  grep '^{' gpurun_out/ring_b$d.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; t=r.get('in_graph_trace',{}); print('defer', $d, d['t_iter_us'], d['value'], d['clocks']['sm_mhz'], t.get('period_us'), t.get('pupdate_us'), t.get('spmv_us'), t.get('update_us'), d['correctness']['ok'])" >> gpurun_out/ring_ab.log 2>&1
done
cat gpurun_out/ring_ab.log
tail -3 gpurun_out/ring_tests.log

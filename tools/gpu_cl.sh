#!/bin/bash
# SpMV cluster partials: parity tests, then an alternating bench A/B
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "spmv_cluster or defer_x or pap_cluster or trips" > gpurun_out/cl_tests.log 2>&1; echo "rc=$?" >> gpurun_out/cl_tests.log
for c in 0 1 0 1 0 1; do
  timeout 300 python bench.py --no-sub-configs --no-cpu-baseline --steps 10 --warmup 3 --spmv-cluster $c ${EXTRA} > gpurun_out/cl_b$c.log 2>&1
  grep '^{' gpurun_out/cl_b$c.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; t=r.get('in_graph_trace',{}); print('cl', $c, d['t_iter_us'], d['value'], d['clocks']['sm_mhz'], d['clocks']['reasons'], t.get('period_us'), t.get('pupdate_us'), t.get('spmv_us'), t.get('update_us'), d['correctness'])" >> gpurun_out/cl_ab.log 2>&1
done
cat gpurun_out/cl_ab.log
tail -3 gpurun_out/cl_tests.log

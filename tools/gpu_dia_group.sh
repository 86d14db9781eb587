#!/bin/bash
# DIA-27 SpMV: slots whose loads are issued together (HPCCG_DIA_GROUP 3 vs 9),
# libraries prebuilt as tools/libhpccg_g<G>.so; bench lines at 128^3 / 256^3.
mkdir -p gpurun_out
L=paper_conf_sc_valero_laragmtv24_b200/libhpccg.so
cp $L /tmp/libhpccg_default.so
for G in 9 3 9 3; do
  cp tools/libhpccg_g$G.so $L
  for W in hpccg128 hpccg256; do
    echo "G=$G $W $(timeout 600 python bench.py --workload $W --spmv-format dia --no-cpu-baseline 2>/dev/null | tail -1)" >> gpurun_out/dia_group.log
  done
done
cp tools/libhpccg_g9.so $L
timeout 600 python -m pytest tests/test_gpu_dia.py -x -q > gpurun_out/pytest_dia_g9.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_dia_g9.log
cp /tmp/libhpccg_default.so $L
tail -n 2 gpurun_out/pytest_dia_g9.log

#!/bin/bash
# DIA-27 SpMV tuning: slots per load group (HPCCG_DIA_GROUP) x resident blocks
# (HPCCG_DIA_MINB), libraries prebuilt as tools/libhpccg_g<G>_m<M>.so (git-ignored);
# bench lines at 128^3 / 256^3, alternating.  Build the variants here first:
#   for v in "9 4" "9 3" "27 2"; do set -- $v; HPCCG_NVCC_EXTRA="-DHPCCG_DIA_GROUP=$1 -DHPCCG_DIA_MINB=$2" \
#     python -c "from paper_conf_sc_valero_laragmtv24_b200 import _build; _build.build(force=True)"; \
#     cp paper_conf_sc_valero_laragmtv24_b200/libhpccg.so tools/libhpccg_g$1_m$2.so; done
# (then rebuild the default library).
mkdir -p gpurun_out
L=paper_conf_sc_valero_laragmtv24_b200/libhpccg.so
cp $L /tmp/libhpccg_default.so
for rep in 1 2; do
  for V in g9_m4 g9_m3 g27_m2; do
    cp tools/libhpccg_$V.so $L
    for W in hpccg128 hpccg256; do
      echo "$V $W $(timeout 600 python bench.py --workload $W --spmv-format dia --no-cpu-baseline --steps 3 2>/dev/null | tail -1)" >> gpurun_out/dia_tune.log
    done
  done
done
cp /tmp/libhpccg_default.so $L

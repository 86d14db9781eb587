#!/bin/bash
# compute-sanitizer passes (memcheck, racecheck, synccheck) over a small slice
# of the GPU tests: every kernel family on small problems.
mkdir -p gpurun_out
SEL="cg_vs_oracle and 20-30-10 or persistent_grid or spmv_loopback or generate_bitwise and 7-5-6 or tri_cg_vs_oracle and 1000- or lbm_bitwise and 17 or lbm_two_step_kernel_bitwise and 3-129 or lbm_two_step_rows_per_cta and 7 or 2d_ddot and 37 or ddot_vs and 257 or nccl_one_rank and 16-12-6 or cg_modes and minb0 or peer_fused_loopback_bitwise and 2-dims0 or serpentine and 24-20-12 or defer_x_bitwise and dims1 or fused_pspmv_bitwise and dims0 or fused_pspmv_spmv or spmv_trips and dims2 or defer_x_fused_loopback and 2"
for tool in memcheck racecheck synccheck initcheck; do
  timeout 1200 /usr/local/cuda/bin/compute-sanitizer --tool $tool --error-exitcode 99 --print-limit 20 \
      python -m pytest tests/test_gpu_parity.py -q -m gpu -x -k "$SEL" -p no:cacheprovider \
      > gpurun_out/sanitize_$tool.log 2>&1
  echo "$tool rc=$?" >> gpurun_out/sanitize_summary.txt
  tail -3 gpurun_out/sanitize_$tool.log >> gpurun_out/sanitize_summary.txt
done
cat gpurun_out/sanitize_summary.txt

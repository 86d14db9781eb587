#!/bin/bash
# Run tools/sanitizer_repro (built here: nvcc -gencode arch=compute_100a,code=sm_100a
# -O3 -lineinfo -o tools/sanitizer_repro tools/sanitizer_repro.cu) under synccheck and
# racecheck in every launch mode and both kernel bodies (run under gpurun).
mkdir -p gpurun_out/sanrep
for tool in synccheck racecheck; do
  for mode in plain pdl graph while; do
    for tail in 0 1; do
      f=gpurun_out/sanrep/$tool.$mode.$tail.log
      timeout 300 /usr/local/cuda/bin/compute-sanitizer --tool $tool --print-limit 5 \
          tools/sanitizer_repro $mode $tail > $f 2>&1
      echo "$tool $mode tail=$tail rc=$? $(grep -m1 -E 'mode=' $f) | $(grep -m1 -E 'ERROR SUMMARY|RACECHECK SUMMARY' $f)"
    done
  done
done
# the library's own CG kernels (tools/rc_case.py: 16x12x6, 20 iterations), the same
# kernels with and without the conditional WHILE node
for tool in synccheck racecheck; do
  for args in "0 0 0 1 3" "0 0 1 1 3" "0 1 0 1 3" "2 0 0 2 3" "2 1 0 2 3"; do
    f="gpurun_out/sanrep/lib.$tool.$(echo $args | tr ' ' '_').log"
    timeout 600 /usr/local/cuda/bin/compute-sanitizer --tool $tool --print-limit 5 \
        python tools/rc_case.py $args > "$f" 2>&1
    echo "lib $tool rc_case($args: HALO_PEER WHILE TIMING P SERP) rc=$? | $(grep -m1 -E 'ERROR SUMMARY|RACECHECK SUMMARY' "$f")"
  done
done

#!/bin/bash
# Round evidence (run under gpurun): profile_round.sh (default bench line,
# ncu launch list, full captures), the other workloads' bench lines, and the
# multi-slab code path on one GPU (1-rank NCCL context and loopback slabs,
# NCCL vs HALO_PEER 1 vs 2).  Everything lands in gpurun_out/.
mkdir -p gpurun_out
bash tools/profile_round.sh
timeout 900 python bench.py --workload hpccg256 > gpurun_out/bench_hpccg256.json 2> gpurun_out/bench_hpccg256.err
timeout 900 python bench.py --workload hpccg512s --steps 3 > gpurun_out/bench_hpccg512s.json 2> gpurun_out/bench_hpccg512s.err
timeout 600 python bench.py --workload hpccg20 > gpurun_out/bench_hpccg20.json 2> gpurun_out/bench_hpccg20.err
{
  PROBE_NCCL=1 timeout 300 python tools/probe.py 128 128 128 300 "peer=0" "peer=1" "peer=2"
  PROBE_NCCL=1 timeout 300 python tools/probe.py 256 256 256 100 "peer=0" "peer=1" "peer=2"
  PROBE_NCCL=1 timeout 300 python tools/trace.py 128 128 128 40 "peer=2"
  PROBE_NCCL=1 timeout 300 python tools/trace.py 256 256 256 30 "peer=2"
  PROBE_P=2 timeout 300 python tools/probe.py 256 256 128 100 "peer=0" "peer=1" "peer=2"
  PROBE_P=4 timeout 300 python tools/probe.py 128 128 32 200 "peer=0" "peer=1" "peer=2"
} > gpurun_out/multislab_probe.log 2>&1
tail -n 2 gpurun_out/*.json gpurun_out/multislab_probe.log

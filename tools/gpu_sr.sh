mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_sr.py -x -q > gpurun_out/sr_tests.log 2>&1; echo "rc=$?" >> gpurun_out/sr_tests.log
timeout 600 python tools/probe.py 128 128 128 500 "" "var=1" "var=1,wu=2" "var=1,unroll=2" "var=1,unroll=1" "timing=1" "var=1,timing=1" > gpurun_out/sr_probe128.log 2>&1
timeout 600 python tools/probe.py 256 256 256 100 "" "var=1" "var=1,unroll=2" "timing=1" "var=1,timing=1" > gpurun_out/sr_probe256.log 2>&1
timeout 600 python tools/probe.py 20 30 10 500 "" "var=1" "persist=0" > gpurun_out/sr_probe_small.log 2>&1
timeout 900 python -m pytest tests -x -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_gpu.log
tail -n 3 gpurun_out/sr_tests.log gpurun_out/pytest_gpu.log; cat gpurun_out/sr_probe*.log

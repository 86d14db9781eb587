mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_sr.py tests/test_gpu_parity.py -x -q > gpurun_out/quick_tests.log 2>&1; echo "rc=$?" >> gpurun_out/quick_tests.log
python tools/probe.py 20 30 10 500 "" "var=1" "smem=0" "persist=0" "persist=0,var=1" > gpurun_out/small_probe.log 2>&1
python tools/probe.py 16 16 16 500 "" "var=1" >> gpurun_out/small_probe.log 2>&1
python tools/probe.py 3 3 3 500 "" "var=1" >> gpurun_out/small_probe.log 2>&1
python tools/probe.py 128 128 128 300 "" >> gpurun_out/small_probe.log 2>&1
python tools/probe.py 256 256 256 60 "" >> gpurun_out/small_probe.log 2>&1
tail -n 3 gpurun_out/quick_tests.log; cat gpurun_out/small_probe.log

# quick GPU check: the given pytest selection, then the full -m gpu suite
mkdir -p gpurun_out
timeout 900 python -m pytest ${SEL:-tests/test_gpu_sr.py} -x -q > gpurun_out/quick_tests.log 2>&1; echo "rc=$?" >> gpurun_out/quick_tests.log
timeout 900 python -m pytest tests -x -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_gpu.log
if [ -n "${PROBE}" ]; then eval "${PROBE}" > gpurun_out/quick_probe.log 2>&1; fi
tail -n 3 gpurun_out/quick_tests.log gpurun_out/pytest_gpu.log

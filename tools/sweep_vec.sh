mkdir -p gpurun_out
python tools/probe.py 256 256 256 60 "" "waves=0" "waves=2" "waves=4" "unroll=2" "unroll=1" "unroll=2,waves=0" "unroll=1,waves=0" "unroll=2,waves=2" > gpurun_out/sweep256.log 2>&1
python tools/probe.py 128 128 128 300 "" "waves=0" "waves=2" "unroll=2" "unroll=1" "unroll=2,waves=0" "unroll=1,waves=0" > gpurun_out/sweep128.log 2>&1
python tools/trace.py 128 128 128 60 "" "ff=0" > gpurun_out/trace128.log 2>&1
python tools/trace.py 256 256 256 30 "" > gpurun_out/trace256.log 2>&1
cat gpurun_out/sweep*.log gpurun_out/trace*.log

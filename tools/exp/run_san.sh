mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_sanitizers.py -x -q -k "split or wcycle or host" > gpurun_out/san_tests.log 2>&1; echo "rc=$?" >> gpurun_out/san_tests.log
tail -5 gpurun_out/san_tests.log
timeout 300 python tools/quick_time.py C3 2>&1 | tail -1
timeout 300 python tools/quick_time.py C3 "" '{"pair_warps": 2}' 2>&1 | tail -1

set -x
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/s6_tests.log 2>&1; echo "rc=$?" >> gpurun_out/s6_tests.log
tail -5 gpurun_out/s6_tests.log
timeout 600 python tools/robustness.py > gpurun_out/robustness_r01.json 2> gpurun_out/robustness_r01.log; tail -8 gpurun_out/robustness_r01.log

set -x
mkdir -p gpurun_out
./tools/evd_probe > gpurun_out/evd_probe2.json 2>&1; cat gpurun_out/evd_probe2.json
timeout 600 python -m pytest tests/test_gpu_l1.py -x -q > gpurun_out/s4_tests.log 2>&1; echo "rc=$?" >> gpurun_out/s4_tests.log
tail -3 gpurun_out/s4_tests.log
for c in C3 C4 C5; do timeout 300 python tools/quick_time.py $c 2>&1 | tail -1; done
timeout 900 python tools/ablation.py > gpurun_out/ablation_r01.json 2> gpurun_out/ablation_r01.log; tail -30 gpurun_out/ablation_r01.log

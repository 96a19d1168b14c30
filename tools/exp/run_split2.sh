set -x
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_l1.py -x -q > gpurun_out/split_tests.log 2>&1; echo "rc=$?" >> gpurun_out/split_tests.log
tail -3 gpurun_out/split_tests.log
for c in C3 C4 C5; do timeout 300 python tools/quick_time.py $c 2>&1 | tail -1; timeout 300 python tools/quick_time.py $c "" '{"pair_warps": 2}' 2>&1 | tail -1; done
timeout 300 bash tools/exp/swap_run.sh tools/exp/libwcsvd_phase.so python tools/exp/phase_tp.py C2 10000 2>&1 | tail -12

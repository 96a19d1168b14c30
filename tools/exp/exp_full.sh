mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; echo tests_rc=$? >> gpurun_out/gpu_tests.log
timeout 300 python bench.py --config C2 --steps 5 --warmup 3 > gpurun_out/bench_C2.json 2> gpurun_out/bench_C2.err
python tools/quick_time.py C1 2>&1 | tail -1 > gpurun_out/c1_new.txt
bash tools/exp/swap_run.sh tools/exp/libwcsvd_notp.so python tools/quick_time.py C1 2>&1 | tail -1 >> gpurun_out/c1_new.txt

# round-2 final-session measurement at HEAD: ncu --set full of the dominant kernel per config, launch
# list of the default bench command, GPU suite, smoke
set -x
ncu --set full --clock-control none --import-source on -k regex:l1_gram -c 1 -o gpurun_out/full_r03_c5 python tools/quick_time.py C5 > gpurun_out/ncu_r03_c5.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:l1_gram -c 1 -o gpurun_out/full_r03_c3 python tools/quick_time.py C3 > gpurun_out/ncu_r03_c3.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:l1_gram -c 1 -o gpurun_out/full_r03_c4 python tools/quick_time.py C4 > gpurun_out/ncu_r03_c4.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:l0tp -c 1 -o gpurun_out/full_r03_c2 python tools/quick_time.py C2 > gpurun_out/ncu_r03_c2.log 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/ncu_launches_r03_c5.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline > gpurun_out/ncu_launches_r03_c5.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q > gpurun_out/gpu_tests_r03.log 2>&1; tail -3 gpurun_out/gpu_tests_r03.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_r03.log 2>&1; tail -1 gpurun_out/smoke_r03.log
ls -la gpurun_out/

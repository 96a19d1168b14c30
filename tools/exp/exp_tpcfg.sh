mkdir -p gpurun_out
timeout 300 python -m pytest tests/test_gpu_l0.py tests/test_gpu_fp32.py -x -q > gpurun_out/tpcfg_tests.log 2>&1; echo rc=$? >> gpurun_out/tpcfg_tests.log
for c in 1 0 2; do
  if [ $c = 1 ]; then L=""; else L="bash tools/exp/swap_run.sh tools/exp/libwcsvd_tp$c.so"; fi
  echo "cfg $c" >> gpurun_out/tpcfg.txt
  $L python tools/quick_time.py C2 2>&1 | tail -1 >> gpurun_out/tpcfg.txt
  $L python tools/quick_time.py C2 10000 '{"compute_uv": false}' 2>&1 | tail -1 >> gpurun_out/tpcfg.txt
done
python tools/quick_time.py C1 2>&1 | tail -1 >> gpurun_out/tpcfg.txt

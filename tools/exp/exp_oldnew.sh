mkdir -p gpurun_out
for L in "" "bash tools/exp/swap_run.sh tools/exp/libwcsvd_notp.so"; do
  echo "== lib: $L"
  $L python tools/quick_time.py C2 10000 '{"compute_uv": false}' 2>&1 | tail -1
  $L python tools/quick_time.py C2 2>&1 | tail -1
done
ncu --set full --clock-control none --import-source on -k regex:l0tp -c 1 -o gpurun_out/full_new_c2x python tools/quick_time.py C2 10000 '{"compute_uv": false}' > /dev/null 2>&1
bash tools/exp/swap_run.sh tools/exp/libwcsvd_notp.so ncu --set full --clock-control none --import-source on -k regex:l0_jacobi -c 1 -o gpurun_out/full_old_c2x python tools/quick_time.py C2 10000 '{"compute_uv": false}' > /dev/null 2>&1

WCSVD_LIBRARY=tools/exp/lib_phase.so timeout 300 python tools/exp/phase.py C3 592
WCSVD_LIBRARY=tools/exp/lib_phase.so timeout 300 python tools/exp/phase.py C4 592
ncu --set full --clock-control none --import-source on -k regex:l1_gram -c 1 -o gpurun_out/full_r02l_c3 python tools/quick_time.py C3 296 > gpurun_out/full_r02l_c3.log 2>&1
ncu -i gpurun_out/full_r02l_c3.ncu-rep --page source --csv > gpurun_out/src_r02l_c3.csv 2>/dev/null
ls -la gpurun_out | tail -5

ncu --set full --clock-control none --import-source on -k regex:l1_gram -c 1 -o gpurun_out/full_r03g_c3 python tools/quick_time.py C3 592 > gpurun_out/ncu_r03g.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:l0tp -c 1 -o gpurun_out/full_r03g_c2 python tools/quick_time.py C2 > gpurun_out/ncu_r03g2.log 2>&1
ls -la gpurun_out/full_r03g*

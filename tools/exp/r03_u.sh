ncu --set full --clock-control none --import-source on -k regex:l0_warp -c 1 -o /tmp/c1w python tools/quick_time.py C1 > /dev/null 2>&1
ncu -i /tmp/c1w.ncu-rep --page source --csv --print-source cuda,sass 2>/dev/null | gzip > gpurun_out/ncu_source_c1w.csv.gz
ncu -i /tmp/c1w.ncu-rep --page details --csv > gpurun_out/ncu_details_c1w.csv 2>/dev/null
ls -la gpurun_out

for i in 1 2; do
timeout 300 python tools/scenarios.py C2 2>&1 | cut -c1-100
WCSVD_LIBRARY=tools/exp/lib_park.so timeout 300 python tools/scenarios.py C2 2>&1 | cut -c1-100
done
M="gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct"
for lib in tools/exp/lib_park.so; do echo $lib; WCSVD_LIBRARY=$lib ncu --metrics $M --clock-control none -k regex:l0tp -c 1 --csv python tools/quick_time.py C2 2>&1 | grep -E "dram__|hit_rate|duration" | awk -F'","' '{print $(NF-2), $NF}'; done

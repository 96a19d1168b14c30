for i in 1 2; do
for lib in paper_conf_sc_xiaopxsmmlzt22_b200/libwcsvd.so tools/exp/lib_l2h1.so tools/exp/lib_l2h2.so tools/exp/lib_l2h3.so tools/exp/lib_l2h4.so; do echo $lib; WCSVD_LIBRARY=$lib timeout 600 python tools/scenarios.py C3 C4 "C5/2:0" 2>&1 | cut -c1-105; done
done
M="gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct"
for lib in paper_conf_sc_xiaopxsmmlzt22_b200/libwcsvd.so tools/exp/lib_l2h1.so tools/exp/lib_l2h3.so; do echo $lib; WCSVD_LIBRARY=$lib ncu --metrics $M --clock-control none -k regex:l1_gram -c 1 --csv python tools/quick_time.py C4 2>&1 | grep -E "dram__|hit_rate|duration" | awk -F'","' '{print $(NF-2), $NF}'; done

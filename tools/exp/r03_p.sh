python tools/exp/dump.py /tmp/b.npz | tail -1
WCSVD_LIBRARY=tools/exp/lib_head.so python tools/exp/dump.py /tmp/a.npz | tail -1
python tools/exp/bitcmp.py /tmp/a.npz /tmp/b.npz
for i in 1 2; do
WCSVD_LIBRARY=tools/exp/lib_head.so timeout 300 python tools/scenarios.py C2 2>&1 | cut -c1-100
timeout 300 python tools/scenarios.py C2 2>&1 | cut -c1-100
done
M="gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct"
for lib in tools/exp/lib_head.so paper_conf_sc_xiaopxsmmlzt22_b200/libwcsvd.so; do echo $lib; WCSVD_LIBRARY=$lib ncu --metrics $M --clock-control none -k regex:l0tp -c 1 --csv python tools/quick_time.py C2 2>&1 | grep -E "dram__|hit_rate|duration" | awk -F'","' '{print $(NF-2), $NF}'; done

# round-2 final measurement at HEAD (reports in /tmp on the box; summaries to gpurun_out)
set -x
R=/tmp/ncu; mkdir -p $R
timeout 2400 python -m pytest tests -m gpu -q > gpurun_out/gpu_tests_r02z.log 2>&1; tail -3 gpurun_out/gpu_tests_r02z.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_r02z.log 2>&1; tail -1 gpurun_out/smoke_r02z.log
timeout 900 python bench.py > gpurun_out/bench_r02z_c5.json 2> gpurun_out/bench_r02z_c5.err; tail -c 300 gpurun_out/bench_r02z_c5.json
timeout 900 python bench.py --impl reference > gpurun_out/bench_r02z_reference.json 2> gpurun_out/bench_r02z_reference.err
for c in C1 C2 C3 C4; do timeout 900 python bench.py --config $c > gpurun_out/bench_r02z_$c.json 2> gpurun_out/bench_r02z_$c.err; done
M="gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active,sm__pipe_shared_cycles_active.avg.pct_of_peak_sustained_active,sm__warps_active.avg.per_cycle_active,lts__t_sector_hit_rate.pct,sm__cycles_elapsed.avg.per_second"
ncu --metrics $M --clock-control none -k regex:l1_gram -c 1 --csv python tools/quick_time.py C5 > gpurun_out/ncu_metrics_r02z_c5.csv 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/ncu_launches_r02z_c5.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline > gpurun_out/ncu_launches_r02z_c5.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:l1_gram -c 1 -o $R/c3 python tools/quick_time.py C3 > /dev/null 2>&1
python tools/ncu_summary.py $R/c3.ncu-rep --json gpurun_out/ncu_summary_r02z.json --key C3 --matrices 2000 > /dev/null
ncu -i $R/c3.ncu-rep --page details --csv > gpurun_out/ncu_details_r02z_c3.csv 2>/dev/null
timeout 900 python tools/robustness.py > gpurun_out/robustness_r02z.json 2> gpurun_out/robustness_r02z.err
du -sh gpurun_out

# round-2 final-session measurement at HEAD (reports stay in /tmp on the box; summaries to gpurun_out)
set -x
R=/tmp/ncu; mkdir -p $R
M="gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active,sm__pipe_shared_cycles_active.avg.pct_of_peak_sustained_active,sm__inst_executed_pipe_dmma.avg.pct_of_peak_sustained_active,sm__warps_active.avg.per_cycle_active,lts__t_sector_hit_rate.pct,sm__cycles_elapsed.avg.per_second"
ncu --metrics $M --clock-control none -k regex:l1_gram -c 1 --csv python tools/quick_time.py C5 > gpurun_out/ncu_metrics_r03_c5.csv 2>&1
ncu --set full --clock-control none --import-source on -k regex:l1_gram -c 1 -o $R/c3 python tools/quick_time.py C3 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:l1_gram -c 1 -o $R/c4 python tools/quick_time.py C4 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:l0tp -c 1 -o $R/c2 python tools/quick_time.py C2 > /dev/null 2>&1
python tools/ncu_summary.py $R/c3.ncu-rep --json gpurun_out/ncu_summary_r02.json --key C3 --matrices 2000 > /dev/null
python tools/ncu_summary.py $R/c4.ncu-rep --json gpurun_out/ncu_summary_r02.json --key C4 --matrices 4000 > /dev/null
python tools/ncu_summary.py $R/c2.ncu-rep --json gpurun_out/ncu_summary_r02.json --key C2 --matrices 10000 > /dev/null
for c in c2 c3 c4; do ncu -i $R/$c.ncu-rep --page details --csv > gpurun_out/ncu_details_r03_$c.csv 2>/dev/null; ncu -i $R/$c.ncu-rep --page source --csv --print-source cuda,sass 2>/dev/null | gzip > gpurun_out/ncu_source_r03_$c.csv.gz; done
python - <<'PY'
import csv, json
rows = [r for r in csv.reader(open("gpurun_out/ncu_metrics_r03_c5.csv")) if len(r) > 10]
hdr = rows[0]; i_n, i_u, i_v = hdr.index("Metric Name"), hdr.index("Metric Unit"), hdr.index("Metric Value")
d = {}
for r in rows[1:]:
    v = float(r[i_v].replace(",", ""))
    u = r[i_u]
    v *= {"Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "usecond": 1e-3, "nsecond": 1e-6, "msecond": 1.0, "ns": 1e-6, "us": 1e-3, "ms": 1.0, "second": 1e3}.get(u, 1.0)
    d[r[i_n]] = v
s = json.load(open("gpurun_out/ncu_summary_r02.json"))
by = d["dram__bytes_read.sum"] + d["dram__bytes_write.sum"]
s["C5"] = {"kernel": "l1_gram_kernel<32, 8> (C5 bucket path 2 variant 13, 1958 matrices)", "matrices": 1958,
           "duration_ms": d["gpu__time_duration.sum"], "dram_bytes_per_launch": by, "dram_bytes_per_matrix": by / 1958,
           "dram_TBps": by / (d["gpu__time_duration.sum"] * 1e-3) / 1e12,
           "fp64_pipe_pct": d.get("sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active"),
           "shared_pipe_pct": d.get("sm__pipe_shared_cycles_active.avg.pct_of_peak_sustained_active"),
           "dmma_inst_pct": d.get("sm__inst_executed_pipe_dmma.avg.pct_of_peak_sustained_active"),
           "warps_active": d.get("sm__warps_active.avg.per_cycle_active"), "l2_hit_pct": d.get("lts__t_sector_hit_rate.pct"),
           "sm_clock_GHz": d.get("sm__cycles_elapsed.avg.per_second", 0) / 1e9,
           "capture": "ncu --metrics (dram, pipes) --clock-control none -k regex:l1_gram -c 1, tools/quick_time.py C5 (first l1_gram launch = the dominant bucket)"}
json.dump(s, open("gpurun_out/ncu_summary_r02.json", "w"), indent=1)
print(json.dumps({k: {kk: s[k].get(kk) for kk in ("duration_ms", "dram_bytes_per_matrix", "fp64_pipe_pct")} for k in s}, indent=0))
PY
cp gpurun_out/ncu_summary_r02.json profiles/ncu_summary_r02.json
ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/ncu_launches_r03_c5.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline > gpurun_out/ncu_launches_r03_c5.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q > gpurun_out/gpu_tests_r03.log 2>&1; tail -3 gpurun_out/gpu_tests_r03.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_r03.log 2>&1; tail -1 gpurun_out/smoke_r03.log
timeout 900 python bench.py > gpurun_out/bench_r03_c5.json 2> gpurun_out/bench_r03_c5.err; tail -c 600 gpurun_out/bench_r03_c5.json
timeout 900 python bench.py --impl reference > gpurun_out/bench_r03_reference.json 2> gpurun_out/bench_r03_reference.err; tail -c 300 gpurun_out/bench_r03_reference.json
for c in C1 C2 C3 C4; do timeout 900 python bench.py --config $c > gpurun_out/bench_r03_$c.json 2> gpurun_out/bench_r03_$c.err; tail -c 200 gpurun_out/bench_r03_$c.json; done
du -sh gpurun_out

set -x
mkdir -p gpurun_out
T=r01g
ncu --set full --clock-control none --import-source on -k regex:l1_gram -c 1 -o gpurun_out/full_${T}_c3 python tools/quick_time.py C3 > gpurun_out/full_${T}_c3.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:l1_gram -c 1 -o gpurun_out/full_${T}_c4 python tools/quick_time.py C4 > gpurun_out/full_${T}_c4.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:l0tp -c 1 -o gpurun_out/full_${T}_c2 python tools/quick_time.py C2 > gpurun_out/full_${T}_c2.log 2>&1
for c in C3 C4 C5; do ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_${T}_${c}.csv python bench.py --config $c --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/launches_${T}_${c}.log 2>&1; done
ls -la gpurun_out

#!/bin/bash
# Profiling pass (run under gpurun, one GPU). Usage: tools/profile.sh <tag>
# 1) ncu launch list of the default bench command (device time per launch; shares, not absolutes)
# 2) ncu --set full of the dominant kernel per config (small batches; one launch)
set -x
TAG=${1:-r01}
mkdir -p gpurun_out
ncu --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file gpurun_out/launches_${TAG}_c2.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline > gpurun_out/launches_${TAG}_c2.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:l0tp -c 1 \
    -o gpurun_out/full_${TAG}_c2 python tools/quick_time.py C2 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:l1_gram -c 1 \
    -o gpurun_out/full_${TAG}_c3 python tools/quick_time.py C3 296 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:l1_gram -c 1 \
    -o gpurun_out/full_${TAG}_c4 python tools/quick_time.py C4 148 > /dev/null 2>&1
ls -la gpurun_out

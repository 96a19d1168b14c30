#!/bin/bash
# ncu --set full captures of the dominant kernels (one launch each). Usage: tools/profile_full.sh TAG
TAG=${1:-x}
ncu --set full --clock-control none --import-source on -k regex:l0_jacobi -c 1 \
    -o gpurun_out/full_${TAG}_c2 python tools/quick_time.py C2 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:l1_gram -c 1 \
    -o gpurun_out/full_${TAG}_c3 python tools/quick_time.py C3 592 > /dev/null 2>&1
ls gpurun_out/full_${TAG}*

mkdir -p gpurun_out
TAG=${1:-tp}
ncu --set full --clock-control none --import-source on -k regex:l0tp -c 1 -o gpurun_out/full_${TAG}_c2 python tools/quick_time.py C2 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:l0tp -c 1 -o gpurun_out/full_${TAG}_c2x python tools/quick_time.py C2 10000 '{"compute_uv": false}' > /dev/null 2>&1
ls gpurun_out/

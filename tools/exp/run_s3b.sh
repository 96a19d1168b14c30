set -x
mkdir -p gpurun_out
./tools/evd_probe > gpurun_out/evd_probe.json 2>&1
./tools/lat_fp64 > gpurun_out/lat_fp64.json 2>&1
cat gpurun_out/evd_probe.json gpurun_out/lat_fp64.json
bash tools/profile.sh r01c

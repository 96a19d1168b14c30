# host pipeline: staging sets x chunk count (e2e), plus host-API bitwise tests and the NS A/B
mkdir -p gpurun_out
timeout 300 python -m pytest tests/test_gpu_host.py -q -x 2>&1 | tail -2
for cfg in "C2 2 20" "C2 3 20" "C2 4 20" "C2 3 32" "C3 2 8" "C3 3 8" "C3 3 16" "C4 3 8" "C4 3 16"; do
  set -- $cfg
  r=$(WCSVD_HOST_SETS=$2 WCSVD_HOST_CHUNKS=$3 timeout 300 python bench.py --config $1 --steps 5 --warmup 3 --no-cpu-baseline 2>/dev/null | tail -1)
  echo "$1 sets=$2 chunks=$3 $(python -c "import json,sys;d=json.loads(sys.argv[1]);print(round(d['value']),round(d['e2e']['value']),d['clocks']['sm_mhz'])" "$r")"
done
bash tools/exp/run_nsab.sh

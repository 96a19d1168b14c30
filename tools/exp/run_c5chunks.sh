# mixed batch (C5) e2e vs chunk count with three staging sets
for k in 1 2 3 4 6; do
  r=$(WCSVD_HOST_CHUNKS=$k timeout 400 python bench.py --config C5 --steps 3 --warmup 3 --no-cpu-baseline 2>/dev/null | tail -1)
  echo "C5 chunks=$k $(python -c "import json,sys;d=json.loads(sys.argv[1]);print(round(d['value']),round(d['e2e']['value']),d['clocks']['sm_mhz'])" "$r")"
done

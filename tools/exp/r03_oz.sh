WCSVD_HOST_OUT_ZC=1 timeout 900 python -m pytest tests/test_gpu_host.py -q 2>&1 | tail -2
for c in C2 C3 C4; do for z in 0 1; do
WCSVD_HOST_OUT_ZC=$z timeout 900 python bench.py --config $c --no-cpu-baseline --steps 3 > /tmp/b.json 2>/dev/null
python -c "import json; d=json.load(open('/tmp/b.json')); print('$c outzc=$z', round(d['value'],1), 'e2e', round(d['e2e']['value'],1), d['clocks']['sm_mhz'])"
done; done

timeout 900 python -m pytest tests/test_gpu_host.py -q 2>&1 | tail -2
for c in C5 C4 C3 C2; do for z in 0 1; do
WCSVD_HOST_ZEROCOPY=$z timeout 900 python bench.py --config $c --no-cpu-baseline --steps 3 > /tmp/b.json 2>/dev/null
python -c "import json; d=json.load(open('/tmp/b.json')); print('$c zc=$z', round(d['value'],1), 'e2e', round(d['e2e']['value'],1), d['clocks']['sm_mhz'])"
done; done

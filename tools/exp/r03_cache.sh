timeout 900 python -m pytest tests/test_gpu_host.py tests/test_gpu_dist.py -q 2>&1 | tail -2
for c in C2 C2 C3 C1; do timeout 900 python bench.py --config $c --no-cpu-baseline --steps 5 > /tmp/b.json 2>/dev/null
python -c "import json; d=json.load(open('/tmp/b.json')); print('$c', round(d['value'],1), 'e2e', round(d['e2e']['value'],1))"; done

for i in 1 2; do timeout 600 python bench.py --config C2 --steps 5 --warmup 3 --no-cpu-baseline 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('C2', round(d['value']), 'e2e', round(d['e2e']['value']))"; done
timeout 600 python -m pytest tests/test_gpu_host.py -q 2>&1 | tail -1

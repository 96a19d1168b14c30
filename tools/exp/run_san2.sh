mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_sanitizers.py tests/test_gpu_host.py -x -q -k "host" > gpurun_out/san2.log 2>&1; echo "rc=$?" >> gpurun_out/san2.log
tail -4 gpurun_out/san2.log
timeout 600 python bench.py --config C2 --steps 5 --warmup 3 --no-cpu-baseline 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('C2', round(d['value']), 'e2e', round(d['e2e']['value']))"

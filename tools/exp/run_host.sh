mkdir -p gpurun_out
export WCSVD_DEBUG=1
timeout 600 python -m pytest tests/test_gpu_host.py -x -q > gpurun_out/host_tests.log 2>&1; echo "rc=$?" >> gpurun_out/host_tests.log
tail -4 gpurun_out/host_tests.log
for c in C2 C3 C4 C5; do timeout 600 python bench.py --config $c --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bh_$c.json 2> gpurun_out/bh_$c.err; python -c "import json; d=json.loads(open('gpurun_out/bh_$c.json').read().strip().splitlines()[-1]); print('$c', round(d['value']), 'e2e', round(d['e2e']['value']))" || tail -5 gpurun_out/bh_$c.err; done

set -x
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/gputests_s3.log 2>&1; echo "tests rc=$?"
tail -3 gpurun_out/gputests_s3.log
for c in C2 C3 C4 C5; do timeout 600 python bench.py --config $c --steps 5 --warmup 3 > gpurun_out/bench_s3_$c.json 2> gpurun_out/bench_s3_$c.err; tail -1 gpurun_out/bench_s3_$c.json; done

set -x
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv
timeout 2400 python -m pytest tests -m gpu -q > gpurun_out/final2_tests.log 2>&1; echo "rc=$?" >> gpurun_out/final2_tests.log
tail -4 gpurun_out/final2_tests.log
for c in C2 C3 C4 C5; do timeout 600 python bench.py --config $c --steps 5 --warmup 3 > gpurun_out/bench_final2_$c.json 2> gpurun_out/bench_final2_$c.err; tail -1 gpurun_out/bench_final2_$c.json | cut -c1-200; done
timeout 300 python bench.py > gpurun_out/bench_default2.json 2> gpurun_out/bench_default2.err; tail -1 gpurun_out/bench_default2.json | cut -c1-300
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke2.log 2>&1; tail -1 gpurun_out/smoke2.log

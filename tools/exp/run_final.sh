set -x
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/final_tests.log 2>&1; echo "rc=$?" >> gpurun_out/final_tests.log
tail -4 gpurun_out/final_tests.log
for c in C2 C3 C4 C5; do timeout 600 python bench.py --config $c --steps 5 --warmup 3 > gpurun_out/bench_final_$c.json 2> gpurun_out/bench_final_$c.err; tail -1 gpurun_out/bench_final_$c.json; done
timeout 300 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err; tail -1 gpurun_out/bench_default.json
timeout 300 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/bench_reference.json 2> gpurun_out/bench_reference.err; tail -1 gpurun_out/bench_reference.json
timeout 600 python tools/robustness.py > gpurun_out/robustness_r01.json 2> gpurun_out/robustness_r01.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; tail -2 gpurun_out/smoke.log

timeout 300 python -m pytest tests/test_gpu_cluster.py tests/test_gpu_l1.py -x -q 2>&1 | tail -3
for f in 1 2 4 8; do WCSVD_TAILOR=$f timeout 600 python tools/scenarios.py "C5/8:0" "C5/4:0" --opts "{\"_f\": $f}" 2>&1 | grep -v Warn; done
timeout 900 python tools/scenarios.py C3 C3 C4 C5 --json gpurun_out/scen_r02c.json

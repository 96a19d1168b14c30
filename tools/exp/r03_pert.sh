timeout 1500 python -m pytest tests/test_gpu_l1.py tests/test_gpu_robust.py tests/test_gpu_cluster.py tests/test_gpu_modes.py tests/test_gpu_fp32.py -q -x 2>&1 | tail -3
for i in 1 2; do
WCSVD_LIBRARY=tools/exp/lib_nopert.so timeout 600 python tools/scenarios.py C3 C4 "C5/2:0" 2>&1 | cut -c1-130
timeout 600 python tools/scenarios.py C3 C4 "C5/2:0" 2>&1 | cut -c1-130
done
timeout 900 python tools/robustness.py > gpurun_out/robust_pert.json 2>/dev/null; python - <<'PY'
import json
d=json.load(open('gpurun_out/robust_pert.json'))
mx={'sigma_err':0,'residual':0,'orth':0}
for m in d['matrices']:
    for path in ('planner','w=8','w=16','wcycle(w1=64,w2=16)'):
        r=m[path]; mx['sigma_err']=max(mx['sigma_err'],r['sigma_err']); mx['residual']=max(mx['residual'],r['residual']); mx['orth']=max(mx['orth'],r['orth_U'],r['orth_V'])
    print(m['name'], [m[p]['sweeps'] for p in ('planner','w=8','w=16','wcycle(w1=64,w2=16)')])
print(mx)
PY

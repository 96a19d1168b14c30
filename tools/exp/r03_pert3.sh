for i in 1 2; do
timeout 600 python tools/scenarios.py C3 C4 "C5/2:0" 2>&1 | cut -c1-130
WCSVD_LIBRARY=tools/exp/lib_pert3.so timeout 600 python tools/scenarios.py C3 C4 "C5/2:0" 2>&1 | cut -c1-130
done
WCSVD_LIBRARY=tools/exp/lib_pert3.so timeout 900 python tools/robustness.py > gpurun_out/robust_pert3.json 2>/dev/null; python - <<'PY'
import json
d=json.load(open('gpurun_out/robust_pert3.json'))
mx={'sigma_err':0,'residual':0,'orth':0}
for m in d['matrices']:
    for path in ('planner','w=8','w=16','wcycle(w1=64,w2=16)'):
        r=m[path]; mx['sigma_err']=max(mx['sigma_err'],r['sigma_err']); mx['residual']=max(mx['residual'],r['residual']); mx['orth']=max(mx['orth'],r['orth_U'],r['orth_V'])
    print(m['name'], [m[p]['sweeps'] for p in ('planner','w=8','w=16','wcycle(w1=64,w2=16)')])
print(mx)
PY

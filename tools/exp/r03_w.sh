WCSVD_LIBRARY=tools/exp/lib_pre.so python tools/exp/dump.py /tmp/a.npz | tail -1
python tools/exp/dump.py /tmp/b.npz | tail -1
python tools/exp/bitcmp.py /tmp/a.npz /tmp/b.npz
python - <<'PY'
import sys, numpy as np, torch
sys.path.insert(0, '.')
import workloads, paper_conf_sc_xiaopxsmmlzt22_b200 as wc
cfg = workloads.get_config("C2", 512)
A = torch.from_numpy(np.stack(cfg.matrices())).cuda()
S, U, V = wc.svd_batched(A); torch.cuda.synchronize()
np.savez("/tmp/c2_new.npz", S=S.cpu().numpy(), U=U.cpu().numpy(), V=V.cpu().numpy())
PY
WCSVD_LIBRARY=tools/exp/lib_pre.so python - <<'PY'
import sys, numpy as np, torch
sys.path.insert(0, '.')
import workloads, paper_conf_sc_xiaopxsmmlzt22_b200 as wc
cfg = workloads.get_config("C2", 512)
A = torch.from_numpy(np.stack(cfg.matrices())).cuda()
S, U, V = wc.svd_batched(A); torch.cuda.synchronize()
np.savez("/tmp/c2_old.npz", S=S.cpu().numpy(), U=U.cpu().numpy(), V=V.cpu().numpy())
PY
python tools/exp/bitcmp.py /tmp/c2_old.npz /tmp/c2_new.npz
timeout 900 python -m pytest tests/test_gpu_l0.py tests/test_gpu_fp32.py tests/test_gpu_modes.py -q 2>&1 | tail -2
for i in 1 2; do WCSVD_LIBRARY=tools/exp/lib_pre.so timeout 300 python tools/scenarios.py C2 | cut -c1-90; timeout 300 python tools/scenarios.py C2 | cut -c1-90; done

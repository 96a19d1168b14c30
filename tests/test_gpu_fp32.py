"""the fp32 variant (wcsvd_batched_f32). Parity with the long-double oracle run on the
same fp32 inputs, at north_star's fp32 bars: sigma 1e-5, residual 1e-5, orthogonality 1e-4 (vector
bars per R-VEC with u = 2^-24). Level 0 iterates in fp32; the Gram path iterates by default on an fp64
working copy (DMMA) and rounds at finalisation, and with f32_compute = 1 in fp32 throughout (FFMA Gram /
update, fp32 EVD and Newton-Schulz on an fp32 working copy)."""
import numpy as np
import pytest
import torch

import oracle
import workloads
import paper_conf_sc_xiaopxsmmlzt22_b200 as wc
from oracle import compare

pytestmark = pytest.mark.gpu
U32 = 2.0 ** -24


def _check(mats32, S, U, V, info):
    mats64 = [np.asarray(a, dtype=np.float64) for a in mats32]
    So, Uo, Vo, _ = oracle.svd_batch(mats64)
    for k, A in enumerate(mats64):
        p = compare.compare(A, S[k].astype(np.float64), U[k].astype(np.float64), V[k].astype(np.float64),
                            So[k], Uo[k], Vo[k], u=U32, vec_tol=compare.FP32_BARS["vec_tol"],
                            proj_tol=compare.FP32_BARS["proj_tol"])
        assert p.ok(**compare.FP32_BARS), (k, A.shape, p.as_dict(), int(info[k]))
        assert info[k] > 0


def _run(mats32, **kw):
    As = [torch.from_numpy(np.ascontiguousarray(a)).cuda() for a in mats32]
    S, U, V, info = wc.svd_batched(As, return_info=True, **kw)
    torch.cuda.synchronize()
    assert S[0].dtype == torch.float32
    return ([s.cpu().numpy() for s in S], [u.cpu().numpy() for u in U], [v.cpu().numpy() for v in V],
            info.cpu().numpy())


@pytest.mark.parametrize("shapes", [
    [(32, 32), (64, 64), (40, 24), (24, 40), (8, 3), (3, 8), (1, 1)],          # Level 0 (fp32)
    [(100, 37), (190, 64), (480, 31), (1000, 16), (1024, 5)],                 # Level 0, tall
    [(97, 97), (256, 256), (300, 170), (170, 300), (1024, 128)],             # Level 1 (fp32 FFMA)
    [(700, 520), (1024, 1024), (150, 900)],                                   # Level 1, large / wide
])
def test_fp32_parity(shapes):
    mats = [workloads.gaussian(workloads.matrix_rng(700 + i, 5), m, n).astype(np.float32)
            for i, (m, n) in enumerate(shapes)]
    _check(mats, *_run(mats))


def test_fp32_c1_prescribed_and_c2_sample():
    # C1 matrices with kappa <= 1e4 (k mod 5 in {0, 1, 2}); kappa >= 1e8 exceeds fp32's 2^-24
    # resolution (sigma_min < u sigma_1): those are checked in fp64 only (test_gpu_l0.py).
    cfg = workloads.get_config("C1", batch=40)
    c1 = [cfg.make(k).astype(np.float32) for k in range(40) if k % 5 in (0, 1, 2)]
    _check(c1, *_run(c1))
    c2 = np.stack(workloads.get_config("C2", batch=64).matrices()).astype(np.float32)
    S, U, V, info = wc.svd_batched(torch.from_numpy(c2).cuda(), return_info=True)
    torch.cuda.synchronize()
    _check(list(c2), [s for s in S.cpu().numpy()], list(U.cpu().numpy()), list(V.cpu().numpy()),
           info.cpu().numpy())


def test_fp32_rank_deficient_and_nonfinite():
    rng = workloads.matrix_rng(710, 0)
    Z = workloads.gaussian(rng, 30, 12).astype(np.float32)
    Z[:, 4] = 0
    R2 = (workloads.gaussian(rng, 40, 2) @ workloads.gaussian(rng, 2, 20)).astype(np.float32)
    _check([Z, R2], *_run([Z, R2]))
    B = workloads.gaussian(rng, 16, 16).astype(np.float32)
    B[2, 3] = np.inf
    S, U, V, info = _run([B])
    assert info[0] == -2 and np.all(np.isnan(S[0]))


@pytest.mark.parametrize("kw", [dict(f32_compute=1), dict(force_path=wc.PATH_GRAM, force_w=8, f32_compute=1),
                                dict(force_path=wc.PATH_WCYCLE, f32_compute=1), dict(cluster_ctas=4, f32_compute=1),
                                dict(cluster_ctas=4), dict(force_path=wc.PATH_GRAM, force_w=8)])
def test_fp32_gram_variants(kw):
    # the 2w = 16 FFMA path (two lanes per column), the W-cycle on fp32, and a 4-CTA cluster
    shapes = [(130, 100), (100, 150), (256, 160), (64, 64), (1024, 128), (300, 700)]
    mats = [workloads.gaussian(workloads.matrix_rng(720 + i, 7), m, n).astype(np.float32)
            for i, (m, n) in enumerate(shapes)]
    _check(mats, *_run(mats, **kw))

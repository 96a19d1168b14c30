"""values-only and single-factor modes. V_x is not accumulated when it is not
requested; the iteration is unchanged, so S (and the vectors, up to the sign rule) are bitwise those
of the full SVD."""
import numpy as np
import pytest
import torch

import workloads
import paper_conf_sc_xiaopxsmmlzt22_b200 as wc
from oracle import compare

pytestmark = pytest.mark.gpu

SHAPES = [(64, 64), (40, 24), (24, 40), (300, 16), (256, 256), (300, 170), (170, 300), (1024, 128)]


def _mats():
    return [workloads.gaussian(workloads.matrix_rng(600 + i, 1), m, n) for i, (m, n) in enumerate(SHAPES)]


def _run(mats, **kw):
    As = [torch.from_numpy(a).cuda() for a in mats]
    out = wc.svd_batched(As, **kw)
    torch.cuda.synchronize()
    return [[None if t is None else t.cpu().numpy() for t in part] if part is not None else None for part in out]


def test_values_only_is_bitwise_full_sigma():
    mats = _mats()
    S, U, V = _run(mats)
    S0, U0, V0 = _run(mats, compute_uv=False)
    assert U0 is None and V0 is None
    for k in range(len(mats)):
        assert np.array_equal(S0[k], S[k])


@pytest.mark.parametrize("want", ["u", "v"])
def test_single_factor_matches_full_up_to_sign(want):
    mats = _mats()
    S, U, V = _run(mats)
    S1, U1, V1 = _run(mats, compute_u=(want == "u"), compute_v=(want == "v"))
    for k, A in enumerate(mats):
        assert np.array_equal(S1[k], S[k])
        X, X0 = (U1[k], U[k]) if want == "u" else (V1[k], V[k])
        assert (U1 is None) == (want == "v") and (V1 is None) == (want == "u")
        sg = np.sign(np.sum(X * X0, axis=0))
        assert np.all(sg != 0)
        assert np.array_equal(X * sg, X0)
        assert compare.orthogonality(X) <= 1e-11

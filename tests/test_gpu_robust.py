"""robustness workload -- the Table VII analogue. Synthetic
stand-ins with the sizes and condition numbers of the paper's five SuiteSparse picks (kappa from 3.1
to 8.08e15, workloads.table7_config) through the planner's path, the forced W-cycle recursion and the
narrow EVD width (Fig 15(b): w changes the sweep count, not the result). Every run must converge and
meet the oracle bars (oracle/compare.py; R-VEC for the clustered / near-null tail of the kappa = 8e15
matrix), and the singular values must match the prescribed spectrum."""
import numpy as np
import pytest

import oracle
import workloads
import paper_conf_sc_xiaopxsmmlzt22_b200 as wc
from tests.gpu_helpers import check_parity, gpu_svd_list

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def t7():
    cfg = workloads.table7_config()
    mats = cfg.matrices()
    return cfg, mats, oracle.svd_batch(mats)


@pytest.mark.parametrize("knob", [{}, {"force_path": 3}, {"force_path": 2, "force_w": 8}],
                         ids=["planner", "wcycle", "gram_w8"])
def test_table7_standins(t7, knob):
    cfg, mats, ref = t7
    S, U, V, info = gpu_svd_list(mats, **knob)
    check_parity(mats, S, U, V, info, oracle_out=ref)
    for k in range(len(mats)):
        s_true = cfg.spectrum(k)
        # the construction itself is exact to a few ulps of sigma_1 = 1
        assert np.abs(S[k] - s_true).max() <= 1e-12, (workloads.TABLE7[k][0], np.abs(S[k] - s_true).max())
        assert 0 < info[k] <= 60

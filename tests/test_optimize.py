"""Batch bandwidth optimisation driver (NEXT-1, paper Section 3.4 / 5.3)."""
import numpy as np
import pytest

import synth
from paper_conf_sigmod_heimelkm15_b200.optimize import QueryRing


def test_query_ring_keeps_last_q_in_order():
    r = QueryRing(3, 2)
    for k in range(5):
        r.push(np.full(2, k, np.float32), np.full(2, k + 1, np.float32), k / 10)
    lo, hi, p = r.arrays()
    assert list(p) == [0.2, 0.3, 0.4]
    assert lo[:, 0].tolist() == [2, 3, 4]
    r2 = QueryRing(4, 1)
    r2.push([1], [2], 0.5)
    assert r2.arrays()[2].tolist() == [0.5]


@pytest.mark.gpu
def test_batch_optimisation_beats_scott():
    """P:L308/L322 protocol on synthetic data: 100 training + 300 test DT queries;
    the optimised bandwidth lowers the training loss and the test absolute error."""
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_sigmod_heimelkm15_b200 as K
    from paper_conf_sigmod_heimelkm15_b200.optimize import optimize_bandwidth
    d = 3
    R = synth.make_data("gauss", 200000, d, seed=60)
    S = R[synth.rng(61).choice(len(R), 4096, replace=False)]
    lo, hi = synth.workload(R, 400, seed=62, kind="DT")
    p = synth.true_selectivity_cpu(R, lo, hi)
    tr, te = slice(0, 100), slice(100, 400)
    m = K.KDEModel.create(S)
    h_scott = m.bandwidth
    err0 = np.mean(np.abs(m.estimate(lo[te], hi[te]) - p[te]))
    res = optimize_bandwidth(m, lo[tr], hi[tr], p[tr], loss=K.LOSS_SQUARED, n_starts=16, n_local=3)
    assert res.loss <= res.loss_start
    assert np.all(res.h > 0) and not np.allclose(res.h, h_scott)
    err1 = np.mean(np.abs(m.estimate(lo[te], hi[te]) - p[te]))
    assert err1 < err0

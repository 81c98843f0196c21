"""The product's offline-phase ridge fit (paper_conf_asplos_wulzj17_b200/calibrate.py) against the
oracle's (oracle/estimates.py) and sklearn — two independent implementations of P:192."""
import numpy as np
import pytest

from oracle import estimates as E
from synth import gen


def _calib():
    from paper_conf_asplos_wulzj17_b200 import calibrate
    return calibrate


@pytest.mark.parametrize("seed", range(5))
def test_ridge_matches_oracle(seed):
    g = gen.rng(900 + seed)
    X = np.column_stack([g.integers(1, 1 << 20, 100), np.full(100, 256), g.integers(1, 1 << 28, 100),
                         g.choice([0, 9216, 201728], 100)]).astype(float)
    y = 0.8 * X[:, 0] + 0.002 * X[:, 2] + g.normal(0, 3000, 100) + 8000
    m_prod = _calib().ridge_fit(X, y, 1.0)
    coef, b = E.ridge_fit(X, y, lam=1.0)
    m_or = E.model_vector(coef, b)
    p1 = _calib().predict(m_prod, X)
    p2 = X @ np.array(m_or[:4]) + m_or[4]
    assert np.allclose(p1, p2, rtol=1e-9, atol=1e-6)


def test_predict_matches_abi_rounding():
    from paper_conf_asplos_wulzj17_b200 import build, flep
    build.build()
    m = [0.5, 1.25, 0.001, 0.0, 1234.4]
    for f in ([100, 256, 10_000, 0], [3, 128, 7, 9216]):
        assert flep.model_predict_ns(m, *f) == E.predict_ns(m, *f)


def _row(c, k, pf, ap, ovh):
    return {"C": c, "K": k, "prefetch": pf, "async_poll": ap, "overhead": ovh}


def test_select_amortizing_factor_smallest_L_under_bound():
    # the smallest L (tried from small to large) whose overhead is below 4 %
    cal = _calib()
    t = [_row(1, 1, False, False, 0.20), _row(2, 1, False, False, 0.05), _row(1, 2, True, True, 0.03),
         _row(2, 1, True, False, 0.039), _row(4, 1, False, False, 0.01), _row(8, 1, False, False, 0.0)]
    c = cal.select_amortizing_factor(t, 0.04)
    assert c["met"] and c["L"] == 2 and (c["C"], c["K"], c["prefetch"], c["async_poll"]) == (2, 1, True, False)
    # a tighter bound moves to the next L; within one L the variant adding the least latency wins
    c = cal.select_amortizing_factor(t + [_row(4, 1, True, True, 0.005)], 0.02)
    assert c["met"] and c["L"] == 4 and not c["prefetch"]


def test_select_amortizing_factor_unmet_bound():
    cal = _calib()
    t = [_row(1, 1, False, False, 0.30), _row(8, 1, True, True, 0.12), _row(16, 1, False, False, 0.12)]
    c = cal.select_amortizing_factor(t, 0.04)
    assert not c["met"] and c["L"] == 8 and c["overhead"] == 0.12
    with pytest.raises(ValueError):
        cal.select_amortizing_factor([], 0.04)

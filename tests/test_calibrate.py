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

"""Pins for oracle/estimates.py and oracle/metrics.py against library routines and closed forms."""
import numpy as np
import pytest

from oracle import estimates as E
from oracle import metrics as M
from synth import gen


def test_ridge_matches_sklearn():
    from sklearn.linear_model import Ridge
    g = gen.rng(21)
    X = np.column_stack([g.integers(1, 5000, 100), g.choice([64, 128, 256, 512], 100),
                         g.integers(1, 10**7, 100), g.choice([0, 4096, 16384], 100)]).astype(float)
    y = 3.0 * X[:, 0] + 0.5 * X[:, 2] / 1000 + 2.0 * X[:, 3] + g.normal(0, 50, 100) + 1000
    coef, b = E.ridge_fit(X, y, lam=1.0)
    mu, sd = X.mean(0), X.std(0)
    Z = (X - mu) / sd
    sk = Ridge(alpha=1.0, fit_intercept=True).fit(Z, y)
    pred_sk = sk.predict(Z)
    pred = X @ coef + b
    assert np.allclose(pred, pred_sk, rtol=1e-9, atol=1e-6)


def test_ridge_exact_recovery_small_lambda():
    g = gen.rng(22)
    X = g.uniform(0, 100, size=(50, 4))
    y = X @ np.array([1.5, -2.0, 0.25, 3.0]) + 7.0
    coef, b = E.ridge_fit(X, y, lam=1e-12)
    assert np.allclose(coef, [1.5, -2.0, 0.25, 3.0], atol=1e-6)
    assert b == pytest.approx(7.0, abs=1e-5)
    m = E.model_vector(coef, b)
    assert E.predict_ns(m, 1, 2, 3, 4) == int(round(1.5 - 4 + 0.75 + 12 + 7))


def test_overhead_mean_and_metrics():
    assert E.overhead_estimate([10, 20, 31]) == 20
    assert M.antt([10, 30], [10, 10]) == 2.0
    assert M.stp([10, 30], [10, 10]) == pytest.approx(1 + 1 / 3)
    assert M.spatial_overhead(110, 100) == pytest.approx(0.1)
    assert M.overhead_reduction(0.069, 0.1) == pytest.approx(0.31)
    assert M.performance_degradation(30, 10) == 4.0

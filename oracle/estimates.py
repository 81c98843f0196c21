"""Offline estimates used by the runtime policy (§4.2).

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

* Kernel-duration model: per-kernel linear regression with an L2-norm penalty on four
  features — grid size, CTA size, input size, shared-memory size — trained on randomly
  generated inputs. Reading A19: features are standardised (mean 0, unit population std; a
  constant feature is left centred with scale 1), the bias is not penalised, lambda = 1.0.
  Closed form: beta = (Z^T Z + lambda*I)^-1 Z^T (y - mean(y)), bias = mean(y) (Z centred).
* Preemption overhead O: the mean of the profiled overheads ("50 runs").
"""
from __future__ import annotations

import numpy as np


def ridge_fit(X: np.ndarray, y: np.ndarray, lam: float = 1.0):
    """Return (coef_raw[4], intercept_raw) such that prediction = X @ coef_raw + intercept_raw,
    i.e. the standardised fit mapped back to raw feature units."""
    X = np.asarray(X, dtype=np.float64)
    y = np.asarray(y, dtype=np.float64)
    mu = X.mean(axis=0)
    sd = X.std(axis=0)
    sd = np.where(sd > 0, sd, 1.0)
    Z = (X - mu) / sd
    ym = y.mean()
    A = Z.T @ Z + lam * np.eye(X.shape[1])
    b = Z.T @ (y - ym)
    beta = np.linalg.solve(A, b)
    coef = beta / sd
    intercept = ym - float(np.dot(coef, mu))
    return coef, intercept


def model_vector(coef, intercept):
    """The 5-vector the C ABI takes (flep_kernel_desc.model: grid, cta, input, smem, bias)."""
    return [float(c) for c in coef] + [float(intercept)]


def predict_ns(model5, grid, cta, input_size, smem) -> int:
    """T_e in integer ns, rounded once (H8): round-half-away-from-zero of the dot product,
    clamped at >= 1 ns."""
    v = (model5[0] * grid + model5[1] * cta + model5[2] * input_size + model5[3] * smem
         + model5[4])
    r = int(np.floor(abs(v) + 0.5)) * (1 if v >= 0 else -1)
    return max(1, r)


def overhead_estimate(samples) -> int:
    """O = mean of the profiled preemption overheads, integer ns (floor)."""
    s = [int(x) for x in samples]
    return sum(s) // len(s)

"""ORACLE -- TEST INFRASTRUCTURE ONLY: the regression pre-process (NEXT-3)
written from PAPER.md §III-C as plain numpy: normalisations phi_V, phi_C
(P:L117), design matrix of Eq. (6) (row-major (i, j), reading C9) and the
least-squares criterion of Eq. (7) solved by numpy.linalg.lstsq (a library
routine serving as the argmin; the product uses the normal equation, Eq. 8)."""
from __future__ import annotations

import numpy as np


def design(v, c, deg_v, deg_c, v_min=0.55, v_max=1.1, c_min=0.5, c_max=128.0):
    x = (np.asarray(v, np.float64) - v_min) / (v_max - v_min)
    z = np.zeros_like(x) if deg_c == 0 else \
        (np.log2(np.asarray(c, np.float64)) - np.log2(c_min)) / (np.log2(c_max) - np.log2(c_min))
    return np.stack([x ** i * z ** j for i in range(deg_v + 1) for j in range(deg_c + 1)], axis=1)


def fit(v, c, y, deg_v, deg_c, **bounds):
    X = design(v, c, deg_v, deg_c, **bounds)
    beta, *_ = np.linalg.lstsq(X, np.asarray(y, np.float64), rcond=None)
    return beta.reshape(deg_v + 1, deg_c + 1)


def evaluate(beta, v, c, **bounds):
    """f(P) of Eq. (4) by the plain double sum (no Horner)."""
    dv, dc = beta.shape[0] - 1, beta.shape[1] - 1
    return design(v, c, dv, dc, **bounds) @ beta.ravel()

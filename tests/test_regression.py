"""NEXT-3 regression pre-process (-m "not gpu"): the library's normal-equation
fit (avfs_fit_delay_polynomial, host code in libavfs) vs the oracle's
numpy.linalg.lstsq, exact recovery of a known polynomial, and Fig. 4-style
error statistics on an alpha-power x logical-effort ground truth."""
import numpy as np
import pytest

from oracle import fit as ofit
from workloads.characterization import make_arcs, paper_grid_samples, eval_grid


@pytest.fixture(scope="module")
def fitlib():
    from paper_conf_date_schneiderw20_b200 import _build
    _build.build()
    from paper_conf_date_schneiderw20_b200 import fit_delay_polynomial
    return fit_delay_polynomial


@pytest.mark.parametrize("dv,dc", [(0, 0), (2, 0), (3, 0), (1, 1), (3, 3), (4, 2)])
def test_exact_recovery_of_known_polynomial(fitlib, dv, dc):
    rng = np.random.default_rng(10 * dv + dc)
    beta = rng.normal(size=(dv + 1, dc + 1)) * 0.3
    arc = make_arcs(1, 1)[0]
    v, c, _ = paper_grid_samples(arc)
    y = ofit.evaluate(beta, v, c)
    got, rms = fitlib(v, c if dc else None, y, dv, dc)
    assert np.allclose(got, beta, rtol=0, atol=1e-8)
    assert rms < 1e-10


@pytest.mark.parametrize("N", [1, 2, 3])
def test_matches_lstsq_on_alpha_power_data(fitlib, N):
    for arc in make_arcs(7, 6):
        v, c, y = paper_grid_samples(arc)
        got, rms = fitlib(v, c, y, N, N)
        want = ofit.fit(v, c, y, N, N)
        vv, cc = eval_grid(64)
        assert np.allclose(ofit.evaluate(got, vv, cc), ofit.evaluate(want, vv, cc), rtol=0, atol=1e-8)
        resid = y - ofit.evaluate(want, v, c)
        assert abs(rms - np.sqrt(np.mean(resid ** 2))) < 1e-9


def test_fig4_error_statistics(fitlib):
    """Fig. 4 / P:L183 on the synthetic ground truth: the error of
    d' = d_nom (1 + f) (Eq. 9) over a 64 x 64 grid shrinks with the order 2N,
    and for N >= 3 the average stddev is below 1 % and the average maximum
    error below 2.7 % (the paper's statements for NanGate 15 nm)."""
    arcs = make_arcs(2024, 24)
    vv, cc = eval_grid(64)
    stats = []
    for N in (1, 2, 3, 4):
        mean_e, std_e, max_e = [], [], []
        for arc in arcs:
            v, c, y = paper_grid_samples(arc)
            beta, _ = fitlib(v, c, y, N, N)
            d_fit = arc.d_nom(cc) * (1.0 + ofit.evaluate(beta, vv, cc))
            err = np.abs(d_fit / arc.delay(vv, cc) - 1.0)
            mean_e.append(err.mean())
            std_e.append(err.std())
            max_e.append(err.max())
        stats.append((np.mean(mean_e), np.mean(std_e), np.mean(max_e)))
    for a, b in zip(stats, stats[1:]):
        assert a[0] > b[0] and a[2] > b[2]
    for N, (m, sd, mx) in zip((1, 2, 3, 4), stats):
        if N >= 3:
            assert sd < 0.01 and mx < 0.027 and m < 0.01


def test_fit_argument_errors(fitlib):
    from paper_conf_date_schneiderw20_b200 import AvfsError
    with pytest.raises(AvfsError):                   # fewer samples than coefficients
        fitlib(np.array([0.6, 0.7]), np.array([1.0, 2.0]), np.array([0.1, 0.2]), 2, 2)
    with pytest.raises(AvfsError):                   # rank deficient (one voltage only)
        fitlib(np.full(20, 0.8), np.full(20, 1.0), np.zeros(20), 2, 0)

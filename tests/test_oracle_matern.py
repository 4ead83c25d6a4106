"""Pins for oracle/matern.py (§III-A): closed forms, mpmath, C(0) = sigma^2."""
import mpmath
import numpy as np
import pytest

from oracle.matern import distance, matern, matern_closed_form

mpmath.mp.dps = 40


def mp_matern(h, sigma2, beta, nu):
    """P:82 written out in 40-digit arithmetic (independent of scipy)."""
    if h == 0:
        return mpmath.mpf(sigma2)
    r = mpmath.mpf(h) / mpmath.mpf(beta)
    nu = mpmath.mpf(nu)
    return mpmath.mpf(sigma2) * 2 ** (1 - nu) / mpmath.gamma(nu) * r**nu * mpmath.besselk(nu, r)


@pytest.mark.parametrize("nu", [0.5, 1.5, 2.5])
def test_closed_form_equals_general_formula(nu):
    h = np.concatenate([np.logspace(-6, 0.5, 200), [0.0]])
    a = matern(h, 1.7, 0.13, nu)
    b = matern_closed_form(h, 1.7, 0.13, nu)
    np.testing.assert_allclose(a, b, rtol=2e-14, atol=0)


@pytest.mark.parametrize("nu", [0.5, 1.5, 2.5])
def test_closed_form_against_mpmath(nu):
    for h in [1e-5, 0.003, 0.05, 0.4, 1.2]:
        ref = float(mp_matern(h, 0.9, 0.07, nu))
        got = float(matern_closed_form(np.array([h]), 0.9, 0.07, nu)[0])
        # r = h/beta carries one rounding, so exp(-r) carries ~ r * eps relative error
        assert abs(got - ref) <= 4e-16 * (2 + h / 0.07) * abs(ref)


@pytest.mark.parametrize("nu", [0.25, 0.8, 1.0, 1.3, 2.0, 3.7])
def test_general_nu_against_mpmath(nu):
    hs = [1e-4, 1e-3, 0.01, 0.05, 0.1, 0.3, 0.7, 1.4]
    got = matern(np.array(hs), 1.3, 0.1, nu)
    for h, g in zip(hs, got):
        ref = float(mp_matern(h, 1.3, 0.1, nu))
        assert abs(g - ref) <= 1e-12 * abs(ref), (nu, h, g, ref)


def test_zero_distance_is_sigma2():
    for nu in [0.3, 0.5, 1.0, 2.5]:
        assert matern(np.array([0.0]), 2.5, 0.3, nu)[0] == 2.5
    # reading C3: near 0 the formula is a genuine r^(2 nu) term, not sigma^2 exactly
    v = matern(np.array([1e-12]), 1.0, 1.0, 0.3)[0]
    assert v < 1.0 and v > 0.99


def test_monotone_decreasing_in_distance():
    h = np.linspace(0, 2, 400)
    for nu in [0.5, 1.0, 2.5]:
        c = matern(h, 1.0, 0.1, nu)
        assert np.all(np.diff(c) <= 0)


def test_distance_is_euclidean():
    assert distance(0.0, 0.0, 3.0, 4.0) == 5.0


def test_sqexp_closed_form_and_limits():
    """C(h) = sigma^2 exp(-h^2/beta); pinned against mpmath and its limits."""
    from oracle.matern import sqexp
    for h in [0.0, 1e-4, 0.01, 0.2, 0.9]:
        ref = float(mpmath.mpf(1.7) * mpmath.exp(-(mpmath.mpf(h) ** 2) / mpmath.mpf(0.05)))
        got = float(sqexp(np.array([h]), 1.7, 0.05)[0])
        assert abs(got - ref) <= 4e-16 * (1 + h * h / 0.05) * ref
    assert sqexp(np.array([0.0]), 2.0, 0.3)[0] == 2.0

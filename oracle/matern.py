"""2D Matérn covariance, PAPER.md:82 (§III-A, item 2).  Oracle: test infrastructure only.

    C(h; theta) = sigma^2 * 2^(1-nu) / Gamma(nu) * (h/beta)^nu * K_nu(h/beta),
    theta = (sigma^2, beta, nu),

with K_nu the modified Bessel function of the second kind.  Readings
(DESIGN.md §Readings):
  C3  C(0) = sigma^2 (the limit h -> 0; the formula itself is 0 * inf).
  C5  h is the Euclidean distance in the unit square.
For nu in {1/2, 3/2, 5/2} K_nu has an elementary closed form; `matern` uses the
general formula for every nu (scipy.special.kv / gamma as the library
primitive), `matern_closed_form` spells the elementary forms out, and the
tests pin one against the other and both against mpmath.
"""
from __future__ import annotations

import numpy as np
from scipy import special


def distance(xi, yi, xj, yj):
    """Euclidean distance (reading C5): sqrt((xi-xj)^2 + (yi-yj)^2)."""
    dx = xi - xj
    dy = yi - yj
    return np.sqrt(dx * dx + dy * dy)


def matern(h, sigma2: float, beta: float, nu: float):
    """C(h; theta) per P:82 with the general-nu formula; C(0) = sigma^2 (reading C3)."""
    h = np.asarray(h, dtype=np.float64)
    r = h / beta
    out = np.full(r.shape, float(sigma2), dtype=np.float64)
    pos = r > 0
    rp = r[pos]
    coef = 2.0 ** (1.0 - nu) / special.gamma(nu)
    out[pos] = sigma2 * coef * rp**nu * special.kv(nu, rp)
    return out


def sqexp(h, sigma2: float, beta: float):
    """2D/3D squared exponential, P:81 (§III-A item 1): C(h; theta) = sigma^2 exp(-h^2 / beta)."""
    h = np.asarray(h, dtype=np.float64)
    return sigma2 * np.exp(-(h * h) / beta)


def covariance(h, theta, kernel: str = "matern"):
    """C(h; theta) for the two covariance families of the paper."""
    if kernel == "matern":
        return matern(h, theta[0], theta[1], theta[2])
    if kernel == "sqexp":
        return sqexp(h, theta[0], theta[1])
    raise ValueError(kernel)


def matern_closed_form(h, sigma2: float, beta: float, nu: float):
    """Elementary forms of P:82 for half-integer nu:
    nu=1/2: e^-r;  nu=3/2: (1+r) e^-r;  nu=5/2: (1 + r + r^2/3) e^-r,  r = h/beta."""
    r = np.asarray(h, dtype=np.float64) / beta
    if nu == 0.5:
        poly = np.ones_like(r)
    elif nu == 1.5:
        poly = 1.0 + r
    elif nu == 2.5:
        poly = 1.0 + r + r * r / 3.0
    else:
        raise ValueError("closed form only for nu in {0.5, 1.5, 2.5}")
    return sigma2 * poly * np.exp(-r)

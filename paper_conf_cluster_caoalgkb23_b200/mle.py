"""Maximum-likelihood driver (§VII-B): maximise l(theta) of Eq. (1) over theta.

The paper uses BOBYQA from NLopt, tolerance 1e-9, every parameter in [0.01, 2], starting from the
lower bounds.  NLopt is not available here; the driver uses SciPy's COBYQA (Powell's
derivative-free, bound-constrained quadratic-model trust-region method, the successor of BOBYQA)
with the same bounds and start, and a final trust-region radius of `tol` (reading C19: the paper's
"tolerance 1e-9" as a relative step tolerance).  Each objective call is one mp_eval on the GPU;
a non-SPD Sigma(theta) (l = -inf) is returned as a large finite penalty so the optimiser can
back off.  This outer loop is host-side Python by design: it is the caller of the hot path, not
part of it.
"""
from __future__ import annotations

import math
import time
from dataclasses import dataclass, field

import numpy as np

from . import MP_MAP_ADAPTIVE, MP_COMM_AUTO, Evaluator

PENALTY = 1e30


@dataclass
class MLEResult:
    theta: np.ndarray
    loglik: float
    nfev: int
    seconds: float
    history: list = field(default_factory=list)
    message: str = ""


def fit(ev: Evaluator, x, y, z, theta0=(0.01, 0.01, 0.01), bounds=((0.01, 2.0),) * 3, u_req: float = 1e-9,
        mode: int = MP_MAP_ADAPTIVE, policy: int = MP_COMM_AUTO, tol: float = 1e-9, maxfev: int = 500,
        fixed_nu: float | None = None, log=None, cache: dict | None = None) -> MLEResult:
    """theta_hat = argmax l(theta).  `fixed_nu` fits (sigma^2, beta) only.  x, y, z: host numpy
    arrays or device tensors (device tensors avoid the per-call host-to-device copy).  `cache`: exact
    {theta: l} values of an earlier identical run (the optimiser and the evaluation are deterministic,
    so a replay retraces it and continues)."""
    from scipy.optimize import Bounds, minimize

    hist = []
    free = 2 if fixed_nu is not None else 3

    def full(t):
        return (float(t[0]), float(t[1]), float(fixed_nu)) if fixed_nu is not None else tuple(float(v) for v in t)

    def obj(t):
        th = full(t)
        if cache and th in cache:
            ll = cache[th]
        else:
            rep = ev.eval(x, y, z, th, u_req=u_req, mode=mode, policy=policy)
            ll = rep.loglik if math.isfinite(rep.loglik) else -PENALTY
        hist.append((th, ll))
        if log:
            log(th, ll)
        return -ll

    lo = np.array([b[0] for b in bounds[:free]])
    hi = np.array([b[1] for b in bounds[:free]])
    t0 = np.clip(np.array(theta0[:free], dtype=np.float64), lo, hi)
    start = time.perf_counter()
    res = minimize(obj, t0, method="COBYQA", bounds=Bounds(lo, hi),
                   options={"maxfev": maxfev, "final_tr_radius": tol, "scale": True})
    th = full(res.x)
    best = max(hist, key=lambda h: h[1]) if hist else (th, -res.fun)
    return MLEResult(theta=np.array(best[0]), loglik=best[1], nfev=len(hist), seconds=time.perf_counter() - start,
                     history=hist, message=str(res.message))

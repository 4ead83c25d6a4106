"""theta recovery, MP vs FP64 (north star: |theta_MP - theta_FP64| <= 1e-3 per component, same data,
optimiser and start).  Z = L(theta_true) e where L is this library's own all-FP64 factor
(validated against the oracle at smaller n); bounds [0.01, 2], start at the lower bounds."""
import json
import os
import sys
import time

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_cluster_caoalgkb23_b200 as mp  # noqa: E402
import synth  # noqa: E402
from paper_conf_cluster_caoalgkb23_b200.mle import fit  # noqa: E402


def sample_z(ev, x, y, theta, seed):
    """Z = L e with L the all-FP64 factor of Sigma(theta): y = L e via the lower tiles."""
    n, nb, M = ev.n, ev.nb, ev.M
    ev.eval(x, y, np.zeros(n), theta, mode=mp.MP_MAP_FP64)  # leaves L in the matrix
    e = synth.normal_vector(n, seed)
    nt = M.nt
    z = np.zeros(n)
    for k in range(nt):
        c0, c1 = k * nb, min(n, (k + 1) * nb)
        for m in range(k, nt):
            r0, r1 = m * nb, min(n, (m + 1) * nb)
            t = M.tile(m, k)[: r1 - r0, : c1 - c0]
            z[r0:r1] += t @ e[c0:c1]
    return z


def main():
    n = int(sys.argv[1]) if len(sys.argv) > 1 else 40000
    modes = (sys.argv[2] if len(sys.argv) > 2 else "fp64,mp").split(",")
    maxfev = int(sys.argv[3]) if len(sys.argv) > 3 else 600
    nb = 2048
    theta_true = (1.0, 0.03, 0.5)
    x, y = synth.locations(n, 0)
    ev = mp.Evaluator(n, nb)
    z = sample_z(ev, x, y, theta_true, 1)
    dx, dy, dz = (torch.from_numpy(a).cuda() for a in (x, y, z))
    out = {"n": n, "nb": nb, "theta_true": theta_true, "optimizer": "COBYQA (BOBYQA family), bounds [0.01,2]^3, "
           "start at the lower bounds, final trust radius 1e-9"}
    os.makedirs("gpurun_out", exist_ok=True)
    for name, mode in [("fp64", mp.MP_MAP_FP64), ("mp", mp.MP_MAP_ADAPTIVE)]:
        if name not in modes:
            continue
        t0 = time.time()
        logf = open(f"gpurun_out/mle_n{n}_{name}.log", "w")

        def log(th, ll, logf=logf):
            logf.write(f"{th[0]:.10f} {th[1]:.10f} {th[2]:.10f} {ll:.10f}\n")
            logf.flush()

        r = fit(ev, dx, dy, dz, mode=mode, u_req=1e-9, maxfev=maxfev, log=log)
        rep = ev.eval(dx, dy, dz, tuple(r.theta), mode=mode)
        out[name] = {"theta": list(r.theta), "loglik": r.loglik, "nfev": r.nfev, "seconds": time.time() - t0,
                     "tiles_fp64_fp32_fp16": list(rep.tiles)}
        print(name, out[name], flush=True)
    if "mp" in out and "fp64" in out:
        out["max_abs_dtheta"] = float(np.max(np.abs(np.array(out["mp"]["theta"]) - np.array(out["fp64"]["theta"]))))
    print(json.dumps(out))
    json.dump(out, open(f"gpurun_out/mle_n{n}_{'_'.join(modes)}.json", "w"), indent=1)


if __name__ == "__main__":
    main()

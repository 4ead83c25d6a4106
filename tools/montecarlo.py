"""Monte-Carlo theta-recovery study, reduced replica count.

For each replica r: locations (jittered grid, seed r), Z = L(theta_true) e_r from the library's own
FP64 factor (mp_gp_sample), then MLE with the FP64 map and with the adaptive MP map at u_req (COBYQA,
bounds [0.01, 2]^3, start at the lower bounds).  Reports every estimate, the per-replica
max |theta_MP - theta_FP64| and the mean / std of both estimators.

  python tools/montecarlo.py [n] [replicas] [u_req] [beta] [nu] [fp64_replicas] [maxfev]

The FP64-map MLE (the MP-vs-FP64 comparison) runs on the first `fp64_replicas` replicas only (default
all); every replica gets the MP estimate.
"""
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


def main():
    n = int(sys.argv[1]) if len(sys.argv) > 1 else 10000
    R = int(sys.argv[2]) if len(sys.argv) > 2 else 4
    u_req = float(sys.argv[3]) if len(sys.argv) > 3 else 1e-9
    nb = 2048 if n >= 40000 else 512
    beta = float(sys.argv[4]) if len(sys.argv) > 4 else 0.03
    nu = float(sys.argv[5]) if len(sys.argv) > 5 else 0.5
    n64 = int(sys.argv[6]) if len(sys.argv) > 6 else R
    maxfev = int(sys.argv[7]) if len(sys.argv) > 7 else 600
    theta_true = (1.0, beta, nu)
    ev = mp.Evaluator(n, nb)
    reps = []
    os.makedirs("gpurun_out", exist_ok=True)
    for r in range(R):
        x, y = synth.locations(n, 100 + r)
        dx, dy = torch.from_numpy(x).cuda(), torch.from_numpy(y).cuda()
        ev.eval(dx, dy, torch.zeros(n, dtype=torch.float64, device="cuda"), theta_true, mode=mp.MP_MAP_FP64)
        de = torch.from_numpy(synth.normal_vector(n, 200 + r)).cuda()
        dz = torch.zeros(n, dtype=torch.float64, device="cuda")
        ev.M.gp_sample(de, dz)
        t0 = time.time()
        fmp = fit(ev, dx, dy, dz, mode=mp.MP_MAP_ADAPTIVE, u_req=u_req, maxfev=maxfev)
        rec = {"replica": r, "mp": list(fmp.theta), "nfev_mp": fmp.nfev, "converged_mp": fmp.nfev < maxfev,
               "loglik_mp": fmp.loglik}
        if r < n64:
            f64 = fit(ev, dx, dy, dz, mode=mp.MP_MAP_FP64, maxfev=maxfev)
            rec.update({"fp64": list(f64.theta), "max_abs_dtheta": float(np.max(np.abs(fmp.theta - f64.theta))),
                        "nfev_fp64": f64.nfev, "converged_fp64": f64.nfev < maxfev, "loglik_fp64": f64.loglik})
        rec["seconds"] = time.time() - t0
        print(json.dumps(rec), flush=True)
        reps.append(rec)
        json.dump({"partial": reps, "theta_true": theta_true, "n": n, "u_req": u_req, "maxfev": maxfev},
                  open(f"gpurun_out/montecarlo_n{n}_R{R}_b{beta}_nu{nu}_f{maxfev}.json", "w"), indent=1)
    a64 = np.array([q["fp64"] for q in reps if "fp64" in q])
    amp = np.array([q["mp"] for q in reps])
    out = {"n": n, "nb": nb, "replicas": R, "fp64_replicas": len(a64), "u_req": u_req, "theta_true": theta_true,
           "maxfev": maxfev, "reps": reps, "mp_mean": amp.mean(0).tolist(), "mp_std": amp.std(0).tolist(),
           "fp64_mean": a64.mean(0).tolist() if len(a64) else None, "fp64_std": a64.std(0).tolist() if len(a64) else None,
           "max_abs_dtheta": float(max(q["max_abs_dtheta"] for q in reps if "max_abs_dtheta" in q)) if len(a64) else None}
    print(json.dumps(out))
    json.dump(out, open(f"gpurun_out/montecarlo_n{n}_R{R}_b{beta}_nu{nu}_f{maxfev}.json", "w"), indent=1)


if __name__ == "__main__":
    main()

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


def sample_z(ev, dx, dy, theta, seed):
    """Z = L(theta) e with L the library's all-FP64 factor of Sigma(theta) (mp_gp_sample, on the device)."""
    n = ev.n
    ev.eval(dx, dy, torch.zeros(n, dtype=torch.float64, device="cuda"), theta, mode=mp.MP_MAP_FP64)
    de = torch.from_numpy(synth.normal_vector(n, seed)).cuda()
    dz = torch.zeros(n, dtype=torch.float64, device="cuda")
    ev.M.gp_sample(de, dz)
    return dz


def main():
    n = int(sys.argv[1]) if len(sys.argv) > 1 else 40000
    modes = (sys.argv[2] if len(sys.argv) > 2 else "fp64,mp").split(",")
    maxfev = int(sys.argv[3]) if len(sys.argv) > 3 else 600
    # replay: the exact (hex) history of an interrupted run of the same workload; COBYQA is deterministic and
    # so is the evaluation, so the optimiser retraces it from the cache and continues live (one GPU call is
    # limited to an hour; a C3 FP64-map MLE from the paper's start takes longer)
    cache = {}
    for path in sys.argv[4:]:
        for line in open(path):
            f = line.split()
            if len(f) == 4 and f[0].startswith(("0x", "-0x")):
                cache[tuple(float.fromhex(v) for v in f[:3])] = float.fromhex(f[3])
    nb = 2048
    theta_true = (1.0, 0.03, 0.5)
    x, y = synth.locations(n, 0)
    ev = mp.Evaluator(n, nb)
    dx, dy = (torch.from_numpy(a).cuda() for a in (x, y))
    dz = sample_z(ev, dx, dy, theta_true, 1)
    out = {"n": n, "nb": nb, "theta_true": theta_true, "optimizer": "COBYQA (BOBYQA family), bounds [0.01,2]^3, "
           "start at the lower bounds, final trust radius 1e-9"}
    os.makedirs("gpurun_out", exist_ok=True)
    for name, mode in [("mp", mp.MP_MAP_ADAPTIVE), ("fp64", mp.MP_MAP_FP64)]:
        if name not in modes:
            continue
        t0 = time.time()
        logf = open(f"gpurun_out/mle_n{n}_{name}.log", "w")

        def log(th, ll, logf=logf):
            logf.write(" ".join(float(v).hex() for v in (*th, ll)) + "\n")
            logf.flush()

        r = fit(ev, dx, dy, dz, mode=mode, u_req=1e-9, maxfev=maxfev, log=log, cache=cache)
        rep = ev.eval(dx, dy, dz, tuple(r.theta), mode=mode)
        out[name] = {"theta": list(r.theta), "loglik": r.loglik, "nfev": r.nfev, "seconds": time.time() - t0,
                     "tiles_fp64_fp32_fp16": list(rep.tiles), "message": r.message}
        print(name, out[name], flush=True)
        json.dump(out, open(f"gpurun_out/mle_n{n}_{'_'.join(modes)}.json", "w"), indent=1)
    if "mp" in out and "fp64" in out:
        out["max_abs_dtheta"] = float(np.max(np.abs(np.array(out["mp"]["theta"]) - np.array(out["fp64"]["theta"]))))
    print(json.dumps(out))
    json.dump(out, open(f"gpurun_out/mle_n{n}_{'_'.join(modes)}.json", "w"), indent=1)


if __name__ == "__main__":
    main()

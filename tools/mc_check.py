"""For a Monte-Carlo replica whose MP and FP64 fits ended apart: evaluate both objectives (adaptive MP map and
all-FP64 map) at both estimates.  If the MP objective is also higher at the FP64 estimate, the gap is the
optimiser's path on the flat sigma^2-beta ridge, not the mixed-precision arithmetic.

  python tools/mc_check.py <montecarlo json> <replica>"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    import torch

    import paper_conf_cluster_caoalgkb23_b200 as mp
    import synth
    d = json.load(open(sys.argv[1]))
    r = int(sys.argv[2])
    rec = [q for q in (d.get("reps") or d["partial"]) if q["replica"] == r][0]
    n = d["n"]
    nb = 2048 if n >= 40000 else 512
    theta_true = tuple(d["theta_true"])
    ev = mp.Evaluator(n, nb)
    x, y = synth.locations(n, 100 + r)
    dx, dy = torch.from_numpy(x).cuda(), torch.from_numpy(y).cuda()
    ev.eval(dx, dy, torch.zeros(n, dtype=torch.float64, device="cuda"), theta_true, mode=mp.MP_MAP_FP64)
    de = torch.from_numpy(synth.normal_vector(n, 200 + r)).cuda()
    dz = torch.zeros(n, dtype=torch.float64, device="cuda")
    ev.M.gp_sample(de, dz)
    out = {"file": sys.argv[1], "replica": r}
    for name, th in (("theta_mp", rec["mp"]), ("theta_fp64", rec["fp64"])):
        for mname, mode in (("mp", mp.MP_MAP_ADAPTIVE), ("fp64", mp.MP_MAP_FP64)):
            out[f"l_{mname}({name})"] = ev.eval(dx, dy, dz, tuple(th), u_req=d.get("u_req", 1e-9), mode=mode).loglik
    print(json.dumps(out))
    os.makedirs("gpurun_out", exist_ok=True)
    json.dump(out, open(f"gpurun_out/mc_check_r{r}.json", "w"), indent=1)


if __name__ == "__main__":
    main()

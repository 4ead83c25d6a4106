"""Reading C7' (four-level maps): fix the FP16_32 class's u_low experimentally, as P:258 says the paper
does ("[23] show FP16_32 has a lower error bound than FP16, so we experimentally determine its machine
epsilon in applications").

Application tiles: the all-FP64 factor of Sigma(theta) at C2 (n = 40,000, nb = 2048, theta = (1, 0.03,
0.5)); for every trailing-update GEMM(m, n, k) whose three-level kernel class is FP16 (the tiles the
FP16 classes would compute), the GEMM L_mk L_nk^T is run with the library's FP16_32 kernel (row-scaled
FP16 operands, FP32 accumulation) and its pure-FP16 kernel (F16 accumulation), and compared with the
FP64 product: e_c = ||C_c - L_mk L_nk^T||_F / (||L_mk||_F ||L_nk||_F).  Then

    eps(FP16_32) = 2^-10 * median(e_FP16_32 / e_FP16)      (FP16's u_low = its machine epsilon 2^-10)

rounded UP to a power of two (the conservative side: a larger eps gives the FP16_32 class fewer
tiles; the value the library ships as MP_EPS_FP16_32).  Output:
gpurun_out/fp16_eps.json.  python tools/fp16_eps.py [n] [samples]"""
import ctypes as C
import json
import math
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    import torch

    import paper_conf_cluster_caoalgkb23_b200 as mp
    import synth
    from paper_conf_cluster_caoalgkb23_b200._lib import lib

    n = int(sys.argv[1]) if len(sys.argv) > 1 else 40000
    samples = int(sys.argv[2]) if len(sys.argv) > 2 else 24
    nb, theta, u_req = 2048, (1.0, 0.03, 0.5), 1e-9
    x, y = synth.locations(n, 0)
    z = synth.normal_vector(n, 1)
    ev = mp.Evaluator(n, nb)
    r = ev.eval(x, y, z, theta, u_req=u_req)  # three-level map: which GEMMs are FP16-class
    km3, _, _ = ev.M.maps()
    nt = ev.nt
    ev.eval(x, y, z, theta, mode=mp.MP_MAP_FP64)  # the FP64 factor
    cand = [(m, n_, k) for k in range(nt) for m in range(k + 2, nt) for n_ in range(k + 1, m) if km3[m, n_] == mp.MP_FP16]
    rng = np.random.default_rng(0)
    pick = [cand[i] for i in rng.choice(len(cand), size=min(samples, len(cand)), replace=False)]
    rows = []
    for (m, n_, k) in pick:
        Lm, Ln = ev.M.tile(m, k), ev.M.tile(n_, k)
        P = np.ascontiguousarray(np.concatenate([Ln, Lm]))  # panel rows: 0 = L_nk, 1 = L_mk
        exact = Lm.astype(np.float32).astype(np.float64) @ Ln.astype(np.float32).astype(np.float64).T
        den = np.linalg.norm(Lm) * np.linalg.norm(Ln)
        err = {}
        for kind in (0, 3):
            dP = torch.from_numpy(P).cuda()
            dC = torch.zeros((nb, nb), dtype=torch.float32, device="cuda")
            assert lib.mp_test_tc_gemm_split(kind, C.c_void_p(dP.data_ptr()), C.c_void_p(dC.data_ptr()), nb, 2, 1, 0, 0) == 0
            err[kind] = float(np.linalg.norm(-dC.cpu().numpy().astype(np.float64) - exact)) / den
        rows.append({"m": m, "n": n_, "k": k, "e_fp16_32": err[0], "e_fp16": err[3], "ratio": err[0] / err[3]})
        print(rows[-1], flush=True)
    ratio = float(np.median([q["ratio"] for q in rows]))
    eps = 2.0**-10 * ratio
    out = {"n": n, "nb": nb, "theta": theta, "u_req": u_req, "three_level_tiles": list(r.tiles), "samples": rows,
           "median_ratio_e16_32_over_e16": ratio, "eps_fp16_32": eps,
           "eps_fp16_32_pow2": 2.0 ** math.ceil(math.log2(eps)),
           "definition": "eps(FP16_32) = 2^-10 * median over FP16-class GEMMs of ||C_16_32 - C|| / ||C_16 - C|| "
                         "(normwise, vs the FP64 product of the FP32-rounded operands)"}
    os.makedirs("gpurun_out", exist_ok=True)
    json.dump(out, open("gpurun_out/fp16_eps.json", "w"), indent=1)
    print(json.dumps({k: v for k, v in out.items() if k != "samples"}))


if __name__ == "__main__":
    main()

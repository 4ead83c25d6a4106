"""Exactly W + 1 evaluations of a bench workload through the public API (no timing, no side legs):
the command to run under ncu for the launch list / a single-kernel capture of the bench's launch
configuration.  Usage: python tools/one_eval.py [c3] [warm=0]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_cluster_caoalgkb23_b200 as mp  # noqa: E402
import synth  # noqa: E402
from bench import CONFIGS  # noqa: E402


def main():
    cfg = CONFIGS[sys.argv[1] if len(sys.argv) > 1 else "c3"]
    warm = int(sys.argv[2]) if len(sys.argv) > 2 else 0
    n, nb = cfg["n"], cfg["nb"]
    x, y = synth.locations(n, seed=0)
    z = synth.normal_vector(n, seed=1)
    dx, dy, dz = (torch.from_numpy(v).cuda() for v in (x, y, z))
    ev = mp.Evaluator(n, nb)
    mode = {"adaptive": mp.MP_MAP_ADAPTIVE, "adaptive4": mp.MP_MAP_ADAPTIVE4, "fp64": mp.MP_MAP_FP64,
            "band": mp.MP_MAP_BAND, "extreme": mp.MP_MAP_EXTREME}[cfg["map"]]
    for _ in range(warm + 1):
        r = ev.eval(dx, dy, dz, cfg["theta"], u_req=1e-9, mode=mode)
    torch.cuda.synchronize()
    print(f"l = {r.loglik:.10f}, launches {r.gpu_launches}, tiles {list(r.tiles)} + pure FP16 {r.tiles_fp16h}")


if __name__ == "__main__":
    main()

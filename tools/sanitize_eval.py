"""One small evaluation per engine, for compute-sanitizer (memcheck / racecheck / synccheck):
FP64 map (Ozaki and DMMA FP64 engines), adaptive MP map (tcgen05 FP32/FP16), general nu (table)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

import paper_conf_cluster_caoalgkb23_b200 as mp  # noqa: E402
import synth  # noqa: E402

n, nb = 2304, 512  # 48^2, NT = 5 with a ragged last tile
x, y = synth.locations(n, 0)
z = synth.normal_vector(n, 1)
ev = mp.Evaluator(n, nb)
out = []
for mode, theta in [(mp.MP_MAP_FP64, (1.0, 0.1, 0.5)), (mp.MP_MAP_ADAPTIVE, (1.0, 0.02, 0.5)),
                    (mp.MP_MAP_EXTREME, (1.0, 0.05, 0.5)), (mp.MP_MAP_FP64, (1.0, 0.1, 0.8))]:
    r = ev.eval(x, y, z, theta, mode=mode)
    out.append(r.loglik)
print("sanitize evals ok", out)

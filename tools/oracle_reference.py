"""Oracle reference values for the studies (calls only oracle/ and synth/): the FP64-definition l of a
bench workload at sizes the host can factor (C1, C2), plus the oracle's wall time and thread count —
the DESIGN.md error columns and the CPU timing of §8(d).  Usage: python tools/oracle_reference.py c2 [theta]"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import synth  # noqa: E402
from oracle.loglik import loglik  # noqa: E402

CONF = {"c1": (1600, 400, (1.0, 0.1, 0.5)), "c2": (40000, 2048, (1.0, 0.03, 0.5))}


def main():
    name = sys.argv[1] if len(sys.argv) > 1 else "c1"
    n, nb, theta = CONF[name]
    if len(sys.argv) > 2:
        theta = tuple(float(v) for v in sys.argv[2].split(","))
    x, y = synth.locations(n, 0)
    z = synth.normal_vector(n, 1)
    t0 = time.perf_counter()
    r = loglik(x, y, z, theta, nb)
    t = time.perf_counter() - t0
    try:
        from threadpoolctl import threadpool_info
        threads = max(i.get("num_threads", 0) for i in threadpool_info() if i.get("user_api") == "blas")
    except Exception:
        threads = os.cpu_count()
    out = {"config": name, "n": n, "nb": nb, "theta": theta, "loglik": r["loglik"], "logdet": r["logdet"],
           "quad": r["quad"], "seconds": t, "tflops": n**3 / 3 / t / 1e12, "blas_threads": threads,
           "omp_num_threads": os.environ.get("OMP_NUM_THREADS")}
    print(json.dumps(out))


if __name__ == "__main__":
    main()

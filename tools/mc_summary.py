"""Summarise Monte-Carlo theta-recovery runs (tools/montecarlo.py outputs) as a markdown table:
per setting (beta, nu), replicas, mean / std of the MP estimates, bias against theta_true, and the
MP-vs-FP64 agreement on the replicas that also ran the FP64 map (Fig. 5 is an image; the
north star's criterion is |theta_MP - theta_FP64| <= 1e-3 per component).

  python tools/mc_summary.py profiles/r02/montecarlo_*.json > profiles/r02/montecarlo_summary.md"""
import json
import sys

import numpy as np


def main():
    print("| beta | nu | maxfev | replicas (FP64 too) | converged (MP / FP64) | mean theta_MP (sigma^2, beta, nu) | std | "
          "bias vs theta_true | max abs(theta_MP - theta_FP64) | s / replica |")
    print("|---|---|---|---|---|---|---|---|---|---|")
    for path in sys.argv[1:]:
        d = json.load(open(path))
        reps = d.get("reps") or d.get("partial") or []
        if not reps:
            continue
        th = np.array(d.get("theta_true") or [1.0, float("nan"), float("nan")])
        amp = np.array([q["mp"] for q in reps])
        d64 = [q["max_abs_dtheta"] for q in reps if "max_abs_dtheta" in q]
        sec = np.mean([q.get("seconds", float("nan")) for q in reps])
        fmt = lambda v: "(" + ", ".join(f"{x:.4f}" for x in v) + ")"  # noqa: E731
        beta, nu = (th[1], th[2]) if len(th) == 3 else ("?", "?")
        mf = d.get("maxfev", "?")
        cm = sum(1 for q in reps if q.get("nfev_mp", 0) < (mf if isinstance(mf, int) else 10**9))
        c64 = sum(1 for q in reps if "nfev_fp64" in q and q["nfev_fp64"] < (mf if isinstance(mf, int) else 10**9))
        print(f"| {beta} | {nu} | {mf} | {len(reps)} ({len(d64)}) | {cm} / {c64} | {fmt(amp.mean(0))} | {fmt(amp.std(0))} | "
              f"{fmt(amp.mean(0) - th)} | {max(d64) if d64 else float('nan'):.2e} | {sec:.0f} |")


if __name__ == "__main__":
    main()

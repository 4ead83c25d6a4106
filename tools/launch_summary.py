"""Per-kernel share of one evaluation from an `ncu --metrics gpu__time_duration.sum --csv` launch list
(serialised, cold-cache per-launch times: shares, not absolutes).  The evaluation is the last one in
the list: launches from the last matern_norm_kernel (generation pass 1) to the end.
Usage: python tools/launch_summary.py launches.csv [title]"""
import csv
import re
import sys
from collections import defaultdict


def main():
    rows = []
    with open(sys.argv[1]) as f:
        lines = [ln for ln in f if ln.startswith('"')]
    for r in csv.reader(lines):
        if len(r) > 14 and r[12] == "gpu__time_duration.sum" and r[14].replace(".", "").isdigit():
            rows.append((r[4], float(r[14]) * (1e-3 if r[13] == "ns" else 1.0 if r[13] == "us" else 1e3)))
    starts = [i for i, (k, _) in enumerate(rows) if k.startswith("matern_norm_kernel")]
    ev = rows[starts[-1]:] if starts else rows
    agg = defaultdict(lambda: [0, 0.0])
    for k, us in ev:
        name = re.sub(r"\(.*", "", k).replace("void ", "")
        agg[name][0] += 1
        agg[name][1] += us
    tot = sum(v[1] for v in agg.values())
    title = sys.argv[2] if len(sys.argv) > 2 else sys.argv[1]
    print(f"# ncu launch list: {title}\n")
    print(f"One evaluation = {len(ev)} launches, serialised total {tot / 1e3:.1f} ms (cold-cache, one at a time).\n")
    print("| kernel | launches | ms | share | us / launch |\n|---|---|---|---|---|")
    for k, (n, us) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
        print(f"| {k} | {n} | {us / 1e3:.1f} | {100 * us / tot:.1f}% | {us / n:.1f} |")


if __name__ == "__main__":
    main()

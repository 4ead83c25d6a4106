"""Top SASS instructions by warp-stall samples with their two dominant stall reasons
(input: `ncu -i X --page source --csv --print-source sass > file.csv`)."""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
n = int(sys.argv[2]) if len(sys.argv) > 2 else 30
h, data = rows[1], rows[2:]
ci = h.index("Warp Stall Sampling (All Samples)")


def f(x):
    try:
        return float(x)
    except ValueError:
        return 0.0


tot = sum(f(r[ci]) for r in data) or 1
stalls = [k for k in h if k.startswith("stall_") and "Not Issued" not in k]
top = sorted(range(len(data)), key=lambda i: -f(data[i][ci]))[:n]
for i in sorted(top):
    r = data[i]
    br = sorted(((k[6:], f(r[h.index(k)])) for k in stalls), key=lambda kv: -kv[1])[:2]
    print(f"{i:5d} {100 * f(r[ci]) / tot:5.1f}% {r[1].strip()[:64]:64s} {br}")

"""Summarise an MPGEO_TIMELINE dump (one block per mp_get_profile call): per-class busy time per
stream, the main stream's idle gaps (waiting for the panel stream) and the panel stream's share of the
critical path.  Usage: python tools/timeline.py <file> [block index, default last]."""
import sys
from collections import defaultdict

CLS = ["upd64", "upd32", "upd16", "potrf", "trsm", "conv", "gen", "solve"]


def blocks(path):
    cur = []
    for line in open(path):
        if line.startswith("--"):
            if cur:
                yield cur
            cur = []
        else:
            c, s, a, b, fl = line.split()
            cur.append((int(c), int(s), float(a), float(b), float(fl)))
    if cur:
        yield cur


def main():
    bl = list(blocks(sys.argv[1]))
    recs = bl[int(sys.argv[2]) if len(sys.argv) > 2 else -1]
    end = max(r[3] for r in recs)
    busy = defaultdict(float)
    for c, s, a, b, fl in recs:
        busy[(s, CLS[c])] += b - a
    print(f"span {end:.1f} ms, {len(recs)} launches")
    for (s, c), t in sorted(busy.items()):
        print(f"  stream {s} {c:6s} {t:9.1f} ms")
    for st in (0, 1):
        ev = sorted((a, b) for c, s, a, b, fl in recs if s == st)
        cov, last, gaps = 0.0, 0.0, []
        for a, b in ev:
            if a > last:
                gaps.append((last, a))
            cov += max(0.0, b - max(a, last))
            last = max(last, b)
        idle = sum(b - a for a, b in gaps)
        print(f"stream {st}: covered {cov:.1f} ms, idle {idle:.1f} ms in {len(gaps)} gaps; largest gaps:",
              ", ".join(f"{b - a:.2f}@{a:.0f}" for a, b in sorted(gaps, key=lambda g: g[0] - g[1])[:6]))


if __name__ == "__main__":
    main()

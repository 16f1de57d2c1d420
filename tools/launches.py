"""Summarise an ncu --metrics gpu__time_duration.sum launch-list CSV (per kernel: count, total, avg)."""
import csv
import sys
from collections import defaultdict


def summarise(path, skip_init=False):
    rows = list(csv.reader(open(path)))
    hi = [i for i, r in enumerate(rows) if r and r[0] == "ID"][0]
    h = rows[hi]
    ki, vi, ui = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Unit")
    agg = defaultdict(lambda: [0, 0.0])
    for r in rows[hi + 1:]:
        if len(r) <= vi:
            continue
        name = r[ki].split("(")[0].replace("cualign::<unnamed>::", "").replace("void ", "")[:70]
        try:
            v = float(r[vi].replace(",", ""))
        except ValueError:
            continue
        scale = {"nsecond": 1e-3, "usecond": 1.0, "msecond": 1e3}.get(r[ui], 1e-3)
        agg[name][0] += 1
        agg[name][1] += v * scale
    out = []
    for k, (n, t) in sorted(agg.items(), key=lambda x: -x[1][1]):
        out.append(f"{n:6d} {t:12.1f} us total {t / n:10.1f} us avg  {k}")
    return "\n".join(out)


if __name__ == "__main__":
    print(summarise(sys.argv[1]))

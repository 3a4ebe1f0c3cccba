"""Aggregate an ncu --metrics gpu__time_duration.sum --csv launch list by kernel name."""
import collections
import csv
import sys


def load(path):
    rows = list(csv.reader(open(path)))
    hi = [i for i, r in enumerate(rows) if "Kernel Name" in r][0]
    h = rows[hi]
    ki, vi, ui = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Unit")
    agg = collections.defaultdict(lambda: [0, 0.0])
    for r in rows[hi + 1:]:
        if len(r) <= vi:
            continue
        v = float(r[vi].replace(",", ""))
        v *= {"ns": 1e-3, "nsecond": 1e-3, "us": 1.0, "usecond": 1.0, "ms": 1e3, "msecond": 1e3,
              "s": 1e6, "second": 1e6}.get(r[ui], 1.0)   # -> microseconds
        name = r[ki].split("(")[0].replace("void ", "")[:58]
        agg[name][0] += 1
        agg[name][1] += v
    return agg


if __name__ == "__main__":
    agg = load(sys.argv[1])
    tot = sum(a[1] for a in agg.values())
    print(f"{'kernel':58s} {'n':>6s} {'total ms':>10s} {'us/launch':>10s} {'share':>6s}")
    for k, (n, t) in sorted(agg.items(), key=lambda x: -x[1][1])[:int(sys.argv[2]) if len(sys.argv) > 2 else 30]:
        print(f"{k:58s} {n:6d} {t / 1e3:10.3f} {t / n:10.2f} {100 * t / tot:5.1f}%")
    print(f"total {tot / 1e3:.3f} ms over {sum(a[0] for a in agg.values())} launches")

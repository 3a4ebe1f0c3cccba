"""Pivot an ncu --csv launch list with several --metrics: per kernel name the
launch count, total / per-launch duration, DRAM read + write bytes per launch
and L2 bytes per launch.  Usage: launch_metrics.py list.csv [top]"""
import collections
import csv
import sys

SCALE = {"ns": 1e-3, "nsecond": 1e-3, "us": 1.0, "usecond": 1.0, "ms": 1e3, "msecond": 1e3, "s": 1e6,
         "second": 1e6, "byte": 1.0, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "KB": 1e3, "MB": 1e6, "GB": 1e9}


def load(path):
    rows = list(csv.reader(open(path)))
    hi = [i for i, r in enumerate(rows) if "Kernel Name" in r][0]
    h = rows[hi]
    ii, ki, mi, vi, ui = (h.index("ID"), h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Value"),
                          h.index("Metric Unit"))
    launches = collections.defaultdict(dict)
    names = {}
    for r in rows[hi + 1:]:
        if len(r) <= vi:
            continue
        v = float(r[vi].replace(",", "")) * SCALE.get(r[ui], 1.0)
        launches[r[ii]][r[mi]] = v
        names[r[ii]] = r[ki].split("(")[0].replace("void ", "")[:56]
    agg = collections.defaultdict(lambda: collections.defaultdict(float))
    for i, m in launches.items():
        a = agg[names[i]]
        a["n"] += 1
        for k, v in m.items():
            a[k] += v
    return agg


if __name__ == "__main__":
    agg = load(sys.argv[1])
    top = int(sys.argv[2]) if len(sys.argv) > 2 else 30
    tot = sum(a["gpu__time_duration.sum"] for a in agg.values())
    print(f"{'kernel':56s} {'n':>5s} {'total ms':>9s} {'us/launch':>10s} {'share':>6s} {'DRAM MB/l':>10s} "
          f"{'GB/s':>7s} {'L2 MB/l':>9s}")
    for k, a in sorted(agg.items(), key=lambda x: -x[1]["gpu__time_duration.sum"])[:top]:
        n, t = a["n"], a["gpu__time_duration.sum"]
        dram = a.get("dram__bytes_read.sum", 0.0) + a.get("dram__bytes_write.sum", 0.0)
        l2 = a.get("lts__t_bytes.sum", 0.0)
        print(f"{k:56s} {int(n):5d} {t / 1e3:9.3f} {t / n:10.2f} {100 * t / tot:5.1f}% {dram / n / 1e6:10.2f} "
              f"{dram / t / 1e3 if t else 0:7.0f} {l2 / n / 1e6:9.2f}")

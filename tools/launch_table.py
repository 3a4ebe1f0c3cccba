"""Per-kernel totals from an ncu --csv launch list (gpu__time_duration.sum)."""
import collections
import csv
import sys

rows = [r for r in csv.reader(open(sys.argv[1])) if len(r) > 14 and r[12] == "gpu__time_duration.sum"]
tot = collections.defaultdict(lambda: [0, 0.0])
for r in rows:
    name = r[4].split("(")[0].replace("void ", "")
    tot[name][0] += 1
    tot[name][1] += float(r[14].replace(",", "")) / 1e3
allus = sum(v[1] for v in tot.values())
print(f"{'kernel':60s} {'n':>6s} {'total us':>10s} {'us/launch':>10s} {'share':>6s}")
for k, (n, us) in sorted(tot.items(), key=lambda kv: -kv[1][1]):
    print(f"{k[:60]:60s} {n:6d} {us:10.1f} {us / n:10.2f} {100 * us / allus:5.1f}%")
print(f"total {allus:.1f} us over {sum(v[0] for v in tot.values())} launches")

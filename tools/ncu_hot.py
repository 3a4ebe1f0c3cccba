"""Summarise an ncu report: warp-stall samples per CUDA source line (needs -lineinfo)."""
import csv
import subprocess
import sys

rep = sys.argv[1]
n = int(sys.argv[2]) if len(sys.argv) > 2 else 30
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass,cuda"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(out.splitlines()))
fname, lst, tot = "?", [], 0
for r in rows:
    if len(r) == 2 and r[0] == "File Path":
        fname = r[1].split("/")[-1]
        continue
    if not r or r[0] in ("Line No", "Function Name") or r[0] == "":
        continue
    try:
        w = int(r[4])
    except (ValueError, IndexError):
        continue
    tot += w
    lst.append((w, f"{fname}:{r[0]}", r[1].strip()[:100]))
print("total samples", tot)
for w, loc, src in sorted(lst, reverse=True)[:n]:
    print(f"{w:8d} {100 * w / max(tot, 1):5.1f}%  {loc:18s} {src}")

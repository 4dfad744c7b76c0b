"""Top SASS instructions by warp-stall samples with context: python tools/ncu_sass_top.py rep [n] [ctx]"""
import csv
import subprocess
import sys

rep = sys.argv[1]
n = int(sys.argv[2]) if len(sys.argv) > 2 else 12
ctx = int(sys.argv[3]) if len(sys.argv) > 3 else 3
src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(src.splitlines()))
hi = next(i for i, r in enumerate(rows) if r and r[0] == "Address")
h = rows[hi]
iS = h.index("Warp Stall Sampling (All Samples)")
data = [r for r in rows[hi + 1:] if len(r) == len(h)]
tot = sum(float(r[iS] or 0) for r in data)
print(f"total samples {tot:.0f}")
for i in sorted(range(len(data)), key=lambda i: -float(data[i][iS] or 0))[:n]:
    print("----", data[i][iS])
    for j in range(max(0, i - ctx), min(len(data), i + 2)):
        print(f"{data[j][iS]:>6} {data[j][1][:100]}")

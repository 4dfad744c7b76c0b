"""Per-CUDA-source-line stall breakdown of an ncu report: python tools/ncu_lines.py rep [n]
(aggregates the SASS-level samples of `--print-source sass,cuda` by CUDA line)."""
import collections
import csv
import subprocess
import sys

rep = sys.argv[1]
n = int(sys.argv[2]) if len(sys.argv) > 2 else 25
src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass,cuda"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(src.splitlines()))
hi = next(i for i, r in enumerate(rows) if r and r[0] == "Line No")
h = rows[hi]
iS = h.index("Warp Stall Sampling (All Samples)")
cols = [i for i, c in enumerate(h) if c.startswith("stall_") and "Not Issued" not in c]
agg = collections.defaultdict(lambda: collections.Counter())
text = {}
for r in rows[hi + 1:]:
    if len(r) != len(h) or not r[0].strip() or r[2] != "-" or not r[iS].replace(".", "").isdigit():
        continue  # keep the per-CUDA-line aggregate rows only
    ln = r[0]
    text.setdefault(ln, r[1])
    agg[ln]["all"] += float(r[iS] or 0)
    for i in cols:
        agg[ln][h[i][6:]] += float(r[i] or 0)
tot = sum(a["all"] for a in agg.values())
print(f"total samples {tot:.0f}")
for ln, a in sorted(agg.items(), key=lambda kv: -kv[1]["all"])[:n]:
    top = sorted(((v, k) for k, v in a.items() if k != "all"), reverse=True)[:3]
    print(f"{a['all']:6.0f} L{ln:>4} {text[ln].strip()[:68]:68s} " + " ".join(f"{k}={v:.0f}" for v, k in top if v > 0))

"""Top stall-sampled SASS instructions of an ncu report: python ncu_hot.py rep [N]."""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
N = int(sys.argv[2]) if len(sys.argv) > 2 else 25
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
lines = out.splitlines()
start = [i for i, l in enumerate(lines) if l.startswith('"Address"')][0]
rows = list(csv.reader(io.StringIO("\n".join(lines[start:]))))
h = rows[0]
si, wi, ai = h.index("Source"), h.index("Warp Stall Sampling (All Samples)"), h.index("Address")
ei = h.index("Instructions Executed")
data = []
for idx, r in enumerate(rows[1:]):
    try:
        data.append((int(r[wi]), idx, r[ai][-5:], int(r[ei] or 0), r[si].strip()[:90]))
    except (ValueError, IndexError):
        pass
tot = sum(d[0] for d in data) or 1
print(f"total samples {tot}")
for s, idx, a, ex, src in sorted(data, reverse=True)[:N]:
    print(f"{s:8d} {100 * s / tot:5.1f}%  #{idx:<5} {a} exec={ex:<10} {src}")

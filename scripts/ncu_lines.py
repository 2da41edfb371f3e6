"""Warp-stall samples of an ncu report aggregated by CUDA source line (needs -lineinfo):
python scripts/ncu_lines.py report.ncu-rep [N]"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
N = int(sys.argv[2]) if len(sys.argv) > 2 else 30
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
res, fname, hdr = [], "", None
for r in rows:
    if len(r) == 2 and r[0] == "File Path":
        fname = r[1].split("/")[-1]
        continue
    if r and r[0] == "Line No":
        hdr = r
        continue
    if hdr is None or len(r) < 6 or not r[0]:
        continue
    try:
        res.append((int(r[4]), int(r[7] or 0), fname, int(r[0]), r[1].strip()[:100]))
    except ValueError:
        pass
tot = sum(x[0] for x in res) or 1
print(f"total samples {tot}")
for s, ex, f, ln, src in sorted(res, reverse=True)[:N]:
    print(f"{s:7d} {100 * s / tot:5.1f}%  {f}:{ln:<5} exec={ex:<9} {src}")

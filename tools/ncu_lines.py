"""Executed warp instructions and stall samples per CUDA source line of an ncu report
(mixed cuda,sass source page): python tools/ncu_lines.py REP [N]"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
n = int(sys.argv[2]) if len(sys.argv) > 2 else 40
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
fname, lines, hdr, tot = None, [], None, 0
for r in rows:
    if len(r) == 2 and r[0] == "File Path":
        fname = r[1].split("/")[-1]
        continue
    if r and r[0] == "Line No":
        hdr = {h: i for i, h in enumerate(r) if h not in ("Source",)}
        continue
    if hdr is None or not r or not r[0] or r[0] == "":
        continue
    try:
        ie = int(r[hdr["Instructions Executed"]])
        st = int(r[hdr["Warp Stall Sampling (All Samples)"]])
    except (ValueError, KeyError, IndexError):
        continue
    tot += ie
    lines.append((ie, st, fname, r[0], r[1].strip()[:110]))
lines.sort(reverse=True)
print(f"total warp instructions {tot:.4e}")
for ie, st, f, ln, src in lines[:n]:
    print(f"{ie / tot * 100:5.1f}% {ie:.3e} st={st:7d} {f}:{ln}  {src}")

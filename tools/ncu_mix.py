"""Instruction mix of an ncu report's SASS (executions per opcode) and the lines with the
most excessive shared-memory wavefronts / stall samples: python tools/ncu_mix.py REP [N]"""
import collections
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
n = int(sys.argv[2]) if len(sys.argv) > 2 else 25
src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(src)))
hi = next(i for i, r in enumerate(rows) if "Address" in r and "Source" in r)
hdr, data = rows[hi], rows[hi + 1:]
col = {h: i for i, h in enumerate(hdr)}
print("columns:", [h for h in hdr if "Wavefront" in h or "Excess" in h or "Stall" in h][:12])
ie, isrc = col["Instructions Executed"], col["Source"]


def num(r, c):
    try:
        return float(r[c] or 0)
    except (ValueError, IndexError):
        return 0.0


mix = collections.Counter()
tot = 0.0
for r in data:
    op = r[isrc].split()
    if not op:
        continue
    k = op[1] if op[0].startswith("@") and len(op) > 1 else op[0]
    k = k.split(".")[0]
    mix[k] += num(r, ie)
    tot += num(r, ie)
print(f"total warp-instructions executed: {tot:.4e}")
for k, v in mix.most_common(30):
    print(f"  {k:12s} {v:.4e}  {v / tot * 100:5.1f}%")
for key in [h for h in hdr if "Shared Excessive" in h or "Excessive" in h]:
    c = col[key]
    s = sum(num(r, c) for r in data)
    print(f"== {key}: total {s:.4e}")
    for r in sorted(data, key=lambda r: -num(r, c))[:n]:
        if num(r, c) <= 0:
            break
        print(f"  {num(r, c):.3e} {r[col['Address']][-5:]} exec={r[ie]:>10} {r[isrc][:90]}")

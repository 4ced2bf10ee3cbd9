"""One-line summary of bench JSON lines: python tools/bline.py FILE..."""
import json
import sys

for fn in sys.argv[1:]:
    for line in open(fn):
        line = line.strip()
        if not line.startswith("{"):
            continue
        d = json.loads(line)
        if "roofline" not in d:
            continue
        r, f = d["roofline"], d.get("finder_roofline") or {}
        e = d.get("e2e") or {}
        print(f"{fn.split('/')[-1]:28s} {d['config']['workload']:4s} {d['ms_per_step']:9.3f} ms {d['value']:9.2f} Gb/s "
              f"cmp/s={d.get('comparisons_per_s', 0):.3e} {r['kernel']:20s} frac={r['frac']:.3f} share={r.get('share_of_step', 0):.2f} "
              f"find={f.get('frac', 0):.2f}/{f.get('ms_per_step', 0):.3f}ms e2e={e.get('value')}")

"""Print the key numbers of bench.py JSON lines (stdin or files)."""
import json
import sys

files = sys.argv[1:] or ["-"]
for f in files:
    text = sys.stdin.read() if f == "-" else open(f).read()
    for line in text.splitlines():
        line = line.strip()
        if not line.startswith("{"):
            continue
        d = json.loads(line)
        r = d.get("roofline") or {}
        fr = d.get("finder_roofline") or {}
        e2e = d.get("e2e") or {}
        print(f"{d['config'].get('workload')} {d['config'].get('comparer')}: {d['ms_per_step']:.2f} ms/step "
              f"{d['value']:.1f} Gbases/s cmp/s={d.get('comparisons_per_s', 0):.3e} "
              f"roof={r.get('kernel')} frac={r.get('frac') or 0:.3f} share={r.get('share_of_step') or 0:.3f} "
              f"finder={fr.get('ms_per_step', 0):.2f}ms frac={fr.get('frac') or 0:.3f} e2e={e2e.get('value')} "
              f"clk={d.get('clocks', {}).get('sm_mhz')}")

"""Summarise the last `search_host_trace` line (COF_TRACE=1) of a log: per-chunk H2D and
device intervals, copy-engine and device busy time, and how much of the H2D overlapped the
kernels.  Experiment tool for the e2e pipeline, not part of the product path."""
import json
import sys


def main(path):
    last = None
    for line in open(path):
        if line.startswith('{"search_host_trace"'):
            last = json.loads(line)["search_host_trace"]
    if last is None:
        print("no trace")
        return
    iv = {}
    for what, j, t in last:
        iv.setdefault(j, {})[what] = t
    rows, h2d, dev = [], [], []
    for j in sorted(iv):
        d = iv[j]
        h = (d["h2d0"], d["h2d1"])
        v = (d["dev0"], d["dev1"])
        h2d.append(h)
        dev.append(v)
        rows.append(f"chunk {j:2d}  h2d {h[0]:8.3f}-{h[1]:8.3f} ({h[1] - h[0]:6.3f})  "
                    f"dev {v[0]:8.3f}-{v[1]:8.3f} ({v[1] - v[0]:6.3f})")
    span = max(b for _, b in h2d + dev) - min(a for a, _ in h2d + dev)
    busy_h = sum(b - a for a, b in h2d)
    busy_d = sum(b - a for a, b in dev)
    ov = sum(max(0.0, min(hb, db) - max(ha, da)) for ha, hb in h2d for da, db in dev)
    print("\n".join(rows))
    print(json.dumps({"span_ms": round(span, 3), "h2d_busy_ms": round(busy_h, 3), "dev_busy_ms": round(busy_d, 3),
                      "h2d_dev_overlap_ms": round(ov, 3), "chunks": len(iv)}))


if __name__ == "__main__":
    main(sys.argv[1])

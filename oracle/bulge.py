"""Bulge search oracle -- TEST INFRASTRUCTURE ONLY (same import rule as oracle.py).

The paper only states the capability: Cas-OFFinder "can also predict off-target sites
with deletions or insertions"; the procedure is not
described.  DESIGN.md §2 readings B1-B6 fix it as follows (a site aligned to a guide with
one gap of b bases):

* DNA bulge of size b at guide offset i: the genome carries b extra bases between guide
  offsets i-1 and i.  Those bases are not compared and the pattern is read around them.
  Allowed for s < i < e, where [s, e) is the guide's compared span (first to last non-N
  letter), and only where the pattern is N at offsets i-1 and i (B1, B2).
* RNA bulge of size b at guide offset i: guide letters [i, i+b) have no DNA partner.  The
  site is L-b bases; the pattern letters [i, i+b) must be N and are dropped.  Allowed for
  s < i and i+b < e (B1, B2).
* The mismatch count over the remaining compared letters must be <= the guide's
  threshold; the bulge itself is not a mismatch (B3).  Every (guide, type, size, offset)
  that aligns a site is reported; there is no deduplication across variants (B4).

Two independent forms:
  ``expand``/``search``   -- rewrite every bulge variant as an ordinary (pattern, guide)
                             pair and run the brute-force oracle (cof_oracle.c) on it;
  ``brute_force``         -- pure Python: for every window and strand, remove / insert the
                             gap explicitly and count mismatches letter by letter.
Tests pin one against the other on small genomes and on hand-built sites.
"""
from __future__ import annotations

import numpy as np

from . import oracle

BULGE_DTYPE = np.dtype([("guide", "<i4"), ("kind", "S1"), ("size", "i1"), ("bpos", "i1"),
                        ("chrom", "<i4"), ("pos", "<i8"), ("strand", "S1"), ("mm", "i1"),
                        ("site", "S40")], align=True)

_SETS = {"A": "A", "C": "C", "G": "G", "T": "T", "R": "AG", "Y": "CT", "S": "CG", "W": "AT",
         "K": "GT", "M": "AC", "B": "CGT", "D": "AGT", "H": "ACT", "V": "ACG", "N": "ACGT"}
_COMP = {"A": "T", "C": "G", "G": "C", "T": "A", "N": "N"}


def _span(guide: str):
    comp = [j for j, c in enumerate(guide.upper()) if c != "N"]
    return (comp[0], comp[-1] + 1) if comp else (0, 0)


def expand(pattern: str, guides, thresholds, dna: int, rna: int):
    """{variant pattern: [(guide, kind, size, bpos, variant guide, threshold), ...]}"""
    pattern = pattern.upper()
    out = {}

    def add(pv, rec):
        out.setdefault(pv, []).append(rec)

    for gi, (g, t) in enumerate(zip(guides, thresholds)):
        g = g.upper()
        add(pattern, (gi, "X", 0, 0, g, int(t)))
        s, e = _span(g)
        for b in range(1, dna + 1):
            for i in range(s + 1, e):
                if pattern[i - 1] != "N" or pattern[i] != "N":
                    continue
                add(pattern[:i] + "N" * b + pattern[i:], (gi, "D", b, i, g[:i] + "N" * b + g[i:], int(t)))
        for b in range(1, rna + 1):
            for i in range(s + 1, e - b):
                if pattern[i:i + b] != "N" * b:
                    continue
                add(pattern[:i] + pattern[i + b:], (gi, "R", b, i, g[:i] + g[i + b:], int(t)))
    return out


def _sort(arr):
    if len(arr) == 0:
        return arr
    key = np.lexsort((arr["bpos"], arr["size"], arr["kind"], arr["guide"], arr["strand"] == b"-",
                      arr["pos"], arr["chrom"]))
    return arr[key]


def search(seqs, pattern, guides, thresholds, dna: int, rna: int) -> np.ndarray:
    """Bulge hits via the variant rewrite + the brute-force oracle, sorted by
    (chrom, pos, strand, guide, kind, size, bpos)."""
    parts = []
    for pv, recs in expand(pattern, guides, thresholds, dna, rna).items():
        h = oracle.search(seqs, pv, [r[4] for r in recs], [r[5] for r in recs])
        if len(h) == 0:
            continue
        o = np.zeros(len(h), dtype=BULGE_DTYPE)
        src = np.array([r[0] for r in recs])[h["guide"]]
        o["guide"] = src
        o["kind"] = np.array([r[1].encode() for r in recs])[h["guide"]]
        o["size"] = np.array([r[2] for r in recs])[h["guide"]]
        o["bpos"] = np.array([r[3] for r in recs])[h["guide"]]
        for f in ("chrom", "pos", "strand", "mm", "site"):
            o[f] = h[f]
        parts.append(o)
    if not parts:
        return np.zeros(0, dtype=BULGE_DTYPE)
    return _sort(np.concatenate(parts))


def _canon(c):
    c = c.upper()
    return c if c in "ACGT" else "N"


def brute_force(seqs, pattern, guides, thresholds, dna: int, rna: int):
    """Pure-Python definition (tiny inputs only): tuples
    (chrom, pos, strand, guide, kind, size, bpos, mm, site)."""
    pattern = pattern.upper()
    L = len(pattern)
    res = []
    for ci, seq in enumerate(seqs):
        s_txt = seq.decode() if isinstance(seq, (bytes, bytearray)) else str(seq)
        s_txt = "".join(_canon(c) for c in s_txt)
        n = len(s_txt)
        for gi, (g, t) in enumerate(zip(guides, thresholds)):
            g = g.upper()
            s, e = _span(g)
            cands = [("X", 0, 0)]
            cands += [("D", b, i) for b in range(1, dna + 1) for i in range(s + 1, e)
                      if pattern[i - 1] == "N" and pattern[i] == "N"]
            cands += [("R", b, i) for b in range(1, rna + 1) for i in range(s + 1, e - b)
                      if pattern[i:i + b] == "N" * b]
            for kind, b, i in cands:
                W = L + b if kind == "D" else L - b if kind == "R" else L
                for p in range(0, n - W + 1):
                    w = s_txt[p:p + W]
                    for strand in "+-":
                        site = w if strand == "+" else "".join(_COMP[c] for c in reversed(w))
                        # align: guide offset j <-> site offset a(j); bulge bases skipped
                        if kind == "D":
                            idx = list(range(i)) + list(range(i + b, W))       # site offsets of guide 0..L-1
                            gl, pl = g, pattern
                        elif kind == "R":
                            idx = list(range(W))
                            gl, pl = g[:i] + g[i + b:], pattern[:i] + pattern[i + b:]
                        else:
                            idx = list(range(W))
                            gl, pl = g, pattern
                        ok = all(pl[j] == "N" or site[idx[j]] in _SETS[pl[j]] for j in range(len(pl)))
                        if not ok:
                            continue
                        mm = 0
                        low = set()
                        for j in range(len(gl)):
                            if gl[j] == "N":
                                continue
                            if site[idx[j]] not in _SETS[gl[j]]:
                                mm += 1
                                low.add(idx[j])
                        if mm <= t:
                            out_site = "".join(c.lower() if k in low else c for k, c in enumerate(site))
                            res.append((ci, p, strand, gi, kind, b, i, mm, out_site))
    res.sort(key=lambda h: (h[0], h[1], h[2] == "-", h[3], h[4], h[5], h[6]))
    return res


def to_tuples(arr):
    return [(int(h["chrom"]), int(h["pos"]), h["strand"].decode(), int(h["guide"]), h["kind"].decode(),
             int(h["size"]), int(h["bpos"]), int(h["mm"]), h["site"].decode()) for h in arr]

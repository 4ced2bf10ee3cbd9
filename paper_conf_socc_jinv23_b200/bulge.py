"""Bulge search: off-target sites aligned to a guide with one DNA or
RNA bulge, through the unchanged find -> compare -> sort path.

The paper states the capability only ("It can also predict off-target sites with
deletions or insertions"); DESIGN.md §2 readings B1-B6 fix the definition.  A
bulge variant is an ordinary (pattern, guide) pair:

* DNA bulge of size b at guide offset i (extra genome bases between guide offsets i-1 and
  i): b 'N' are inserted at offset i into the pattern and the guide -- the inserted bases
  are matched by the pattern's N and never compared;
* RNA bulge of size b at offset i (guide letters [i, i+b) unpaired): those b letters are
  dropped from the guide and the b 'N' at [i, i+b) from the pattern.

Bulges stay strictly inside the guide's compared span and only where the pattern is N
(B1, B2).  Inserting N into (or dropping N from) the pattern's N run gives the same variant
pattern for every offset i, so a search with bulges up to size D (DNA) and R (RNA) is
1 + D + R ordinary searches, each over all guides x offsets of its kind -- many guides per
launch, which is the comparer's best case.  Hits map back to (guide, kind, size, offset).
"""
from __future__ import annotations

import numpy as np

from . import cof
from . import search as _search

BULGE_DTYPE = np.dtype([("guide", "<u4"), ("kind", "S1"), ("size", "u1"), ("bpos", "u1"),
                        ("chrom", "<u4"), ("pos", "<u8"), ("strand", "S1"), ("mm", "u1"),
                        ("site", "S66")], align=True)


def compared_span(guide: str):
    """[first, last + 1) of the guide's non-N letters ((0, 0) for an all-N guide)."""
    first = last = -1
    for j, ch in enumerate(guide):
        if ch not in "Nn":
            if first < 0:
                first = j
            last = j
    return (first, last + 1) if first >= 0 else (0, 0)


def variants(pattern: str, guides, thresholds, dna: int = 0, rna: int = 0):
    """Variant groups: {variant pattern: (guide strings, thresholds, meta)} with meta rows
    (original guide, kind 'X'|'D'|'R', size, offset)."""
    P = pattern.upper()
    groups: dict = {}

    def put(pv, gv, t, meta):
        gs, ts, ms = groups.setdefault(pv, ([], [], []))
        gs.append(gv)
        ts.append(min(t, len(pv)))   # a threshold >= the variant length admits every PAM site either way
        ms.append(meta)

    for gi, (g0, t) in enumerate(zip(guides, thresholds)):
        g = g0.upper()
        put(P, g, int(t), (gi, b"X", 0, 0))
        lo, hi = compared_span(g)
        for size in range(1, int(dna) + 1):
            for i in range(lo + 1, hi):
                if P[i - 1] == "N" and P[i] == "N":
                    put(P[:i] + "N" * size + P[i:], g[:i] + "N" * size + g[i:], int(t), (gi, b"D", size, i))
        for size in range(1, int(rna) + 1):
            for i in range(lo + 1, hi - size):
                if all(P[k] == "N" for k in range(i, i + size)):
                    put(P[:i] + P[i + size:], g[:i] + g[i + size:], int(t), (gi, b"R", size, i))
    return groups


def search(seqs, pattern, guides, thresholds, dna: int = 0, rna: int = 0, device="cuda", chunk_bases=None,
           pack_bases=None):
    """Bulge search of ``seqs`` on one GPU: one device search per variant pattern, hits
    mapped back and ordered by (chrom, pos, strand, guide, kind, size, offset)."""
    arrs = [np.frombuffer(s, dtype=np.uint8) if isinstance(s, (bytes, bytearray)) else
            (np.frombuffer(s.encode(), dtype=np.uint8) if isinstance(s, str) else s) for s in seqs]
    parts = []
    for pv, (gs, ts, ms) in variants(pattern, guides, thresholds, dna, rna).items():
        if len(pv) > cof.COF_MAX_L:
            raise ValueError(f"bulge variant pattern of length {len(pv)} exceeds {cof.COF_MAX_L}")
        chunks = _search.plan_chunks([len(a) for a in arrs], len(pv), chunk_bases, pack_bases)
        host = _search.HostGenome(arrs, chunks)
        srch = _search.Searcher(pv, gs, ts, device)
        h = srch.search_host(host)
        if len(h) == 0:
            continue
        meta = np.array(ms, dtype=[("guide", "<u4"), ("kind", "S1"), ("size", "u1"), ("bpos", "u1")])
        m = meta[h["guide"]]
        o = np.empty(len(h), dtype=BULGE_DTYPE)
        for f in ("guide", "kind", "size", "bpos"):
            o[f] = m[f]
        for f in ("chrom", "pos", "strand", "mm", "site"):
            o[f] = h[f]
        parts.append(o)
    if not parts:
        return np.zeros(0, dtype=BULGE_DTYPE)
    out = np.concatenate(parts)
    order = np.lexsort((out["bpos"], out["size"], out["kind"], out["guide"], out["strand"] == b"-", out["pos"],
                        out["chrom"]))
    return out[order]


def to_tuples(arr):
    return [(int(h["chrom"]), int(h["pos"]), h["strand"].decode(), int(h["guide"]), h["kind"].decode(),
             int(h["size"]), int(h["bpos"]), int(h["mm"]), h["site"].decode()) for h in arr]

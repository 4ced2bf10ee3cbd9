"""Second, independent oracle in pure Python -- TEST INFRASTRUCTURE ONLY.

Written separately from ``cof_oracle.c`` (different tables, different loops) so that
the two can check each other by brute force on tiny inputs ("Exhaustive
tiny brute force ... compared with a second pure-Python oracle written separately").
Only for small inputs: it is quadratic-ish pure Python.

Definition followed: PAPER.md P:L29 (search, then compare, output fields) and
Listing 1 P:L204-L246 (non-N index list, IUPAC mismatch rows, inclusive threshold,
'+' and '-' handled as two independent comparisons).  Readings G2/G4/G5/G6/G13 as
in DESIGN.md.
"""
from __future__ import annotations

# IUPAC nucleotide nomenclature, spelled as sets of the bases each letter stands for.
IUPAC_SETS = {
    "A": frozenset("A"), "C": frozenset("C"), "G": frozenset("G"), "T": frozenset("T"),
    "R": frozenset("AG"), "Y": frozenset("CT"), "S": frozenset("GC"), "W": frozenset("AT"),
    "K": frozenset("GT"), "M": frozenset("AC"),
    "B": frozenset("CGT"), "D": frozenset("AGT"), "H": frozenset("ACT"), "V": frozenset("ACG"),
    "N": frozenset("ACGT"),
}
_WC = str.maketrans("ACGTN", "TGCAN")


def _canon_text(s: str) -> str:
    s = s.upper()
    return "".join(ch if ch in "ACGT" else "N" for ch in s)


def _revcomp(s: str) -> str:
    return s[::-1].translate(_WC)


def search(chroms, pattern, guides, thresholds):
    """chroms: list of str.  Returns sorted list of (chrom, pos, strand, guide, mm, site)."""
    pattern = pattern.upper()
    guides = [g.upper() for g in guides]
    L = len(pattern)
    out = []
    for ci, raw in enumerate(chroms):
        text = _canon_text(raw)
        for p in range(0, len(text) - L + 1):
            fwd = text[p:p + L]
            for strand, read in (("+", fwd), ("-", _revcomp(fwd))):
                if any(pc != "N" and read[j] not in IUPAC_SETS[pc] for j, pc in enumerate(pattern)):
                    continue
                for gi, g in enumerate(guides):
                    miss = [gc != "N" and read[j] not in IUPAC_SETS[gc] for j, gc in enumerate(g)]
                    mm = sum(miss)
                    if mm <= thresholds[gi]:
                        site = "".join(c.lower() if m else c for c, m in zip(read, miss))
                        out.append((ci, p, strand, gi, mm, site))
    out.sort(key=lambda h: (h[0], h[1], h[2] == "-", h[3]))
    return out

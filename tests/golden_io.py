"""Readers for the hand-written fixtures under tests/golden/ (each cites its source)."""
import os

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


def _rows(name):
    with open(os.path.join(GOLDEN, name)) as f:
        for line in f:
            line = line.rstrip("\n")
            if line and not line.startswith("#"):
                yield line.split("\t")


def listing1_rows():
    """{code: set of genome bases counted as mismatch} (Listing 1)."""
    return {r[0]: set(r[1]) for r in _rows("listing1_mismatch_rows.tsv")}


def iupac_sets():
    """{code: (member set, complement code)}."""
    return {r[0]: (set(r[1]), r[2]) for r in _rows("iupac_sets.tsv")}


def worked_example():
    d = {"chroms": [], "names": [], "guides": [], "thr": [], "hits": []}
    for r in _rows("worked_example.txt"):
        if r[0] == "pattern":
            d["pattern"] = r[1]
        elif r[0] == "chrom":
            d["names"].append(r[1])
            d["chroms"].append(r[2])
        elif r[0] == "guide":
            d["guides"].append(r[1])
            d["thr"].append(int(r[2]))
        elif r[0] == "hit":
            d["hits"].append((int(r[1]), int(r[2]), r[3], int(r[4]), int(r[5]), r[6]))
    return d

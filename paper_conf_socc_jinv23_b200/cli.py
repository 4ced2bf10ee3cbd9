"""Cas-OFFinder-style command line (I/O compatibility).

    python -m paper_conf_socc_jinv23_b200 INPUT [G] OUTPUT [--chunk-bases N] [--device cuda:0] [--gpus N]

INPUT follows the tool's input file ("the desired pattern, query sequences, and maximum
mismatch number", P:L158 via [17]):

    /path/to/genome.fa            (a FASTA or UCSC .2bit file, or a directory of
                                  .fa/.fasta/.fna/.2bit files)
    NNNNNNNNNNNNNNNNNNNNNRG [D R] (pattern; N = any base, PAM letters in IUPAC; optional
                                  maximum DNA / RNA bulge sizes)
    GGCCGACCTGTCGCTGACGCNNN 5     (query and its maximum mismatch count, one per line)
    ...

OUTPUT is tab-separated, one hit per line ("chromosome number, position, direction,
the number of mismatched bases and potential off-target DNA sequence with mismatched
bases"): query, chromosome name, 0-based position, site (mismatches lower-case),
strand, mismatches — in (chromosome, position, strand, query) order (reading G13).
The second positional argument (the original tool's C/G/A device letter) is accepted and
ignored: the search always runs on the GPU.  With bulges (D or R > 0) three columns follow:
bulge type (X = none, DNA, RNA), bulge size and the guide offset of the bulge (bulge.py).
"""
from __future__ import annotations

import argparse
import dataclasses
import os
import sys

import numpy as np


@dataclasses.dataclass
class InputSpec:
    genome: str
    pattern: str
    queries: list
    thresholds: list
    dna_bulge: int = 0
    rna_bulge: int = 0


def parse_input(text: str, base_dir: str = ".") -> InputSpec:
    lines = [ln.strip() for ln in text.splitlines()]
    lines = [ln for ln in lines if ln and not ln.startswith("#")]
    if len(lines) < 3:
        raise ValueError("input needs a genome path, a pattern and at least one query line")
    genome = lines[0]
    if not os.path.isabs(genome):
        genome = os.path.join(base_dir, genome)
    pl = lines[1].split()
    pattern = pl[0]
    dna_b = int(pl[1]) if len(pl) > 1 else 0
    rna_b = int(pl[2]) if len(pl) > 2 else 0
    if dna_b < 0 or rna_b < 0:
        raise ValueError(f"negative bulge size in {lines[1]!r}")
    queries, thr = [], []
    for ln in lines[2:]:
        parts = ln.split()
        if len(parts) < 2:
            raise ValueError(f"query line needs a sequence and a mismatch count: {ln!r}")
        q, t = parts[0], int(parts[1])
        if len(q) != len(pattern):
            raise ValueError(f"query {q} has length {len(q)}, pattern has {len(pattern)}")
        if t < 0:
            raise ValueError(f"negative mismatch count in {ln!r}")
        queries.append(q)
        thr.append(min(t, len(pattern)))   # t >= L admits every PAM site; the C ABI wants t <= L
    return InputSpec(genome, pattern, queries, thr, dna_b, rna_b)


def genome_files(path: str):
    if os.path.isdir(path):
        ext = (".fa", ".fasta", ".fna", ".fa.txt", ".2bit")
        return sorted(os.path.join(path, f) for f in os.listdir(path) if f.lower().endswith(ext))
    return [path]


def format_hits(hits, queries, names) -> str:
    """TSV lines for a cof.HIT_DTYPE array."""
    out = []
    for h in hits:
        out.append(f"{queries[int(h['guide'])]}\t{names[int(h['chrom'])]}\t{int(h['pos'])}\t"
                   f"{h['site'].decode()}\t{h['strand'].decode()}\t{int(h['mm'])}")
    return "\n".join(out) + ("\n" if out else "")


def format_bulge_hits(hits, queries, names) -> str:
    """TSV lines for a bulge.BULGE_DTYPE array (three bulge columns appended)."""
    kinds = {b"X": "X", b"D": "DNA", b"R": "RNA"}
    out = []
    for h in hits:
        out.append(f"{queries[int(h['guide'])]}\t{names[int(h['chrom'])]}\t{int(h['pos'])}\t"
                   f"{h['site'].decode()}\t{h['strand'].decode()}\t{int(h['mm'])}\t"
                   f"{kinds[h['kind']]}\t{int(h['size'])}\t{int(h['bpos'])}")
    return "\n".join(out) + ("\n" if out else "")


def run_bulge(spec: InputSpec, device: str = "cuda", chunk_bases: int | None = None):
    """Bulge search (bulge.py) of the genome of ``spec``; returns (hits, names)."""
    import torch
    from . import bulge, cof

    names, seqs = [], []
    for f in genome_files(spec.genome):
        fa = cof.open_genome(f)
        for i in range(len(fa)):
            names.append(fa.name(i))
            seqs.append(fa.read(i))
    hits = bulge.search(seqs, spec.pattern, spec.queries, spec.thresholds, spec.dna_bulge, spec.rna_bulge,
                        device=device, chunk_bases=chunk_bases)
    torch.cuda.synchronize()
    return hits, names


def run(spec: InputSpec, device: str = "cuda", chunk_bases: int | None = None, gpus: int = 1):
    """Search the genome of ``spec``; returns (hits, chromosome names).  ``gpus`` > 1: the
    single-process multi-GPU path (search.search_multi: one pipeline per GPU over a shared
    queue of <= 64 Mbp work units, merge by concatenation in genome order)."""
    import torch
    from . import cof, search

    fastas = [cof.open_genome(f) for f in genome_files(spec.genome)]
    names, recs = [], []
    for fi, fa in enumerate(fastas):
        for i in range(len(fa)):
            names.append(fa.name(i))
            recs.append((fi, i, fa.length(i)))
    L = len(spec.pattern)
    if gpus > 1 and chunk_bases is None:
        chunk_bases = search.MULTI_CHUNK_BASES
    chunks = search.plan_chunks([r[2] for r in recs], L, chunk_bases)
    host = search.HostGenome.from_packer(chunks, lambda c, first, n, lo, hi, nm:
                                         fastas[recs[c][0]].pack(recs[c][1], first, n, lo, hi, nm))
    if gpus > 1:
        n_dev = torch.cuda.device_count()
        devices = [f"cuda:{k % n_dev}" for k in range(gpus)]
        hits = search.search_multi(None, spec.pattern, spec.queries, spec.thresholds, devices=devices, host=host)
    else:
        srch = search.Searcher(spec.pattern, spec.queries, spec.thresholds, device=device)
        hits = srch.search_host(host)
    torch.cuda.synchronize()
    return hits, names


def main(argv=None) -> int:
    ap = argparse.ArgumentParser(prog="python -m paper_conf_socc_jinv23_b200", description=__doc__.split("\n")[0])
    ap.add_argument("input")
    ap.add_argument("args", nargs="+", help="[C|G|A] OUTPUT")
    ap.add_argument("--chunk-bases", type=int, default=None)
    ap.add_argument("--device", default="cuda")
    ap.add_argument("--gpus", type=int, default=1,
                    help="GPUs of this node to shard the genome over (one pipeline per GPU, one process)")
    a = ap.parse_args(argv)
    output = a.args[-1]
    with open(a.input) as f:
        spec = parse_input(f.read(), os.path.dirname(os.path.abspath(a.input)))
    if spec.dna_bulge or spec.rna_bulge:
        hits, names = run_bulge(spec, a.device, a.chunk_bases)
        text = format_bulge_hits(hits, spec.queries, names)
    else:
        hits, names = run(spec, a.device, a.chunk_bases, gpus=a.gpus)
        text = format_hits(hits, spec.queries, names)
    if output == "-":
        sys.stdout.write(text)
    else:
        with open(output, "w") as f:
            f.write(text)
    return 0

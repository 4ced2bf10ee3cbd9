"""Seeded synthetic inputs shared by the CUDA path and the oracle.

This module only *constructs inputs*: genome text, guide strings, thresholds and
planted sites.  It holds none of the method's arithmetic -- no IUPAC set
membership, no PAM test, no mismatch counting -- so that it can serve both sides
(DESIGN.md "Input recipe").  The only biology it knows is the Watson-Crick
complement of the four concrete bases, needed to write a planted site onto the
reverse strand.

Workload shapes follow SURVEY.md §8(d) and BASELINE.json `configs`:

* C1  1 Mbp single chromosome, SpCas9 ``N*21 RG``, 1 guide, <=4 mismatches
* C2  chr22-shaped 50.8 Mbp with N-runs (~23% N), ``N*21 GG``, 10 guides, <=5
* C3  hg38-shaped 3.09 Gbp / 24 chromosomes, ``N*21 RG``, 100 guides, <=6
* C4  hg38-shaped, Cas12a ``TTTV N*23`` with 23-nt guides, 100 guides, <=5
* C5  hg38-shaped, ``N*21 RG``, 1000 guides, <=6 (the 1/2/4/8-GPU config)

Composition is i.i.d. A=T=0.295, C=G=0.205 (GC 41%), ~50% soft-masked
lowercase in geometric runs (mean 300 bp), rare non-ACGT IUPAC letters, hg38-like
N-runs.  Every random draw comes from ``numpy.random.PCG64`` seeded per config
and per chromosome, so the same (config, scale) always yields the same bytes.
"""
from __future__ import annotations

import dataclasses
import hashlib
import math
from concurrent.futures import ThreadPoolExecutor

import numpy as np

# UCSC hg38 chrom.sizes, primary chromosomes.
HG38 = [
    ("chr1", 248956422), ("chr2", 242193529), ("chr3", 198295559),
    ("chr4", 190214555), ("chr5", 181538259), ("chr6", 170805979),
    ("chr7", 159345973), ("chr8", 145138636), ("chr9", 138394717),
    ("chr10", 133797422), ("chr11", 135086622), ("chr12", 133275309),
    ("chr13", 114364328), ("chr14", 107043718), ("chr15", 101991189),
    ("chr16", 90338345), ("chr17", 83257441), ("chr18", 80373285),
    ("chr19", 58617616), ("chr20", 64444167), ("chr21", 46709983),
    ("chr22", 50818468), ("chrX", 156040895), ("chrY", 57227415),
]
# Acrocentric p-arm N blocks (bp, unscaled) and the chrY heterochromatin block.
_ACRO = {"chr13": 16_000_000, "chr14": 16_000_000, "chr15": 17_000_000,
         "chr21": 5_000_000, "chr22": 10_500_000}
_CHRY_BLOCK = (26_600_000, 30_000_000)  # (start, length), unscaled

COMPOSITION = (0.295, 0.205, 0.205, 0.295)  # A, C, G, T
_BASES = np.frombuffer(b"ACGT", dtype=np.uint8)
_COMP = {ord("A"): ord("T"), ord("C"): ord("G"), ord("G"): ord("C"), ord("T"): ord("A")}
_RARE = np.frombuffer(b"RYMK", dtype=np.uint8)

# 65536-entry lookup: uniform uint16 -> base with the target composition.
_U16_LUT = np.empty(65536, dtype=np.uint8)
_edges = np.round(np.cumsum(COMPOSITION) * 65536).astype(np.int64)
_U16_LUT[: _edges[0]] = ord("A")
_U16_LUT[_edges[0]: _edges[1]] = ord("C")
_U16_LUT[_edges[1]: _edges[2]] = ord("G")
_U16_LUT[_edges[2]:] = ord("T")


@dataclasses.dataclass(frozen=True)
class GenomeSpec:
    """Shape of a synthetic genome."""
    chroms: tuple            # ((name, length), ...)
    n_layout: str            # "none" | "chr22" | "hg38"
    softmask: bool = True
    rare_per_bp: float = 1e-8   # ~1 rare IUPAC letter per 100 Mbp


@dataclasses.dataclass(frozen=True)
class Config:
    """One workload of BASELINE.json `configs`."""
    name: str
    genome: GenomeSpec
    genome_seed: int
    seed: int                # guides / thresholds / planting
    pattern: str
    n_guides: int
    core_len: int            # compared guide letters
    guide_prefix: str        # N placeholders before the core (Cas12a: "NNNN")
    guide_suffix: str        # N placeholders after the core (SpCas9: "NNN")
    pam_instances: tuple     # concrete PAM strings used when planting
    threshold: int
    description: str

    @property
    def L(self) -> int:
        return len(self.pattern)


def _scaled(chroms, scale):
    if scale == 1.0:
        return tuple(chroms)
    return tuple((n, max(2000, int(round(l * scale)))) for n, l in chroms)


def config(name: str, scale: float = 1.0) -> Config:
    """Return config C1..C5; ``scale`` < 1 shrinks chromosome lengths (tests)."""
    nrg = "N" * 21 + "RG"
    ngg = "N" * 21 + "GG"
    tttv = "TTTV" + "N" * 23
    hg38 = GenomeSpec(_scaled(HG38, scale), "hg38",
                      rare_per_bp=1e-8 if scale == 1.0 else 2e-6)
    if name == "C1":
        g = GenomeSpec(_scaled([("chrS", 1_000_000)], scale), "none", rare_per_bp=0.0)
        return Config("C1", g, 101, 101, nrg, 1, 20, "", "NNN",
                      ("AGG", "CAG", "GGG", "TAG"), 4,
                      "synthetic 1 Mbp single-chromosome genome, SpCas9 NNNNNNNNNNNNNNNNNNNNNRG, 1 guide, <=4 mismatches")
    if name == "C2":
        g = GenomeSpec(_scaled([("chr22", 50_818_468)], scale), "chr22",
                       rare_per_bp=1e-8 if scale == 1.0 else 2e-6)
        return Config("C2", g, 202, 202, ngg, 10, 20, "", "NNN",
                      ("AGG", "CGG", "GGG", "TGG"), 5,
                      "synthetic chr22-sized genome (51 Mbp, with N-runs) SpCas9 NGG, 10 guides, <=5 mismatches")
    if name == "C3":
        return Config("C3", hg38, 303, 303, nrg, 100, 20, "", "NNN",
                      ("AGG", "CAG", "GGG", "TAG"), 6,
                      "synthetic hg38-shaped genome (3.1 Gbp, 24 chromosomes) SpCas9 NRG, 100 guides, <=6 mismatches on 1 B200")
    if name == "C4":
        return Config("C4", hg38, 303, 404, tttv, 100, 23, "NNNN", "",
                      ("TTTA", "TTTC", "TTTG"), 5,
                      "synthetic hg38-shaped genome, Cas12a 5' TTTV PAM with 23-nt guides, 100 guides, <=5 mismatches")
    if name == "C5":
        return Config("C5", hg38, 303, 505, nrg, 1000, 20, "", "NNN",
                      ("AGG", "CAG", "GGG", "TAG"), 6,
                      "synthetic hg38-shaped genome, 1000 guides, <=6 mismatches, chromosome-sharded across 1/2/4/8 B200")
    # Long-window parity cases (not BASELINE configs): patterns with
    # 32 < L <= 64 on a chr22-shaped genome.
    if name == "X1":   # 37-nt spacers + NGG: compared span 37 > 32 (two-word comparer windows)
        g = GenomeSpec(_scaled([("chr22", 50_818_468)], scale), "chr22",
                       rare_per_bp=1e-8 if scale == 1.0 else 2e-6)
        return Config("X1", g, 202, 606, "N" * 38 + "GG", 20, 37, "", "NNN",
                      ("AGG", "CGG", "GGG", "TGG"), 8,
                      "synthetic chr22-sized genome, 37-nt guides + NGG (L = 40), 20 guides, <=8 mismatches")
    if name == "X2":   # CjCas9-like 8-letter PAM after 30-nt spacers: L = 38, PAM offsets >= 32
        g = GenomeSpec(_scaled([("chr22", 50_818_468)], scale), "chr22",
                       rare_per_bp=1e-8 if scale == 1.0 else 2e-6)
        return Config("X2", g, 202, 707, "N" * 34 + "RYAC", 20, 30, "", "NNNNNNNN",
                      ("AGCTGCAC", "TTAAATAC", "CCGGACAC", "GATCGTAC"), 6,
                      "synthetic chr22-sized genome, 30-nt guides + NNNNRYAC (L = 38), 20 guides, <=6 mismatches")
    raise KeyError(name)


CONFIG_NAMES = ("C1", "C2", "C3", "C4", "C5")
EXTRA_CONFIG_NAMES = ("X1", "X2")


# --------------------------------------------------------------------------- genome
def _n_runs(name, length, layout, rng, scale):
    """List of (start, length) N-runs for one chromosome."""
    runs = []
    if layout == "none":
        return runs
    tel = max(1, int(10_000 * scale))
    if layout == "chr22":
        lead = int(length * 0.2066)           # ~10.5 Mbp of 50.8
        runs.append((0, lead))
        runs.append((length - tel, tel))
        for frac in (0.45, 0.72):             # two interior gaps of ~0.6 Mbp
            gl = int(length * 0.0118)
            runs.append((int(length * frac), gl))
        return runs
    # hg38 layout
    runs.append((0, tel))
    runs.append((length - tel, tel))
    if name in _ACRO:
        runs.append((tel, int(_ACRO[name] * scale)))
    if name == "chrY":
        s, l = _CHRY_BLOCK
        runs.append((int(s * scale), int(l * scale)))
    n_gaps = rng.poisson(length / 40e6) if scale == 1.0 else rng.poisson(max(length / 40e6, 0.5))
    for _ in range(n_gaps):
        gl = int(math.exp(rng.uniform(math.log(50_000), math.log(3_000_000))) * scale)
        gl = max(gl, 1)
        st = int(rng.integers(0, max(1, length - gl)))
        runs.append((st, gl))
    return runs


def _make_chrom(name, length, spec, seed_seq, scale):
    rng = np.random.Generator(np.random.PCG64(seed_seq))
    seq = np.empty(length, dtype=np.uint8)
    block = 1 << 24
    for s in range(0, length, block):
        e = min(length, s + block)
        seq[s:e] = _U16_LUT[rng.integers(0, 65536, e - s, dtype=np.uint16)]
    # rare non-ACGT IUPAC letters (assembly ambiguity codes)
    n_rare = rng.poisson(length * spec.rare_per_bp)
    if n_rare:
        pos = rng.integers(0, length, n_rare)
        seq[pos] = _RARE[rng.integers(0, len(_RARE), n_rare)]
    # soft-mask: alternating runs, geometric lengths with mean 300 bp
    if spec.softmask:
        n_runs = int(length / 300 * 1.2) + 16
        lens = rng.geometric(1.0 / 300.0, n_runs).astype(np.int64)
        while lens.sum() < length:
            lens = np.concatenate([lens, rng.geometric(1.0 / 300.0, n_runs)])
        ends = np.cumsum(lens)
        keep = int(np.searchsorted(ends, length)) + 1
        lens = lens[:keep]
        bits = np.where(np.arange(keep) % 2 == int(rng.integers(0, 2)), 0x20, 0).astype(np.uint8)
        seq |= np.repeat(bits, lens)[:length]
    # N-runs (upper- or lower-case N, as assemblies have both)
    for st, ln in _n_runs(name, length, spec.n_layout, rng, scale):
        seq[st:st + ln] = ord("N")
    return seq


def make_genome(cfg: Config, scale: float = 1.0, threads: int = 8):
    """Return ``[(name, uint8 ASCII array), ...]`` for ``cfg``'s genome (unplanted)."""
    spec = cfg.genome
    seqs = np.random.SeedSequence(cfg.genome_seed).spawn(len(spec.chroms))
    with ThreadPoolExecutor(max_workers=threads) as ex:
        futs = [ex.submit(_make_chrom, n, l, spec, s, scale)
                for (n, l), s in zip(spec.chroms, seqs)]
        return [(n, f.result()) for (n, _), f in zip(spec.chroms, futs)]


# --------------------------------------------------------------------------- guides
def _draw_core(rng, n):
    return _U16_LUT[rng.integers(0, 65536, n, dtype=np.uint16)].tobytes().decode()


def make_guides(cfg: Config, genome, rng):
    """Half the guide cores are copied from random genome positions (upper-cased,
    concrete bases only), half are i.i.d.; each core gets the config's N padding."""
    lens = np.array([len(s) for _, s in genome], dtype=np.float64)
    cores = []
    n_from_genome = cfg.n_guides // 2 + (cfg.n_guides % 2)
    tries = 0
    while len(cores) < n_from_genome and tries < 100000:
        tries += 1
        c = int(rng.choice(len(genome), p=lens / lens.sum()))
        seq = genome[c][1]
        if len(seq) <= cfg.core_len:
            continue
        p = int(rng.integers(0, len(seq) - cfg.core_len))
        core = (seq[p:p + cfg.core_len] & 0xDF).tobytes().decode()
        if set(core) <= set("ACGT"):
            cores.append(core)
    while len(cores) < cfg.n_guides:
        cores.append(_draw_core(rng, cfg.core_len))
    order = rng.permutation(len(cores))
    cores = [cores[i] for i in order]
    return [cfg.guide_prefix + c + cfg.guide_suffix for c in cores]


# --------------------------------------------------------------------------- planting
@dataclasses.dataclass(frozen=True)
class Plant:
    chrom: int
    pos: int          # 0-based leftmost base of the window on the '+' strand
    strand: str       # '+' or '-'
    guide: int
    k: int            # substitutions at compared (core) positions


def _revcomp_concrete(b: bytes) -> bytes:
    return bytes(_COMP[x] for x in reversed(b))


def _site_bytes(cfg, guide, rng, k):
    core = guide[len(cfg.guide_prefix): len(cfg.guide_prefix) + cfg.core_len].encode()
    core = bytearray(core)
    for i in rng.choice(cfg.core_len, size=k, replace=False):
        alts = [x for x in b"ACGT" if x != core[i]]
        core[i] = alts[int(rng.integers(0, 3))]
    pam = cfg.pam_instances[int(rng.integers(0, len(cfg.pam_instances)))].encode()
    if cfg.guide_suffix:          # PAM 3' of the protospacer (SpCas9)
        return bytes(core) + pam
    return pam + bytes(core)      # PAM 5' of the protospacer (Cas12a)


class _Occupancy:
    def __init__(self):
        self.iv = {}

    def free(self, c, s, e):
        for (a, b) in self.iv.get(c, ()):
            if s < b and a < e:
                return False
        return True

    def take(self, c, s, e):
        self.iv.setdefault(c, []).append((s, e))


def plant_sites(cfg: Config, genome, guides, rng, boundaries=(), edges=True):
    """Write, for every guide and k = 0..t+1, one '+' and one '-' copy with exactly
    k core substitutions.  Also plants at position 0, at len-L, right next to an
    N-run, in lowercase, and straddling each ``(chrom, offset)`` in ``boundaries``.
    Mutates ``genome`` in place; returns the list of :class:`Plant`."""
    L = cfg.L
    occ = _Occupancy()
    plants = []
    seqs = [s for _, s in genome]
    lens = np.array([len(s) for s in seqs], dtype=np.float64)

    def put(c, p, strand, gi, k, lower=False):
        site = _site_bytes(cfg, guides[gi], rng, k)
        if strand == "-":
            site = _revcomp_concrete(site)
        arr = np.frombuffer(site, dtype=np.uint8).copy()
        if lower:
            arr |= 0x20
        seqs[c][p:p + L] = arr
        occ.take(c, p - L, p + 2 * L)
        plants.append(Plant(c, p, strand, gi, k))

    def random_slot():
        for _ in range(1000):
            c = int(rng.choice(len(seqs), p=lens / lens.sum()))
            if len(seqs[c]) < 3 * L:
                continue
            p = int(rng.integers(L, len(seqs[c]) - 2 * L))
            w = seqs[c][p:p + L] & 0xDF
            if (w == ord("N")).any() or not occ.free(c, p - L, p + 2 * L):
                continue
            return c, p
        return None

    for gi in range(len(guides)):
        for k in range(cfg.threshold + 2):
            for strand in "+-":
                slot = random_slot()
                if slot is not None:
                    put(slot[0], slot[1], strand, gi, k, lower=bool(rng.integers(0, 4) == 0))
    if edges and len(guides):
        c0 = 0
        n0 = len(seqs[c0])
        cand = [(c0, 0, "+"), (c0, n0 - L, "-")]
        # next to an N-run: first run end after position L
        isn = (seqs[c0] & 0xDF) == ord("N")
        if isn.any():
            d = np.flatnonzero(np.diff(isn.astype(np.int8)))
            for x in d[:4]:
                x = int(x)
                if isn[x] and x + 1 + L < n0:      # run ends at x -> plant at x+1
                    cand.append((c0, x + 1, "+"))
                elif not isn[x] and x + 1 - L >= 0:  # run starts at x+1 -> plant ending at x
                    cand.append((c0, x + 1 - L, "-"))
        for c, off in boundaries:
            for p in (off - L // 2, off - 1, off, off - L + 1):
                if 0 <= p <= len(seqs[c]) - L:
                    cand.append((c, p, "+" if p % 2 else "-"))
        for c, p, strand in cand:
            if occ.free(c, p, p + L):
                put(c, p, strand, int(rng.integers(0, len(guides))),
                    int(rng.integers(0, cfg.threshold + 1)))
    return plants


@dataclasses.dataclass
class Workload:
    cfg: Config
    names: list
    seqs: list            # uint8 ASCII arrays
    guides: list          # str, length L
    thresholds: list      # int per guide
    plants: list

    @property
    def total_bases(self) -> int:
        return int(sum(len(s) for s in self.seqs))

    def sha256(self) -> str:
        h = hashlib.sha256()
        for n, s in zip(self.names, self.seqs):
            h.update(n.encode())
            h.update(s.tobytes())
        for g, t in zip(self.guides, self.thresholds):
            h.update(f"{g}:{t};".encode())
        return h.hexdigest()


def make_workload(name: str, scale: float = 1.0, boundaries=(), threads: int = 8,
                  n_guides: int | None = None) -> Workload:
    """Genome + guides + thresholds + planted sites for config ``name``."""
    cfg = config(name, scale)
    if n_guides is not None:
        cfg = dataclasses.replace(cfg, n_guides=n_guides)
    genome = make_genome(cfg, scale, threads)
    rng = np.random.Generator(np.random.PCG64(cfg.seed))
    guides = make_guides(cfg, genome, rng)
    plants = plant_sites(cfg, genome, guides, rng, boundaries=boundaries)
    return Workload(cfg, [n for n, _ in genome], [s for _, s in genome],
                    guides, [cfg.threshold] * len(guides), plants)


def random_genome_text(rng, n, alphabet=b"ACGT", p=None):
    """Small i.i.d. sequence over ``alphabet`` (tests)."""
    a = np.frombuffer(alphabet, dtype=np.uint8)
    return a[rng.choice(len(a), size=n, p=p)].copy()


def write_fasta(path, names, seqs, width: int = 60):
    """FASTA with ``width``-column lines (whole lines laid out with numpy: a 3 Gbp genome
    in seconds)."""
    with open(path, "wb") as f:
        for n, s in zip(names, seqs):
            f.write(b">" + n.encode() + b"\n")
            a = np.frombuffer(s, dtype=np.uint8) if isinstance(s, (bytes, bytearray)) else np.asarray(s, np.uint8)
            full = len(a) // width
            if full:
                lines = np.empty((full, width + 1), dtype=np.uint8)
                lines[:, :width] = a[:full * width].reshape(full, width)
                lines[:, width] = 10
                f.write(lines.tobytes())
            if len(a) % width:
                f.write(a[full * width:].tobytes() + b"\n")

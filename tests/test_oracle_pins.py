"""Pins for the oracle (tests that tie it to the paper and to mathematics, not to itself).

Each test names what fixes the expected value: a golden fixture written by hand from
the paper, a closed form, an invariant, a special case, or a second independent
implementation (pyoracle) run by brute force on tiny inputs.
"""
import itertools
import math

import numpy as np
import pytest

from oracle import oracle, pyoracle
from paper_conf_socc_jinv23_b200 import synth
from tests import golden_io

BASES = "ACGT"


# ----------------------------------------------------------------- truth tables
def test_listing1_rows():
    """Pin: the mismatch rows printed in Listing 1 + reading G1."""
    rows = golden_io.listing1_rows()
    assert len(rows) == 14
    for code, mism in rows.items():
        for b in BASES:
            assert oracle.contains(code, b) == (b not in mism), (code, b)
            assert (b not in pyoracle.IUPAC_SETS[code]) == (b in mism), (code, b)


def test_iupac_standard_table():
    """Pin: the IUPAC nomenclature table (golden), incl. that a genome N/other is in no set."""
    tab = golden_io.iupac_sets()
    assert set(tab) == set("ACGTRYSWKMBDHVN")
    for code, (members, _) in tab.items():
        for b in BASES:
            assert oracle.contains(code, b) == (b in members)
            assert oracle.contains(code.lower(), b.lower()) == (b in members)   # G4
        for other in "NnRYX-":
            assert not oracle.contains(code, other)                               # G2
        assert set(pyoracle.IUPAC_SETS[code]) == members


def test_complement_table():
    """Pin: Watson-Crick complement and the identity x in S <=> comp(x) in comp(S)."""
    tab = golden_io.iupac_sets()
    for b in BASES:
        assert oracle.complement_base(b) == tab[b][1]
        assert oracle.complement_base(oracle.complement_base(b)) == b
    assert oracle.complement_base("N") == "N"
    for code, (members, comp) in tab.items():
        assert tab[comp][1] == code                      # involution on codes
        for b in BASES:
            assert (b in members) == (tab[b][1] in tab[comp][0])


def test_canon():
    for c in "ACGT":
        assert oracle.canon(c) == c and oracle.canon(c.lower()) == c
    for c in "NnRYrykmX.":
        assert oracle.canon(c) == "N"


# ----------------------------------------------------------------- worked example
def test_worked_example_c_oracle():
    """Pin: hand-derived expected hits in tests/golden/worked_example.txt."""
    d = golden_io.worked_example()
    got = oracle.hits_to_tuples(oracle.search(d["chroms"], d["pattern"], d["guides"], d["thr"]))
    assert got == d["hits"]


def test_worked_example_pyoracle():
    d = golden_io.worked_example()
    assert pyoracle.search(d["chroms"], d["pattern"], d["guides"], d["thr"]) == d["hits"]


# ----------------------------------------------------------------- brute force
def test_exhaustive_tiny_two_oracles():
    """Pin: every 4^7 genome of length 7 (each as its own chromosome), pattern NNRG-like,
    C oracle == independent pure-Python oracle, incl. degenerate guide letters."""
    chroms = ["".join(t) for t in itertools.product(BASES, repeat=7)]
    pattern = "NNNRG"
    guides = ["ACGNN", "TTKNN", "NNNNN", "RYSWN", "GGGGG"]
    thr = [1, 0, 0, 2, 3]
    a = oracle.hits_to_tuples(oracle.search(chroms, pattern, guides, thr))
    b = pyoracle.search(chroms, pattern, guides, thr)
    assert len(a) > 1000
    assert a == b


@pytest.mark.parametrize("seed", range(6))
def test_random_two_oracles(seed):
    """Random IUPAC patterns/guides, genomes with N, lowercase and rare IUPAC letters."""
    rng = np.random.default_rng(1000 + seed)
    L = int(rng.integers(3, 12))
    codes = "ACGTRYSWKMBDHVN"
    pat = "".join(rng.choice(list("NNNNNN" + codes), L))
    guides = ["".join(rng.choice(list("ACGTACGTN" + "RYKM"), L)) for _ in range(4)]
    thr = [int(rng.integers(0, L + 1)) for _ in guides]
    chroms = [synth.random_genome_text(rng, int(rng.integers(0, 400)), b"ACGTacgtNnRy",
                                       p=[.2, .15, .15, .2, .06, .06, .06, .06, .03, .01, .01, .01]).tobytes().decode()
              for _ in range(3)]
    a = oracle.hits_to_tuples(oracle.search(chroms, pat, guides, thr))
    b = pyoracle.search(chroms, pat, guides, thr)
    assert a == b


def test_thread_count_invariance():
    rng = np.random.default_rng(7)
    seq = synth.random_genome_text(rng, 300_000)
    g = ["ACGTACGTACGTACGTACGTNNN", "NNNTTTTGGGGCCCCAAAANNN"[:20] + "NNN"]
    a = oracle.search([seq], "N" * 21 + "RG", g, [8, 8], threads=1)
    b = oracle.search([seq], "N" * 21 + "RG", g, [8, 8], threads=8)
    assert oracle.hits_to_tuples(a) == oracle.hits_to_tuples(b)


# ----------------------------------------------------------------- planted sites
def test_planted_sites():
    """Pin by construction: every planted copy with k <= t substitutions is reported
    for its guide at exactly mm == k; every k = t+1 copy is not."""
    w = synth.make_workload("C1", scale=0.2)
    cfg = w.cfg
    hits = oracle.search(w.seqs, cfg.pattern, w.guides, w.thresholds)
    found = {(int(h["chrom"]), int(h["pos"]), h["strand"].decode(), int(h["guide"])): int(h["mm"])
             for h in hits}
    n_checked = 0
    for pl in w.plants:
        key = (pl.chrom, pl.pos, pl.strand, pl.guide)
        if pl.k <= cfg.threshold:
            assert found.get(key) == pl.k, pl
        else:
            assert key not in found, pl
        n_checked += 1
    assert n_checked >= 2 * (cfg.threshold + 2)


def test_planted_sites_cas12a():
    w = synth.make_workload("C4", scale=0.001, n_guides=3)
    cfg = w.cfg
    hits = oracle.search(w.seqs, cfg.pattern, w.guides, w.thresholds)
    found = {(int(h["chrom"]), int(h["pos"]), h["strand"].decode(), int(h["guide"])): int(h["mm"])
             for h in hits}
    for pl in w.plants:
        key = (pl.chrom, pl.pos, pl.strand, pl.guide)
        if pl.k <= cfg.threshold:
            assert found.get(key) == pl.k, pl
        else:
            assert key not in found, pl


# ----------------------------------------------------------------- invariants
def _rc_text(s):
    return s[::-1].translate(str.maketrans("ACGTacgtNn", "TGCAtgcaNn"))


def test_reverse_complement_symmetry():
    """Invariant: searching rc(genome) gives each hit at p' = len-L-p on the other strand
    with the same guide, mm and site string (the site reads 5'->3' along the strand)."""
    rng = np.random.default_rng(11)
    seq = synth.random_genome_text(rng, 50_000, b"ACGTacgtN", p=[.2, .2, .2, .2, .04, .04, .04, .04, .04])
    s = seq.tobytes().decode()
    pat, L = "N" * 21 + "RG", 23
    guides = ["".join(rng.choice(list("ACGT"), 20)) + "NNN" for _ in range(4)] + ["N" * 23]
    thr = [9, 9, 9, 9, 0]
    a = oracle.hits_to_tuples(oracle.search([s], pat, guides, thr))
    b = oracle.hits_to_tuples(oracle.search([_rc_text(s)], pat, guides, thr))
    flip = {"+": "-", "-": "+"}
    mapped = sorted(((c, len(s) - L - p, flip[st], g, mm, site) for c, p, st, g, mm, site in a),
                    key=lambda h: (h[0], h[1], h[2] == "-", h[3]))
    assert len(a) > 100
    assert mapped == b


def test_threshold_monotone():
    rng = np.random.default_rng(12)
    seq = synth.random_genome_text(rng, 100_000)
    g = ["".join(rng.choice(list("ACGT"), 20)) + "NNN" for _ in range(3)]
    prev = set()
    for t in range(0, 12):
        cur = {(h[0], h[1], h[2], h[3]) for h in
               oracle.hits_to_tuples(oracle.search([seq], "N" * 21 + "NGG"[1:], g, [t] * 3))}
        assert prev <= cur
        prev = cur


def test_all_n_pattern_every_window():
    """Special case: all-N pattern + all-N guide at t=0 -> every valid window, both strands."""
    rng = np.random.default_rng(13)
    chroms = [synth.random_genome_text(rng, n, b"ACGTN") for n in (0, 4, 5, 6, 997)]
    L = 5
    hits = oracle.search(chroms, "N" * L, ["N" * L], [0])
    expect = sum(2 * max(0, len(c) - L + 1) for c in chroms)
    assert len(hits) == expect
    assert (hits["mm"] == 0).all()


def test_threshold_at_least_compared_is_pam_list():
    """Special case: t >= #compared letters -> hits == PAM candidate list, each strand."""
    rng = np.random.default_rng(14)
    seq = synth.random_genome_text(rng, 20_000, b"ACGTN", p=[.24, .24, .24, .24, .04])
    pat = "TTTV" + "N" * 6
    g = "NNNN" + "ACGTAC"
    hits = oracle.search([seq], pat, [g], [6])
    for st in "+-":
        pos = hits["pos"][hits["strand"] == st.encode()]
        assert np.array_equal(pos, oracle.pam_sites(seq, pat, st))


def test_pam_sites_against_pyoracle():
    rng = np.random.default_rng(15)
    s = synth.random_genome_text(rng, 3000, b"ACGTacgtN").tobytes().decode()
    for pat in ("NNNNRG", "TTTVNNNN", "NGGN", "NNNNNN"):
        L = len(pat)
        ref = pyoracle.search([s], pat, ["N" * L], [0])
        for st in "+-":
            exp = [h[1] for h in ref if h[2] == st]
            assert oracle.pam_sites(s, pat, st).tolist() == exp


def test_short_and_empty():
    assert len(oracle.search([], "NNRG", ["ACNN"], [1])) == 0
    assert len(oracle.search(["ACG", ""], "NNRG", ["ACNN"], [4])) == 0
    with pytest.raises(ValueError):
        oracle.search(["ACGT"], "NNRG", ["ACN"], [1])           # guide length != L (G11)
    with pytest.raises(ValueError):
        oracle.search(["ACGT"], "NNRU", ["ACNN"], [1])          # not an IUPAC letter (G18)
    with pytest.raises(ValueError):
        oracle.search(["ACGT"], "N" * 65, ["N" * 65], [1])      # L > 64 (COF_ORACLE_MAX_L)


@pytest.mark.parametrize("seed", range(4))
def test_long_patterns_two_oracles(seed):
    """32 < L <= 64: the C oracle against the independent pure-Python
    oracle on random long IUPAC patterns and guides (brute force on small genomes)."""
    rng = np.random.default_rng(2000 + seed)
    L = int(rng.integers(33, 65))
    codes = "ACGTRYSWKMBDHV"
    pat = "".join(rng.choice(list("N" * 30 + codes), L))
    guides = ["".join(rng.choice(list("ACGTACGTN" + "RYKM"), L)) for _ in range(3)]
    thr = [int(rng.integers(L // 3, L // 2)) for _ in guides]
    chroms = [synth.random_genome_text(rng, int(rng.integers(0, 1500)), b"ACGTacgtNnRy",
                                       p=[.2, .15, .15, .2, .06, .06, .06, .06, .03, .01, .01, .01]).tobytes().decode()
              for _ in range(3)]
    a = oracle.hits_to_tuples(oracle.search(chroms, pat, guides, thr))
    b = pyoracle.search(chroms, pat, guides, thr)
    assert a == b


def test_planted_sites_long():
    """Pin by construction at L = 40 (36-nt cores + NGG, a two-word compared span) and
    L = 38 (CjCas9-like 8-letter PAM): every planted k <= t copy is found at mm == k."""
    for name in ("X1", "X2"):
        w = synth.make_workload(name, scale=0.01, n_guides=3)
        cfg = w.cfg
        assert cfg.L > 32
        hits = oracle.search(w.seqs, cfg.pattern, w.guides, w.thresholds)
        found = {(int(h["chrom"]), int(h["pos"]), h["strand"].decode(), int(h["guide"])): int(h["mm"])
                 for h in hits}
        for pl in w.plants:
            key = (pl.chrom, pl.pos, pl.strand, pl.guide)
            if pl.k <= cfg.threshold:
                assert found.get(key) == pl.k, pl
            else:
                assert key not in found, pl


def test_ranges_restrict_window_starts():
    rng = np.random.default_rng(16)
    seq = synth.random_genome_text(rng, 40_000)
    g = ["".join(rng.choice(list("ACGT"), 20)) + "NNN"]
    full = oracle.search([seq], "N" * 21 + "RG", g, [10])
    part = oracle.search([seq], "N" * 21 + "RG", g, [10], ranges=[(1234, 30001)])
    sel = full[(full["pos"] >= 1234) & (full["pos"] < 30001)]
    assert oracle.hits_to_tuples(part) == oracle.hits_to_tuples(sel)


# ----------------------------------------------------------------- statistics
def _poisson_binomial_cdf(q_match, t):
    """P(#mismatches <= t) for independent positions with match probabilities q_match."""
    dp = np.zeros(len(q_match) + 1)
    dp[0] = 1.0
    for q in q_match:
        nxt = np.zeros_like(dp)
        nxt[:] += dp * q              # match: count unchanged
        nxt[1:] += dp[:-1] * (1 - q)  # mismatch: count + 1
        dp = nxt
    return dp[: t + 1].sum()


def test_binomial_hit_rate():
    """Closed form: on an i.i.d. genome (A=T=.295, C=G=.205) the expected number of
    '+'/'-' NRG items is 2(n-L+1)*P(R)*P(G) and the expected hits add the
    Poisson-binomial P(mm <= t) per guide; the oracle's counts sit within 5 sigma."""
    comp = dict(zip("ACGT", synth.COMPOSITION))
    rng = np.random.default_rng(17)
    n = 1_500_000
    seq = synth.random_genome_text(rng, n, b"ACGT", p=list(synth.COMPOSITION))
    guides = ["".join(rng.choice(list("ACGT"), 20)) + "NNN" for _ in range(4)]
    t = 8
    L = 23
    p_item = (comp["A"] + comp["G"]) * comp["G"]
    e_items = 2 * (n - L + 1) * p_item
    n_items = len(oracle.pam_sites(seq, "N" * 21 + "RG", "+")) + len(oracle.pam_sites(seq, "N" * 21 + "RG", "-"))
    assert abs(n_items - e_items) < 5 * 1.5 * math.sqrt(e_items)
    hits = oracle.search([seq], "N" * 21 + "RG", guides, [t] * 4)
    for gi, g in enumerate(guides):
        p_hit = _poisson_binomial_cdf([comp[c] for c in g[:20]], t)
        e = e_items * p_hit
        got = int((hits["guide"] == gi).sum())
        assert abs(got - e) < 5 * 1.5 * math.sqrt(e) + 3, (gi, got, e)

"""Bulge search (DESIGN.md §2 readings B1-B6).

CPU: the variant-rewrite oracle (oracle/bulge.search) is pinned against the explicit
gap-alignment brute force (oracle/bulge.brute_force) and against hand-built sites; the
product's host-side variant expansion is checked against the oracle's.
GPU: the product bulge search (paper_conf_socc_jinv23_b200.bulge, through the CUDA path)
equals the oracle element by element.
"""
import numpy as np
import pytest

from oracle import bulge as obulge
from paper_conf_socc_jinv23_b200 import bulge as pbulge

PAT = "NNNNNNNNNNGG"          # 10 guide positions + NGG-like PAM (L = 12)
GUIDE = "ACGTTGCAGTNN"


def _find(res, **kw):
    keys = ("chrom", "pos", "strand", "guide", "kind", "size", "bpos", "mm", "site")
    out = []
    for h in res:
        d = dict(zip(keys, h))
        if all(d[k] == v for k, v in kw.items()):
            out.append(d)
    return out


def test_hand_built_dna_bulge():
    # the genome carries an extra 'C' between guide offsets 3 and 4, then the PAM 'GG'
    site = "ACGT" + "C" + "TGCAGT" + "GG"           # 13 bases: L + 1
    seq = "TTTT" + site + "TTTT"
    res = obulge.brute_force([seq], PAT, [GUIDE], [0], dna=1, rna=0)
    hit = _find(res, kind="D", size=1, bpos=4, pos=4, strand="+")
    assert len(hit) == 1 and hit[0]["mm"] == 0 and hit[0]["site"] == site
    assert not _find(res, kind="X", pos=4)          # no ungapped alignment with 0 mismatches
    assert obulge.to_tuples(obulge.search([seq], PAT, [GUIDE], [0], 1, 0)) == res


def test_hand_built_rna_bulge_and_mismatch():
    # guide letter 5 ('G') has no partner; one substitution at guide offset 1 (C -> a)
    g_wo = GUIDE[:5] + GUIDE[6:]                     # guide without offset 5: 11 letters
    site = "A" + "A" + g_wo[2:9] + "GG"             # L - 1 = 11 bases, PAM 'GG' at the end
    seq = "CCCCC" + site + "CCCCC"
    res = obulge.brute_force([seq], PAT, [GUIDE], [1], dna=0, rna=1)
    hit = _find(res, kind="R", size=1, bpos=5, pos=5, strand="+")
    assert len(hit) == 1 and hit[0]["mm"] == 1
    assert hit[0]["site"][1] == "a"
    assert obulge.to_tuples(obulge.search([seq], PAT, [GUIDE], [1], 0, 1)) == res


def test_bulges_only_inside_span_and_pattern_n():
    v = obulge.expand(PAT, [GUIDE], [2], dna=2, rna=2)
    for recs in v.values():
        for gi, kind, size, bpos, gv, t in recs:
            if kind == "D":
                assert 0 < bpos < 10
            if kind == "R":
                assert 0 < bpos and bpos + size < 10
    # a guide whose compared span is one letter has no bulge variants
    v1 = obulge.expand("NNNNGG", ["NNANNN"], [0], dna=2, rna=2)
    assert sum(len(r) for r in v1.values()) == 1


def test_reverse_strand_dna_bulge():
    site = "ACGT" + "C" + "TGCAGT" + "GG"
    comp = {"A": "T", "C": "G", "G": "C", "T": "A"}
    rc = "".join(comp[c] for c in reversed(site))
    seq = "GGGG" + rc + "GGGG"
    res = obulge.brute_force([seq], PAT, [GUIDE], [0], dna=1, rna=0)
    hit = _find(res, kind="D", size=1, bpos=4, pos=4, strand="-")
    assert len(hit) == 1 and hit[0]["site"] == site


@pytest.mark.parametrize("seed", range(4))
def test_variant_oracle_equals_brute_force(seed):
    rng = np.random.default_rng(900 + seed)
    L = int(rng.integers(6, 11))
    pam = "".join(rng.choice(list("ACGTRN"), 2))
    pat = "N" * (L - 2) + pam
    guides = ["".join(rng.choice(list("ACGTACGTNRY"), L - 2)) + "NN" for _ in range(3)]
    thr = [int(rng.integers(0, 3)) for _ in guides]
    seqs = ["".join(rng.choice(list("ACGTACGTacgtN"), int(rng.integers(30, 200)))) for _ in range(2)]
    bf = obulge.brute_force(seqs, pat, guides, thr, dna=2, rna=2)
    vo = obulge.to_tuples(obulge.search(seqs, pat, guides, thr, 2, 2))
    assert vo == bf


def test_product_variant_expansion_matches_oracle():
    rng = np.random.default_rng(77)
    guides = ["".join(rng.choice(list("ACGTN"), 20)) + "NNN" for _ in range(5)] + ["NNNNACGTNN" + "N" * 13]
    pat = "N" * 21 + "RG"
    ov = obulge.expand(pat, guides, [3] * len(guides), dna=2, rna=2)
    pv = pbulge.variants(pat, guides, [3] * len(guides), dna=2, rna=2)
    assert set(ov) == set(pv)
    for k in ov:
        o = sorted((r[0], r[1], r[2], r[3], r[4], r[5]) for r in ov[k])
        gs, ts, ms = pv[k]
        p = sorted((m[0], m[1].decode(), m[2], m[3], g, t) for g, t, m in zip(gs, ts, ms))
        assert o == p


# ---------------------------------------------------------------- GPU parity
@pytest.mark.gpu
@pytest.mark.parametrize("seed", range(3))
def test_gpu_bulge_search_matches_oracle(seed):
    from paper_conf_socc_jinv23_b200 import synth
    rng = np.random.default_rng(1200 + seed)
    L = 23
    guides = ["".join(rng.choice(list("ACGT"), 20)) + "NNN" for _ in range(6)]
    thr = [3] * len(guides)
    pat = "N" * 21 + "RG"
    seqs = [synth.random_genome_text(rng, int(n)) for n in (50_000, 31_337)]
    # plant bulged copies of each guide on both strands
    comp = {"A": "T", "C": "G", "G": "C", "T": "A"}
    s0 = bytearray(seqs[0])
    off = 100
    for g in guides:
        core = g[:20]
        for site in (core[:7] + "T" + core[7:] + "AGG", core[:9] + core[10:] + "TGG"):
            for strand in "+-":
                txt = site if strand == "+" else "".join(comp[c] for c in reversed(site))
                s0[off:off + len(txt)] = txt.encode()
                off += len(txt) + 37
    seqs[0] = bytes(s0)
    exp = obulge.to_tuples(obulge.search(seqs, pat, guides, thr, 1, 1))
    assert any(h[4] == "D" and h[7] == 0 for h in exp) and any(h[4] == "R" and h[7] == 0 for h in exp)
    got = pbulge.to_tuples(pbulge.search(seqs, pat, guides, thr, dna=1, rna=1))
    assert got == exp
    # chunked + packed layouts give the same list
    got2 = pbulge.to_tuples(pbulge.search(seqs, pat, guides, thr, dna=1, rna=1, chunk_bases=7001,
                                          pack_bases=20_000))
    assert got2 == exp


@pytest.mark.gpu
def test_gpu_bulge_degenerate_and_sizes():
    rng = np.random.default_rng(1300)
    pat = "TTTV" + "N" * 14
    guides = ["NNNN" + "".join(rng.choice(list("ACGTRYN"), 14)) for _ in range(4)]
    thr = [2, 3, 1, 4]
    from paper_conf_socc_jinv23_b200 import synth
    seqs = [synth.random_genome_text(rng, 40_000, b"ACGTacgtN", p=[.22, .22, .22, .22, .03, .03, .03, .02, .01])]
    exp = obulge.to_tuples(obulge.search(seqs, pat, guides, thr, 2, 2))
    assert len(exp) > 0
    assert pbulge.to_tuples(pbulge.search(seqs, pat, guides, thr, dna=2, rna=2)) == exp

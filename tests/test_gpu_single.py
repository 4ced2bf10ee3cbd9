"""GPU parity of the single-pass find + compare kernel (single.cu, SURVEY §8(f) f1 as ONE
streaming kernel: PAM test, per-warp site queues, filter + exact verification) against
the CPU oracle, element by element.  The single pass is forced (path="single") wherever
the plan's shape allows it -- every compared position of both strands inside one
31-position window -- including plans whose filter is not selective (thresholds near the
pair count), where nearly every comparison goes through the verification."""
import numpy as np
import pytest

from oracle import oracle
from paper_conf_socc_jinv23_b200 import cof, search, synth

pytestmark = pytest.mark.gpu


def single_shape_ok(pattern, guides):
    """Python restatement of the shape condition (single.cu single_shape_ok)."""
    L = len(pattern)
    if L > 32:
        return False
    care = [j for j in range(L) if any(g[j].upper() != "N" for g in guides)]
    return not care or care[-1] - care[0] + 1 <= 31


def ref_hits(seqs, pattern, guides, thr, ranges=None):
    return oracle.hits_to_tuples(oracle.search(seqs, pattern, guides, thr, ranges=ranges))


def gpu_single(seqs, pattern, guides, thr, **kw):
    return cof.hits_to_tuples(search.search(seqs, pattern, guides, thr, path="single", **kw))


@pytest.mark.parametrize("seed", range(12))
def test_random_small_single(seed):
    """Random IUPAC patterns (incl. all-N and degenerate letters), guides with degenerate
    letters and Ns (non-contiguous compared positions: the generic pair path), genomes with
    N / lowercase / rare IUPAC letters, one or many chunks, multi-segment chunks."""
    rng = np.random.default_rng(900 + seed)
    L = int(rng.integers(1, 33))
    pat = "".join(rng.choice(list("NNNNNNNNACGTRYSWKMBDHV"), L))
    for _ in range(50):
        guides = ["".join(rng.choice(list("ACGTACGTACGTNNRYKMSWBDHV"), L)) for _ in range(int(rng.integers(1, 90)))]
        if single_shape_ok(pat, guides):
            break
        guides = [("N" + g[1:]) if L > 31 else g for g in guides]
        if single_shape_ok(pat, guides):
            break
    assert single_shape_ok(pat, guides)
    thr = [int(rng.integers(0, L + 1)) for _ in guides]
    lens = [int(rng.integers(0, 3)) if i == 0 else int(rng.integers(L, 60_000)) for i in range(4)]
    seqs = [synth.random_genome_text(rng, n, b"ACGTacgtNnRy",
                                     p=[.22, .15, .15, .22, .05, .05, .05, .05, .04, .01, .005, .005]) for n in lens]
    exp = ref_hits(seqs, pat, guides, thr)
    assert gpu_single(seqs, pat, guides, thr) == exp
    assert gpu_single(seqs, pat, guides, thr, pack_bases=0) == exp
    assert gpu_single(seqs, pat, guides, thr, chunk_bases=9973, pack_bases=30_000) == exp


@pytest.mark.parametrize("shape", ["spcas9", "cas12a", "ngg"])
@pytest.mark.parametrize("n_guides", [1, 33, 100, 1000])
def test_uniform_threshold_single(shape, n_guides):
    """The configs' shapes (uniform thresholds: the specialised filter; 20-nt + NRG / NGG,
    Cas12a TTTV + 23 nt) with planted exact and near sites of every guide, genomes with N
    runs, lowercase and rare letters; one to 32 guide blocks in one launch."""
    rng = np.random.default_rng(31 + n_guides + 7 * len(shape))
    if shape == "cas12a":
        pat, mk, t = "TTTV" + "N" * 23, lambda: "NNNN" + "".join(rng.choice(list("ACGT"), 23)), 5
    else:
        pat = "N" * 21 + ("RG" if shape == "spcas9" else "GG")
        mk, t = (lambda: "".join(rng.choice(list("ACGT"), 20)) + "NNN"), 6
    guides = [mk() for _ in range(n_guides)]
    lens = [0, 7, 600_011 if n_guides < 500 else 120_007, 77_777]
    seqs = [synth.random_genome_text(rng, n, b"ACGTacgtNnRy",
                                     p=[.23, .17, .17, .23, .04, .04, .04, .04, .02, .01, .005, .005]) for n in lens]
    s2 = seqs[2]
    for gi, g in enumerate(guides[:60]):
        core = g.replace("N", "")
        site = list((core + "AGG") if shape != "cas12a" else ("TTTA" + core))
        for k in range(gi % (t + 2)):      # k substitutions (k = t + 1: must not be reported)
            j = (3 + 5 * k) % len(core) + (0 if shape != "cas12a" else 4)
            site[j] = {"A": "C", "C": "G", "G": "T", "T": "A"}[site[j]]
        p = 1000 + gi * 997
        s2[p:p + len(site)] = np.frombuffer("".join(site).encode(), np.uint8)
    thr = [t] * len(guides)
    exp = ref_hits(seqs, pat, guides, thr)
    assert len(exp) >= min(20, n_guides)
    p = search.Searcher(pat, guides, thr)
    assert p.path == "single"          # the product picks the single pass for these shapes
    assert gpu_single(seqs, pat, guides, thr) == exp
    assert gpu_single(seqs, pat, guides, thr, chunk_bases=99_991, pack_bases=300_000) == exp


def test_many_guides_several_launches():
    """2,100 guides with per-guide thresholds: more guide blocks than one launch's shared
    memory holds (several launches, each re-streaming the planes)."""
    rng = np.random.default_rng(5)
    pat = "N" * 21 + "RG"
    guides = ["".join(rng.choice(list("ACGT"), 20)) + "NNN" for _ in range(2100)]
    thr = [int(x) for x in rng.integers(3, 7, len(guides))]
    seqs = [synth.random_genome_text(rng, 150_000, b"ACGTN", p=[.24, .24, .24, .24, .04])]
    for gi in range(0, 2100, 37):     # exact copies of every 37th guide
        site = guides[gi][:20] + "AGG"
        p = 100 + gi * 60
        seqs[0][p:p + 23] = np.frombuffer(site.encode(), np.uint8)
    exp = ref_hits(seqs, pat, guides, thr)
    assert len(exp) >= 2100 // 37
    assert gpu_single(seqs, pat, guides, thr) == exp


def test_single_capacity_retry_and_counts():
    """A hit buffer far too small: COF_E_CAPACITY with the needed count, the Searcher grows
    it and re-runs; the PAM-site counts equal the oracle's candidate counts."""
    w = synth.make_workload("C3", scale=0.002, n_guides=64)
    cfg = w.cfg
    exp = ref_hits(w.seqs, cfg.pattern, w.guides, w.thresholds)
    srch = search.Searcher(cfg.pattern, w.guides, w.thresholds)
    assert srch.path == "single"
    host = search.HostGenome(w.seqs, search.plan_chunks([len(s) for s in w.seqs], cfg.L, None, 0))
    srch.reserve(host.chunks[0].n_bases, 16)
    got = cof.hits_to_tuples(srch.search_host(host))
    assert got == exp and len(exp) > 16
    dch = srch.device_chunk(host.chunks[0], segs=host.segs[0])
    cof.cof_load_chunk(host.chunk_struct(0), dch, srch.stream)
    small = srch.d_hits[:8]
    with pytest.raises(cof.CofError) as ei:
        cof.cof_search_single(srch.plan, srch.plan_dev, dch, srch.d_find_ws, small, 8, srch.stream)
    assert ei.value.status == cof.COF_E_CAPACITY
    nf, nr, nh = cof.cof_read_counts(srch.plan, srch.plan_dev, srch.stream)
    assert nh == len(exp)
    n_plus = sum(len(oracle.pam_sites(s, cfg.pattern, "+")) for s in w.seqs)
    n_minus = sum(len(oracle.pam_sites(s, cfg.pattern, "-")) for s in w.seqs)
    assert (nf, nr) == (n_plus, n_minus)


def test_single_refuses_wide_shapes():
    """L > 32 (two-word windows) is not the single pass's shape: COF_E_ARG, and the product
    chooses another path."""
    pat = "N" * 38 + "GG"
    guides = ["N" + "".join(np.random.default_rng(1).choice(list("ACGT"), 36)) + "NNN"]
    srch = search.Searcher(pat, guides, [8])
    assert srch.path != "single"
    seq = synth.random_genome_text(np.random.default_rng(2), 10_000, b"ACGT")
    with pytest.raises(cof.CofError) as ei:
        search.search([seq], pat, guides, [8], path="single")
    assert ei.value.status == cof.COF_E_ARG

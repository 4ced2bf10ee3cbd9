"""Genome-resident searches (search.ResidentGenome + Searcher.search_resident): the
planes cross PCIe once, then several guide sets are searched against them; every result
must equal the oracle's list (and the host-pipeline result) element by element."""
import numpy as np
import pytest

from oracle import oracle
from paper_conf_socc_jinv23_b200 import cof, search, synth

pytestmark = pytest.mark.gpu


def test_resident_genome_several_guide_sets():
    w = synth.make_workload("C3", scale=0.004, n_guides=60)
    cfg = w.cfg
    chunks = search.plan_chunks([len(s) for s in w.seqs], cfg.L, 3_000_001, 5_000_000)
    host = search.HostGenome(w.seqs, chunks)
    rg = search.ResidentGenome(host, "cuda")
    rng = np.random.default_rng(3)
    sets = [(cfg.pattern, w.guides[:40], w.thresholds[:40]),
            (cfg.pattern, w.guides[20:], [5] * 40),
            ("N" * 21 + "GG", w.guides[:10], [6] * 10),
            (cfg.pattern, ["".join(rng.choice(list("ACGTRY"), 20)) + "NNN" for _ in range(7)],
             [int(x) for x in rng.integers(3, 9, 7)])]
    for pat, guides, thr in sets:
        srch = search.Searcher(pat, guides, thr)
        got = cof.hits_to_tuples(srch.search_resident(rg))
        exp = oracle.hits_to_tuples(oracle.search(w.seqs, pat, guides, thr))
        assert got == exp and len(exp) > 0
        assert got == cof.hits_to_tuples(srch.search_host(host))
    # the caller's pinned result buffer
    srch = search.Searcher(*sets[0])
    out = np.zeros(10**5, dtype=srch.hit_dtype)
    got = srch.search_resident(rg, out=out)
    assert cof.hits_to_tuples(got) == oracle.hits_to_tuples(oracle.search(w.seqs, *sets[0]))


@pytest.mark.parametrize("path", ["single", "fused", "twocall"])
def test_pipelines_restart_on_overflow(path):
    """search_host and search_resident read each chunk's hit count only after later chunks
    are queued; a count above the (deliberately tiny) buffers restarts the call with larger
    ones.  The result must still equal the oracle's -- for a list of chunks, an iterator of
    chunk indices (search_multi's shared queue: the chunks already taken are replayed) and
    the resident genome."""
    w = synth.make_workload("C3", scale=0.004, n_guides=60)
    cfg = w.cfg
    chunks = search.plan_chunks([len(s) for s in w.seqs], cfg.L, 2_000_003, 4_000_000)
    host = search.HostGenome(w.seqs, chunks)
    exp = oracle.hits_to_tuples(oracle.search(w.seqs, cfg.pattern, w.guides, w.thresholds))
    assert len(exp) > 2000 and len(host.chunks) > 3

    def fresh():
        srch = search.Searcher(cfg.pattern, w.guides, w.thresholds)
        srch.path = path if path != "fused" or cof.cof_find_compare_supported(srch.plan) else "twocall"
        srch.reserve(max(ch.n_bases for ch in host.chunks), 64)    # far too small
        return srch

    assert cof.hits_to_tuples(fresh().search_host(host)) == exp
    assert cof.hits_to_tuples(fresh().search_host(host, indices=iter(range(len(host.chunks))))) == exp
    rg = search.ResidentGenome(host, "cuda")
    assert cof.hits_to_tuples(fresh().search_resident(rg)) == exp

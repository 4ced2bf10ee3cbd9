"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle, element by element.

Bar: bit-exact -- every hit record (chrom, pos, strand, guide, mm, site)
and every finder candidate list must equal the oracle's.  Sizes span many finder tiles
(8192 starts) and comparer tiles plus ragged tails; full-size configs are checked on
sampled window ranges that the oracle recomputes one by one.
"""
import numpy as np
import pytest
import torch

from oracle import oracle
from paper_conf_socc_jinv23_b200 import cof, search, synth
from tests import golden_io

pytestmark = pytest.mark.gpu
IMPLS = ["table", "popc"]


@pytest.fixture(autouse=True)
def _impl_reset():
    yield
    cof.cof_set_comparer("table")


def gpu_hits(seqs, pattern, guides, thr, chunk_bases=None, impl="table", pack_bases=None, fused=None):
    cof.cof_set_comparer(impl)
    return cof.hits_to_tuples(search.search(seqs, pattern, guides, thr, chunk_bases=chunk_bases,
                                            pack_bases=pack_bases, fused=fused))


def ref_hits(seqs, pattern, guides, thr, ranges=None):
    return oracle.hits_to_tuples(oracle.search(seqs, pattern, guides, thr, ranges=ranges))


@pytest.mark.parametrize("impl", IMPLS)
def test_worked_example(impl):
    d = golden_io.worked_example()
    got = gpu_hits([c.encode() for c in d["chroms"]], d["pattern"], d["guides"], d["thr"], impl=impl)
    assert got == d["hits"]


@pytest.mark.parametrize("impl", IMPLS)
@pytest.mark.parametrize("seed", range(8))
def test_random_small(impl, seed):
    """Random IUPAC patterns (incl. all-N and degenerate letters), guides with degenerate
    letters and Ns, genomes with N / lowercase / rare IUPAC letters, lengths around tiles."""
    rng = np.random.default_rng(500 + seed)
    L = int(rng.integers(1, 33))
    pat = "".join(rng.choice(list("NNNNNNNNACGTRYSWKMBDHV"), L))
    guides = ["".join(rng.choice(list("ACGTACGTACGTNNRYKMSWBDHV"), L)) for _ in range(int(rng.integers(1, 70)))]
    thr = [int(rng.integers(0, L + 1)) for _ in guides]
    lens = [int(rng.integers(0, 3)) if i == 0 else int(rng.integers(L, 40_000)) for i in range(4)]
    seqs = [synth.random_genome_text(rng, n, b"ACGTacgtNnRy",
                                     p=[.22, .15, .15, .22, .05, .05, .05, .05, .04, .01, .005, .005]) for n in lens]
    exp = ref_hits(seqs, pat, guides, thr)
    assert gpu_hits(seqs, pat, guides, thr, impl=impl) == exp
    # the same genome as one multi-segment chunk and as packed pieces
    assert gpu_hits(seqs, pat, guides, thr, impl=impl, pack_bases=0) == exp
    assert gpu_hits(seqs, pat, guides, thr, impl=impl, chunk_bases=9973, pack_bases=30_000) == exp
    if impl == "table":   # both table paths: fused (masks) and two-call (item lists)
        assert gpu_hits(seqs, pat, guides, thr, impl=impl, fused=False) == exp
        assert gpu_hits(seqs, pat, guides, thr, impl=impl, fused=False, pack_bases=0) == exp
        assert gpu_hits(seqs, pat, guides, thr, impl=impl, fused=True) == exp
        assert gpu_hits(seqs, pat, guides, thr, impl=impl, fused=True, chunk_bases=9973, pack_bases=30_000) == exp


@pytest.mark.parametrize("impl", IMPLS)
def test_c1_full(impl):
    w = synth.make_workload("C1")
    cfg = w.cfg
    exp = ref_hits(w.seqs, cfg.pattern, w.guides, w.thresholds)
    assert len(exp) >= cfg.threshold + 1
    assert gpu_hits(w.seqs, cfg.pattern, w.guides, w.thresholds, impl=impl) == exp


@pytest.mark.parametrize("name,scale,chunk,pack", [("C2", 0.1, None, None), ("C3", 0.004, 1_000_003, None),
                                                   ("C4", 0.004, 333_333, 0), ("C5", 0.002, None, 0),
                                                   ("C3", 0.003, None, 2_000_000)])
def test_configs_scaled(name, scale, chunk, pack):
    w = synth.make_workload(name, scale=scale, n_guides=None if name != "C5" else 200)
    cfg = w.cfg
    exp = ref_hits(w.seqs, cfg.pattern, w.guides, w.thresholds)
    assert gpu_hits(w.seqs, cfg.pattern, w.guides, w.thresholds, chunk_bases=chunk, pack_bases=pack) == exp
    assert gpu_hits(w.seqs, cfg.pattern, w.guides, w.thresholds, chunk_bases=chunk, pack_bases=pack,
                    fused=False) == exp
    assert gpu_hits(w.seqs, cfg.pattern, w.guides, w.thresholds, chunk_bases=chunk, pack_bases=pack,
                    fused=True) == exp


@pytest.mark.parametrize("shape", ["spcas9", "cas12a"])
@pytest.mark.parametrize("n_guides", [1, 37, 512, 600])
def test_uniform_threshold_paths(shape, n_guides):
    """The uniform-threshold specializations (20-nt SpCas9 guides: 10 pairs; 23-nt Cas12a:
    12 pairs) on genomes with N runs, lowercase and rare letters, one to 19 guide blocks
    (one fused launch, or two for 600 guides of Cas12a), fused and two-call paths."""
    rng = np.random.default_rng(77 + n_guides + (shape == "cas12a"))
    if shape == "spcas9":
        pat, mk = "N" * 21 + "RG", lambda: "".join(rng.choice(list("ACGT"), 20)) + "NNN"
    else:
        pat, mk = "TTTV" + "N" * 23, lambda: "NNNN" + "".join(rng.choice(list("ACGT"), 23))
    guides = [mk() for _ in range(n_guides)]
    t = 6 if shape == "spcas9" else 5
    lens = [0, 5, 1_000_003 if n_guides < 100 else 200_003, 77_777]
    seqs = [synth.random_genome_text(rng, n, b"ACGTacgtNnRy",
                                     p=[.23, .17, .17, .23, .04, .04, .04, .04, .02, .01, .005, .005]) for n in lens]
    # plant exact and near copies of every guide so every guide block sees hits
    s2 = seqs[2]
    for gi, g in enumerate(guides[:64]):
        core = g.replace("N", "")
        site = (core + "AGG") if shape == "spcas9" else ("TTTA" + core)
        p = 1000 + gi * 997
        s2[p:p + len(site)] = np.frombuffer(site.encode(), np.uint8)
    thr = [t] * len(guides)
    exp = ref_hits(seqs, pat, guides, thr)
    assert len(exp) >= min(64, n_guides)
    assert gpu_hits(seqs, pat, guides, thr, fused=True) == exp
    assert gpu_hits(seqs, pat, guides, thr, fused=True, pack_bases=0) == exp
    assert gpu_hits(seqs, pat, guides, thr, fused=True, chunk_bases=99_991, pack_bases=300_000) == exp
    assert gpu_hits(seqs, pat, guides, thr, fused=False) == exp


@pytest.mark.parametrize("seed", range(6))
def test_random_long(seed):
    """32 < L <= 64: random long IUPAC patterns (PAM letters at window
    offsets >= 32: the finder's three-word slices), guides whose compared span is either
    <= 32 or up to 63 (two-word comparer windows, padded pair tables), degenerate letters,
    genome N / lowercase; fused and two-call paths, one chunk and packed pieces; the popc
    selection falls back to the table comparer."""
    rng = np.random.default_rng(900 + seed)
    L = int(rng.integers(33, 65))
    pat = "".join(rng.choice(list("N" * 24 + "ACGTRYSWKMBDHV"), L))
    span = int(rng.integers(8, 33)) if seed % 2 else int(rng.integers(33, min(L, 63) + 1))
    off = int(rng.integers(0, L - span + 1))
    guides = []
    for _ in range(int(rng.integers(1, 70))):
        g = ["N"] * L
        for j in range(off, off + span):
            g[j] = str(rng.choice(list("ACGTACGTACGTNRYKMSWBDHV")))
        g[off] = str(rng.choice(list("ACGT")))
        g[off + span - 1] = str(rng.choice(list("ACGT")))
        guides.append("".join(g))
    thr = [int(rng.integers(span // 4, span // 2 + 2)) for _ in guides]
    lens = [int(rng.integers(0, 3)) if i == 0 else int(rng.integers(L, 40_000)) for i in range(4)]
    seqs = [synth.random_genome_text(rng, n, b"ACGTacgtNnRy",
                                     p=[.22, .15, .15, .22, .05, .05, .05, .05, .04, .01, .005, .005]) for n in lens]
    exp = ref_hits(seqs, pat, guides, thr)
    assert gpu_hits(seqs, pat, guides, thr) == exp
    assert gpu_hits(seqs, pat, guides, thr, pack_bases=0) == exp
    assert gpu_hits(seqs, pat, guides, thr, chunk_bases=9973, pack_bases=30_000) == exp
    assert gpu_hits(seqs, pat, guides, thr, fused=False) == exp
    assert gpu_hits(seqs, pat, guides, thr, fused=True, pack_bases=0) == exp
    assert gpu_hits(seqs, pat, guides, thr, impl="popc") == exp


@pytest.mark.parametrize("name,scale,n_guides", [("X1", 0.05, None), ("X2", 0.05, None), ("X1", 0.01, 300)])
def test_long_configs(name, scale, n_guides):
    """Long-window configs X1 (37-nt spacers + NGG, L = 40) and X2 (30-nt + NNNNRYAC,
    L = 38) with planted sites, through the device decoration (cof_decorate64)."""
    w = synth.make_workload(name, scale=scale, n_guides=n_guides)
    cfg = w.cfg
    exp = ref_hits(w.seqs, cfg.pattern, w.guides, w.thresholds)
    assert len(exp) >= cfg.threshold + 1
    for fused in (False, True):
        assert gpu_hits(w.seqs, cfg.pattern, w.guides, w.thresholds, fused=fused) == exp
        assert gpu_hits(w.seqs, cfg.pattern, w.guides, w.thresholds, fused=fused, pack_bases=0,
                        chunk_bases=1_000_003) == exp


def test_chunk_size_invariance():
    w = synth.make_workload("C2", scale=0.02)
    cfg = w.cfg
    base = gpu_hits(w.seqs, cfg.pattern, w.guides, w.thresholds)
    for cb in (8192, 8191, 100_003, 7):
        assert gpu_hits(w.seqs, cfg.pattern, w.guides, w.thresholds, chunk_bases=cb) == base


def test_finder_candidates_match_oracle():
    """Finder output (ordered per-strand item lists) == oracle PAM candidate lists."""
    rng = np.random.default_rng(9)
    n = 300_001
    seq = synth.random_genome_text(rng, n, b"ACGTacgtN", p=[.23, .23, .23, .23, .02, .02, .02, .01, .01])
    for pat in ("N" * 21 + "RG", "TTTV" + "N" * 23, "NGG", "N" * 8, "N" * 34 + "RYAC", "TTTV" + "N" * 40 + "GA"):
        L = len(pat)
        plan = cof.cof_plan_create(pat, ["N" * L], [0])
        s = torch.cuda.current_stream()
        pd = torch.empty(cof.cof_plan_device_bytes(plan) + 256, dtype=torch.uint8, device="cuda")
        cof.cof_plan_upload(plan, pd, s)
        for start, owned in ((0, n - L + 1), (12345, 100_000), (n - L - 40, 41)):
            nb = owned + L - 1
            w = cof.cof_plane_words(nb)
            host = np.zeros((3, w), np.uint32)
            cof.cof_pack(np.ascontiguousarray(seq[start:start + nb]), nb, host[0], host[1], host[2])
            d = torch.from_numpy(host.view(np.int32)).cuda()
            dch = cof.make_chunk(0, start, nb, owned, d[0], d[1], d[2])
            items = torch.empty((2, owned), dtype=torch.int32, device="cuda")
            ws = torch.empty(cof.cof_find_workspace_bytes(nb), dtype=torch.uint8, device="cuda")
            nf, nr = cof.cof_find_pam(plan, pd, dch, ws, items[0], items[1], owned, s)
            for k, st in enumerate("+-"):
                exp = oracle.pam_sites(seq, pat, st, start, start + owned) - start
                got = items[k, : (nf, nr)[k]].cpu().numpy().astype(np.int64)
                assert np.array_equal(got, exp), (pat, start, st)


def test_capacity_overflow_and_device_counts():
    rng = np.random.default_rng(10)
    seq = synth.random_genome_text(rng, 50_000)
    pat = "N" * 10
    guides = ["N" * 10, "A" * 10]
    thr = [0, 10]
    exp = ref_hits([seq], pat, guides, thr)
    srch = search.Searcher(pat, guides, thr)
    srch.fused = False            # this test drives the two-call API (item lists) directly
    srch.reserve(len(seq), 64)    # far too small: forces COF_E_CAPACITY + retry
    host = search.HostGenome([seq], search.plan_chunks([len(seq)], 10))
    got = cof.hits_to_tuples(srch.search_host(host))
    assert got == exp
    # items capacity too small -> COF_E_CAPACITY with the needed count
    dch = srch.device_chunk(host.chunks[0])
    cof.cof_load_chunk(host.chunk_struct(0), dch, srch.stream)
    with pytest.raises(cof.CofError) as ei:
        cof.cof_find_pam(srch.plan, srch.plan_dev, dch, srch.d_find_ws, srch.d_items[0], srch.d_items[1], 100,
                         srch.stream)
    assert ei.value.status == cof.COF_E_CAPACITY
    # counts left on the device are used by compare / sort without a host round trip
    cof.cof_find_pam(srch.plan, srch.plan_dev, dch, srch.d_find_ws, srch.d_items[0], srch.d_items[1],
                     host.chunks[0].n_owned, srch.stream, sync=False)
    cof.cof_compare(srch.plan, srch.plan_dev, dch, srch.d_items[0], cof.COF_COUNT_ON_DEVICE, srch.d_items[1],
                    cof.COF_COUNT_ON_DEVICE, srch.d_hits, srch._hits_cap, srch.stream, sync=False)
    cof.cof_sort_hits(srch.plan, srch.plan_dev, dch, srch.d_hits, srch.d_tmp, srch._hits_cap,
                      cof.COF_COUNT_ON_DEVICE, srch.d_sort_ws, srch.stream)
    nf, nr, nh = cof.cof_read_counts(srch.plan, srch.plan_dev, srch.stream)
    assert nh == len(exp)
    got2 = cof.hits_to_tuples(cof.cof_collect(srch.plan, host.chunk_struct(0), srch.d_hits, nh, srch.stream))
    assert got2 == exp


def test_sorted_keys_and_determinism():
    w = synth.make_workload("C3", scale=0.002, n_guides=64)
    cfg = w.cfg
    a = gpu_hits(w.seqs, cfg.pattern, w.guides, w.thresholds)
    b = gpu_hits(w.seqs, cfg.pattern, w.guides, w.thresholds)
    assert a == b
    assert a == sorted(a, key=lambda h: (h[0], h[1], h[2] == "-", h[3]))


@pytest.mark.parametrize("name", ["C5", "C3", "C4"])
def test_full_size_sampled(name):
    """C5 / C3 / C4 at full size on one GPU, in the bench's launch configuration (the whole
    genome as one multi-segment chunk, device-resident planes, counts on device; the single
    pass -- one launch, the sparse-PAM geometry for C4); the oracle recomputes sampled
    window ranges one by one, every planted site is found with its exact count, and the
    single pass's PAM-site counts equal the separate search kernel's (cof_find_pam)."""
    from bench import run_device_pipeline, prepare_workload, time_search_kernel   # the bench's code
    wl, plan_obj = prepare_workload(name)
    assert plan_obj.path_name == "single"
    res = run_device_pipeline(wl, plan_obj, collect=True)
    time_search_kernel(plan_obj, 1)    # raises unless its item counts equal the step's
    rng = np.random.default_rng(77)
    cfg = wl.cfg
    n_samples = 0
    for c in rng.choice(len(wl.seqs), 6, replace=False):
        n = len(wl.seqs[c])
        for s0 in list(rng.integers(0, n - 200_000, 2)) + [0, n - 60_000]:
            rng_ = [(0, 0)] * len(wl.seqs)
            rng_[c] = (int(s0), int(s0) + 60_000)
            exp = ref_hits(wl.seqs, cfg.pattern, wl.guides, wl.thresholds, ranges=rng_)
            h = res[(res["chrom"] == c) & (res["pos"] >= s0) & (res["pos"] < s0 + 60_000)]
            assert cof.hits_to_tuples(h) == exp
            n_samples += 1
    # planted sites at full size: every k <= t copy present with its exact mismatch count
    found = {(int(h["chrom"]), int(h["pos"]), h["strand"].decode(), int(h["guide"])): int(h["mm"]) for h in res}
    for pl in wl.plants:
        key = (pl.chrom, pl.pos, pl.strand, pl.guide)
        if pl.k <= cfg.threshold:
            assert found.get(key) == pl.k
        else:
            assert key not in found
    assert n_samples >= 20


@pytest.mark.parametrize("decorate", ["device", "host"])
def test_search_host_into_caller_buffer_and_chunk_pipeline(decorate):
    """The pipelined public path (double-buffered H2D, device or host decoration) writing
    straight into a caller buffer equals the oracle; a too-small buffer falls back to merge."""
    w = synth.make_workload("C3", scale=0.003, n_guides=40)
    cfg = w.cfg
    exp = ref_hits(w.seqs, cfg.pattern, w.guides, w.thresholds)
    chunks = search.plan_chunks([len(s) for s in w.seqs], cfg.L, 200_003)
    host = search.HostGenome(w.seqs, chunks)
    srch = search.Searcher(cfg.pattern, w.guides, w.thresholds)
    out = np.empty(len(exp) + 10, dtype=cof.HIT_DTYPE)
    got = srch.search_host(host, out=out, decorate=decorate)
    assert got.base is out or np.shares_memory(got, out)
    assert cof.hits_to_tuples(got) == exp
    small = np.empty(max(1, len(exp) // 3), dtype=cof.HIT_DTYPE)
    assert cof.hits_to_tuples(srch.search_host(host, out=small, decorate=decorate)) == exp
    # multi-segment chunks through the same path
    packed = search.HostGenome(w.seqs, search.plan_chunks([len(s) for s in w.seqs], cfg.L, 150_001,
                                                          pack_bases=1_000_000))
    assert any(c.multi for c in packed.chunks)
    assert cof.hits_to_tuples(srch.search_host(packed, decorate=decorate)) == exp


@pytest.mark.parametrize("impl", ["table"])
def test_many_guides_multiple_table_launches(impl):
    """> 4096 guides: the table comparer splits the guides into launches of 128 blocks
    (thresholds in the parameter space) and tiles them through shared memory."""
    rng = np.random.default_rng(21)
    seq = synth.random_genome_text(rng, 30_000)
    n_g = 4096 + 300
    guides = ["".join(rng.choice(list("ACGT"), 20)) + "NNN" for _ in range(n_g)]
    thr = [int(t) for t in rng.integers(4, 8, n_g)]
    exp = ref_hits([seq], "N" * 21 + "RG", guides, thr)
    assert len(exp) > 0
    assert gpu_hits([seq], "N" * 21 + "RG", guides, thr, impl=impl) == exp
    if impl == "table":   # fused (several launches per strand) and two-call paths
        assert gpu_hits([seq], "N" * 21 + "RG", guides, thr, impl=impl, fused=True) == exp
        assert gpu_hits([seq], "N" * 21 + "RG", guides, thr, impl=impl, fused=False) == exp
    thr_u = [7] * n_g
    assert gpu_hits([seq], "N" * 21 + "RG", guides, thr_u, impl=impl) == ref_hits([seq], "N" * 21 + "RG", guides, thr_u)


@pytest.mark.parametrize("multi", [False, True])
def test_load_chunk_runs_equals_copy(multi):
    """cof_load_chunk_runs (lo/hi over PCIe, nm rebuilt from N runs and vs from the segment
    table on the device) yields exactly the planes cof_load_chunk copies: runs at offset 0,
    at the chunk end, within one word, whole words, and n_bases both a multiple of 32 and not."""
    rng = np.random.default_rng(61 + multi)
    lens = [64_000, 33, 5_001, 96] if multi else [100_003]
    seqs = [synth.random_genome_text(rng, n, b"ACGTacgtNnRy",
                                     p=[.23, .17, .17, .23, .04, .04, .04, .04, .02, .01, .005, .005]) for n in lens]
    seqs[0][:40] = ord("N")
    seqs[0][1000:1003] = ord("n")
    seqs[0][2048:4096] = ord("N")
    seqs[-1][-9:] = ord("N")
    chunks = search.plan_chunks(lens, 23, None, 0 if multi else None)
    host = search.HostGenome(seqs, chunks)
    srch = search.Searcher("N" * 21 + "RG", ["A" * 20 + "NNN"], [3])
    for i, ch in enumerate(chunks):
        w = cof.cof_plane_words(ch.n_bases)
        a = torch.zeros((4, w), dtype=torch.int32, device="cuda")
        b = torch.full((4, w), -1, dtype=torch.int32, device="cuda")   # garbage the rebuild must overwrite
        da = srch.device_chunk(ch, a, host.segs[i])
        db = srch.device_chunk(ch, b, host.segs[i])
        c = torch.full((4, w), -1, dtype=torch.int32, device="cuda")
        dc = srch.device_chunk(ch, c, host.segs[i])
        cof.cof_load_chunk(host.chunk_struct(i), da, srch.stream)
        cof.cof_load_chunk_runs(host.chunk_struct(i), host.runs[i], db, srch.stream)
        side = torch.cuda.Stream()
        torch.cuda.synchronize()
        # the two halves on two streams (DMA on a side stream, fills on the main one)
        cof.cof_load_chunk_runs_split(host.chunk_struct(i), host.runs[i], dc, side, srch.stream)
        torch.cuda.synchronize()
        n = 4 if ch.multi else 3
        assert torch.equal(a[:n], b[:n]), i
        assert torch.equal(a[:n], c[:n]), i
    # this genome is N-fragmented (4% scattered N letters): load() keeps copying its planes
    assert host.h2d_bytes <= host.bytes

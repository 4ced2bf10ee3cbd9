"""CPU tests of the C ABI library: it loads, exports every declared symbol, and its host
logic (pack/unpack, plan validation, FASTA, collect/decorate, merge) is right.  No CUDA
compute call is made here."""
import ctypes
import os
import re

import numpy as np
import pytest

from oracle import oracle
from paper_conf_socc_jinv23_b200 import cof, search, synth

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared_symbols():
    text = open(os.path.join(ROOT, "include", "cof.h")).read()
    text = re.sub(r"/\*.*?\*/", "", text, flags=re.S)
    return sorted(set(re.findall(r"\b(cof_[a-z_0-9]+)\s*\(", text)))


def test_library_exports_every_declared_symbol():
    names = declared_symbols()
    assert len(names) >= 25
    lib = ctypes.CDLL(cof.LIB_PATH)
    for n in names:
        assert hasattr(lib, n), n
    assert set(cof.EXPORTS) <= set(names)


def test_version_and_counter():
    assert "sm_100a" in cof.cof_version()
    assert cof.cof_launch_count() >= 0


def test_plane_words():
    for n in (0, 1, 31, 32, 33, 8191, 8192, 8193, 10**6):
        w = cof.cof_plane_words(n)
        assert w >= (n + 31) // 32 + 1 and (w - 4) % 512 == 0


def _canon(b: bytes) -> bytes:
    return bytes(c if c in b"ACGT" else ord("N") for c in b.upper())


@pytest.mark.parametrize("n", [0, 1, 31, 32, 33, 1000, 70001])
def test_pack_roundtrip(n):
    rng = np.random.default_rng(n)
    seq = synth.random_genome_text(rng, n, b"ACGTacgtNnRYmk.-") if n else np.zeros(0, np.uint8)
    w = cof.cof_plane_words(n)
    lo, hi, nm = (np.zeros(w, np.uint32) for _ in range(3))
    cof.cof_pack(seq, n, lo, hi, nm)
    out = np.zeros(n, np.uint8)
    cof.cof_unpack(lo, hi, nm, 0, n, out)
    assert out.tobytes() == _canon(seq.tobytes())
    # padding: past the last base every position is N (lo = hi = 0)
    last = n // 32
    if n % 32:
        assert nm[last] >> (n % 32) == (0xFFFFFFFF >> (n % 32))
        last += 1
    assert (nm[last:] == 0xFFFFFFFF).all() and (lo[last:] == 0).all() and (hi[last:] == 0).all()
    assert not (lo & nm).any() and not (hi & nm).any()


def test_plan_validation():
    good = "N" * 21 + "RG"
    p = cof.cof_plan_create(good, ["ACGT" * 5 + "NNN"], [3])
    assert p.L == 23 and p.n_guides == 1
    assert cof.cof_plan_device_bytes(p) > 0
    bad = [
        (good, ["ACGT" * 5 + "NN"], [3]),          # length mismatch (G11)
        ("N" * 21 + "RU", ["A" * 23], [3]),        # non-IUPAC pattern letter (G18)
        (good, ["ACGT" * 5 + "NNX"], [3]),         # non-IUPAC guide letter
        ("N" * 65, ["N" * 65], [1]),               # L > COF_MAX_L (64)
        ("N" * 64, ["A" * 64], [1]),               # 64 compared letters (6-bit counts)
        ("", [""], [0]),                           # L = 0
        (good, [], []),                            # no guides
        (good, ["ACGT" * 5 + "NNN"], [24]),        # max_mm > L
    ]
    for pat, g, t in bad:
        with pytest.raises(cof.CofError) as ei:
            cof.cof_plan_create(pat, g, t)
        assert ei.value.status == cof.COF_E_ARG
    # two-word windows: 32 < L <= 64
    assert cof.cof_plan_create("N" * 60 + "NRG", ["A" * 62 + "N"], [5]).L == 63
    assert cof.cof_plan_create("N" * 64, ["N" + "C" * 63], [5]).L == 64
    # lower case accepted (G4 / G18)
    assert cof.cof_plan_create(good.lower(), [("acgt" * 5) + "nnn"], [2]).L == 23


def _keys_from_oracle(hits):
    return np.array([(int(h["pos"]) << 32) | ((1 if h["strand"] == b"-" else 0) << 31) |
                     (int(h["guide"]) << 7) | int(h["mm"]) for h in hits], dtype=np.uint64)


def test_collect_decorates_like_the_oracle():
    """cof_collect (host decoration: site string, lower-case mismatches, '-' as reverse
    complement, chrom/abs position) against the oracle's records, from host keys."""
    rng = np.random.default_rng(3)
    seq = synth.random_genome_text(rng, 20000, b"ACGTacgtN", p=[.22, .22, .22, .22, .02, .02, .02, .02, .04])
    pat = "N" * 21 + "RG"
    guides = ["".join(rng.choice(list("ACGT"), 20)) + "NNN" for _ in range(3)] + ["RYNNKMSWACGTACGTACGTNNN"]
    thr = [12, 12, 12, 14]
    ref = oracle.search([seq], pat, guides, thr)
    assert len(ref) > 20
    plan = cof.cof_plan_create(pat, guides, thr)
    start = 0
    w = cof.cof_plane_words(len(seq))
    planes = np.zeros((3, w), np.uint32)
    cof.cof_pack(seq, len(seq), planes[0], planes[1], planes[2])
    host = cof.make_chunk(0, start, len(seq), len(seq) - 22, planes[0], planes[1], planes[2])
    keys = _keys_from_oracle(ref)
    shuffled = keys[rng.permutation(len(keys))]
    got = cof.cof_collect(plan, host, None, len(keys), host_keys=shuffled)
    assert cof.hits_to_tuples(got) == oracle.hits_to_tuples(ref)
    # a key whose mismatch count disagrees with the genome is rejected
    badk = keys.copy()
    badk[0] ^= 1
    with pytest.raises(cof.CofError) as ei:
        cof.cof_collect(plan, host, None, len(badk), host_keys=badk)
    assert ei.value.status == cof.COF_E_STATE


@pytest.mark.parametrize("L", [33, 41, 64])
def test_collect64_decorates_like_the_oracle(L):
    """cof_collect64 (L > 32: 64-bit windows, cof_hit64 records) against the oracle, incl.
    windows whose start sits late in a plane word (three-word slices)."""
    rng = np.random.default_rng(30 + L)
    seq = synth.random_genome_text(rng, 30000, b"ACGTacgtN", p=[.22, .22, .22, .22, .02, .02, .02, .02, .04])
    pat = "N" * (L - 3) + "NRG"
    core = L - 4
    guides = ["N" + "".join(rng.choice(list("ACGT"), core)) + "NNN" for _ in range(3)]
    guides.append("N" + "RYNNKMSWAC" + "".join(rng.choice(list("ACGT"), core - 10)) + "NNN")
    thr = [int(core * 0.6)] * 4
    ref = oracle.search([seq], pat, guides, thr)
    assert len(ref) > 20
    plan = cof.cof_plan_create(pat, guides, thr)
    w = cof.cof_plane_words(len(seq))
    planes = np.zeros((3, w), np.uint32)
    cof.cof_pack(seq, len(seq), planes[0], planes[1], planes[2])
    host = cof.make_chunk(0, 0, len(seq), len(seq) - L + 1, planes[0], planes[1], planes[2])
    keys = _keys_from_oracle(ref)
    got = cof.cof_collect(plan, host, None, len(keys), host_keys=keys[rng.permutation(len(keys))])
    assert got.dtype == cof.HIT64_DTYPE
    assert cof.hits_to_tuples(got) == oracle.hits_to_tuples(ref)
    # the 56-byte record cannot hold the site: cof_collect itself refuses
    with pytest.raises(cof.CofError) as ei:
        out = np.zeros(len(keys), dtype=cof.HIT_DTYPE)
        cof._check(cof.lib.cof_collect(plan.handle, ctypes.addressof(host), None, keys.ctypes.data, len(keys),
                                       out.ctypes.data, None))
    assert ei.value.status == cof.COF_E_ARG
    # cof_merge64 of the record halves gives the whole list back
    m = cof.cof_merge([got[len(got) // 2:], got[:len(got) // 2]])
    assert cof.hits_to_tuples(m) == cof.hits_to_tuples(got)


def test_merge_orders_lists():
    rng = np.random.default_rng(4)
    lists = []
    for _ in range(5):
        n = int(rng.integers(0, 50))
        a = np.zeros(n, dtype=cof.HIT_DTYPE)
        a["chrom"] = rng.integers(0, 3, n)
        a["pos"] = rng.integers(0, 100, n)
        a["strand"] = rng.choice([b"+", b"-"], n)
        a["guide"] = rng.integers(0, 4, n)
        a = a[np.lexsort((a["guide"], a["strand"] == b"-", a["pos"], a["chrom"]))]
        lists.append(a)
    m = cof.cof_merge(lists)
    cat = np.concatenate(lists)
    exp = cat[np.lexsort((cat["guide"], cat["strand"] == b"-", cat["pos"], cat["chrom"]))]
    key = lambda x: list(zip(x["chrom"], x["pos"], x["strand"], x["guide"]))
    assert key(m) == key(exp)
    with pytest.raises(cof.CofError):
        cof.cof_merge([lists[0][::-1]] if len(lists[0]) > 1 and (lists[0][0] != lists[0][-1]) else [np.array(
            [(0, 0, 5, b"+", 0, b""), (0, 0, 1, b"+", 0, b"")], dtype=cof.HIT_DTYPE)])


def test_fasta_reader(tmp_path):
    rng = np.random.default_rng(5)
    seqs = [synth.random_genome_text(rng, n, b"ACGTacgtN") for n in (0, 5, 61, 1000, 4097)]
    names = [f"chr{i}" for i in range(len(seqs))]
    for width in (60, 7):
        path = tmp_path / f"g{width}.fa"
        synth.write_fasta(path, names, seqs, width)
        fa = cof.Fasta(path)
        assert len(fa) == len(seqs)
        for i, s in enumerate(seqs):
            assert fa.name(i) == names[i] and fa.length(i) == len(s)
            for first, n in ((0, len(s)), (min(3, len(s)), max(0, len(s) - 6))):
                w = cof.cof_plane_words(n)
                a = np.zeros((3, w), np.uint32)
                b = np.zeros((3, w), np.uint32)
                fa.pack(i, first, n, a[0], a[1], a[2])
                cof.cof_pack(np.ascontiguousarray(s[first:first + n]), n, b[0], b[1], b[2])
                assert (a == b).all()
        fa.close()
    # irregular line lengths fall back to a streaming read
    path = tmp_path / "irr.fa"
    path.write_bytes(b">x desc\nACG\nTTTTT\nA\n>y\nNNNNacgt\n")
    fa = cof.Fasta(path)
    assert [fa.name(0), fa.name(1)] == ["x", "y"] and [fa.length(0), fa.length(1)] == [9, 8]
    w = cof.cof_plane_words(9)
    a = np.zeros((3, w), np.uint32)
    fa.pack(0, 0, 9, a[0], a[1], a[2])
    out = np.zeros(9, np.uint8)
    cof.cof_unpack(a[0], a[1], a[2], 0, 9, out)
    assert out.tobytes() == b"ACGTTTTTA"
    with pytest.raises(cof.CofError):
        cof.Fasta(tmp_path / "missing.fa")


@pytest.mark.parametrize("eol", [b"\n", b"\r\n"])
def test_fasta_layouts_against_plain_canonicalisation(tmp_path, eol):
    """The line-geometry reader (regular records) and the byte-walk reader (everything else)
    both give canon(sequence) for any (first, n): line widths around the 32-base word,
    CR/LF, a missing final newline, blank lines, bytes that differ from ACGT in bit 5 only."""
    rng = np.random.default_rng(11)
    alphabet = np.frombuffer(b"ACGTacgtNnRy\xc1\xe3-*", np.uint8)
    seqs = [rng.choice(alphabet, n).tobytes() for n in (0, 1, 31, 32, 33, 95, 1000, 2049)]
    for width in (1, 31, 32, 33, 60):
        for tail in (b"", b"nofinal", b"blank"):
            text = b""
            for k, s in enumerate(seqs):
                text += b">r%d some description" % k + eol
                text += b"".join(s[o:o + width] + eol for o in range(0, len(s), width))
                if tail == b"blank" and k == 2:
                    text += eol
            if tail == b"nofinal" and text.endswith(eol):
                text = text[: -len(eol)]
            path = tmp_path / f"w{width}{tail.decode()}.fa"
            path.write_bytes(text)
            fa = cof.Fasta(path)
            assert len(fa) == len(seqs)
            for i, s in enumerate(seqs):
                assert fa.name(i) == f"r{i}" and fa.length(i) == len(s)
                for first, n in ((0, len(s)), (min(5, len(s)), max(0, len(s) - 7)), (len(s) // 3, len(s) // 2)):
                    w = cof.cof_plane_words(n)
                    a = np.zeros((3, w), np.uint32)
                    fa.pack(i, first, n, a[0], a[1], a[2])
                    out = np.zeros(n, np.uint8)
                    cof.cof_unpack(a[0], a[1], a[2], 0, n, out)
                    assert out.tobytes() == _canon(s[first:first + n]), (width, tail, i, first, n)
                    full = (n + 31) // 32
                    assert (a[2][full:] == 0xFFFFFFFF).all() and not a[0][full:].any()
                    if n % 32:
                        assert a[2][n // 32] >> (n % 32) == (1 << (32 - n % 32)) - 1
            fa.close()


def test_fasta_mixed_line_endings(tmp_path):
    """One CRLF line inside an LF record: its newline still sits where the line geometry
    expects one, so the fast reader must notice the CR and hand the record to the byte
    walk (otherwise the CR is packed as an N and every later coordinate shifts by one)."""
    rng = np.random.default_rng(12)
    s = rng.choice(np.frombuffer(b"ACGT", np.uint8), 49).tobytes()
    lines = [s[0:10], s[10:19], s[19:29], s[29:39], s[39:49]]
    text = b">m\n" + lines[0] + b"\n" + lines[1] + b"\r\n" + b"".join(x + b"\n" for x in lines[2:])
    path = tmp_path / "mixed.fa"
    path.write_bytes(text)
    fa = cof.Fasta(path)
    assert fa.length(0) == len(s)
    assert fa.read(0).tobytes() == s
    fa.close()


def test_plan_chunks_cover_every_window_once():
    L = 23
    lengths = [0, 10, 23, 24, 100_000, 77_777]
    for cb in (None, 1, 1000, 7919, 10**6):
        chunks = search.plan_chunks(lengths, L, cb)
        for c, n in enumerate(lengths):
            starts = []
            for ch in chunks:
                if ch.chrom != c:
                    continue
                assert ch.n_bases == ch.n_owned + L - 1
                assert ch.start + ch.n_bases <= n
                starts.append((ch.start, ch.start + ch.n_owned))
            starts.sort()
            covered = sum(e - s for s, e in starts)
            assert covered == max(0, n - L + 1)
            for (s0, e0), (s1, e1) in zip(starts, starts[1:]):
                assert e0 == s1


def test_split_pieces_matches_plan_chunks():
    """Re-cutting whole-chromosome pieces gives exactly the pieces plan_chunks makes
    directly at that size (same ownership, same L-1 overlap)."""
    L = 23
    lengths = [0, 10, 23, 24, 100_000, 77_777]
    whole = [p for ch in search.plan_chunks(lengths, L, None) for p in ch.pieces]
    for cb in (1, 1000, 7919, 10**6):
        direct = [p for ch in search.plan_chunks(lengths, L, cb) for p in ch.pieces]
        assert search.split_pieces(whole, cb, L) == direct


def test_shard_lpt_assigns_each_chunk_once():
    chunks = search.plan_chunks([l for _, l in synth.HG38], 23, None)
    for world in (1, 2, 4, 8):
        shards = search.shard_lpt(chunks, world)
        flat = sorted([c for s in shards for c in s], key=lambda c: (c.chrom, c.start))
        assert flat == sorted(chunks, key=lambda c: (c.chrom, c.start))
        loads = [sum(c.n_owned for c in s) for s in shards]
        ideal = sum(loads) / world
        assert max(loads) <= max(ideal * 1.05, max(c.n_owned for c in chunks) + 1)


def test_valid_starts_plane():
    segs_rows = [(0, 0, 0, 5), (1, 10, 0, 40), (2, 60, 7, 33), (3, 100, 0, 0), (4, 200, 3, 64)]
    n = 300
    segs = cof.make_segments(segs_rows)
    vs = np.zeros(cof.cof_plane_words(n), np.uint32)
    cof.cof_valid_starts(segs, len(segs_rows), n, vs)
    bits = np.unpackbits(vs.view(np.uint8), bitorder="little")
    exp = np.zeros(len(bits), np.uint8)
    for _, off, _, owned in segs_rows:
        exp[off:off + owned] = 1
    assert np.array_equal(bits, exp)
    with pytest.raises(cof.CofError):
        cof.cof_valid_starts(cof.make_segments([(0, 290, 0, 20)]), 1, n, vs)


def test_collect_maps_multi_segment_chunks():
    """Chunk coordinates of a multi-segment chunk map back to (chromosome, position)."""
    rng = np.random.default_rng(8)
    seqs = [synth.random_genome_text(rng, n, b"ACGTacgtN", p=[.22, .22, .22, .22, .02, .02, .02, .02, .04])
            for n in (5000, 30, 7000, 4000)]
    pat = "N" * 21 + "RG"
    guides = ["".join(rng.choice(list("ACGT"), 20)) + "NNN" for _ in range(3)]
    thr = [12, 12, 12]
    ref = oracle.search(seqs, pat, guides, thr)
    chunks = search.plan_chunks([len(s) for s in seqs], 23, 2500, pack_bases=0)
    assert len(chunks) == 1 and chunks[0].multi
    ch = chunks[0]
    host = search.HostGenome(seqs, chunks, pin=False)
    segs = ch.segments()
    keys = []
    for h in ref:   # oracle record -> chunk coordinate of its window start
        c, p = int(h["chrom"]), int(h["pos"])
        off = [co + (p - so) for (cc, co, so, no) in segs if cc == c and so <= p < so + no]
        assert len(off) == 1
        keys.append((off[0] << 32) | ((1 if h["strand"] == b"-" else 0) << 31) | (int(h["guide"]) << 7) | int(h["mm"]))
    keys = np.array(keys, dtype=np.uint64)
    plan = cof.cof_plan_create(pat, guides, thr)
    got = cof.cof_collect(plan, host.chunk_struct(0), None, len(keys), host_keys=np.sort(keys))
    assert cof.hits_to_tuples(got) == oracle.hits_to_tuples(ref)


def test_plan_chunks_packed():
    L = 23
    lengths = [100_000, 10, 77_777, 5000]
    for cb, pb in ((None, 0), (7919, 0), (7919, 50_000), (None, 1)):
        chunks = search.plan_chunks(lengths, L, cb, pack_bases=pb)
        cover = {}
        for ch in chunks:
            off = 0
            for p in ch.pieces:
                cover.setdefault(p.chrom, []).append((p.chrom_off, p.chrom_off + p.n_owned))
                assert p.length == p.n_owned + L - 1 and p.chrom_off + p.length <= lengths[p.chrom]
                off += p.length
            assert ch.n_bases == off
            if pb:
                assert ch.n_bases <= pb or len(ch.pieces) == 1
        for c, n in enumerate(lengths):
            iv = sorted(cover.get(c, []))
            assert sum(e - s for s, e in iv) == max(0, n - L + 1)
            assert all(a[1] == b[0] for a, b in zip(iv, iv[1:]))


def test_path_selection_by_pam_density():
    """search.use_fused: fused from 256 guides, or when PAM sites are dense (NRG, NGG);
    the two-call path for sparse PAMs with few guides (TTTV)."""
    assert search.pam_density("N" * 21 + "RG") == pytest.approx(0.125)
    assert search.pam_density("TTTV" + "N" * 23) == pytest.approx(0.75 / 64)
    nrg = cof.cof_plan_create("N" * 21 + "RG", ["A" * 20 + "NNN"] * 3, [3] * 3)
    tttv = cof.cof_plan_create("TTTV" + "N" * 23, ["NNNN" + "A" * 23] * 3, [3] * 3)
    assert search.use_fused(nrg, 3) and not search.use_fused(tttv, 100) and search.use_fused(tttv, 300)


@pytest.mark.parametrize("n", [0, 1, 31, 32, 33, 64, 1000, 70_001])
def test_n_runs_match_numpy(n):
    """cof_n_runs: maximal N intervals of the packed nm plane, checked against numpy
    run boundaries of the canonical text (runs at 0, at the end, across words)."""
    rng = np.random.default_rng(40 + n)
    seq = synth.random_genome_text(rng, n, b"ACGTN", p=[.2, .2, .2, .2, .2]) if n else np.zeros(0, np.uint8)
    if n > 40:
        seq[:7] = ord("N")
        seq[-5:] = ord("N")
        seq[32:64] = ord("N")
    w = cof.cof_plane_words(n)
    lo, hi, nm = (np.zeros(w, np.uint32) for _ in range(3))
    cof.cof_pack(seq, n, lo, hi, nm)
    runs = cof.cof_n_runs(nm, n)
    isn = np.frombuffer(_canon(seq.tobytes()), np.uint8) == ord("N") if n else np.zeros(0, bool)
    d = np.diff(np.concatenate([[0], isn.astype(np.int8), [0]]))
    exp = np.stack([np.flatnonzero(d == 1), np.flatnonzero(d == -1)], axis=1) if n else np.zeros((0, 2))
    assert runs.shape == exp.shape and (runs == exp).all()


def test_n_runs_parallel_ranges_join():
    """A plane long enough for the threaded scan (> 2^20 words): runs that straddle the
    word-range boundaries of any thread count 2..64 come back whole."""
    n = 40_000_003
    seq = np.full(n, ord("A"), np.uint8)
    words = (n + 31) // 32
    for nt in range(2, 65):
        per = -(-words // nt)
        for t in range(1, nt):
            b = t * per * 32
            if b < n:
                seq[max(0, b - 3 - nt):b + 2 * nt] = ord("N")
    rng = np.random.default_rng(7)
    for s0 in rng.integers(0, n, 300):
        seq[s0:s0 + int(rng.integers(1, 5000))] = ord("n")
    seq[-1] = ord("N")
    w = cof.cof_plane_words(n)
    lo, hi, nm = (np.zeros(w, np.uint32) for _ in range(3))
    cof.cof_pack(seq, n, lo, hi, nm)
    runs = cof.cof_n_runs(nm, n)
    d = np.diff(np.concatenate([[0], ((seq | 0x20) == ord("n")).astype(np.int8), [0]]))
    exp = np.stack([np.flatnonzero(d == 1), np.flatnonzero(d == -1)], axis=1)
    assert runs.shape == exp.shape and (runs == exp).all()


def test_host_genome_h2d_bytes_with_runs():
    """An assembly-shaped genome (few long N runs) crosses PCIe as lo/hi + its N runs:
    about 2/3 of the plane bytes (3 planes; 1/2 of them with the valid-start plane)."""
    w = synth.make_workload("C2", scale=0.05)
    chunks = search.plan_chunks([len(s) for s in w.seqs], w.cfg.L, None, 0)
    host = search.HostGenome(w.seqs, chunks, pin=False)
    assert all(len(r) < 200 for r in host.runs)
    assert host.h2d_bytes < 0.7 * host.bytes

"""UCSC .2bit reader: planes from cof_2bit_pack equal cof_pack of the
same ASCII bases; the file is written here by an independent writer following the UCSC
format description (header, index, N / mask blocks, 4 bases per byte, T=0 C=1 A=2 G=3)."""
import struct

import numpy as np
import pytest

from paper_conf_socc_jinv23_b200 import cli, cof, synth

CODE = {"T": 0, "C": 1, "A": 2, "G": 3}


def runs(mask):
    """(start, size) runs of True in a bool array."""
    out = []
    i, n = 0, len(mask)
    while i < n:
        if mask[i]:
            j = i
            while j < n and mask[j]:
                j += 1
            out.append((i, j - i))
            i = j
        else:
            i += 1
    return out


def write_2bit(path, names, seqs, big_endian=False, version=0):
    e = ">" if big_endian else "<"
    recs = []
    for s in seqs:
        txt = bytes(s).decode() if not isinstance(s, str) else s
        up = txt.upper()
        nmask = np.array([c not in "ACGT" for c in up], dtype=bool)
        lmask = np.array([c.islower() for c in txt], dtype=bool)
        nb, mb = runs(nmask), runs(lmask)
        packed = bytearray()
        for k in range(0, len(up), 4):
            byte = 0
            for j in range(4):
                c = up[k + j] if k + j < len(up) else "T"
                byte |= CODE.get(c, 0) << (6 - 2 * j)
            packed.append(byte)
        body = struct.pack(e + "II", len(up), len(nb))
        body += b"".join(struct.pack(e + "I", a) for a, _ in nb) + b"".join(struct.pack(e + "I", z) for _, z in nb)
        body += struct.pack(e + "I", len(mb))
        body += b"".join(struct.pack(e + "I", a) for a, _ in mb) + b"".join(struct.pack(e + "I", z) for _, z in mb)
        body += struct.pack(e + "I", 0) + bytes(packed)
        recs.append(body)
    osz = 8 if version == 1 else 4
    index_len = sum(1 + len(nm) + osz for nm in names)
    off = 16 + index_len
    hdr = struct.pack(e + "IIII", 0x1A412743, version, len(names), 0)
    idx = b""
    for nm, body in zip(names, recs):
        idx += bytes([len(nm)]) + nm.encode() + struct.pack(e + ("Q" if version == 1 else "I"), off)
        off += len(body)
    with open(path, "wb") as f:
        f.write(hdr + idx + b"".join(recs))


def planes_of(ascii_bytes):
    n = len(ascii_bytes)
    w = cof.cof_plane_words(n)
    p = np.zeros((3, w), np.uint32)
    cof.cof_pack(np.frombuffer(ascii_bytes, np.uint8).copy(), n, p[0], p[1], p[2])
    return p


@pytest.mark.parametrize("big_endian,version", [(False, 0), (True, 0), (False, 1)])
def test_2bit_pack_equals_ascii_pack(tmp_path, big_endian, version):
    rng = np.random.default_rng(5)
    seqs = [bytes(synth.random_genome_text(rng, n, b"ACGTacgtN", p=[.2, .2, .2, .2, .04, .04, .04, .04, .04]))
            for n in (1, 3, 4, 33, 1000, 70_001)]
    seqs[-1] = seqs[-1][:500] + b"N" * 3000 + seqs[-1][3500:]
    names = [f"s{i}" for i in range(len(seqs))]
    path = tmp_path / "g.2bit"
    write_2bit(path, names, seqs, big_endian, version)
    tb = cof.TwoBit(path)
    assert len(tb) == len(seqs)
    for i, s in enumerate(seqs):
        assert tb.name(i) == names[i] and tb.length(i) == len(s)
        ranges = [(0, len(s))] + [tuple(sorted(rng.integers(0, len(s) + 1, 2))) for _ in range(6)]
        for a, b in ranges:
            n = b - a
            w = cof.cof_plane_words(n)
            got = np.zeros((3, w), np.uint32)
            tb.pack(i, a, n, got[0], got[1], got[2])
            exp = planes_of(bytes(s[a:b]))
            assert np.array_equal(got, exp), (i, a, b)
        assert bytes(tb.read(i)) == bytes(s).upper()


def test_2bit_rejects_bad_files(tmp_path):
    p = tmp_path / "bad.2bit"
    p.write_bytes(b"\x00" * 32)
    with pytest.raises(cof.CofError):
        cof.TwoBit(p)
    write_2bit(tmp_path / "ok.2bit", ["a"], [b"ACGTACGT"])
    raw = (tmp_path / "ok.2bit").read_bytes()
    (tmp_path / "trunc.2bit").write_bytes(raw[:-1])
    with pytest.raises(cof.CofError):
        cof.TwoBit(tmp_path / "trunc.2bit")
    tb = cof.TwoBit(tmp_path / "ok.2bit")
    z = np.zeros((3, 8), np.uint32)
    with pytest.raises(cof.CofError):
        tb.pack(0, 4, 5, z[0], z[1], z[2])


@pytest.mark.gpu
def test_cli_with_2bit_genome(tmp_path):
    from oracle import oracle
    rng = np.random.default_rng(41)
    seqs = [bytes(synth.random_genome_text(rng, n, b"ACGTacgtN", p=[.23, .2, .2, .23, .03, .03, .03, .03, .02]))
            for n in (30_000, 9_999)]
    names = ["chrX", "chrY"]
    write_2bit(tmp_path / "genome.2bit", names, seqs)
    guides = ["".join(rng.choice(list("ACGT"), 20)) + "NNN" for _ in range(4)]
    inp = tmp_path / "input.txt"
    inp.write_text("genome.2bit\n" + "N" * 21 + "RG\n" + "".join(f"{g} 8\n" for g in guides))
    out = tmp_path / "out.txt"
    assert cli.main([str(inp), "G", str(out)]) == 0
    ref = oracle.search(seqs, "N" * 21 + "RG", guides, [8] * 4)
    assert len(ref) > 5
    assert out.read_text() == cli.format_hits(
        np.array([(h["guide"], h["chrom"], h["pos"], h["strand"], h["mm"], h["site"]) for h in ref],
                 dtype=cof.HIT_DTYPE), guides, names)

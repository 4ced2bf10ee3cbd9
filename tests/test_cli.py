"""Cas-OFFinder-style input file / TSV output."""
import os

import numpy as np
import pytest

from oracle import oracle
from paper_conf_socc_jinv23_b200 import cli, cof, synth


def test_parse_input(tmp_path):
    spec = cli.parse_input("genome.fa\nNNNNNRG\nACGTANN 1\n# comment\nTTTTTNN 0\n", str(tmp_path))
    assert spec.genome == os.path.join(str(tmp_path), "genome.fa")
    assert spec.pattern == "NNNNNRG" and spec.queries == ["ACGTANN", "TTTTTNN"] and spec.thresholds == [1, 0]
    for bad in ("g\nNNRG\n", "g\nNNRG\nACG 1\n", "g\nNNRG\nACGT\n", "g\nNNRG\nACGT -1\n"):
        with pytest.raises(ValueError):
            cli.parse_input(bad)


def test_format_hits():
    h = np.zeros(2, dtype=cof.HIT_DTYPE)
    h[0] = (1, 0, 12, b"+", 2, b"ACgTaGG")
    h[1] = (0, 1, 7, b"-", 0, b"ACGTAGG")
    txt = cli.format_hits(h, ["Q0NNNNN", "Q1NNNNN"], ["chrA", "chrB"])
    assert txt == "Q1NNNNN\tchrA\t12\tACgTaGG\t+\t2\nQ0NNNNN\tchrB\t7\tACGTAGG\t-\t0\n"


@pytest.mark.gpu
def test_cli_end_to_end(tmp_path):
    rng = np.random.default_rng(31)
    seqs = [synth.random_genome_text(rng, n, b"ACGTacgtN", p=[.23, .2, .2, .23, .03, .03, .03, .03, .02])
            for n in (40_000, 25_001, 500)]
    names = ["chr1", "chr2", "chrM"]
    gdir = tmp_path / "genome"
    gdir.mkdir()
    synth.write_fasta(gdir / "a.fa", names[:2], seqs[:2])
    synth.write_fasta(gdir / "b.fa", names[2:], seqs[2:], width=70)
    guides = ["".join(rng.choice(list("ACGT"), 20)) + "NNN" for _ in range(5)]
    inp = tmp_path / "input.txt"
    inp.write_text("genome\n" + "N" * 21 + "RG\n" + "".join(f"{g} 9\n" for g in guides))
    out = tmp_path / "out.txt"
    assert cli.main([str(inp), "G", str(out), "--chunk-bases", "9999"]) == 0
    ref = oracle.search(seqs, "N" * 21 + "RG", guides, [9] * 5)
    exp = "".join(f"{guides[int(h['guide'])]}\t{names[int(h['chrom'])]}\t{int(h['pos'])}\t{h['site'].decode()}\t"
                  f"{h['strand'].decode()}\t{int(h['mm'])}\n" for h in ref)
    assert len(ref) > 10
    assert out.read_text() == exp
    # --gpus 2: one pipeline per GPU (both on the one GPU of the test box), same TSV
    out2 = tmp_path / "out2.txt"
    assert cli.main([str(inp), "G", str(out2), "--chunk-bases", "7777", "--gpus", "2"]) == 0
    assert out2.read_text() == exp


def test_parse_input_bulges():
    spec = cli.parse_input("genome.fa\nNNNNNRG 2 1\nACGTANN 1\n")
    assert (spec.dna_bulge, spec.rna_bulge) == (2, 1)
    assert cli.parse_input("g\nNNRG\nACGN 0\n").dna_bulge == 0
    with pytest.raises(ValueError):
        cli.parse_input("g\nNNRG -1 0\nACGN 0\n")


@pytest.mark.gpu
def test_cli_bulge_end_to_end(tmp_path):
    from oracle import bulge as obulge
    rng = np.random.default_rng(32)
    seqs = [synth.random_genome_text(rng, n) for n in (30_000, 12_345)]
    names = ["chrA", "chrB"]
    synth.write_fasta(tmp_path / "g.fa", names, seqs)
    guides = ["".join(rng.choice(list("ACGT"), 20)) + "NNN" for _ in range(3)]
    inp = tmp_path / "input.txt"
    inp.write_text("g.fa\n" + "N" * 21 + "RG 1 1\n" + "".join(f"{g} 5\n" for g in guides))
    out = tmp_path / "out.txt"
    assert cli.main([str(inp), "G", str(out)]) == 0
    ref = obulge.search(seqs, "N" * 21 + "RG", guides, [5] * 3, 1, 1)
    kinds = {b"X": "X", b"D": "DNA", b"R": "RNA"}
    exp = "".join(f"{guides[int(h['guide'])]}\t{names[int(h['chrom'])]}\t{int(h['pos'])}\t{h['site'].decode()}\t"
                  f"{h['strand'].decode()}\t{int(h['mm'])}\t{kinds[h['kind']]}\t{int(h['size'])}\t{int(h['bpos'])}\n"
                  for h in ref)
    assert len(ref) > 0
    assert out.read_text() == exp


def test_format_hits_long():
    """cof_hit64 records (L > 32) format like cof_hit ones."""
    h = np.zeros(1, dtype=cof.HIT64_DTYPE)
    site = b"ACGT" * 9 + b"AgG"
    h[0]["guide"], h[0]["chrom"], h[0]["pos"], h[0]["strand"], h[0]["mm"], h[0]["site"] = 0, 0, 5, b"-", 1, site
    txt = cli.format_hits(h, ["Q" * 39], ["chrA"])
    assert txt == "Q" * 39 + "\tchrA\t5\t" + site.decode() + "\t-\t1\n"


@pytest.mark.gpu
def test_cli_long_pattern_end_to_end(tmp_path):
    """A 40-letter pattern (two-word windows) through the CLI: .2bit-free FASTA input,
    TSV output equal to the oracle's."""
    rng = np.random.default_rng(33)
    seqs = [synth.random_genome_text(rng, n, b"ACGTacgtN", p=[.23, .2, .2, .23, .03, .03, .03, .03, .02])
            for n in (60_000, 9_001)]
    names = ["chr1", "chr2"]
    synth.write_fasta(tmp_path / "g.fa", names, seqs)
    pat = "N" * 38 + "GG"
    guides = ["".join(rng.choice(list("ACGT"), 37)) + "NNN" for _ in range(4)]
    inp = tmp_path / "input.txt"
    inp.write_text("g.fa\n" + pat + "\n" + "".join(f"{g} 21\n" for g in guides))
    out = tmp_path / "out.txt"
    assert cli.main([str(inp), "G", str(out)]) == 0
    ref = oracle.search(seqs, pat, guides, [21] * 4)
    exp = "".join(f"{guides[int(h['guide'])]}\t{names[int(h['chrom'])]}\t{int(h['pos'])}\t{h['site'].decode()}\t"
                  f"{h['strand'].decode()}\t{int(h['mm'])}\n" for h in ref)
    assert len(ref) > 10
    assert out.read_text() == exp

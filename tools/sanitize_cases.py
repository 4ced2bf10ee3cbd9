"""Small searches that launch every kernel of libcof.so once or more, for the CUDA
sanitizers (memcheck, racecheck, synccheck, initcheck):

    compute-sanitizer --tool <tool> python tools/sanitize_cases.py

Covers the single pass (uniform-threshold concrete kernel and the generic one, several
launches, multi-segment chunks), the masks path (finder pass 1 + mask-expanding
comparer), the two-call path (cooperative finder with dense and sparse pass 2 + pair-
table comparer), long patterns (WIDE finder, W64 comparer), the loads (full copy, N-run
rebuild, split), the radix sort and device decoration.  Every result is checked against
the CPU oracle (test infrastructure), so a sanitizer run is also a parity run."""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

from oracle import oracle  # noqa: E402
from paper_conf_socc_jinv23_b200 import cof, search, synth  # noqa: E402


def check(name, got, seqs, pat, guides, thr):
    exp = oracle.hits_to_tuples(oracle.search(seqs, pat, guides, thr))
    g = cof.hits_to_tuples(got)
    status = "ok" if g == exp else "MISMATCH"
    print(f"{name}: {len(g)} hits ({status})", flush=True)
    if g != exp:
        raise SystemExit(1)


def main():
    import torch
    rng = np.random.default_rng(2024)
    seqs = [synth.random_genome_text(rng, n, b"ACGTacgtNnRy", p=[.23, .17, .17, .23, .04, .04, .04, .04, .02, .01,
                                                                .005, .005]) for n in (5, 70_001, 33_333)]
    s1 = seqs[1]
    spc = "N" * 21 + "RG"
    g20 = ["".join(rng.choice(list("ACGT"), 20)) + "NNN" for _ in range(40)]
    for gi, g in enumerate(g20[:10]):
        s1[500 + gi * 901: 500 + gi * 901 + 23] = np.frombuffer((g[:20] + "AGG").encode(), np.uint8)
    # single pass: uniform thresholds (concrete kernel), per-guide thresholds (generic), one chunk
    # and packed pieces (multi-segment: vs plane)
    check("single uniform", search.search(seqs, spc, g20, [6] * 40, path="single"), seqs, spc, g20, [6] * 40)
    thr = [int(x) for x in rng.integers(2, 8, 40)]
    check("single generic packed", search.search(seqs, spc, g20, thr, path="single", chunk_bases=9973,
                                                 pack_bases=30_000), seqs, spc, g20, thr)
    deg = ["RYNNKMSWACGTACGTACGTNNN", "ACGTACGTACGTACGTACGTNNN"]
    check("single degenerate", search.search(seqs, spc, deg, [8, 5], path="single"), seqs, spc, deg, [8, 5])
    # masks path and two-call path (dense NRG: CTA pass 2; sparse TTTV: warp pass 2)
    check("fused masks", search.search(seqs, spc, g20, [6] * 40, path="fused"), seqs, spc, g20, [6] * 40)
    check("two-call dense", search.search(seqs, spc, g20, [6] * 40, path="twocall", pack_bases=0), seqs, spc, g20,
          [6] * 40)
    c12 = "TTTV" + "N" * 23
    g23 = ["NNNN" + "".join(rng.choice(list("ACGT"), 23)) for _ in range(8)]
    check("two-call sparse", search.search(seqs, c12, g23, [5] * 8, path="twocall"), seqs, c12, g23, [5] * 8)
    check("single cas12a", search.search(seqs, c12, g23, [5] * 8, path="single"), seqs, c12, g23, [5] * 8)
    # long patterns: WIDE finder + W64 comparer (L = 40)
    lp = "N" * 38 + "GG"
    g40 = ["N" + "".join(rng.choice(list("ACGT"), 36)) + "NNN" for _ in range(4)]
    check("long L=40", search.search(seqs, lp, g40, [9] * 4), seqs, lp, g40, [9] * 4)
    # the pipelined host path (H2D with N-run rebuild, device decoration, D2H) over several chunks
    host = search.HostGenome(seqs, search.plan_chunks([len(s) for s in seqs], 23, 20_011))
    srch = search.Searcher(spc, g20, [6] * 40)
    check("search_host pipeline", srch.search_host(host), seqs, spc, g20, [6] * 40)
    os.environ["COF_SPLIT_FILL"] = "1"
    search.SPLIT_FILL = True
    check("search_host split fill", srch.search_host(host), seqs, spc, g20, [6] * 40)
    torch.cuda.synchronize()
    print("all cases ok")


if __name__ == "__main__":
    main()

"""Stress the one-pass finder (cof_find_pam): repeated launches on an idle GPU and next to a
busy stream; every result is checked against the CPU oracle's PAM sites."""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from oracle import oracle  # noqa: E402
from paper_conf_socc_jinv23_b200 import cof, search, synth  # noqa: E402


def main():
    rng = np.random.default_rng(9)
    seq = synth.random_genome_text(rng, 3_000_000, b"ACGTN", p=[.24, .24, .24, .24, .04])
    bad = 0
    for pat in ("TTTV" + "N" * 23, "N" * 21 + "RG"):
        L = len(pat)
        srch = search.Searcher(pat, ["N" * L], [0])
        host = search.HostGenome([seq], search.plan_chunks([len(seq)], L))
        srch.fused = False
        srch.reserve(host.chunks[0].n_bases, 1 << 16)
        dch = srch.device_chunk(host.chunks[0])
        cof.cof_load_chunk(host.chunk_struct(0), dch, srch.stream)
        n = host.chunks[0].n_owned
        exp = [oracle.pam_sites(seq, pat, st, 0, n) for st in "+-"]
        busy = torch.cuda.Stream()
        a = torch.randn(8192, 8192, device="cuda", dtype=torch.bfloat16)
        for it in range(60):
            if it % 2:
                with torch.cuda.stream(busy):
                    for _ in range(4):
                        a = (a @ a).clamp_(-1, 1)
            got = cof.cof_find_pam(srch.plan, srch.plan_dev, dch, srch.d_find_ws, srch.d_items[0], srch.d_items[1], n,
                                   srch.stream)
            ok = got == (len(exp[0]), len(exp[1]))
            if ok:
                for k in range(2):
                    g = srch.d_items[k][: got[k]].cpu().numpy().astype(np.int64)
                    ok &= np.array_equal(g, exp[k])
            if not ok:
                bad += 1
                print(f"{pat} it {it}: got {got} expected {(len(exp[0]), len(exp[1]))}")
        torch.cuda.synchronize()
        print(pat, "done, bad so far", bad, flush=True)
    print("BAD", bad)


if __name__ == "__main__":
    main()

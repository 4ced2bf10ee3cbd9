"""Multi-GPU product paths (north_star: chromosomes or fixed-size chunks
sharded over the GPUs, the host merging the per-GPU hit lists) on the one GPU of the test
box: two pipelines (search_multi: one host thread per GPU, shared chunk queue) or two
torchrun ranks (search_dist: LPT shards, merge_dist through shared memory) share it.
The merged list must equal the oracle's element by element, and at full size the
single-GPU bench pipeline's list."""
import os
import socket
import subprocess
import sys

import numpy as np
import pytest

from oracle import oracle
from paper_conf_socc_jinv23_b200 import cof, search, synth

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def ref_hits(w, ranges=None):
    return oracle.hits_to_tuples(oracle.search(w.seqs, w.cfg.pattern, w.guides, w.thresholds, ranges=ranges))


@pytest.mark.parametrize("name,scale,chunk,ng", [("C3", 0.004, 500_003, None), ("C5", 0.002, 300_007, 200),
                                                 ("C4", 0.004, 700_001, None), ("X1", 0.03, 400_009, None)])
def test_search_multi_two_pipelines_one_gpu(name, scale, chunk, ng):
    w = synth.make_workload(name, scale=scale, n_guides=ng)
    exp = ref_hits(w)
    assert len(exp) > 10
    got = search.search_multi(w.seqs, w.cfg.pattern, w.guides, w.thresholds, devices=["cuda:0", "cuda:0"],
                              chunk_bases=chunk)
    assert cof.hits_to_tuples(got) == exp
    # three pipelines and one-chunk-per-chromosome work units give the same list
    got3 = search.search_multi(w.seqs, w.cfg.pattern, w.guides, w.thresholds, devices=["cuda:0"],
                               streams_per_device=3, chunk_bases=None)
    assert cof.hits_to_tuples(got3) == exp


def _port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


@pytest.mark.parametrize("name,scale,chunk,ng", [("C3", 0.004, 400_009, None), ("C5", 0.002, 250_007, 300)])
def test_search_dist_two_ranks_one_gpu(tmp_path, name, scale, chunk, ng):
    """torchrun, world size 2 (gloo; both ranks on cuda:0): LPT shards of the chunks, per-rank
    search_host, merge_dist (per-chunk counts -> offsets -> each rank writes its slices of
    one shared-memory file) == the oracle, record by record."""
    out = tmp_path / "merged.npy"
    env = dict(os.environ, COF_DIST_BACKEND="gloo")
    args = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node=2",
            "--master-addr=127.0.0.1", f"--master-port={_port()}", os.path.join(ROOT, "tests", "dist_worker.py"),
            name, str(scale), str(chunk), str(out)] + ([str(ng)] if ng else [])
    r = subprocess.run(args, cwd=ROOT, capture_output=True, text=True, timeout=900, env=env)
    assert r.returncode == 0, r.stderr[-3000:]
    w = synth.make_workload(name, scale=scale, n_guides=ng)
    got = np.load(out)
    exp = ref_hits(w)
    assert len(exp) > 10
    assert cof.hits_to_tuples(got) == exp


def test_search_multi_full_size_equals_single_gpu():
    """C3 at full size (3.09 Gbp, 100 guides): two pipelines over 64 Mbp work units give
    exactly the single-GPU bench pipeline's list (the whole genome as one chunk); sampled
    window ranges are recomputed by the oracle."""
    from bench import prepare_workload, run_device_pipeline
    wl, st = prepare_workload("C3")
    one = run_device_pipeline(wl, st, collect=True)
    del st
    cfg = wl.cfg
    multi = search.search_multi(wl.seqs, cfg.pattern, wl.guides, wl.thresholds, devices=["cuda:0", "cuda:0"])
    assert len(multi) == len(one) and len(one) > 10**6
    for f in ("chrom", "pos", "strand", "guide", "mm", "site"):
        assert (multi[f] == one[f]).all(), f
    rng = np.random.default_rng(5)
    for c in rng.choice(len(wl.seqs), 4, replace=False):
        n = len(wl.seqs[c])
        s0 = int(rng.integers(0, n - 100_000))
        ranges = [(0, 0)] * len(wl.seqs)
        ranges[c] = (s0, s0 + 50_000)
        h = multi[(multi["chrom"] == c) & (multi["pos"] >= s0) & (multi["pos"] < s0 + 50_000)]
        assert cof.hits_to_tuples(h) == ref_hits(wl, ranges)


def test_finder_grid_exchange_next_to_a_busy_stream():
    """The two-call finder's grid-wide exchange runs under a cooperative launch (every CTA
    co-resident); with another stream keeping SMs busy (back-to-back GEMMs) it must still
    finish and give the same ordered item lists as when the GPU is idle."""
    import torch
    rng = np.random.default_rng(9)
    seq = synth.random_genome_text(rng, 3_000_000, b"ACGTN", p=[.24, .24, .24, .24, .04])
    pat = "TTTV" + "N" * 23                       # sparse PAM
    guides = ["NNNN" + "".join(rng.choice(list("ACGT"), 23)) for _ in range(4)]
    srch = search.Searcher(pat, guides, [5] * 4)
    srch.fused = False            # the two-call path: item lists sized for cof_find_pam
    host = search.HostGenome([seq], search.plan_chunks([len(seq)], len(pat)))
    srch.reserve(host.chunks[0].n_bases, 1 << 16)
    dch = srch.device_chunk(host.chunks[0])
    cof.cof_load_chunk(host.chunk_struct(0), dch, srch.stream)
    n = host.chunks[0].n_owned
    ref = cof.cof_find_pam(srch.plan, srch.plan_dev, dch, srch.d_find_ws, srch.d_items[0], srch.d_items[1], n,
                           srch.stream)
    ref_items = [srch.d_items[k][: ref[k]].clone() for k in range(2)]
    busy = torch.cuda.Stream()
    a = torch.randn(8192, 8192, device="cuda", dtype=torch.bfloat16)
    with torch.cuda.stream(busy):
        for _ in range(20):
            a = (a @ a).clamp_(-1, 1)
    got = cof.cof_find_pam(srch.plan, srch.plan_dev, dch, srch.d_find_ws, srch.d_items[0], srch.d_items[1], n,
                           srch.stream)
    torch.cuda.synchronize()
    assert got == ref and ref[0] > 1000
    for k in range(2):
        assert torch.equal(srch.d_items[k][: got[k]], ref_items[k])

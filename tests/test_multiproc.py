"""World-size-2 (gloo, CPU) test of the multi-GPU host logic: LPT sharding of chunks over
ranks, per-rank independent search, merge on rank 0 == single-process search.  The
per-rank search is the oracle here (no GPU on this box); the sharding and merge code is
the product's (search.shard_indices / merge_dist / gather_and_merge / cof_merge).  The
GPU twins are in tests/test_gpu_multi.py."""
import os
import socket

import numpy as np
import pytest
import torch.distributed as dist
import torch.multiprocessing as mp

from oracle import oracle
from paper_conf_socc_jinv23_b200 import cof, search, synth


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _oracle_chunk_hits(wl, ch):
    cfg = wl.cfg
    ranges = [(0, 0)] * len(wl.seqs)
    ranges[ch.chrom] = (ch.start, ch.start + ch.n_owned)
    h = oracle.search(wl.seqs, cfg.pattern, wl.guides, wl.thresholds, ranges=ranges)
    out = np.zeros(len(h), dtype=cof.hit_dtype(cfg.L))
    for f in ("guide", "chrom", "pos", "strand", "mm", "site"):
        out[f] = h[f]
    return out


def _worker(rank, world, port, q, name="C3"):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    wl = synth.make_workload(name, scale=0.0005 if name == "C3" else 0.003, n_guides=8)
    chunks = search.plan_chunks([len(s) for s in wl.seqs], wl.cfg.L, 40_000)
    # the product's merge (merge_dist): per-chunk lists of this rank's LPT share -> offsets
    # from the summed per-chunk counts -> slices of one shared-memory file
    mine = search.shard_indices(chunks, world)[rank]
    per = {i: _oracle_chunk_hits(wl, chunks[i]) for i in mine}
    merged = search.merge_dist(per, len(chunks), cof.hit_dtype(wl.cfg.L))
    # the older per-rank-list gather (host objects) gives the same list
    local = search.merge_hit_lists([per[i] for i in mine], cof.hit_dtype(wl.cfg.L))
    merged2 = search.gather_and_merge(local)
    if rank == 0:
        ref = oracle.search(wl.seqs, wl.cfg.pattern, wl.guides, wl.thresholds)
        q.put((cof.hits_to_tuples(merged), oracle.hits_to_tuples(ref), len(mine), len(chunks),
               cof.hits_to_tuples(merged2)))
    else:
        assert merged is None and merged2 is None
        q.put(("rank1", len(mine)))
    dist.destroy_process_group()


@pytest.mark.parametrize("name", ["C3", "X1"])
def test_two_rank_shard_gather_merge(name):
    """C3 (cof_hit records) and X1 (L = 40: cof_hit64 records, cof_merge64)."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker, args=(r, 2, port, q, name)) for r in range(2)]
    for p in ps:
        p.start()
    res = [q.get(timeout=300) for _ in range(2)]
    for p in ps:
        p.join(timeout=60)
        assert p.exitcode == 0
    r0 = [r for r in res if r[0] != "rank1"][0]
    r1 = [r for r in res if r[0] == "rank1"][0]
    got, exp, n0, n_all, got2 = r0
    assert got == exp and len(exp) > 0
    assert got2 == exp
    assert n0 + r1[1] == n_all and n0 > 0 and r1[1] > 0


def test_chunk_queue_hands_out_each_index_once():
    import threading
    qq = search.ChunkQueue(5000)
    seen = []
    lock = threading.Lock()

    def pop():
        for i in qq:
            with lock:
                seen.append(i)

    ts = [threading.Thread(target=pop) for _ in range(6)]
    for t in ts:
        t.start()
    for t in ts:
        t.join()
    assert sorted(seen) == list(range(5000))

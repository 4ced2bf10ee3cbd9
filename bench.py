"""Benchmark of the B200 Cas-OFFinder hot path (bench contract: one JSON line on rank 0).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config C5] [--impl ours|reference]

One *step* = one pass of the whole hot path over the synthetic genome: the rank's
chromosomes as one chunk through the finder, the comparer, the device hit sort and the
device decoration into output records (SURVEY.md §8(a) rows a3-a7 on the device; a1 pack,
a2 H2D and the D2H of the records are outside ``value`` because the inputs are resident
in HBM, and inside ``e2e``).  ``value`` = genome bases of the whole job /
max-over-ranks device time; comparisons/s are reported beside it.  Multi-GPU: chunks
are LPT-sharded over ranks (no collective on the data path), strong scaling.

``e2e`` runs the same search through the public API from pinned HOST planes every step:
cof_load_chunk (H2D) -> find -> compare -> sort -> cof_collect (D2H + decorate) ->
cof_merge.  ``--impl reference`` times the CPU oracle (the only other program that
computes this path) on a bounded sample of the same workload.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

from paper_conf_socc_jinv23_b200 import synth  # noqa: E402


E2E_CHUNK_BASES = int(os.environ.get("COF_E2E_CHUNK_BASES", 250_000_000))  # e2e: pieces packed into chunks of <= this
# e2e: chromosomes cut into pieces of <= this many window starts first (0 = whole chromosomes)
E2E_PIECE_BASES = int(os.environ.get("COF_E2E_PIECE_BASES", 0))
E2E_FIRST_BASES = int(os.environ.get("COF_E2E_FIRST_BASES", 0))   # e2e: first chunk <= this (0: no limit)
SHARD_PIECE_BASES = 16_000_000   # N > 1: chromosome pieces LPT-assigned to ranks
RESIDENT_CHUNK_BASES = int(os.environ.get("COF_RESIDENT_CHUNK_BASES", 800_000_000))   # e2e_resident chunks


def _peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            return json.load(f), "measured"
    except Exception:
        return {"hbm_gbs": 6650.0, "sm_max_mhz": 1965.0}, "fallback"


# ----------------------------------------------------------------------------- clocks
class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled every 100 ms during the timed region."""

    FIELDS = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,"
              "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
              "clocks_event_reasons.sw_power_cap")

    def __init__(self, index):
        self.index = index
        self.proc = None
        self.lines = []

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.FIELDS}", "--format=csv,noheader,nounits",
                 "-lms", "100"], stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.thread = threading.Thread(target=self._read, daemon=True)
            self.thread.start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        self.thread.join(timeout=2)
        sm, mx, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            parts = [p.strip() for p in ln.split(",")]
            if len(parts) < 6:
                continue
            try:
                sm.append(float(parts[0]))
                mx.append(float(parts[1]))
            except ValueError:
                continue
            for nme, v in zip(names, parts[2:6]):
                if v.lower().startswith("active"):
                    reasons.add(nme)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(sm),
                "window": "warm-up (>= W steps and >= 0.5 s) + timed region, every 100 ms"}


# ----------------------------------------------------------------------------- workload
def prepare_workload(name: str, scale: float = 1.0, chunks=None, device=None, wl=None, query=None, n_guides=None):
    """Synthetic workload + the device state the timed step runs on: resident planes of
    every chunk, one plan_dev per chunk (its counters), shared item buffers, per-chunk
    hit buffers sized from a first (untimed) pass.  ``wl``: reuse a generated workload;
    ``query``: (pattern, guides, thresholds) replacing the workload's (bulge variants)."""
    import torch
    from paper_conf_socc_jinv23_b200 import cof, search

    if wl is None:
        wl = synth.make_workload(name, scale=scale, threads=max(1, min(16, os.cpu_count() or 1)), n_guides=n_guides)
    pattern, guides, thresholds = query if query is not None else (wl.cfg.pattern, wl.guides, wl.thresholds)
    L = len(pattern)
    if chunks is None:   # the whole genome as one multi-segment chunk (the bench's default)
        chunks = [search.pack_shard(search.plan_chunks([len(s) for s in wl.seqs], L, None))]
    st = type("State", (), {})()
    st.device = device or torch.device("cuda", torch.cuda.current_device())
    st.stream = torch.cuda.current_stream(st.device)
    st.chunks = chunks
    st.plan = cof.cof_plan_create(pattern, guides, thresholds)
    st.n_guides = len(guides)
    nbytes = cof.cof_plan_device_bytes(st.plan)
    st.host = search.HostGenome(wl.seqs, chunks)
    st.d_planes, st.d_chunks, st.plan_devs = [], [], []
    for i, ch in enumerate(chunks):
        d = st.host.planes[i].to(st.device, non_blocking=True)
        st.d_planes.append(d)
        if ch.multi:
            st.d_chunks.append(cof.make_chunk(0, 0, ch.n_bases, ch.n_owned, d[0], d[1], d[2], d[3], st.host.segs[i]))
        else:
            st.d_chunks.append(cof.make_chunk(ch.chrom, ch.start, ch.n_bases, ch.n_owned, d[0], d[1], d[2]))
        pd = torch.empty(nbytes + 256, dtype=torch.uint8, device=st.device)
        cof.cof_plan_upload(st.plan, pd, st.stream)
        st.plan_devs.append(pd)
    max_owned = max(ch.n_owned for ch in chunks)
    # fused find+compare (finder masks -> comparer, no item lists) unless the guide table is
    # too large for it or COF_FUSED=0; the two-call path writes / reads ordered item lists
    st.path_name = search.choose_path(st.plan, len(guides))   # single pass / fused masks / two-call
    st.fused = st.path_name != "twocall"
    st.items = torch.empty((2, 1 if st.fused else max_owned), dtype=torch.int32, device=st.device)
    st.find_ws = torch.empty(cof.cof_find_compare_workspace_bytes(max(ch.n_bases for ch in chunks)),
                             dtype=torch.uint8, device=st.device)
    # first pass with host counts: exact item / hit counts per chunk
    st.counts = []
    tmp_cap = 1 << 20
    tmp_hits = torch.empty(tmp_cap, dtype=torch.int64, device=st.device)
    for i, ch in enumerate(chunks):
        try:
            if st.path_name == "single":
                nh = cof.cof_search_single(st.plan, st.plan_devs[i], st.d_chunks[i], st.find_ws, tmp_hits, tmp_cap,
                                           st.stream)
            elif st.fused:
                cof.cof_find_masks(st.plan, st.plan_devs[i], st.d_chunks[i], st.find_ws, st.stream)
                nh = cof.cof_compare_masks(st.plan, st.plan_devs[i], st.d_chunks[i], st.find_ws, tmp_hits, tmp_cap,
                                           st.stream)
            else:
                nf, nr = cof.cof_find_pam(st.plan, st.plan_devs[i], st.d_chunks[i], st.find_ws, st.items[0],
                                          st.items[1], max_owned, st.stream)
                nh = cof.cof_compare(st.plan, st.plan_devs[i], st.d_chunks[i], st.items[0], nf, st.items[1], nr,
                                     tmp_hits, tmp_cap, st.stream)
        except cof.CofError as e:
            if e.status != cof.COF_E_CAPACITY:
                raise
        nf, nr, nh = cof.cof_read_counts(st.plan, st.plan_devs[i], st.stream)
        st.counts.append((nf, nr, nh))
    del tmp_hits
    st.caps = [max(1024, int(c[2] * 1.1) + 1024) for c in st.counts]
    st.hits = [torch.empty(c, dtype=torch.int64, device=st.device) for c in st.caps]
    st.tmp = torch.empty(max(st.caps), dtype=torch.int64, device=st.device)
    st.sort_ws = torch.empty(cof.cof_sort_workspace_bytes(max(st.caps)), dtype=torch.uint8, device=st.device)
    # device decoration (the device half of a7 collect): records per chunk
    st.recs = [torch.empty(c * cof.hit_dtype(st.plan.L).itemsize, dtype=torch.uint8, device=st.device) for c in st.caps]
    st.dec_ws = torch.empty((len(chunks), cof.cof_decorate_workspace_bytes(max(len(ch.pieces) for ch in chunks))),
                            dtype=torch.uint8, device=st.device)
    st.max_owned = max_owned
    torch.cuda.synchronize(st.device)
    return wl, st


GRAPH_STEP_MS = 1.0   # steps shorter than this (eager) are timed as CUDA-graph replays


def capture_step(wl, st):
    """One device step captured into a CUDA graph on a side stream (every call of the step
    is asynchronous, counts stay on the device).  Returns (graph, kernels per step)."""
    import torch
    from paper_conf_socc_jinv23_b200 import cof
    g = torch.cuda.CUDAGraph()
    s0 = st.stream
    cs = torch.cuda.Stream(st.device)
    cs.wait_stream(s0)
    n0 = cof.cof_launch_count()
    try:
        with torch.cuda.graph(g, stream=cs):
            st.stream = torch.cuda.current_stream(st.device)
            run_device_pipeline(wl, st)
    finally:
        st.stream = s0
    s0.wait_stream(cs)
    return g, cof.cof_launch_count() - n0


def run_device_pipeline(wl, st, collect=False, events=None, fevents=None):
    """One step on the device: per chunk find -> compare -> sort, counts kept on the
    device (no host round trip between kernels).  ``events`` / ``fevents``: lists to append
    (start, end) CUDA event pairs bracketing each comparer / finder call.  With ``collect``
    returns the merged, decorated hit array (cof_collect + cof_merge)."""
    import torch
    from paper_conf_socc_jinv23_b200 import cof, search

    ON = cof.COF_COUNT_ON_DEVICE
    s = st.stream

    def ev():
        e = torch.cuda.Event(enable_timing=True)
        e.record(s)
        return e

    for i in range(len(st.chunks)):
        dch, pd = st.d_chunks[i], st.plan_devs[i]
        if st.path_name != "single":   # (the single pass has no separate search kernel)
            f0 = ev() if fevents is not None else None
            if st.fused:
                cof.cof_find_masks(st.plan, pd, dch, st.find_ws, s)
            else:
                cof.cof_find_pam(st.plan, pd, dch, st.find_ws, st.items[0], st.items[1], st.max_owned, s, sync=False)
            if fevents is not None:
                fevents.append((f0, ev()))
        e0 = ev() if events is not None else None
        if st.path_name == "single":
            cof.cof_search_single(st.plan, pd, dch, st.find_ws, st.hits[i], st.caps[i], s, sync=False)
        elif st.fused:
            cof.cof_compare_masks(st.plan, pd, dch, st.find_ws, st.hits[i], st.caps[i], s, sync=False)
        else:
            cof.cof_compare(st.plan, pd, dch, st.items[0], ON, st.items[1], ON, st.hits[i], st.caps[i], s, sync=False)
        if events is not None:
            events.append((e0, ev()))
        cof.cof_sort_hits(st.plan, pd, dch, st.hits[i], st.tmp, st.caps[i], ON, st.sort_ws, s)
        cof.cof_decorate(st.plan, pd, dch, st.hits[i], ON, st.recs[i], st.dec_ws[i], s, cap=st.caps[i])
    if not collect:
        return None
    out = []
    for i in range(len(st.chunks)):
        nf, nr, nh = cof.cof_read_counts(st.plan, st.plan_devs[i], s)
        if nh > st.caps[i]:
            raise RuntimeError(f"chunk {i}: {nh} hits exceed capacity {st.caps[i]}")
        out.append(cof.cof_collect(st.plan, st.host.chunk_struct(i), st.hits[i], nh, s))
    return search.merge_hit_lists(out)


def step_counts(st):
    from paper_conf_socc_jinv23_b200 import cof
    tot = [0, 0, 0]
    for i in range(len(st.chunks)):
        cof.cof_decorate_check(st.dec_ws[i], st.stream)     # every key matched its chunk / plan
        c = cof.cof_read_counts(st.plan, st.plan_devs[i], st.stream)
        if c[2] > st.caps[i]:
            raise RuntimeError(f"chunk {i}: {c[2]} hits exceed capacity {st.caps[i]}")
        for k in range(3):
            tot[k] += c[k]
    return tot


def run_e2e_step(wl, st, searcher, out=None):
    """Public-API end-to-end step from pinned host planes; returns (hits, h2d, d2h bytes).
    ``out``: the caller's result buffer (reused between steps, as an application would)."""
    hits = searcher.search_host(st.e2e_host, out=out)
    h2d = st.e2e_host.h2d_bytes
    d2h = len(hits) * hits.dtype.itemsize + 24 * len(st.e2e_host.chunks)   # decorated records + per-chunk counts
    return hits, h2d, d2h


def measure_from_fasta(wl, dev, runs: int = 2):
    """whole search from a FASTA file through the CLI's path
    (cli.run: mmap + index, OpenMP pack of <= 250 Mbp chunks straight from the file into
    pinned planes, the pipelined search, records in host memory), wall clock, best of
    ``runs``.  The paper's elapsed time likewise includes the genome read; the
    TSV formatting is not included.  The file is written to /tmp first (untimed)."""
    import tempfile
    import torch
    from paper_conf_socc_jinv23_b200 import cli

    d = tempfile.mkdtemp(prefix="cof_fa_")
    path = os.path.join(d, "genome.fa")
    synth.write_fasta(path, wl.names, wl.seqs)
    spec = cli.InputSpec(path, wl.cfg.pattern, list(wl.guides), list(wl.thresholds))
    best, nh = None, 0
    try:
        for _ in range(runs):
            torch.cuda.synchronize(dev)
            t0 = time.perf_counter()
            hits, _names = cli.run(spec, device=str(dev), chunk_bases=E2E_CHUNK_BASES)
            dt = time.perf_counter() - t0
            nh = len(hits)
            best = dt if best is None else min(best, dt)
        size = os.path.getsize(path)
    finally:
        try:
            os.remove(path)
            os.rmdir(d)
        except OSError:
            pass
    return {"value": round(wl.total_bases / best / 1e9, 4), "unit": "Gbases/s", "s": round(best, 4),
            "fasta_bytes": int(size), "hits": int(nh), "runs": runs,
            "path": "cli.run: FASTA mmap/index -> cof_fasta_pack (OpenMP) into pinned planes of <= 250 Mbp "
                    "chunks -> Searcher.search_host (H2D lo/hi + N runs, find/compare, sort, device "
                    "decoration, D2H of the records); wall clock, best of runs"}


def input_sha256(wl):
    """SHA-256 over the synthetic input exactly as the search sees it: every chromosome's
    name and ASCII bases, then the pattern and each (guide, threshold)."""
    import hashlib
    h = hashlib.sha256()
    for name, seq in zip(wl.names, wl.seqs):
        h.update(name.encode() + b"\n")
        h.update(memoryview(np.ascontiguousarray(seq)))
        h.update(b"\n")
    h.update(wl.cfg.pattern.encode() + b"\n")
    for g, t in zip(wl.guides, wl.thresholds):
        h.update(f"{g} {int(t)}\n".encode())
    return h.hexdigest()


def host_info():
    """CPU model and core counts of the box (record the lscpu model)."""
    model = None
    try:
        with open("/proc/cpuinfo") as f:
            for ln in f:
                if ln.startswith("model name"):
                    model = ln.split(":", 1)[1].strip()
                    break
    except OSError:
        pass
    return {"cpu_model": model, "cpus": os.cpu_count(), "affinity_cpus": len(os.sched_getaffinity(0))}


def oracle_single_thread():
    """the oracle on ONE thread over the whole C1 and C2 workloads (seconds
    each), wall clock, with the hit counts it found."""
    from oracle import oracle as orc
    out = {}
    for name in ("C1", "C2"):
        w = synth.make_workload(name)
        t = time.perf_counter()
        h = orc.search(w.seqs, w.cfg.pattern, w.guides, w.thresholds, threads=1)
        dt = time.perf_counter() - t
        out[name] = {"s": round(dt, 3), "Gbases_per_s": round(w.total_bases / dt / 1e9, 6), "hits": int(len(h)),
                     "genome_bases": int(w.total_bases), "guides": len(w.guides)}
    return out


# ----------------------------------------------------------------------------- oracle arm
def oracle_sample(wl, target_s: float, threads: int):
    """Bounded sample for the CPU oracle: the first B window starts after the leading
    telomere of every chromosome in turn, B calibrated to ~target_s of CPU time."""
    from oracle import oracle as orc
    cfg = wl.cfg
    c = int(np.argmax([len(s) for s in wl.seqs]))
    s0 = 1_000_000 if len(wl.seqs[c]) > 3_000_000 else 0
    probe = 100_000
    t = time.perf_counter()
    orc.search([wl.seqs[c]], cfg.pattern, wl.guides, wl.thresholds, ranges=[(s0, s0 + probe)], threads=threads)
    dt = max(time.perf_counter() - t, 1e-3)
    n = int(min(len(wl.seqs[c]) - s0 - cfg.L, max(probe, probe * target_s / dt)))
    return c, s0, n


def run_oracle(wl, c, s0, n, threads):
    from oracle import oracle as orc
    cfg = wl.cfg
    t = time.perf_counter()
    h = orc.search([wl.seqs[c]], cfg.pattern, wl.guides, wl.thresholds, ranges=[(s0, s0 + n)], threads=threads)
    return time.perf_counter() - t, len(h)


def items_per_base_estimate(st, wl):
    tot_items = sum(c[0] + c[1] for c in st.counts)
    return tot_items / max(1, sum(ch.n_owned for ch in st.chunks))


# ----------------------------------------------------------------------------- bulge search
def main_bulge(args, cfgname):
    """--bulge D,R: the bulge search (bulge.py) of the config's genome on
    one GPU: one device step = find -> compare -> sort -> decorate for every variant
    pattern (X, DNA 1..D, RNA 1..R), each over all its guide variants; Gbases/s = genome
    bases / device time of the whole step."""
    import torch
    from paper_conf_socc_jinv23_b200 import bulge, cof, search

    dna, rna = (int(x) for x in args.bulge.split(","))
    dev = torch.device("cuda", 0)
    torch.cuda.set_device(dev)
    cof.cof_set_comparer(args.comparer)
    wl = synth.make_workload(cfgname, scale=args.scale, threads=max(1, min(16, os.cpu_count() or 1)))
    groups = bulge.variants(wl.cfg.pattern, wl.guides, wl.thresholds, dna, rna)
    states = []
    for pv, (gs, ts, ms) in groups.items():
        chunks = [search.pack_shard(search.plan_chunks([len(x) for x in wl.seqs], len(pv), None))]
        _, st = prepare_workload(cfgname, args.scale, chunks=chunks, device=dev, wl=wl, query=(pv, gs, ts))
        states.append((pv, st))
    for _ in range(max(args.warmup, 3)):
        for _, st in states:
            run_device_pipeline(wl, st)
    torch.cuda.synchronize(dev)
    s = states[0][1].stream
    t0, t1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    launches0 = cof.cof_launch_count()
    t0.record(s)
    for _ in range(args.steps):
        for _, st in states:
            run_device_pipeline(wl, st)
    t1.record(s)
    torch.cuda.synchronize(dev)
    launches = cof.cof_launch_count() - launches0
    ms = t0.elapsed_time(t1) / args.steps
    comps = items = hits = 0
    per = []
    for pv, st in states:
        c = step_counts(st)
        items += c[0] + c[1]
        comps += (c[0] + c[1]) * st.n_guides
        hits += c[2]
        per.append({"pattern": pv, "guide_variants": st.n_guides, "items": int(c[0] + c[1]), "hits": int(c[2])})
    line = {"metric": "genome Gbases/s, bulge search (X + DNA<=%d + RNA<=%d)" % (dna, rna),
            "value": round(wl.total_bases / (ms * 1e-3) / 1e9, 4), "unit": "Gbases/s", "n_gpus": 1,
            "steps": args.steps, "warmup": max(args.warmup, 3), "ms_per_step": round(ms, 4),
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "u32", "dtype_note": "2-bit bases in u32 bit-planes, bitwise integer arithmetic (exact)",
            "data": "synthetic (seeded hg38-shaped genome, synth.py)", "comparisons_per_s": comps / (ms * 1e-3),
            "hits_per_step": int(hits), "items_per_step": int(items),
            "config": {"workload": cfgname, "genome_bases": wl.total_bases, "guides": len(wl.guides),
                       "threshold": wl.cfg.threshold, "pattern": wl.cfg.pattern, "dna_bulge": dna, "rna_bulge": rna,
                       "variant_searches": per, "comparer": args.comparer,
                       "l2": "inputs larger than L2, no flush"},
            "gpu_launches": int(launches // max(1, args.steps))}
    print(json.dumps(line))
    return 0


# ----------------------------------------------------------------------------- main
def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="C5")
    ap.add_argument("--scale", type=float, default=1.0)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--comparer", default="table", choices=["table", "popc"])
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--e2e-steps", type=int, default=2)
    ap.add_argument("--no-fasta", action="store_true",
                    help="skip the search from a FASTA file (SURVEY §8(d) (iii), fasta_e2e; it writes the "
                         "genome as FASTA under /tmp first)")
    ap.add_argument("--from-fasta", action="store_true", help=argparse.SUPPRESS)   # the default now
    ap.add_argument("--no-single-thread", action="store_true",
                    help="skip the single-thread oracle times of C1 and C2 (SURVEY §8(d))")
    ap.add_argument("--bulge", default=None, help="D,R: time the bulge search (max DNA, RNA bulge sizes)")
    ap.add_argument("--n-guides", type=int, default=None, help="override the config's guide count (scaling study)")
    args = ap.parse_args()

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    cfgname = args.config
    metric = "genome Gbases/s (and guide x site comparisons/s)"

    if args.impl == "reference":
        if rank != 0:
            return 0
        return main_reference(args, cfgname, metric)
    if args.bulge:
        return main_bulge(args, cfgname)

    import torch
    import torch.distributed as dist
    from paper_conf_socc_jinv23_b200 import cof, search

    # one process per GPU; COF_DIST_BACKEND=gloo lets several ranks share a device (tests)
    local_dev = local % max(1, torch.cuda.device_count())
    torch.cuda.set_device(local_dev)
    dev = torch.device("cuda", local_dev)
    backend = os.environ.get("COF_DIST_BACKEND", "nccl")
    coll_dev = dev if backend == "nccl" else torch.device("cpu")
    if world > 1:
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group(backend)
    cof.cof_set_comparer(args.comparer)
    if world > 1:   # torchrun sets OMP_NUM_THREADS=1: share the node's cores among the ranks instead
        nthr = max(1, len(os.sched_getaffinity(0)) // int(os.environ.get("LOCAL_WORLD_SIZE", world)))
        torch.set_num_threads(nthr)
        cof.cof_set_host_threads(nthr)
    cfg = synth.config(cfgname, args.scale)
    L = cfg.L
    # N > 1: chromosomes cut into <= 16 Mbp pieces before the LPT assignment (max/ideal load
    # 1.0025 at 8 ranks instead of 1.036 with whole chromosomes); N = 1: whole chromosomes
    all_chunks = search.plan_chunks([l for _, l in cfg.genome.chroms], L, SHARD_PIECE_BASES if world > 1 else None)
    shards = search.shard_lpt(all_chunks, world)
    mine = [search.pack_shard(shards[rank])]          # this rank's pieces as ONE chunk
    wl, st = prepare_workload(cfgname, args.scale, chunks=mine, device=dev, n_guides=args.n_guides)
    genome_bases = wl.total_bases
    sha = None
    if rank == 0:   # SHA-256 of the input (genome text, pattern, guides, thresholds), off the timed path
        import concurrent.futures
        sha = concurrent.futures.ThreadPoolExecutor(1).submit(input_sha256, wl)
    my_items = sum(c[0] + c[1] for c in st.counts)
    comps_mine = my_items * len(wl.guides)

    def barrier():
        if world > 1:
            dist.barrier()

    # the clock sampler (nvidia-smi every 100 ms) starts with the warm-up, which runs at least
    # W steps and at least 0.5 s, so short timed regions (C1, C2, C4) still get samples under load
    clocks = ClockSampler(local)
    clocks.start()
    t_w, n_w = time.perf_counter(), 0
    while n_w < max(args.warmup, 3) or time.perf_counter() - t_w < 0.5:
        run_device_pipeline(wl, st)
        n_w += 1
        if n_w >= max(args.warmup, 3):
            torch.cuda.synchronize(dev)
    torch.cuda.synchronize(dev)
    barrier()
    torch.cuda.synchronize(dev)
    # launch-bound steps (small genomes: the host's ~15 launches per step outlast the
    # kernels) are captured once into a CUDA graph and replayed; long steps run eagerly
    step_ms_est = (time.perf_counter() - t_w) * 1e3 / max(1, n_w)
    graph, graph_note, graph_launches = None, None, 0
    if step_ms_est < GRAPH_STEP_MS and os.environ.get("COF_GRAPH", "1") != "0":
        try:
            graph, graph_launches = capture_step(wl, st)
            for _ in range(3):
                graph.replay()
            torch.cuda.synchronize(dev)
        except Exception as e:   # (a capture the runtime refuses: eager steps)
            graph, graph_note = None, f"eager (graph capture failed: {e})"
    events, fevents = [], []
    launches0 = cof.cof_launch_count()
    t_start, t_end = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    t_start.record(st.stream)
    for _ in range(args.steps):
        if graph is not None:
            graph.replay()
        else:
            run_device_pipeline(wl, st, events=events, fevents=fevents)
    t_end.record(st.stream)
    torch.cuda.synchronize(dev)
    launches = (cof.cof_launch_count() - launches0) if graph is None else graph_launches * args.steps
    clk = clocks.stop()
    barrier()
    ms_total = t_start.elapsed_time(t_end)
    totals = step_counts(st)   # verifies capacities and every decorated key (graph replays too)
    if graph is not None:
        # the dominant kernel's own time cannot be bracketed inside a graph: K eager steps
        # after the timed region, events around its launches
        for _ in range(args.steps):
            run_device_pipeline(wl, st, events=events, fevents=fevents)
        torch.cuda.synchronize(dev)
        step_counts(st)
        graph_note = (f"CUDA graph of one step ({graph_launches} kernels) replayed K times in the timed region; "
                      "kernel times from K eager steps after it")
    cmp_ms = sum(a.elapsed_time(b) for a, b in events)
    find_ms = sum(a.elapsed_time(b) for a, b in fevents)

    # max over ranks
    t = torch.tensor([ms_total, cmp_ms, float(comps_mine), float(totals[2]), float(my_items)],
                     dtype=torch.float64, device=coll_dev)
    if world > 1:
        tmax = t.clone()
        dist.all_reduce(tmax[:2], op=dist.ReduceOp.MAX)
        tsum = t.clone()
        dist.all_reduce(tsum[2:], op=dist.ReduceOp.SUM)
        ms_total, cmp_ms_max = float(tmax[0]), float(tmax[1])
        comps_all, hits_all, items_all = float(tsum[2]), float(tsum[3]), float(tsum[4])
    else:
        cmp_ms_max = cmp_ms
        comps_all, hits_all, items_all = float(comps_mine), float(totals[2]), float(my_items)
    ms_step = ms_total / args.steps
    gbases = genome_bases / (ms_step * 1e-3) / 1e9
    comps_s = comps_all / (ms_step * 1e-3)

    # roofline of the dominant kernel (comparer): comparisons/s vs the ALU/LDS roof
    peaks, peak_src = _peaks()
    sm_max = float(peaks.get("sm_max_mhz", 1965.0))
    n_sm = torch.cuda.get_device_properties(dev).multi_processor_count
    roof = comparer_roof(st.plan, n_sm, sm_max, args.comparer, st.path_name)
    cmp_rate = comps_mine * args.steps / (cmp_ms * 1e-3) if cmp_ms > 0 else 0.0
    n_cmp_launch = len(events)
    traffic_k = traffic_for("cof_single_kernel" if st.path_name == "single" else "cof_comparer", st, cfgname)
    kname = {"single": "cof_single_kernel", "fused": "cof_comparer_fused"}.get(st.path_name,
                                                                              f"cof_comparer_{args.comparer}")
    roofline = {"bound": "alu", "kernel": kname,
                "achieved": cmp_rate, "peak": roof["peak"], "unit": "comparisons/s",
                "frac": cmp_rate / roof["peak"] if roof["peak"] else None,
                "traffic": traffic_k[0], "traffic_capture": traffic_k[1],
                "peak_basis": roof["basis"], "launches": n_cmp_launch,
                "share_of_step": cmp_ms_max / ms_total if ms_total else None,
                # the same rate against SURVEY §8(d)'s roof (one POPC per comparison)
                "frac_popc_roof": cmp_rate / popc_roof(n_sm, sm_max),
                "popc_roof": popc_roof(n_sm, sm_max)}

    # finder roofline (HBM): algorithmic bytes of the search kernel per step
    plane_bytes = sum(cof.cof_plane_words(ch.n_bases) * 4 * (4 if ch.multi else 3) for ch in st.chunks)
    words = sum(cof.cof_plane_words(ch.n_bases) for ch in st.chunks)
    if st.path_name == "single":
        # the single pass has no separate search kernel: the paper's search step (ordered PAM
        # item lists, cof_find_pam -> cof_finder_kernel) is timed on its own, after the step
        find_ms, n_items_sk = time_search_kernel(st, args.steps)
        find_bytes = plane_bytes + 4 * n_items_sk
        find_basis = ("search kernel alone (cof_find_pam: count pass, grid exchange, ordered item lists; the "
                      "single pass fuses the PAM test into cof_single_kernel): planes (+ valid-start plane) read + "
                      f"4 B per item written, timed {args.steps} times after the step's timed region")
    elif st.fused:      # planes (+ valid-start plane) read, {fwd, rev} masks written
        find_bytes = plane_bytes + words * 8
        find_basis = "planes read + 8 B of PAM masks per plane word written (fused path)"
    else:             # planes read, 4 B per item written
        find_bytes = plane_bytes + 4 * my_items
        find_basis = "planes read + 4 B per item written (two-call path)"
    find_gbs = find_bytes * args.steps / (find_ms * 1e-3) / 1e9 if find_ms > 0 else 0.0
    hbm_peak = float(peaks.get("hbm_gbs", 6650.0))
    traffic_f = traffic_for("cof_finder_kernel", st, cfgname, path="twocall" if st.path_name == "single" else None)
    finder_roof = {"bound": "hbm", "kernel": "cof_finder_kernel",
                   "achieved": round(find_gbs, 1),
                   "peak": hbm_peak, "unit": "GB/s", "frac": find_gbs / hbm_peak,
                   "bytes_per_step": int(find_bytes), "basis": find_basis,
                   "ms_per_step": find_ms / args.steps, "traffic": traffic_f[0], "traffic_capture": traffic_f[1]}

    masks_roof = None
    if st.path_name == "single" and cof.cof_find_compare_supported(st.plan):
        m_ms, m_bytes = time_masks_kernel(st, args.steps)
        m_gbs = m_bytes * args.steps / (m_ms * 1e-3) / 1e9 if m_ms > 0 else 0.0
        masks_roof = {"bound": "hbm", "kernel": "cof_finder_kernel (masks)", "achieved": round(m_gbs, 1),
                      "peak": hbm_peak, "unit": "GB/s", "frac": m_gbs / hbm_peak, "bytes_per_step": int(m_bytes),
                      "ms_per_step": m_ms / args.steps,
                      "basis": "search kernel writing per-word PAM masks (cof_find_masks, the fused path's finder): "
                               "planes (+ valid-start plane) read + 8 B of masks per plane word written; timed "
                               f"{args.steps} times after the step's timed region"}
    e2e = None
    resident = None
    if not args.no_e2e:
        e2e = measure_e2e(wl, st, dev, args, world, genome_bases, coll_dev)
        if world == 1:
            resident = measure_resident(wl, st, dev, args, genome_bases)

    fasta = None
    if rank == 0 and world == 1 and not args.no_fasta:
        fasta = measure_from_fasta(wl, dev)

    single = None
    if rank == 0 and world == 1 and not args.no_cpu and not args.no_single_thread:
        single = oracle_single_thread()

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu:
        threads = len(os.sched_getaffinity(0))
        c, s0, n = oracle_sample(wl, 15.0, threads)
        dt, nh = run_oracle(wl, c, s0, n, threads)
        ipb = items_per_base_estimate(st, wl)
        cpu = {"value": n / dt / 1e9, "unit": "Gbases/s", "cores": threads, "kind": "oracle",
               "comparisons_per_s": n * ipb * len(wl.guides) / dt,
               "sample": f"{n} window starts of {wl.names[c]} from offset {s0}, both strands, all "
                         f"{len(wl.guides)} guides ({dt:.1f} s, {nh} hits)"}

    if rank == 0:
        line = {
            "metric": metric, "value": round(gbases, 4), "unit": "Gbases/s", "n_gpus": world,
            "steps": args.steps, "warmup": max(args.warmup, 3), "warmup_steps_run": n_w,
            "ms_per_step": round(ms_step, 4),
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "u32", "dtype_note": "2-bit bases in u32 bit-planes, bitwise integer arithmetic (exact)",
            "data": "synthetic (seeded hg38-shaped genome, synth.py)",
            "comparisons_per_s": comps_s, "hits_per_step": int(hits_all), "items_per_step": int(items_all),
            "config": {"workload": cfgname if not args.n_guides else f"{cfgname} with {args.n_guides} guides",
                       "description": cfg.description, "genome_bases": genome_bases,
                       "chromosomes": len(wl.seqs), "guides": len(wl.guides), "threshold": cfg.threshold,
                       "pattern": cfg.pattern,
                       "chunking": "device: this rank's chromosomes as one multi-segment chunk; "
                                   f"e2e: packed chunks of <= {E2E_CHUNK_BASES / 1e6:g} Mbp"
                                   + (f" (pieces <= {E2E_PIECE_BASES / 1e6:g} Mbp)" if E2E_PIECE_BASES else "")
                                   + ", pipelined",
                       "parallelism": (f"LPT shards of <= {SHARD_PIECE_BASES // 10**6} Mbp chromosome pieces over "
                                       f"{world} GPUs" if world > 1 else "one GPU, whole genome as one chunk"),
                       "comparer": args.comparer,
                       "l2": "inputs larger than L2 (1.16 GB planes + item lists), no flush"},
            "roofline": roofline,
            "finder_roofline": finder_roof,
            "finder_masks_roofline": masks_roof,
            "gpu_launches": int(launches // args.steps) if args.steps else 0,
            "step_launch": graph_note or "eager launches",
            "gpu_launches_timed_region": int(launches),
            "clocks": clk,
            "e2e": e2e,
            "e2e_resident": resident,
            "fasta_e2e": fasta,
            "cpu_baseline": cpu,
            "oracle_single_thread": single,
            "peaks_source": peak_src,
            "host": host_info(),
            "input_sha256": sha.result() if sha is not None else None,
        }
        print(json.dumps(line))
    if world > 1:
        dist.destroy_process_group()
    return 0


def time_search_kernel(st, steps):
    """The search kernel alone (cof_find_pam: ordered PAM item lists of every chunk) on the
    resident planes, ``steps`` launches per chunk after one warm-up, CUDA events on the
    launching stream.  Returns (ms per step, items per step)."""
    import torch
    from paper_conf_socc_jinv23_b200 import cof
    s = st.stream
    total_ms, n_items = 0.0, 0
    for i in range(len(st.chunks)):
        nf, nr = st.counts[i][0], st.counts[i][1]
        cap = max(nf, nr) + 1024
        items = torch.empty((2, cap), dtype=torch.int32, device=st.device)
        ws = torch.empty(cof.cof_find_workspace_bytes(st.chunks[i].n_bases), dtype=torch.uint8, device=st.device)
        got = cof.cof_find_pam(st.plan, st.plan_devs[i], st.d_chunks[i], ws, items[0], items[1], cap, s)
        if tuple(got) != (nf, nr):
            raise RuntimeError(f"search kernel counts {got} != the step's {(nf, nr)}")
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        for _ in range(steps):
            cof.cof_find_pam(st.plan, st.plan_devs[i], st.d_chunks[i], ws, items[0], items[1], cap, s, sync=False)
        e1.record(s)
        torch.cuda.synchronize(st.device)
        total_ms += e0.elapsed_time(e1)
        n_items += nf + nr
        del items, ws
    return total_ms, n_items


def time_masks_kernel(st, steps):
    """The search kernel in its masks form (cof_find_masks: per plane word {fwd, rev} PAM
    masks, the fused path's finder) alone on the resident planes, ``steps`` launches per
    chunk; returns (ms per step, algorithmic bytes per step: planes read + 8 B per word)."""
    import torch
    from paper_conf_socc_jinv23_b200 import cof
    s = st.stream
    total_ms, nbytes = 0.0, 0
    for i, ch in enumerate(st.chunks):
        ws = torch.empty(cof.cof_find_compare_workspace_bytes(ch.n_bases), dtype=torch.uint8, device=st.device)
        cof.cof_find_masks(st.plan, st.plan_devs[i], st.d_chunks[i], ws, s)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        for _ in range(steps):
            cof.cof_find_masks(st.plan, st.plan_devs[i], st.d_chunks[i], ws, s)
        e1.record(s)
        torch.cuda.synchronize(st.device)
        total_ms += e0.elapsed_time(e1)
        words = cof.cof_plane_words(ch.n_bases)
        nbytes += words * 4 * (4 if ch.multi else 3) + words * 8
        del ws
    return total_ms, nbytes


def traffic_for(kernel, st, cfgname, path=None):
    """DRAM bytes per launch of ``kernel`` on THIS config and path from a committed ncu
    --set full capture (profiles/roofline_traffic.json, keyed "<config>:<kernel>_<path>"),
    or None when no capture of that config and path is committed.  Returns (bytes, capture)."""
    try:
        with open(os.path.join(ROOT, "profiles", "roofline_traffic.json")) as f:
            d = json.load(f)
        key = f"{cfgname}:{kernel}_{path or st.path_name}"
        e = d.get(key)
        return (None, None) if e is None else (int(e["dram_bytes_per_launch"]), e.get("capture"))
    except Exception:
        return None, None


def popc_roof(n_sm, sm_mhz):
    """SURVEY §8(d)'s comparer roof: one POPC per comparison on the quarter-rate POPC pipe,
    16/clk/SM (measured 4.54e12 POPC/s = 15.6/clk/SM at 1965 MHz,
    profiles/microbench_pipes_r2.txt: 15.65/clk/SM at 1956 MHz)."""
    return 16.0 * n_sm * sm_mhz * 1e6


def single_roof(plan, n_sm, sm_mhz):
    """Peak comparisons/s of the single-pass kernel's filter: per site and
    32-guide block, NP one-word shared-memory lookups (one wavefront per warp each, 1 per
    clk per SM) and the nz_count carry-save tree (gen_csa.gen_count: FA / HA counts for
    this plan's NP) + a 4-step comparator + the valid mask, all LOP3 at 64 /clk/SM.
    Verification of the filter's survivors, site setup and queueing are not in this roof."""
    import importlib.util
    spec = importlib.util.spec_from_file_location(
        "gen_csa", os.path.join(ROOT, "paper_conf_socc_jinv23_b200", "csrc", "gen_csa.py"))
    g = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(g)
    care = 0
    for gs in plan.guides:
        for j, ch in enumerate(gs):
            if ch.upper() != "N":
                care |= 1 << j
    npairs = max(1, (bin(care).count("1") + 1) // 2)
    hdr = g.gen_count(npairs).splitlines()[0]
    fa = int(hdr.split(":")[1].split("full")[0])
    ha = int(hdr.split(",")[1].split("half")[0])
    alu_ops = 2 * fa + 2 * ha + 4 + 1
    # hand-reduced count-vs-threshold circuits (csrc/filter_circuit.cuh; LOP3 per 32 comparisons,
    # incl. the survivor mask): uniform thresholds of the configs' shapes
    ts = set(int(t) for t in plan.max_mm)
    if len(ts) == 1:
        alu_ops = {(10, 4): 16, (10, 5): 15, (10, 6): 16, (12, 5): 18}.get((npairs, ts.pop()), alu_ops)
    alu_rate = 64.0 * 32 / alu_ops
    lds_rate = 32.0 * 32 / npairs
    per_clk = min(alu_rate, lds_rate)
    return {"peak": per_clk * n_sm * sm_mhz * 1e6,
            "basis": f"single-pass filter: min(ALU {alu_rate:.1f}, LDS {lds_rate:.1f}) comparisons/clk/SM for "
                     f"{npairs} pairs ({alu_ops} LOP3 and {npairs} one-word lookups per 32 comparisons; survivor "
                     f"verification excluded) x {n_sm} SMs x {sm_mhz:.0f} MHz"}


def comparer_roof(plan, n_sm, sm_mhz, impl, path="fused"):
    if path == "single":
        return single_roof(plan, n_sm, sm_mhz)
    return table_roof(plan, n_sm, sm_mhz, impl)


def table_roof(plan, n_sm, sm_mhz, impl):
    """Peak comparisons/s of the comparer's binding pipe.
    popc: 1 POPC per comparison, POPC = 16/clk/SM (measured, tools/microbench_pipes.cu).
    table: per item and 32-guide block, the minimal carry-save tree (FA/HA count from
    gen_csa for this plan's pair count) + 6-step borrow chain + 1 mask op, all LOP3 on
    the 64/clk/SM ALU pipe (profiles/microbench_pipes_r2.txt); co-bound by shared memory: NP 64-bit lookups per item and
    block = 2*NP wavefronts per 32 items x 32 guides at 1 wavefront/clk/SM."""
    clk = sm_mhz * 1e6
    if impl == "popc":
        return {"peak": popc_roof(n_sm, sm_mhz), "basis": "POPC pipe 16/clk/SM x SMs x max SM clock"}
    import importlib.util
    spec = importlib.util.spec_from_file_location(
        "gen_csa", os.path.join(ROOT, "paper_conf_socc_jinv23_b200", "csrc", "gen_csa.py"))
    g = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(g)
    import ctypes
    from paper_conf_socc_jinv23_b200 import cof
    # pair count from the plan's guides (union of compared positions)
    L = plan.L
    care = 0
    for gs in plan.guides:
        for j, ch in enumerate(gs):
            if ch.upper() != "N":
                care |= 1 << j
    npairs = max(1, (bin(care).count("1") + 1) // 2)
    hdr = g.gen(npairs).splitlines()[0]
    fa = int(hdr.split(":")[1].split("full")[0])
    ha = int(hdr.split(",")[1].split("half")[0])
    alu_ops = 2 * fa + 2 * ha + 6 + 1
    # 64 LOP3/clk/SM: the ALU pipe issues one warp instruction per 2 cycles per SMSP
    # (B300_MICROARCH.md "Pipe rates"); measured 1.855e13 LOP3/s = 63.8/clk/SM at the
    # 1965 MHz max clock (profiles/microbench_pipes_r2.txt: 63.94 LOP3/clk/SM at a globaltimer-measured 1955 MHz)
    alu_rate = 64.0 * 32 / alu_ops           # comparisons / clk / SM
    lds_rate = 32.0 * 32 / (2 * npairs)      # comparisons / clk / SM
    per_clk = min(alu_rate, lds_rate)
    return {"peak": per_clk * n_sm * clk,
            "basis": f"min(ALU {alu_rate:.1f}, LDS {lds_rate:.1f}) comparisons/clk/SM for {npairs} pairs "
                     f"({alu_ops} LOP3 per 32 comparisons) x {n_sm} SMs x {sm_mhz:.0f} MHz"}


def measure_e2e(wl, st, dev, args, world, genome_bases, coll_dev=None):
    """``e2e``: the same search through the public API from pinned packed HOST planes,
    wall clock, H2D + kernels + D2H of the decorated records inside the timed region.
    N = 1: Searcher.search_host over packed chunks of <= 250 Mbp into the caller's pinned
    result buffer.  N > 1: search.search_dist's path -- the genome cut into <= 64 Mbp work
    units (genome order), LPT-assigned to the ranks, each rank's search_host pipeline, then
    merge_dist (per-chunk counts all-reduced -> offsets -> every rank writes its records
    into one shared-memory result): the merge is inside the timed step."""
    import torch
    import torch.distributed as dist
    from paper_conf_socc_jinv23_b200 import search
    L = len(wl.cfg.pattern)
    if world > 1:
        rank = dist.get_rank()
        gchunks = search.plan_chunks([len(x) for x in wl.seqs], L, search.MULTI_CHUNK_BASES)
        mine = search.shard_indices(gchunks, world)[rank]
        host = search.HostGenome(wl.seqs, [gchunks[i] for i in mine])
        srch = search.Searcher(wl.cfg.pattern, wl.guides, wl.thresholds, device=dev)
        srch.reserve(max(ch.n_bases for ch in host.chunks), max(st.caps))

        def step():
            per = {}
            srch.search_host(host, sink=lambda j, r: per.__setitem__(mine[j], r))
            merged = search.merge_dist(per, len(gchunks), srch.hit_dtype)
            d2h = sum(len(r) for r in per.values()) * srch.hit_dtype.itemsize + 24 * len(mine)
            return merged, host.h2d_bytes, d2h

        step()                                   # warm-up
        torch.cuda.synchronize(dev)
        dist.barrier()
        t0 = time.perf_counter()
        nh = 0
        for _ in range(args.e2e_steps):
            merged, h2d, d2h = step()
            nh = len(merged) if merged is not None else 0
        torch.cuda.synchronize(dev)
        dt = (time.perf_counter() - t0) / args.e2e_steps
        t = torch.tensor([dt], dtype=torch.float64, device=coll_dev if coll_dev is not None else dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        dt = float(t[0])
        return {"value": round(genome_bases / dt / 1e9, 4), "unit": "Gbases/s", "h2d_bytes_per_step": int(h2d),
                "d2h_bytes_per_step": int(d2h), "s_per_step": dt, "hits": nh, "bytes_per_step_per_rank": "rank 0",
                "path": "search_dist: <= 64 Mbp work units LPT-assigned to ranks -> per-rank Searcher.search_host "
                        "(H2D lo/hi + N runs, find/compare, sort, device decoration, D2H of the records) -> "
                        "merge_dist (per-chunk counts all-reduced, each rank writes its records at their "
                        "genome-order offsets into one shared-memory result); wall clock, max over ranks"}
    pieces = [p for ch in st.chunks for p in ch.pieces]
    if E2E_PIECE_BASES:
        pieces = search.split_pieces(pieces, E2E_PIECE_BASES, L)
    if E2E_FIRST_BASES:   # a short first chunk: cut the first piece
        pieces = search.split_pieces(pieces[:1], E2E_FIRST_BASES, L) + pieces[1:]
    chunks = search.pack_pieces(pieces, E2E_CHUNK_BASES, E2E_FIRST_BASES)
    st.e2e_host = search.HostGenome(wl.seqs, chunks)
    srch = search.Searcher(wl.cfg.pattern, wl.guides, wl.thresholds, device=dev)
    srch.reserve(max(ch.n_bases for ch in chunks), max(st.caps))
    hits0, _, _ = run_e2e_step(wl, st, srch)     # warm-up; sizes the caller's result buffer
    n_out = int(len(hits0) * 1.05) + 1024
    # the caller's result buffer: pinned host memory, so the device-decorated records DMA
    # straight into it (allocated and touched once, outside the timed steps)
    hd = srch.hit_dtype
    out = torch.zeros(n_out * hd.itemsize, dtype=torch.uint8, pin_memory=True).numpy().view(hd)
    del hits0
    torch.cuda.synchronize(dev)
    t0 = time.perf_counter()
    h2d = d2h = 0
    nh = 0
    for _ in range(args.e2e_steps):
        hits, a, b = run_e2e_step(wl, st, srch, out=out)
        h2d, d2h, nh = a, b, len(hits)
    torch.cuda.synchronize(dev)
    dt = (time.perf_counter() - t0) / args.e2e_steps
    return {"value": round(genome_bases / dt / 1e9, 4), "unit": "Gbases/s", "h2d_bytes_per_step": int(h2d),
            "d2h_bytes_per_step": int(d2h), "s_per_step": dt, "hits": nh,
            "path": "Searcher.search_host: cof_load_chunk (copy stream, double-buffered) -> find/compare "
                    "(fused masks path or item lists) -> cof_sort_hits -> cof_decorate (device) -> D2H of the "
                    "records (D2H stream) into the caller's pinned buffer, from pinned packed host planes "
                    "(wall clock)"}


def measure_resident(wl, st, dev, args, genome_bases):
    """``e2e_resident``: the public API on a genome already resident in HBM
    (search.ResidentGenome, uploaded once outside the timed steps -- the CRISPR-design loop
    of many guide sets against one genome): per step Searcher.search_resident over the
    e2e chunks (find / compare, sort, device decoration) with the records' D2H into the
    caller's pinned buffer inside the timed region; wall clock."""
    import torch
    from paper_conf_socc_jinv23_b200 import search
    # a few large chunks (the genome is resident: no H2D to overlap, only the records' D2H,
    # which overlaps the next chunk's kernels; fewer chunks = fewer per-chunk round trips)
    pieces = [p for ch in st.chunks for p in ch.pieces]
    host = search.HostGenome(wl.seqs, search.pack_pieces(pieces, RESIDENT_CHUNK_BASES))
    rg = search.ResidentGenome(host, dev)
    del host
    srch = search.Searcher(wl.cfg.pattern, wl.guides, wl.thresholds, device=dev)
    srch.reserve(max(ch.n_bases for ch in rg.chunks), max(st.caps))
    h0 = srch.search_resident(rg)
    hd = srch.hit_dtype
    out = torch.zeros((int(len(h0) * 1.05) + 1024) * hd.itemsize, dtype=torch.uint8,
                      pin_memory=True).numpy().view(hd)
    del h0
    torch.cuda.synchronize(dev)
    t0 = time.perf_counter()
    nh = 0
    for _ in range(args.e2e_steps):
        nh = len(srch.search_resident(rg, out=out))
    torch.cuda.synchronize(dev)
    dt = (time.perf_counter() - t0) / args.e2e_steps
    return {"value": round(genome_bases / dt / 1e9, 4), "unit": "Gbases/s", "h2d_bytes_per_step": 0,
            "d2h_bytes_per_step": int(nh * hd.itemsize + 24 * len(rg.chunks)), "s_per_step": dt, "hits": nh,
            "resident_bytes": int(rg.bytes), "chunks": len(rg.chunks),
            "path": "ResidentGenome (planes uploaded once, untimed) -> Searcher.search_resident per step: "
                    "find/compare, sort, device decoration, D2H of the records (second stream) into the "
                    "caller's pinned buffer; wall clock"}


def main_reference(args, cfgname, metric):
    """CPU oracle arm: each step = the oracle on a bounded sample of the workload."""
    threads = len(os.sched_getaffinity(0))
    cfg = synth.config(cfgname, args.scale)
    wl = synth.make_workload(cfgname, scale=args.scale, threads=max(1, min(16, os.cpu_count() or 1)))
    c, s0, n = oracle_sample(wl, 8.0, threads)
    for _ in range(args.warmup):
        run_oracle(wl, c, s0, min(n, 20_000), threads)
    times = []
    for _ in range(args.steps):
        dt, nh = run_oracle(wl, c, s0, n, threads)
        times.append(dt)
    dt = statistics.mean(times)
    v = n / dt / 1e9
    line = {"impl": "reference", "metric": metric, "value": v, "unit": "Gbases/s", "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": dt * 1e3, "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "ascii chars", "data": "synthetic",
            "config": {"workload": cfgname, "description": cfg.description},
            "cpu_baseline": {"value": v, "unit": "Gbases/s", "cores": threads, "kind": "oracle",
                             "sample": f"{n} window starts of {wl.names[c]} from offset {s0}, both strands, "
                                       f"all {len(wl.guides)} guides per step"},
            "e2e": {"value": v, "unit": "Gbases/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line))
    return 0


if __name__ == "__main__":
    sys.exit(main())

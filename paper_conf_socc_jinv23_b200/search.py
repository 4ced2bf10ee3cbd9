"""Driver of the hot path: chunk planning (M3), the per-chunk device pipeline
(load -> find -> compare -> sort -> collect, M5-M11), multi-GPU sharding (M19) and the
final merge.  Every step of the path runs in libcof.so; this module only allocates
memory (torch), orders the calls on a stream and moves counts.

Paper: P:L29 -- the host "divides the genome data into chunks that can fit the memory of
a heterogeneous device", runs the search kernel, hands the PAM sites to the compare
kernel, and "the interaction ... continues until all chunks are processed".
"""
from __future__ import annotations

import dataclasses
import heapq
import itertools
import os

import numpy as np
import torch

from . import cof


@dataclasses.dataclass(frozen=True)
class Piece:
    """Window starts [chrom_off, chrom_off + n_owned) of chromosome ``chrom`` plus the
    L-1 bases their last window needs (length = n_owned + L - 1, reading G12)."""
    chrom: int
    chrom_off: int
    n_owned: int
    length: int


@dataclasses.dataclass(frozen=True)
class Chunk:
    """One device work unit: one or more pieces laid back to back (chunk coordinates)."""
    pieces: tuple

    @property
    def n_bases(self):
        return sum(p.length for p in self.pieces)

    @property
    def n_owned(self):
        return sum(p.n_owned for p in self.pieces)

    @property
    def multi(self):
        return len(self.pieces) > 1

    # single-segment conveniences
    @property
    def chrom(self):
        return self.pieces[0].chrom

    @property
    def start(self):
        return self.pieces[0].chrom_off

    def segments(self):
        """(chrom, chunk_off, chrom_off, n_owned) per piece."""
        rows, off = [], 0
        for p in self.pieces:
            rows.append((p.chrom, off, p.chrom_off, p.n_owned))
            off += p.length
        return rows


FUSED_MIN_GUIDES = 256     # fused path from this many guides on, whatever the PAM
FUSED_MIN_DENSITY = 0.03   # ... and below it when PAM sites are at least this dense per strand
_SET_SIZE = {c: len(v) for c, v in {"A": "A", "C": "C", "G": "G", "T": "T", "R": "AG", "Y": "CT", "S": "CG",
                                    "W": "AT", "K": "GT", "M": "AC", "B": "CGT", "D": "AGT", "H": "ACT",
                                    "V": "ACG", "N": "ACGT"}.items()}


def pam_density(pattern: str) -> float:
    """Expected PAM sites per window start and strand on a uniform random genome."""
    d = 1.0
    for c in pattern.upper():
        d *= _SET_SIZE[c] / 4.0
    return d


def use_fused(plan, n_guides: int) -> bool:
    """Fused find+compare (finder masks, no item lists) or the two-call path.  Measured on
    B200 (round 1, final kernels): C3 (NRG, density 0.125, 100 guides) fused 9.67 ms vs
    two-call 11.71 ms; C5 (1000 guides) 51.8 vs 57.5 ms; C2 (NGG 0.0625, 10 guides) 0.172 vs
    0.180 ms; C4 (TTTV 0.0117, 100 guides) 3.82 vs 3.14 ms -- with sparse PAM sites the
    per-strand mask expansion and the unprefetched window loads cost more than the item
    lists save.  COF_FUSED=0/1 overrides."""
    env = os.environ.get("COF_FUSED")
    if not cof.cof_find_compare_supported(plan):
        return False
    if env is not None:
        return env != "0"
    return n_guides >= FUSED_MIN_GUIDES or pam_density(plan.pattern) >= FUSED_MIN_DENSITY


PATHS = ("single", "fused", "twocall")


def choose_path(plan, n_guides: int) -> str:
    """The device path of a plan: "single" (one streaming find + compare kernel, filter +
    verify comparer; cof_single_supported), else "fused" (finder masks -> mask-expanding
    pair-table comparer) or "twocall" (ordered item lists, the paper's two kernels).
    COF_PATH=single|fused|twocall overrides (falling back when unsupported)."""
    env = os.environ.get("COF_PATH")
    if env == "twocall":
        return "twocall"
    if env in (None, "single") and cof.cof_single_supported(plan):
        return "single"
    if env == "fused" or use_fused(plan, n_guides):
        return "fused" if cof.cof_find_compare_supported(plan) else "twocall"
    return "twocall"


def plan_chunks(lengths, L: int, chunk_bases: int | None = None, pack_bases: int | None = None):
    """Split chromosomes into pieces of at most ``chunk_bases`` owned window starts (whole
    chromosomes if None): every valid start 0 <= p <= len-L belongs to exactly one piece.
    Without ``pack_bases`` each piece is its own chunk; with it, consecutive pieces are
    packed into multi-segment chunks of at most ``pack_bases`` bases (a piece longer than
    that gets a chunk of its own); ``pack_bases=0`` packs everything into one chunk."""
    pieces = []
    for c, n in enumerate(lengths):
        n_starts = int(n) - L + 1
        if n_starts <= 0:
            continue
        step = int(chunk_bases) if chunk_bases else n_starts
        for s in range(0, n_starts, step):
            owned = min(step, n_starts - s)
            pieces.append(Piece(c, s, owned, owned + L - 1))
    if pack_bases is None:
        return [Chunk((p,)) for p in pieces]
    return pack_pieces(pieces, pack_bases)


def split_pieces(pieces, max_owned: int, L: int):
    """Cut every piece into pieces of at most ``max_owned`` window starts (same ownership
    rule as plan_chunks: consecutive pieces overlap by L-1 bases)."""
    out = []
    for p in pieces:
        for s in range(0, p.n_owned, max_owned):
            owned = min(max_owned, p.n_owned - s)
            out.append(Piece(p.chrom, p.chrom_off + s, owned, owned + L - 1))
    return out


def pack_pieces(pieces, pack_bases: int, first_bases: int = 0):
    """Consecutive pieces -> multi-segment chunks of at most ``pack_bases`` bases (0: one);
    the first chunk at most ``first_bases`` if given (a short first chunk starts the
    pipelined search sooner: its H2D is the only one nothing overlaps)."""
    out, cur, cur_bases = [], [], 0
    for p in pieces:
        limit = first_bases if (first_bases and not out) else pack_bases
        if cur and limit and cur_bases + p.length > limit:
            out.append(Chunk(tuple(cur)))
            cur, cur_bases = [], 0
        cur.append(p)
        cur_bases += p.length
    if cur:
        out.append(Chunk(tuple(cur)))
    return out


def shard_lpt(chunks, world: int):
    """Longest-processing-time-first assignment of chunks to ``world`` ranks (cost =
    owned window starts).  Returns one chunk list per rank, each in genome order."""
    loads = [(0, r) for r in range(world)]
    heapq.heapify(loads)
    out = [[] for _ in range(world)]
    for i in sorted(range(len(chunks)), key=lambda i: (-chunks[i].n_owned, i)):
        load, r = heapq.heappop(loads)
        out[r].append(i)
        heapq.heappush(loads, (load + chunks[i].n_owned, r))
    return [[chunks[i] for i in sorted(lst)] for lst in out]


def pack_shard(chunks):
    """All pieces of a list of chunks as ONE multi-segment chunk (a rank's whole shard)."""
    return Chunk(tuple(p for ch in chunks for p in ch.pieces))


def merge_hit_lists(lists, dtype=None):
    """Order (chrom, pos, strand, guide) across chunk / rank lists (cof_merge / cof_merge64)."""
    if dtype is None:
        dtype = next((x.dtype for x in lists if hasattr(x, "dtype")), cof.HIT_DTYPE)
    lists = [x for x in lists if len(x)]
    if not lists:
        return np.zeros(0, dtype=dtype)
    return cof.cof_merge(lists)


class HostGenome:
    """Packed bit-planes of every chunk in pinned host memory (a1: chunk & pack); multi-
    segment chunks also get their valid-start plane and segment table, every chunk the
    list of its N runs (cof_n_runs: only lo/hi cross PCIe, nm and vs are rebuilt on the
    device by cof_load_chunk_runs)."""

    def __init__(self, seqs, chunks, pin: bool = True):
        self.chunks = chunks
        self.planes = []
        self.segs = []
        self.runs = []
        pin = pin and torch.cuda.is_available()
        for ch in chunks:
            words = cof.cof_plane_words(ch.n_bases)
            buf = torch.empty((4 if ch.multi else 3, words), dtype=torch.int32, pin_memory=pin)
            if ch.multi:
                text = np.concatenate([np.asarray(seqs[p.chrom][p.chrom_off: p.chrom_off + p.length])
                                       for p in ch.pieces])
                segs = cof.make_segments(ch.segments())
                cof.cof_valid_starts(segs, len(ch.pieces), ch.n_bases, buf[3])
            else:
                p = ch.pieces[0]
                text = np.ascontiguousarray(seqs[p.chrom][p.chrom_off: p.chrom_off + p.length])
                segs = None
            cof.cof_pack(text, ch.n_bases, buf[0], buf[1], buf[2])
            self.planes.append(buf)
            self.segs.append(segs)
            self.runs.append(cof.cof_n_runs(buf[2], ch.n_bases))

    @classmethod
    def from_packer(cls, chunks, pack, pin: bool = True):
        """Single-segment chunks packed by ``pack(chrom, first, n, lo, hi, nm)`` (e.g. straight
        from an indexed FASTA file, cof_fasta_pack) without materialising the ASCII."""
        self = cls.__new__(cls)
        self.chunks, self.planes, self.segs, self.runs = chunks, [], [], []
        pin = pin and torch.cuda.is_available()
        for ch in chunks:
            if ch.multi:
                raise ValueError("from_packer builds single-segment chunks")
            words = cof.cof_plane_words(ch.n_bases)
            buf = torch.empty((3, words), dtype=torch.int32, pin_memory=pin)
            pack(ch.chrom, ch.start, ch.n_bases, buf[0], buf[1], buf[2])
            self.planes.append(buf)
            self.segs.append(None)
            self.runs.append(cof.cof_n_runs(buf[2], ch.n_bases))
        return self

    def chunk_struct(self, i) -> cof.cof_chunk:
        ch, buf, segs = self.chunks[i], self.planes[i], self.segs[i]
        if ch.multi:
            return cof.make_chunk(0, 0, ch.n_bases, ch.n_owned, buf[0], buf[1], buf[2], buf[3], segs)
        return cof.make_chunk(ch.chrom, ch.start, ch.n_bases, ch.n_owned, buf[0], buf[1], buf[2])

    @property
    def bytes(self):
        return sum(p.numel() * 4 for p in self.planes)

    def _use_runs(self, i) -> bool:
        # the run list replaces the nm (and vs) planes when it is smaller than they are
        return self.runs[i].nbytes < (self.planes[i].shape[0] - 2) * self.planes[i].shape[1] * 4

    @property
    def h2d_bytes(self):
        """Bytes load() moves per pass over all chunks (lo, hi and the N runs, or all planes)."""
        return sum(2 * p.shape[1] * 4 + r.nbytes if self._use_runs(i) else p.numel() * 4
                   for i, (p, r) in enumerate(zip(self.planes, self.runs)))

    def load(self, i, dev: cof.cof_chunk, stream, fill_stream=None):
        """H2D of chunk i into the device chunk ``dev``: lo/hi copied and nm/vs rebuilt on the
        device from the N runs / segments (cof_load_chunk_runs; the fill kernels on
        ``fill_stream`` if given), or every plane copied (cof_load_chunk) when the genome is
        so N-fragmented that the runs are larger."""
        if self._use_runs(i) and fill_stream is not None:
            cof.cof_load_chunk_runs_split(self.chunk_struct(i), self.runs[i], dev, stream, fill_stream)
        elif self._use_runs(i):
            cof.cof_load_chunk_runs(self.chunk_struct(i), self.runs[i], dev, stream)
        else:
            cof.cof_load_chunk(self.chunk_struct(i), dev, stream)


class ResidentGenome:
    """A genome's packed chunks resident in one GPU's memory (all planes, incl. the N and
    valid-start planes), uploaded once from a HostGenome: searches with different guide
    sets then move no genome bytes over PCIe (Searcher.search_resident)."""

    def __init__(self, host: HostGenome, device="cuda", stream=None):
        self.device = torch.device(device)
        self.chunks = host.chunks
        self.segs = host.segs
        self.d_planes, self.d_chunks = [], []
        stream = stream or torch.cuda.current_stream(self.device)
        with torch.cuda.device(self.device):
            for i, ch in enumerate(host.chunks):
                d = torch.empty((4, host.planes[i].shape[1]), dtype=torch.int32, device=self.device)
                dch = (cof.make_chunk(0, 0, ch.n_bases, ch.n_owned, d[0], d[1], d[2], d[3], host.segs[i]) if ch.multi
                       else cof.make_chunk(ch.chrom, ch.start, ch.n_bases, ch.n_owned, d[0], d[1], d[2]))
                host.load(i, dch, stream)                       # the chunk's one H2D
                self.d_planes.append(d)
                self.d_chunks.append(dch)
            stream.synchronize()

    @property
    def bytes(self):
        return sum(d.numel() * 4 for d in self.d_planes)


# search_host pipeline: the N / valid-start fills on the compute stream (on the
# copy stream they queue behind the persistent kernel that holds every SM), three device
# plane sets (the H2D runs two chunks ahead) and three record buffers (a chunk's hit count
# is read two chunks late, so the host never idles the GPU)
SPLIT_FILL = os.environ.get("COF_SPLIT_FILL", "1") == "1"
PLANE_BUFS = int(os.environ.get("COF_PLANE_BUFS", 3))
REC_BUFS = int(os.environ.get("COF_REC_BUFS", 3))
if PLANE_BUFS < 2:
    # with one plane set chunk j+1's H2D would overwrite the planes chunk j is searched on
    raise ValueError(f"COF_PLANE_BUFS={PLANE_BUFS}: the search_host pipeline needs at least 2 device plane sets")


class Searcher:
    """One GPU's pipeline for a fixed (pattern, guides, thresholds) plan."""

    def __init__(self, pattern, guides, thresholds, device="cuda", stream=None):
        self.device = torch.device(device)
        self.plan = cof.cof_plan_create(pattern, guides, thresholds)
        self.hit_dtype = cof.hit_dtype(self.plan.L)   # cof_hit (L <= 32) or cof_hit64
        self.L = self.plan.L
        self.stream = stream or torch.cuda.current_stream(self.device)
        nbytes = cof.cof_plan_device_bytes(self.plan)
        self.plan_dev = torch.empty(nbytes + 256, dtype=torch.uint8, device=self.device)
        cof.cof_plan_upload(self.plan, self.plan_dev, self.stream)
        self._cap_bases = 0
        self._hits_cap = 0
        self._rec_cap = 0
        self.d_records = None
        # single pass, fused (masks) or two-call (item lists): choose_path
        self.path = choose_path(self.plan, len(guides))

    @property
    def fused(self) -> bool:
        """No item lists (single pass or the masks path)."""
        return self.path != "twocall"

    @fused.setter
    def fused(self, on: bool):
        # True: the masks path (the single pass is chosen with .path = "single")
        self.path = "fused" if on and cof.cof_find_compare_supported(self.plan) else "twocall"

    # ---- device buffers sized for the largest chunk seen so far
    def reserve(self, max_bases: int, hits_cap: int):
        if max_bases > self._cap_bases:
            words = cof.cof_plane_words(max_bases)
            self.d_planes = torch.empty((4, words), dtype=torch.int32, device=self.device)
            # item lists only for the two-call path (the fused path never materialises them)
            self.d_items = torch.empty((2, 1 if self.fused else max(max_bases, 1)), dtype=torch.int32,
                                       device=self.device)
            self.d_find_ws = torch.empty(cof.cof_find_compare_workspace_bytes(max_bases), dtype=torch.uint8,
                                         device=self.device)
            self._cap_bases = max_bases
        if hits_cap > self._hits_cap:
            self.d_hits = torch.empty(hits_cap, dtype=torch.int64, device=self.device)
            self.d_tmp = torch.empty(hits_cap, dtype=torch.int64, device=self.device)
            self.d_sort_ws = torch.empty(cof.cof_sort_workspace_bytes(hits_cap), dtype=torch.uint8,
                                         device=self.device)
            self._hits_cap = hits_cap

    def device_chunk(self, ch: Chunk, planes=None, segs=None) -> cof.cof_chunk:
        p = self.d_planes if planes is None else planes
        if ch.multi:
            return cof.make_chunk(0, 0, ch.n_bases, ch.n_owned, p[0], p[1], p[2], p[3],
                                  segs if segs is not None else cof.make_segments(ch.segments()))
        return cof.make_chunk(ch.chrom, ch.start, ch.n_bases, ch.n_owned, p[0], p[1], p[2])

    def run_device_chunk(self, dchunk: cof.cof_chunk, items_cap: int, counts: bool = True):
        """find -> compare -> sort on the device; returns (n_fwd, n_rev, n_hits) (item counts
        None on the fused path with ``counts=False``).  Grows the hit buffer and re-runs
        compare on capacity overflow."""
        s = self.stream
        if not self.fused and self.d_items.shape[1] < items_cap:   # path switched after reserve()
            self.d_items = torch.empty((2, items_cap), dtype=torch.int32, device=self.device)
        if self.path == "fused":
            cof.cof_find_masks(self.plan, self.plan_dev, dchunk, self.d_find_ws, s)
        elif self.path == "twocall":
            nf, nr = cof.cof_find_pam(self.plan, self.plan_dev, dchunk, self.d_find_ws, self.d_items[0],
                                      self.d_items[1], items_cap, s)
        while True:
            try:
                if self.path == "single":
                    nh = cof.cof_search_single(self.plan, self.plan_dev, dchunk, self.d_find_ws, self.d_hits,
                                               self._hits_cap, s)
                elif self.fused:
                    nh = cof.cof_compare_masks(self.plan, self.plan_dev, dchunk, self.d_find_ws, self.d_hits,
                                               self._hits_cap, s)
                else:
                    nh = cof.cof_compare(self.plan, self.plan_dev, dchunk, self.d_items[0], nf, self.d_items[1],
                                         nr, self.d_hits, self._hits_cap, s)
                break
            except cof.CofError as e:
                if e.status != cof.COF_E_CAPACITY:
                    raise
                _, _, need = cof.cof_read_counts(self.plan, self.plan_dev, s)
                self.reserve(self._cap_bases, int(need * 1.25) + 1024)
        if self.fused:
            # item counts: compare's count read left the stream idle, so this sync is short;
            # after the sort it would block the host until the sort is done (a pipeline bubble)
            nf, nr = cof.cof_read_counts(self.plan, self.plan_dev, s)[:2] if counts else (None, None)
        cof.cof_sort_hits(self.plan, self.plan_dev, dchunk, self.d_hits, self.d_tmp, self._hits_cap, nh,
                          self.d_sort_ws, s)
        return nf, nr, nh

    def enqueue_device_chunk(self, dchunk: cof.cof_chunk, items_cap: int):
        """find -> compare -> sort on the device with every count left on the device: no
        host synchronisation (a capacity overflow shows in the device hit count, which the
        caller reads later, cof_counts_async)."""
        s = self.stream
        ON = cof.COF_COUNT_ON_DEVICE
        if not self.fused and self.d_items.shape[1] < items_cap:
            self.d_items = torch.empty((2, items_cap), dtype=torch.int32, device=self.device)
        if self.path == "single":
            cof.cof_search_single(self.plan, self.plan_dev, dchunk, self.d_find_ws, self.d_hits, self._hits_cap, s,
                                  sync=False)
        elif self.path == "fused":
            cof.cof_find_masks(self.plan, self.plan_dev, dchunk, self.d_find_ws, s)
            cof.cof_compare_masks(self.plan, self.plan_dev, dchunk, self.d_find_ws, self.d_hits, self._hits_cap, s,
                                  sync=False)
        else:
            cof.cof_find_pam(self.plan, self.plan_dev, dchunk, self.d_find_ws, self.d_items[0], self.d_items[1],
                             items_cap, s, sync=False)
            cof.cof_compare(self.plan, self.plan_dev, dchunk, self.d_items[0], ON, self.d_items[1], ON, self.d_hits,
                            self._hits_cap, s, sync=False)
        cof.cof_sort_hits(self.plan, self.plan_dev, dchunk, self.d_hits, self.d_tmp, self._hits_cap, ON,
                          self.d_sort_ws, s)

    def search_host(self, host: HostGenome, indices=None, out=None, decorate="device", sink=None):
        """End-to-end over host-resident packed chunks.  Per chunk: H2D on a copy stream
        (double-buffered device planes, overlapping the previous chunk's kernels), find,
        compare, device sort, device decoration (cof_decorate) and an async D2H of the
        finished records; nothing waits on the host except the item/hit counts.

        ``indices``: the chunks to search, in order -- a list, or any iterable (e.g. a shared
        work queue that several Searchers on several GPUs pop from, search_multi); it is
        consumed one chunk ahead of the device.  Returns the sorted hit array.  If ``out``
        (a ``Searcher.hit_dtype`` array, ideally in pinned memory) is large enough and the
        chunks come in genome order, each chunk's records land straight in its slice of
        ``out`` and a view of ``out`` is returned; otherwise per-chunk arrays are merged
        with cof_merge.  ``sink(i, records)``: called once per chunk with its sorted records
        (after the final synchronisation); then the merged array is not built and None is
        returned.  ``decorate="host"`` decorates on CPU threads instead (cof_collect)."""
        if decorate == "host":
            if sink is not None:
                raise ValueError("sink needs device decoration")
            return self._search_host_cpu_decorate(host, indices, out)
        listed = indices is None or isinstance(indices, (list, tuple, range))
        it = iter(range(len(host.chunks)) if indices is None else indices)
        # device buffers: sized for every chunk this call may see (an iterator may yield any)
        cand = list(indices) if listed and indices is not None else range(len(host.chunks))
        max_bases = max((host.chunks[i].n_bases for i in cand), default=1)
        max_segs = max((len(host.chunks[i].pieces) for i in cand), default=1)
        self.reserve(max_bases, max(self._hits_cap, 1 << 16))
        if getattr(self, "_planes_more_shape", None) != tuple(self.d_planes.shape):
            # PLANE_BUFS device plane sets: the H2D of chunk j+1 waits only for the
            # decoration of chunk j+1-PLANE_BUFS, not for the chunk just before it
            self.d_planes_more = [torch.empty_like(self.d_planes) for _ in range(PLANE_BUFS - 1)]
            self._planes_more_shape = tuple(self.d_planes.shape)
            self.copy_stream = torch.cuda.Stream(self.device)
            self.d2h_stream = torch.cuda.Stream(self.device)
        planes = [self.d_planes] + self.d_planes_more
        nb = len(planes)
        rec_free = [None] * REC_BUFS
        use_out = out is not None and sink is None
        ws_bytes = cof.cof_decorate_workspace_bytes(max_segs)
        ws = []                    # one decoration workspace (key-check flag) per chunk
        results = []               # (chunk index, records)
        total = 0
        overflow = False
        last_i = -1
        with torch.cuda.device(self.device):
            loaded = [None] * nb
            freed = [None] * nb

            trace = [] if os.environ.get("COF_TRACE") else None   # (what, chunk, stream, event)

            def mark(what, j, stream):
                if trace is not None:
                    e = torch.cuda.Event(enable_timing=True)
                    e.record(stream)
                    trace.append((what, j, e))

            def load(j, i, k):
                with torch.cuda.stream(self.copy_stream):
                    if freed[k] is not None:
                        self.copy_stream.wait_event(freed[k])
                    mark("h2d0", j, self.copy_stream)
                    dch = self.device_chunk(host.chunks[i], planes[k], host.segs[i])
                    # fills on the compute stream: that stream last used this plane set, and on
                    # the copy stream they would queue behind the running persistent kernels
                    # (COF_TRACE showed H2D intervals ~40% longer than the bytes need)
                    host.load(i, dch, self.copy_stream, fill_stream=self.stream if SPLIT_FILL else None)
                    mark("h2d1", j, self.copy_stream)
                    ev = torch.cuda.Event()
                    ev.record(self.copy_stream)
                    loaded[k] = ev
                    return dch

            dchs = [None] * nb
            # Chunk j's kernels, sort and decoration run with every count on the device; its
            # hit count reaches pinned host memory asynchronously and is read only after chunk
            # j + 1 is queued, so the host never idles the GPU between chunks.  A count above
            # the hit / record capacity restarts the call with larger buffers.
            cnt_host = torch.zeros((REC_BUFS, 3), dtype=torch.int64, pin_memory=True)
            consumed = []              # chunk indices taken from ``it`` (a restart replays them)
            pending = []               # (chunk index, record buffer, event) awaiting their counts
            need = 0

            def finish(p):
                nonlocal total, overflow, last_i, need
                i_, kr_, ev_ = p
                ev_.synchronize()
                nh = int(cnt_host[kr_][2])
                if nh > self._hits_cap or nh > self._rec_cap:
                    need = max(need, nh)
                    return
                dst = None
                if use_out and not overflow:
                    if i_ > last_i and total + nh <= len(out):
                        dst = out[total:total + nh]
                    else:
                        overflow = True
                if dst is None:
                    dst = torch.empty(max(nh, 1) * self.hit_dtype.itemsize, dtype=torch.uint8,
                                      pin_memory=True).numpy().view(self.hit_dtype)[:nh]
                if nh:   # D2H on its own stream: overlaps the next chunks' kernels (and H2D)
                    self.d2h_stream.wait_event(ev_)
                    with torch.cuda.stream(self.d2h_stream):
                        torch.from_numpy(dst.view(np.uint8)).copy_(self.d_records[kr_][: nh * self.hit_dtype.itemsize],
                                                                   non_blocking=True)
                        e2 = torch.cuda.Event()
                        e2.record(self.d2h_stream)
                    rec_free[kr_] = e2
                results.append((i_, dst))
                total += nh
                last_i = i_

            if self.d_records is None:
                self._reserve_records(self._hits_cap)
            cur = next(it, None)
            if cur is not None:
                consumed.append(cur)
                dchs[0] = load(0, cur, 0)
            j = 0
            while cur is not None:
                i = cur
                nxt = next(it, None)
                if nxt is not None:
                    consumed.append(nxt)
                k, kr = j % nb, j % REC_BUFS
                self.stream.wait_event(loaded[k])
                if nxt is not None:
                    if host.chunks[nxt].n_bases > self._cap_bases:
                        raise ValueError(f"chunk {nxt} is larger than the chunks this call was sized for")
                    dchs[(j + 1) % nb] = load(j + 1, nxt, (j + 1) % nb)
                mark("dev0", j, self.stream)
                self.enqueue_device_chunk(dchs[k], host.chunks[i].n_owned)
                if rec_free[kr] is not None:         # the D2H of chunk j-2 from this buffer is done
                    self.stream.wait_event(rec_free[kr])
                ws.append(torch.empty(ws_bytes, dtype=torch.uint8, device=self.device))
                cof.cof_decorate(self.plan, self.plan_dev, dchs[k], self.d_hits, cof.COF_COUNT_ON_DEVICE,
                                 self.d_records[kr], ws[-1], self.stream, cap=min(self._rec_cap, self._hits_cap))
                cof.cof_counts_async(self.plan, self.plan_dev, cnt_host[kr], self.stream)
                mark("dev1", j, self.stream)
                fr = torch.cuda.Event()
                fr.record(self.stream)
                freed[k] = fr
                pending.append((i, kr, fr))
                # finish every chunk that is done (its records' D2H starts at once), and block
                # only when all record buffers are in flight -- or for the first chunk, whose
                # count sizes the buffers before more chunks are queued on a guess
                while pending and not need and (len(pending) >= REC_BUFS or j == 0 or pending[0][2].query()):
                    finish(pending.pop(0))
                if need:
                    # (scaled to the largest chunk: chunk sizes differ)
                    need = int(need * max(1.0, max_bases / max(1, host.chunks[i].n_bases)))
                    break
                cur = nxt
                j += 1
            while pending and not need:
                finish(pending.pop(0))
            if need:   # a chunk's hits exceeded the buffers: grow them, replay every chunk taken
                self.d2h_stream.synchronize()
                self.stream.synchronize()
                self.copy_stream.synchronize()
                self.reserve(self._cap_bases, max(self._hits_cap, 2 * need + 1024))
                self._reserve_records(2 * need)
                return self.search_host(host, indices if listed else itertools.chain(consumed, it),
                                        out=out, decorate=decorate, sink=sink)
            self.d2h_stream.synchronize()
            self.stream.synchronize()
            if trace:   # COF_TRACE=1: per-chunk H2D / device intervals in ms from the first mark
                import json
                import sys
                t0 = trace[0][2]
                print(json.dumps({"search_host_trace": [(w, jj, round(t0.elapsed_time(e), 3)) for w, jj, e in trace]}),
                      file=sys.stderr)
            for w in ws:
                cof.cof_decorate_check(w, self.stream)
        if sink is not None:
            for i, r in results:
                sink(i, r)
            return None
        if use_out and not overflow:
            return out[:total]
        return merge_hit_lists([r for _, r in sorted(results, key=lambda x: x[0])], self.hit_dtype)

    def search_resident(self, rg: "ResidentGenome", out=None):
        """The search over a genome already resident in this GPU's memory (ResidentGenome:
        planes uploaded once, then searched with any number of guide sets -- the usual
        CRISPR-design loop): per chunk find / compare, device sort and decoration, and the
        records' D2H on a second stream that overlaps the next chunk's kernels.  ``out``:
        as in search_host.  Returns the sorted hit array."""
        if rg.device != self.device:
            raise ValueError(f"resident genome on {rg.device}, searcher on {self.device}")
        max_bases = max((ch.n_bases for ch in rg.chunks), default=1)
        self.reserve(max_bases, max(self._hits_cap, 1 << 16))
        if not hasattr(self, "d2h_stream"):
            self.d2h_stream = torch.cuda.Stream(self.device)
        ws_bytes = cof.cof_decorate_workspace_bytes(max((len(ch.pieces) for ch in rg.chunks), default=1))
        ws, results = [], []
        rec_free = [None] * REC_BUFS
        total, overflow, need = 0, False, 0
        cnt_host = torch.zeros((REC_BUFS, 3), dtype=torch.int64, pin_memory=True)
        pending = []
        if self.d_records is None:
            self._reserve_records(self._hits_cap)

        def finish(p):   # as in search_host: the chunk is done, its count is in pinned memory
            nonlocal total, overflow, need
            kr_, ev_ = p
            ev_.synchronize()
            nh = int(cnt_host[kr_][2])
            if nh > self._hits_cap or nh > self._rec_cap:
                need = max(need, nh)
                return
            dst = None
            if out is not None and not overflow:
                if total + nh <= len(out):
                    dst = out[total:total + nh]
                else:
                    overflow = True
            if dst is None:
                dst = torch.empty(max(nh, 1) * self.hit_dtype.itemsize, dtype=torch.uint8,
                                  pin_memory=True).numpy().view(self.hit_dtype)[:nh]
            if nh:
                self.d2h_stream.wait_event(ev_)
                with torch.cuda.stream(self.d2h_stream):
                    torch.from_numpy(dst.view(np.uint8)).copy_(self.d_records[kr_][: nh * self.hit_dtype.itemsize],
                                                               non_blocking=True)
                    e2 = torch.cuda.Event()
                    e2.record(self.d2h_stream)
                rec_free[kr_] = e2
            results.append(dst)
            total += nh

        with torch.cuda.device(self.device):
            for j, (ch, dch) in enumerate(zip(rg.chunks, rg.d_chunks)):
                kr = j % REC_BUFS
                self.enqueue_device_chunk(dch, ch.n_owned)
                if rec_free[kr] is not None:
                    self.stream.wait_event(rec_free[kr])
                ws.append(torch.empty(ws_bytes, dtype=torch.uint8, device=self.device))
                cof.cof_decorate(self.plan, self.plan_dev, dch, self.d_hits, cof.COF_COUNT_ON_DEVICE,
                                 self.d_records[kr], ws[-1], self.stream, cap=min(self._rec_cap, self._hits_cap))
                cof.cof_counts_async(self.plan, self.plan_dev, cnt_host[kr], self.stream)
                fr = torch.cuda.Event()
                fr.record(self.stream)
                pending.append((kr, fr))
                while pending and not need and (len(pending) >= REC_BUFS or pending[0][1].query()):
                    finish(pending.pop(0))
                if need:
                    break
            while pending and not need:
                finish(pending.pop(0))
            self.d2h_stream.synchronize()
            self.stream.synchronize()
            if need:   # grow the buffers and search again
                self.reserve(self._cap_bases, max(self._hits_cap, 2 * need + 1024))
                self._reserve_records(2 * need)
                return self.search_resident(rg, out=out)
            for w in ws:
                cof.cof_decorate_check(w, self.stream)
        if out is not None and not overflow:
            return out[:total]
        return merge_hit_lists(results, self.hit_dtype)

    def _reserve_records(self, n):
        # REC_BUFS device record buffers: chunk j decorates into one while the D2H of earlier
        # chunks drains the others
        self.d2h_stream.synchronize() if hasattr(self, "d2h_stream") else None
        cap = int(n * 1.25 + 1024)
        self.d_records = [torch.empty(cap * self.hit_dtype.itemsize, dtype=torch.uint8, device=self.device)
                          for _ in range(REC_BUFS)]
        self._rec_cap = cap

    def _search_host_cpu_decorate(self, host: HostGenome, indices=None, out=None):
        """As search_host, decorating on CPU threads (cof_collect) overlapped with the GPU."""
        import queue
        import threading

        idx = list(range(len(host.chunks)) if indices is None else indices)
        max_bases = max((host.chunks[i].n_bases for i in idx), default=1)
        self.reserve(max_bases, max(self._hits_cap, 1 << 16))
        results = {}
        errors = []
        work = queue.Queue()
        ordered = all(a < b for a, b in zip(idx, idx[1:]))
        use_out = out is not None and ordered

        def collector():
            while True:
                job = work.get()
                if job is None:
                    return
                i, ev, keys, nh, dst = job
                try:
                    ev.synchronize()
                    if dst is not None:
                        if nh:
                            cof.cof_collect_into(self.plan, host.chunk_struct(i), keys, nh, dst)
                        results[i] = dst
                    else:
                        results[i] = cof.cof_collect(self.plan, host.chunk_struct(i), None, nh, host_keys=keys)
                except Exception as e:      # surfaced after the join
                    errors.append(e)

        th = threading.Thread(target=collector, daemon=True)
        th.start()
        total = 0
        overflow = False
        try:
            with torch.cuda.device(self.device):
                for i in idx:
                    dch = self.device_chunk(host.chunks[i], None, host.segs[i])
                    host.load(i, dch, self.stream)
                    _, _, nh = self.run_device_chunk(dch, host.chunks[i].n_owned)
                    keys = torch.empty(max(nh, 1), dtype=torch.int64, pin_memory=True)
                    with torch.cuda.stream(self.stream):
                        if nh:
                            keys[:nh].copy_(self.d_hits[:nh], non_blocking=True)
                        ev = torch.cuda.Event()
                        ev.record(self.stream)
                    dst = None
                    if use_out and not overflow:
                        if total + nh <= len(out):
                            dst = out[total:total + nh]
                        else:
                            overflow = True
                    total += nh
                    work.put((i, ev, keys.numpy().view(np.uint64), nh, dst))
                    self.stream.synchronize()    # the single plane buffer is reused next chunk
        finally:
            work.put(None)
            th.join()
        if errors:
            raise errors[0]
        if use_out and not overflow:
            return out[:total]
        return merge_hit_lists([results[i] for i in idx], self.hit_dtype)

def _as_arrays(seqs):
    return [np.frombuffer(s, dtype=np.uint8) if isinstance(s, (bytes, bytearray)) else
            (np.frombuffer(s.encode(), dtype=np.uint8) if isinstance(s, str) else s) for s in seqs]


def search(seqs, pattern, guides, thresholds, chunk_bases=None, device="cuda", pack_bases=None, fused=None,
           path=None):
    """Convenience: whole search of ``seqs`` (list of uint8 ASCII arrays / bytes) on one GPU.
    ``pack_bases`` packs chromosome pieces into multi-segment chunks (0 = one chunk);
    ``fused`` False forces the two-call path (item lists), True the masks path;
    ``path`` = "single" | "fused" | "twocall" picks the device path explicitly (the single
    pass is then run even when its filter is not selective, if the plan's shape allows)."""
    L = len(pattern)
    arrs = _as_arrays(seqs)
    chunks = plan_chunks([len(a) for a in arrs], L, chunk_bases, pack_bases)
    host = HostGenome(arrs, chunks)
    srch = Searcher(pattern, guides, thresholds, device)
    if fused is not None:
        srch.fused = bool(fused)
    if path is not None:
        srch.path = path
    return srch.search_host(host)


# ----------------------------------------------------------------------------- multi-GPU
# The path shards: chromosomes -- and pieces of a chromosome that overlap by L-1 bases --
# are independent (reading G12), and the global order (chrom, pos, strand, guide) is a
# property of the records, so results do not depend on which GPU searched which piece.
# The host concatenates per-chunk lists in genome order (the host collects the
# results; the paper ran one GPU).  No collective touches the data path.

MULTI_CHUNK_BASES = 64_000_000   # owned window starts per work unit (<= 64 Mbp chunk queue)


class ChunkQueue:
    """Thread-safe iterator over chunk indices in genome order: the shared work queue the
    per-GPU pipelines of search_multi pop from (dynamic balance: a GPU that finishes early
    takes the next chunk)."""

    def __init__(self, n: int):
        import threading
        self._it = iter(range(n))
        self._lock = threading.Lock()

    def __iter__(self):
        return self

    def __next__(self):
        with self._lock:
            return next(self._it)


def search_multi(seqs, pattern, guides, thresholds, devices=None, chunk_bases=MULTI_CHUNK_BASES, host=None,
                 streams_per_device: int = 1):
    """Single-process multi-GPU search: the genome cut into chunks of <= ``chunk_bases``
    owned window starts, one host thread per GPU (``devices``; default every visible GPU;
    a device may repeat) running its own Searcher pipeline over chunks popped from one
    shared queue in genome order; the merge is the concatenation of the per-chunk lists in
    chunk order (cof_merge's parallel fast path).  ``host``: a prebuilt HostGenome."""
    import threading
    if host is None:
        arrs = _as_arrays(seqs)
        host = HostGenome(arrs, plan_chunks([len(a) for a in arrs], len(pattern), chunk_bases))
    if devices is None:
        devices = [f"cuda:{k}" for k in range(torch.cuda.device_count())]
    devices = [torch.device(d) for d in devices for _ in range(max(1, streams_per_device))]
    if not devices:
        raise RuntimeError("search_multi: no CUDA device")
    queue = ChunkQueue(len(host.chunks))
    per_chunk = [None] * len(host.chunks)
    errors = []

    def sink(i, recs):
        per_chunk[i] = recs

    def worker(dev):
        try:
            torch.cuda.set_device(dev)
            srch = Searcher(pattern, guides, thresholds, device=dev, stream=torch.cuda.Stream(dev))
            srch.search_host(host, indices=queue, sink=sink)
        except BaseException as e:   # surfaced after the join
            errors.append(e)

    threads = [threading.Thread(target=worker, args=(d,), daemon=True) for d in devices]
    for t in threads:
        t.start()
    for t in threads:
        t.join()
    if errors:
        raise errors[0]
    missing = [i for i, r in enumerate(per_chunk) if r is None]
    if missing:
        raise RuntimeError(f"search_multi: chunks {missing[:5]} were not searched")
    return merge_hit_lists(per_chunk, cof.hit_dtype(len(pattern)))


def shard_for_rank(chunks, rank: int, world: int):
    """This rank's chunks (LPT over owned window starts; ranks are independent)."""
    return shard_lpt(chunks, world)[rank]


def shard_indices(chunks, world: int):
    """LPT shards as chunk INDEX lists (genome order inside each shard)."""
    idx = {id(c): i for i, c in enumerate(chunks)}
    return [[idx[id(c)] for c in sh] for sh in shard_lpt(chunks, world)]


def _coll_device(group=None):
    import torch.distributed as dist
    return torch.device("cuda", torch.cuda.current_device()) if dist.get_backend(group) == "nccl" else torch.device("cpu")


_MERGE_ARENAS = {}   # per process group: the shared-memory result buffer every rank keeps mapped


def _merge_arena(nbytes: int, group, dst: int, shm_dir=None):
    """The group's shared result buffer, at least ``nbytes``: one file in /dev/shm created by
    ``dst``, mapped by every rank and unlinked at once (the mappings keep it alive).  It is
    reused by later merges of the same group, so its pages are faulted in once -- mapping a
    fresh file per merge cost ~0.1 s per 100 MB in page faults."""
    import tempfile
    import uuid
    import torch.distributed as dist
    key = id(group) if group is not None else None
    arena = _MERGE_ARENAS.get(key)
    need = [arena is None or arena.size < nbytes]
    # every rank sees the same counts, hence the same decision; no collective needed for it
    if need[0]:
        size = max(int(nbytes * 1.25), 1 << 20)
        name = [None]
        if dist.get_rank(group) == dst:
            d = shm_dir
            if d is None:   # /dev/shm when it has room (a container's may be 64 MB), else the temp dir
                d = tempfile.gettempdir()
                if os.path.isdir("/dev/shm"):
                    st = os.statvfs("/dev/shm")
                    if st.f_bavail * st.f_frsize >= size + (64 << 20):
                        d = "/dev/shm"
            name[0] = os.path.join(d, f"cof_merge_{uuid.uuid4().hex}.bin")
            with open(name[0], "wb") as f:
                f.truncate(size)
        dist.broadcast_object_list(name, src=dst, group=group)
        arena = np.memmap(name[0], dtype=np.uint8, mode="r+", shape=(size,))
        dist.barrier(group=group)
        if dist.get_rank(group) == dst:
            os.unlink(name[0])
        _MERGE_ARENAS[key] = arena
    return arena


def merge_dist(per_chunk: dict, n_chunks: int, dtype, group=None, dst: int = 0, shm_dir=None):
    """Host merge of a torchrun job (one process per GPU): ``per_chunk`` maps this rank's
    global chunk indices to their sorted records.  Per-chunk hit counts are summed over
    the ranks (one small all-reduce), their exclusive prefix gives every chunk's offset in
    the genome-ordered result, and every rank copies its records straight into that slice
    of one shared-memory buffer (all ranks of a torchrun job share the node; the buffer is
    kept mapped across merges) -- the merge is a parallel concatenation, no record crosses
    the process group.  Returns the merged array on ``dst`` (a view of the shared buffer,
    valid until the group's next merge_dist) and None elsewhere."""
    import torch.distributed as dist
    rank = dist.get_rank(group)
    cd = _coll_device(group)
    counts = torch.zeros(n_chunks, dtype=torch.int64)
    for i, r in per_chunk.items():
        counts[i] = len(r)
    counts = counts.to(cd)
    dist.all_reduce(counts, group=group)
    counts = counts.cpu().numpy()
    offs = np.zeros(n_chunks + 1, dtype=np.int64)
    np.cumsum(counts, out=offs[1:])
    total = int(offs[-1])
    isz = dtype.itemsize
    arena = _merge_arena(max(1, total) * isz, group, dst, shm_dir)
    out = arena[: total * isz].view(dtype) if total else np.zeros(0, dtype=dtype)
    for i, r in per_chunk.items():
        if len(r):   # (a byte copy -- torch's is multi-threaded; numpy's field-wise one was 4x slower)
            torch.from_numpy(arena[offs[i] * isz:(offs[i] + len(r)) * isz]).copy_(
                torch.from_numpy(np.ascontiguousarray(r).view(np.uint8)))
    dist.barrier(group=group)
    return out if rank == dst else None


def search_dist(seqs, pattern, guides, thresholds, chunk_bases=MULTI_CHUNK_BASES, group=None, device=None,
                dst: int = 0):
    """Multi-process multi-GPU search (torchrun, one rank per GPU): every rank plans the
    same chunks, packs and searches its LPT share (search_host pipeline on its GPU) and
    the ranks merge through merge_dist.  Returns the merged list on ``dst``, None elsewhere."""
    import torch.distributed as dist
    rank, world = dist.get_rank(group), dist.get_world_size(group)
    arrs = _as_arrays(seqs)
    chunks = plan_chunks([len(a) for a in arrs], len(pattern), chunk_bases)
    mine = shard_indices(chunks, world)[rank]
    dev = torch.device(device) if device is not None else torch.device("cuda", torch.cuda.current_device())
    per = {}
    if mine:
        host = HostGenome(arrs, [chunks[i] for i in mine])
        srch = Searcher(pattern, guides, thresholds, device=dev)
        srch.search_host(host, sink=lambda j, r: per.__setitem__(mine[j], r))
    return merge_dist(per, len(chunks), cof.hit_dtype(len(pattern)), group=group, dst=dst)


def gather_and_merge(local_hits: np.ndarray, group=None, dst: int = 0):
    """Merge of per-rank hit lists that each cover whole genome-ordered chunks (host
    objects over the process group; kept for callers with one list per rank -- the
    product path is merge_dist)."""
    import torch.distributed as dist
    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    buf = [None] * world if rank == dst else None
    dist.gather_object(local_hits.tobytes(), buf, dst=dst, group=group)
    if rank != dst:
        return None
    lists = [np.frombuffer(b, dtype=local_hits.dtype) for b in buf]
    return merge_hit_lists(lists, local_hits.dtype)

"""Thin Python binding of ``libcof.so`` (include/cof.h) -- argument marshalling only.

Every function here has the name of the C entry point it calls and does no arithmetic of
the method: it converts torch tensors / numpy arrays to pointers, CUDA streams to
handles, and non-zero status codes to :class:`CofError`.  There is no CPU fallback: if
the shared library is missing the import fails loudly.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
# (COF_LIB: an alternative build of the same library, for A/B measurements of kernel variants)
LIB_PATH = os.environ.get("COF_LIB") or os.path.join(HERE, "libcof.so")

COF_OK = 0
COF_E_ARG = -1
COF_E_CAPACITY = -2
COF_E_CUDA = -3
COF_E_STATE = -4
COF_E_IO = -5
COF_COUNT_ON_DEVICE = (1 << 64) - 1

HIT_DTYPE = np.dtype([("guide", "<u4"), ("chrom", "<u4"), ("pos", "<u8"), ("strand", "S1"),
                      ("mm", "u1"), ("site", "S34")], align=True)
# cof_hit64: the record of patterns with 32 < L <= COF_MAX_L
HIT64_DTYPE = np.dtype([("guide", "<u4"), ("chrom", "<u4"), ("pos", "<u8"), ("strand", "S1"),
                        ("mm", "u1"), ("site", "S66"), ("_pad", "V4")], align=True)
COF_MAX_L = 64
assert HIT_DTYPE.itemsize == 56 and HIT64_DTYPE.itemsize == 88


def hit_dtype(L: int) -> np.dtype:
    """Record dtype of a plan with pattern length L (cof_hit for L <= 32, else cof_hit64)."""
    return HIT_DTYPE if L <= 32 else HIT64_DTYPE


class CofError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"cof status {status}: {msg}")
        self.status = status


class cof_segment(ctypes.Structure):
    _fields_ = [("chrom", ctypes.c_uint32), ("reserved", ctypes.c_uint32), ("chunk_off", ctypes.c_uint64),
                ("chrom_off", ctypes.c_uint64), ("n_owned", ctypes.c_uint64)]


class cof_chunk(ctypes.Structure):
    _fields_ = [("chrom", ctypes.c_uint32), ("n_segs", ctypes.c_uint32), ("start", ctypes.c_uint64),
                ("n_bases", ctypes.c_uint64), ("n_owned", ctypes.c_uint64),
                ("lo", ctypes.c_void_p), ("hi", ctypes.c_void_p), ("nm", ctypes.c_void_p),
                ("vs", ctypes.c_void_p), ("segs", ctypes.c_void_p)]


def _load():
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} is missing: run `python -m paper_conf_socc_jinv23_b200.build` "
                          "(there is no CPU fallback)")
    L = ctypes.CDLL(LIB_PATH)
    P, U32, U64, SZ, I32 = ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint64, ctypes.c_size_t, ctypes.c_int32
    sig = {
        "cof_last_error": (ctypes.c_char_p, []),
        "cof_version": (ctypes.c_char_p, []),
        "cof_set_host_threads": (I32, [I32]),
        "cof_launch_count": (U64, []),
        "cof_plan_create": (I32, [ctypes.c_char_p, U32, P, P, P]),
        "cof_plan_destroy": (None, [P]),
        "cof_plan_length": (U32, [P]),
        "cof_plan_n_guides": (U32, [P]),
        "cof_plan_device_bytes": (SZ, [P]),
        "cof_plan_upload": (I32, [P, P, P]),
        "cof_plane_words": (U64, [U64]),
        "cof_pack": (I32, [P, U64, P, P, P]),
        "cof_unpack": (I32, [P, P, P, U64, U64, P]),
        "cof_load_chunk": (I32, [P, P, P]),
        "cof_valid_starts": (I32, [P, U32, U64, P]),
        "cof_fasta_open": (I32, [ctypes.c_char_p, P]),
        "cof_fasta_close": (None, [P]),
        "cof_fasta_count": (U32, [P]),
        "cof_fasta_name": (ctypes.c_char_p, [P, U32]),
        "cof_fasta_length": (U64, [P, U32]),
        "cof_fasta_pack": (I32, [P, U32, U64, U64, P, P, P]),
        "cof_find_workspace_bytes": (SZ, [U64]),
        "cof_find_pam": (I32, [P, P, P, P, P, P, U64, P, P, P]),
        "cof_compare": (I32, [P, P, P, P, U64, P, U64, P, U64, P, P]),
        "cof_sort_workspace_bytes": (SZ, [U64]),
        "cof_sort_hits": (I32, [P, P, P, P, P, U64, U64, P, P]),
        "cof_read_counts": (I32, [P, P, P, P]),
        "cof_counts_async": (I32, [P, P, P, P]),
        "cof_n_runs": (I32, [P, U64, P, U64, P]),
        "cof_load_chunk_runs": (I32, [P, P, U64, P, P]),
        "cof_load_chunk_runs_split": (I32, [P, P, U64, P, P, P]),
        "cof_collect": (I32, [P, P, P, P, U64, P, P]),
        "cof_collect64": (I32, [P, P, P, P, U64, P, P]),
        "cof_merge": (I32, [P, P, U32, P]),
        "cof_merge64": (I32, [P, P, U32, P]),
        "cof_decorate_workspace_bytes": (SZ, [U32]),
        "cof_decorate": (I32, [P, P, P, P, U64, U64, P, P, P]),
        "cof_decorate64": (I32, [P, P, P, P, U64, U64, P, P, P]),
        "cof_decorate_check": (I32, [P, P]),
        "cof_find_compare_supported": (ctypes.c_int, [P]),
        "cof_single_supported": (ctypes.c_int, [P]),
        "cof_search_single": (I32, [P, P, P, P, P, U64, P, P]),
        "cof_find_compare_workspace_bytes": (SZ, [U64]),
        "cof_find_compare": (I32, [P, P, P, P, P, U64, P, P]),
        "cof_find_masks": (I32, [P, P, P, P, P]),
        "cof_compare_masks": (I32, [P, P, P, P, P, U64, P, P]),
        "cof_2bit_open": (I32, [ctypes.c_char_p, P]),
        "cof_2bit_close": (None, [P]),
        "cof_2bit_count": (U32, [P]),
        "cof_2bit_name": (ctypes.c_char_p, [P, U32]),
        "cof_2bit_length": (U64, [P, U32]),
        "cof_2bit_pack": (I32, [P, U32, U64, U64, P, P, P]),
        "cof_set_comparer": (I32, [ctypes.c_int]),
    }
    for name, (res, args) in sig.items():
        f = getattr(L, name)
        f.restype = res
        f.argtypes = args
    return L


lib = _load()

# names the header declares (checked by tests/test_abi_host.py)
EXPORTS = [n for n in ("cof_last_error", "cof_version", "cof_set_host_threads", "cof_launch_count", "cof_plan_create",
                       "cof_plan_destroy", "cof_plan_length", "cof_plan_n_guides",
                       "cof_plan_device_bytes", "cof_plan_upload", "cof_plane_words", "cof_pack",
                       "cof_unpack", "cof_valid_starts", "cof_load_chunk", "cof_fasta_open", "cof_fasta_close",
                       "cof_fasta_count", "cof_fasta_name", "cof_fasta_length", "cof_fasta_pack",
                       "cof_find_workspace_bytes", "cof_find_pam", "cof_compare",
                       "cof_sort_workspace_bytes", "cof_sort_hits", "cof_read_counts", "cof_counts_async",
                       "cof_n_runs", "cof_load_chunk_runs", "cof_load_chunk_runs_split", "cof_collect", "cof_collect64", "cof_merge", "cof_merge64",
                       "cof_decorate_workspace_bytes", "cof_decorate", "cof_decorate64",
                       "cof_decorate_check", "cof_find_compare_supported",
                       "cof_find_compare_workspace_bytes", "cof_find_compare", "cof_find_masks",
                       "cof_compare_masks", "cof_single_supported", "cof_search_single", "cof_set_comparer", "cof_2bit_open",
                       "cof_2bit_close", "cof_2bit_count", "cof_2bit_name", "cof_2bit_length",
                       "cof_2bit_pack")]


def _check(st):
    if st != COF_OK:
        raise CofError(st, lib.cof_last_error().decode(errors="replace"))


def _ptr(x):
    """Address of a tensor / ndarray / int / None."""
    if x is None:
        return None
    if isinstance(x, int):
        return x
    if hasattr(x, "data_ptr"):
        return x.data_ptr()
    if isinstance(x, np.ndarray):
        return x.ctypes.data
    if isinstance(x, (ctypes.Array, ctypes.Structure)):
        return ctypes.addressof(x)
    raise TypeError(f"cannot take the address of {type(x)}")


def _stream(s):
    if s is None:
        return None
    if isinstance(s, int):
        return s
    return s.cuda_stream


def cof_last_error() -> str:
    return lib.cof_last_error().decode(errors="replace")


def cof_version() -> str:
    return lib.cof_version().decode()


def cof_set_host_threads(n: int) -> int:
    """Threads of the library's host OpenMP regions (n <= 0: unchanged); returns the setting."""
    return int(lib.cof_set_host_threads(int(n)))


def cof_launch_count() -> int:
    return int(lib.cof_launch_count())


class Plan:
    """Owns a ``cof_plan*``."""

    def __init__(self, handle, pattern, guides, max_mm):
        self.handle = handle
        self.pattern = pattern
        self.guides = list(guides)
        self.max_mm = list(max_mm)

    @property
    def L(self):
        return int(lib.cof_plan_length(self.handle))

    @property
    def n_guides(self):
        return int(lib.cof_plan_n_guides(self.handle))

    def __del__(self):
        h, self.handle = getattr(self, "handle", None), None
        if h and lib is not None:
            lib.cof_plan_destroy(h)


def cof_plan_create(pattern: str, guides, max_mm) -> Plan:
    gs = [g.encode() for g in guides]
    arr = (ctypes.c_char_p * max(len(gs), 1))(*gs)
    mm = np.ascontiguousarray(np.asarray(max_mm, dtype=np.uint8))
    out = ctypes.c_void_p()
    _check(lib.cof_plan_create(pattern.encode(), len(gs), ctypes.addressof(arr), mm.ctypes.data,
                               ctypes.addressof(out)))
    return Plan(out.value, pattern, guides, max_mm)


def cof_plan_device_bytes(plan: Plan) -> int:
    return int(lib.cof_plan_device_bytes(plan.handle))


def cof_plan_upload(plan: Plan, plan_dev, stream=None):
    _check(lib.cof_plan_upload(plan.handle, _ptr(plan_dev), _stream(stream)))


def cof_plane_words(n_bases: int) -> int:
    return int(lib.cof_plane_words(int(n_bases)))


def cof_pack(ascii_arr, n, lo, hi, nm):
    _check(lib.cof_pack(_ptr(ascii_arr), int(n), _ptr(lo), _ptr(hi), _ptr(nm)))


def cof_unpack(lo, hi, nm, first, n, out):
    _check(lib.cof_unpack(_ptr(lo), _ptr(hi), _ptr(nm), int(first), int(n), _ptr(out)))


def make_chunk(chrom, start, n_bases, n_owned, lo, hi, nm, vs=None, segs=None) -> cof_chunk:
    """Single-segment chunk (segs None) or multi-segment chunk (segs = cof_segment array, vs plane)."""
    c = cof_chunk(int(chrom), 0 if segs is None else len(segs), int(start), int(n_bases), int(n_owned),
                  _ptr(lo), _ptr(hi), _ptr(nm), _ptr(vs), None if segs is None else ctypes.addressof(segs))
    c._keep = segs          # the host segment table must outlive the struct
    return c


def make_segments(rows):
    """rows = [(chrom, chunk_off, chrom_off, n_owned), ...] -> cof_segment array."""
    arr = (cof_segment * max(len(rows), 1))()
    for k, (c, co, so, no) in enumerate(rows):
        arr[k] = cof_segment(int(c), 0, int(co), int(so), int(no))
    return arr


def cof_valid_starts(segs, n_segs, n_bases, vs):
    _check(lib.cof_valid_starts(ctypes.addressof(segs), int(n_segs), int(n_bases), _ptr(vs)))


def cof_load_chunk(host: cof_chunk, dev: cof_chunk, stream=None):
    _check(lib.cof_load_chunk(ctypes.addressof(host), ctypes.addressof(dev), _stream(stream)))


def cof_n_runs(nm, n_bases: int) -> np.ndarray:
    """[begin, end) runs of N bases of an nm plane, as an (n, 2) uint64 array."""
    cnt = ctypes.c_uint64(0)
    cap = 4096
    while True:
        runs = np.empty((cap, 2), dtype=np.uint64)
        st = lib.cof_n_runs(_ptr(nm), int(n_bases), runs.ctypes.data, cap, ctypes.byref(cnt))
        if st == COF_E_CAPACITY:
            cap = int(cnt.value)
            continue
        _check(st)
        return runs[: int(cnt.value)]


def cof_load_chunk_runs(host: cof_chunk, runs: np.ndarray, dev: cof_chunk, stream=None):
    """cof_load_chunk with nm (from ``runs``) and vs (from the segments) built on the device."""
    runs = np.ascontiguousarray(runs, dtype=np.uint64)
    _check(lib.cof_load_chunk_runs(ctypes.addressof(host), runs.ctypes.data if len(runs) else None, len(runs),
                                   ctypes.addressof(dev), _stream(stream)))


def cof_load_chunk_runs_split(host: cof_chunk, runs: np.ndarray, dev: cof_chunk, copy_stream, fill_stream):
    """cof_load_chunk_runs with the lo/hi DMA on ``copy_stream`` and the fills on ``fill_stream``."""
    runs = np.ascontiguousarray(runs, dtype=np.uint64)
    _check(lib.cof_load_chunk_runs_split(ctypes.addressof(host), runs.ctypes.data if len(runs) else None, len(runs),
                                         ctypes.addressof(dev), _stream(copy_stream), _stream(fill_stream)))


def cof_find_workspace_bytes(n_bases: int) -> int:
    return int(lib.cof_find_workspace_bytes(int(n_bases)))


def cof_find_pam(plan, plan_dev, dev: cof_chunk, workspace, items_fwd, items_rev, items_cap,
                 stream=None, sync=True):
    """Returns (n_fwd, n_rev) if ``sync`` else None (counts stay on the device)."""
    if sync:
        a, b = ctypes.c_uint64(), ctypes.c_uint64()
        _check(lib.cof_find_pam(plan.handle, _ptr(plan_dev), ctypes.addressof(dev), _ptr(workspace),
                                _ptr(items_fwd), _ptr(items_rev), int(items_cap), ctypes.addressof(a),
                                ctypes.addressof(b), _stream(stream)))
        return int(a.value), int(b.value)
    _check(lib.cof_find_pam(plan.handle, _ptr(plan_dev), ctypes.addressof(dev), _ptr(workspace),
                            _ptr(items_fwd), _ptr(items_rev), int(items_cap), None, None, _stream(stream)))
    return None


def cof_compare(plan, plan_dev, dev: cof_chunk, items_fwd, n_fwd, items_rev, n_rev, hits, hits_cap,
                stream=None, sync=True):
    """Returns n_hits if ``sync`` else None.  n_fwd/n_rev may be COF_COUNT_ON_DEVICE."""
    if sync:
        n = ctypes.c_uint64()
        _check(lib.cof_compare(plan.handle, _ptr(plan_dev), ctypes.addressof(dev), _ptr(items_fwd),
                               int(n_fwd), _ptr(items_rev), int(n_rev), _ptr(hits), int(hits_cap),
                               ctypes.addressof(n), _stream(stream)))
        return int(n.value)
    _check(lib.cof_compare(plan.handle, _ptr(plan_dev), ctypes.addressof(dev), _ptr(items_fwd), int(n_fwd),
                           _ptr(items_rev), int(n_rev), _ptr(hits), int(hits_cap), None, _stream(stream)))
    return None


def cof_find_compare_supported(plan) -> bool:
    return bool(lib.cof_find_compare_supported(plan.handle))


def cof_find_compare_workspace_bytes(n_bases: int) -> int:
    return int(lib.cof_find_compare_workspace_bytes(int(n_bases)))


def cof_find_compare(plan, plan_dev, dev: cof_chunk, workspace, hits, hits_cap, stream=None, sync=True):
    """Fused finder + comparer; returns n_hits if ``sync`` else None (count stays on the device)."""
    if sync:
        n = ctypes.c_uint64()
        _check(lib.cof_find_compare(plan.handle, _ptr(plan_dev), ctypes.addressof(dev), _ptr(workspace),
                                    _ptr(hits), int(hits_cap), ctypes.addressof(n), _stream(stream)))
        return int(n.value)
    _check(lib.cof_find_compare(plan.handle, _ptr(plan_dev), ctypes.addressof(dev), _ptr(workspace),
                                _ptr(hits), int(hits_cap), None, _stream(stream)))
    return None


def cof_single_supported(plan) -> bool:
    return bool(lib.cof_single_supported(plan.handle))


def cof_search_single(plan, plan_dev, dev: cof_chunk, workspace, hits, hits_cap, stream=None, sync=True):
    """Single-pass find + compare (one streaming kernel); returns n_hits if ``sync`` else None."""
    if sync:
        n = ctypes.c_uint64()
        _check(lib.cof_search_single(plan.handle, _ptr(plan_dev), ctypes.addressof(dev), _ptr(workspace),
                                     _ptr(hits), int(hits_cap), ctypes.addressof(n), _stream(stream)))
        return int(n.value)
    _check(lib.cof_search_single(plan.handle, _ptr(plan_dev), ctypes.addressof(dev), _ptr(workspace),
                                 _ptr(hits), int(hits_cap), None, _stream(stream)))
    return None


def cof_find_masks(plan, plan_dev, dev: cof_chunk, workspace, stream=None):
    _check(lib.cof_find_masks(plan.handle, _ptr(plan_dev), ctypes.addressof(dev), _ptr(workspace), _stream(stream)))


def cof_compare_masks(plan, plan_dev, dev: cof_chunk, workspace, hits, hits_cap, stream=None, sync=True):
    if sync:
        n = ctypes.c_uint64()
        _check(lib.cof_compare_masks(plan.handle, _ptr(plan_dev), ctypes.addressof(dev), _ptr(workspace),
                                     _ptr(hits), int(hits_cap), ctypes.addressof(n), _stream(stream)))
        return int(n.value)
    _check(lib.cof_compare_masks(plan.handle, _ptr(plan_dev), ctypes.addressof(dev), _ptr(workspace),
                                 _ptr(hits), int(hits_cap), None, _stream(stream)))
    return None


def cof_sort_workspace_bytes(cap: int) -> int:
    return int(lib.cof_sort_workspace_bytes(int(cap)))


def cof_sort_hits(plan, plan_dev, dev: cof_chunk, hits, tmp, cap, n_hits, workspace, stream=None):
    _check(lib.cof_sort_hits(plan.handle, _ptr(plan_dev), ctypes.addressof(dev), _ptr(hits), _ptr(tmp),
                             int(cap), int(n_hits), _ptr(workspace), _stream(stream)))


def cof_read_counts(plan, plan_dev, stream=None):
    out = (ctypes.c_uint64 * 3)()
    _check(lib.cof_read_counts(plan.handle, _ptr(plan_dev), ctypes.addressof(out), _stream(stream)))
    return int(out[0]), int(out[1]), int(out[2])


def cof_counts_async(plan, plan_dev, out_host, stream=None):
    """Async copy of the three device counters into ``out_host`` (a pinned uint64 tensor or
    array of >= 3 elements) on ``stream``; read it after an event recorded behind it."""
    _check(lib.cof_counts_async(plan.handle, _ptr(plan_dev), _ptr(out_host), _stream(stream)))


def _collect_fn(plan):
    return lib.cof_collect if plan.L <= 32 else lib.cof_collect64


def cof_collect(plan, host: cof_chunk, hits_dev, n_hits, stream=None, host_keys=None) -> np.ndarray:
    """cof_collect (L <= 32, cof_hit records) or cof_collect64 (L > 32, cof_hit64)."""
    out = np.empty(int(n_hits), dtype=hit_dtype(plan.L))
    if n_hits:
        _check(_collect_fn(plan)(plan.handle, ctypes.addressof(host), _ptr(hits_dev), _ptr(host_keys),
                                 int(n_hits), out.ctypes.data, _stream(stream)))
    return out


def cof_collect_into(plan, host: cof_chunk, host_keys, n_hits, out: np.ndarray):
    """cof_collect from host keys into a caller-provided (contiguous) record array."""
    if not out.flags["C_CONTIGUOUS"] or out.dtype != hit_dtype(plan.L) or len(out) < n_hits:
        raise ValueError("out must be a contiguous hit_dtype(L) array of >= n_hits records")
    if n_hits:
        _check(_collect_fn(plan)(plan.handle, ctypes.addressof(host), None, _ptr(host_keys), int(n_hits),
                                 out.ctypes.data, None))
    return out


def cof_decorate_workspace_bytes(n_segs: int) -> int:
    return int(lib.cof_decorate_workspace_bytes(int(n_segs)))


def cof_decorate(plan, plan_dev, dev: cof_chunk, hits_dev, n_hits, out_dev, workspace, stream=None, cap=0):
    """Device decoration: n_hits keys -> n_hits cof_hit records in the device buffer out_dev
    (n_hits = COF_COUNT_ON_DEVICE: the device count clamped to ``cap``); cof_hit64 records
    (cof_decorate64) when L > 32."""
    fn = lib.cof_decorate if plan.L <= 32 else lib.cof_decorate64
    _check(fn(plan.handle, _ptr(plan_dev), ctypes.addressof(dev), _ptr(hits_dev), int(n_hits),
                            int(cap), _ptr(out_dev), _ptr(workspace), _stream(stream)))


def cof_decorate_check(workspace, stream=None):
    _check(lib.cof_decorate_check(_ptr(workspace), _stream(stream)))


def cof_merge(lists) -> np.ndarray:
    """cof_merge (cof_hit lists) or cof_merge64 (cof_hit64 lists, any list of HIT64_DTYPE)."""
    wide = any(getattr(x, "dtype", None) == HIT64_DTYPE for x in lists)
    dt = HIT64_DTYPE if wide else HIT_DTYPE
    lists = [np.ascontiguousarray(x, dtype=dt) for x in lists]
    total = sum(len(x) for x in lists)
    out = np.empty(total, dtype=dt)
    ptrs = (ctypes.c_void_p * max(len(lists), 1))(*[x.ctypes.data for x in lists])
    lens = (ctypes.c_uint64 * max(len(lists), 1))(*[len(x) for x in lists])
    fn = lib.cof_merge64 if wide else lib.cof_merge
    _check(fn(ctypes.addressof(ptrs), ctypes.addressof(lens), len(lists), out.ctypes.data))
    return out


def cof_set_comparer(impl: str):
    """'table' (bit-sliced pair tables, default) or 'popc' (POPC per comparison)."""
    _check(lib.cof_set_comparer({"popc": 0, "table": 1}[impl]))


class Fasta:
    def __init__(self, path):
        out = ctypes.c_void_p()
        _check(lib.cof_fasta_open(str(path).encode(), ctypes.addressof(out)))
        self.handle = out.value

    def __len__(self):
        return int(lib.cof_fasta_count(self.handle))

    def name(self, i):
        return lib.cof_fasta_name(self.handle, i).decode()

    def length(self, i):
        return int(lib.cof_fasta_length(self.handle, i))

    def pack(self, i, first, n, lo, hi, nm):
        _check(lib.cof_fasta_pack(self.handle, i, int(first), int(n), _ptr(lo), _ptr(hi), _ptr(nm)))

    def read(self, i) -> np.ndarray:
        """Record i in canonical form (upper-case ACGT, N for anything else) as uint8 ASCII:
        packed to planes and unpacked (the same canonicalisation as the device path)."""
        n = self.length(i)
        w = cof_plane_words(n)
        planes = np.zeros((3, max(w, 1)), dtype=np.uint32)
        out = np.empty(n, dtype=np.uint8)
        if n:
            self.pack(i, 0, n, planes[0], planes[1], planes[2])
            cof_unpack(planes[0], planes[1], planes[2], 0, n, out)
        return out

    def close(self):
        if self.handle:
            lib.cof_fasta_close(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class TwoBit(Fasta):
    """UCSC .2bit genome (same interface as Fasta: len, name, length, pack, read)."""

    def __init__(self, path):
        out = ctypes.c_void_p()
        _check(lib.cof_2bit_open(str(path).encode(), ctypes.addressof(out)))
        self.handle = out.value

    def __len__(self):
        return int(lib.cof_2bit_count(self.handle))

    def name(self, i):
        return lib.cof_2bit_name(self.handle, i).decode()

    def length(self, i):
        return int(lib.cof_2bit_length(self.handle, i))

    def pack(self, i, first, n, lo, hi, nm):
        _check(lib.cof_2bit_pack(self.handle, i, int(first), int(n), _ptr(lo), _ptr(hi), _ptr(nm)))

    def close(self):
        if self.handle:
            lib.cof_2bit_close(self.handle)
            self.handle = None


def open_genome(path):
    """Fasta or TwoBit by file name (.2bit -> TwoBit)."""
    return TwoBit(path) if str(path).lower().endswith(".2bit") else Fasta(path)


def hits_to_tuples(arr):
    """(chrom, pos, strand, guide, mm, site) tuples (same serialization as the tests use)."""
    return [(int(h["chrom"]), int(h["pos"]), h["strand"].decode(), int(h["guide"]), int(h["mm"]),
             h["site"].decode()) for h in arr]

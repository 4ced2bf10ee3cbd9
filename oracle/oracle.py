"""ctypes wrapper around ``oracle/cof_oracle.c`` -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (cpu_baseline and
``--impl reference``) may import this module.  The product path
(``paper_conf_socc_jinv23_b200``) never does.

See the header of ``cof_oracle.c`` for the definition it computes and the paper
passages it follows.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
SRC = os.path.join(HERE, "cof_oracle.c")
LIB = os.path.join(HERE, "liboracle.so")

HIT_DTYPE = np.dtype([("guide", "<i4"), ("chrom", "<i4"), ("pos", "<i8"),
                      ("strand", "S1"), ("mm", "i1"), ("site", "S66")], align=True)


def build(force: bool = False) -> str:
    """Compile the oracle with gcc/OpenMP (building the checker is not using it)."""
    if force or not os.path.exists(LIB) or os.path.getmtime(LIB) < os.path.getmtime(SRC):
        tmp = LIB + f".{os.getpid()}.tmp"
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-shared", "-fPIC", "-std=c11",
                               "-Wall", "-o", tmp, SRC])
        os.replace(tmp, LIB)
    return LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(LIB)
        L.cof_oracle_search.restype = ctypes.c_int64
        L.cof_oracle_search.argtypes = [
            ctypes.c_int32, ctypes.POINTER(ctypes.c_char_p), ctypes.POINTER(ctypes.c_int64),
            ctypes.POINTER(ctypes.c_int64), ctypes.POINTER(ctypes.c_int64),
            ctypes.c_char_p, ctypes.c_int32, ctypes.POINTER(ctypes.c_char_p),
            ctypes.POINTER(ctypes.c_int32), ctypes.c_int32, ctypes.POINTER(ctypes.c_void_p)]
        L.cof_oracle_pam_sites.restype = ctypes.c_int64
        L.cof_oracle_pam_sites.argtypes = [
            ctypes.c_char_p, ctypes.c_int64, ctypes.c_int64, ctypes.c_int64,
            ctypes.c_char_p, ctypes.c_char, ctypes.POINTER(ctypes.c_void_p)]
        L.cof_oracle_free.argtypes = [ctypes.c_void_p]
        L.cof_oracle_contains.restype = ctypes.c_int
        L.cof_oracle_contains.argtypes = [ctypes.c_char, ctypes.c_char]
        L.cof_oracle_canon.restype = ctypes.c_char
        L.cof_oracle_canon.argtypes = [ctypes.c_char]
        L.cof_oracle_complement_base.restype = ctypes.c_char
        L.cof_oracle_complement_base.argtypes = [ctypes.c_char]
        L.cof_oracle_max_threads.restype = ctypes.c_int32
        assert L.cof_oracle_hit_size() == HIT_DTYPE.itemsize, "oracle_hit layout"
        _lib = L
    return _lib


def _as_bytes(s):
    if isinstance(s, np.ndarray):
        return s.tobytes()
    if isinstance(s, str):
        return s.encode()
    return bytes(s)


def search(seqs, pattern, guides, thresholds, ranges=None, threads: int = 0) -> np.ndarray:
    """Brute-force hit list as a structured array (``HIT_DTYPE``), sorted by
    (chrom, pos, strand '+' before '-', guide).  ``ranges`` = optional list of
    (begin, end) window-start ranges, one per chromosome."""
    L = lib()
    keep = [np.ascontiguousarray(s) if isinstance(s, np.ndarray) else _as_bytes(s) for s in seqs]
    n = len(keep)
    addrs = [ctypes.cast(k.ctypes.data, ctypes.c_char_p) if isinstance(k, np.ndarray) else k for k in keep]
    cseqs = (ctypes.c_char_p * max(n, 1))(*addrs)
    lens = (ctypes.c_int64 * max(n, 1))(*[len(k) for k in keep])
    beg = end = None
    if ranges is not None:
        beg = (ctypes.c_int64 * n)(*[r[0] for r in ranges])
        end = (ctypes.c_int64 * n)(*[r[1] for r in ranges])
    gs = (ctypes.c_char_p * max(len(guides), 1))(*[g.encode() for g in guides])
    th = (ctypes.c_int32 * max(len(guides), 1))(*[int(t) for t in thresholds])
    out = ctypes.c_void_p()
    cnt = L.cof_oracle_search(n, cseqs, lens, beg, end, pattern.encode(), len(guides), gs, th,
                              int(threads), ctypes.byref(out))
    if cnt == -1:
        raise ValueError("oracle: bad arguments")
    if cnt < 0:
        raise MemoryError("oracle: out of memory")
    if cnt == 0:
        return np.zeros(0, dtype=HIT_DTYPE)
    buf = (ctypes.c_char * (cnt * HIT_DTYPE.itemsize)).from_address(out.value)
    arr = np.frombuffer(buf, dtype=HIT_DTYPE).copy()
    L.cof_oracle_free(out)
    return arr


def pam_sites(seq, pattern, strand, begin=0, end=None) -> np.ndarray:
    """Ascending window starts whose strand reading passes the PAM pattern."""
    L = lib()
    b = _as_bytes(seq)
    out = ctypes.c_void_p()
    cnt = L.cof_oracle_pam_sites(b, len(b), int(begin), int(end if end is not None else len(b)),
                                 pattern.encode(), strand.encode(), ctypes.byref(out))
    if cnt < 0:
        raise ValueError("oracle: bad arguments")
    if cnt == 0:
        return np.zeros(0, dtype=np.int64)
    arr = np.frombuffer((ctypes.c_int64 * cnt).from_address(out.value), dtype=np.int64).copy()
    L.cof_oracle_free(out)
    return arr


def contains(code: str, base: str) -> bool:
    return bool(lib().cof_oracle_contains(code.encode(), base.encode()))


def canon(c: str) -> str:
    return lib().cof_oracle_canon(c.encode()).decode()


def complement_base(c: str) -> str:
    return lib().cof_oracle_complement_base(c.encode()).decode()


def max_threads() -> int:
    return int(lib().cof_oracle_max_threads())


def hits_to_tuples(arr: np.ndarray):
    """(chrom, pos, strand, guide, mm, site) tuples, the serialized comparison form."""
    return [(int(h["chrom"]), int(h["pos"]), h["strand"].decode(), int(h["guide"]),
             int(h["mm"]), h["site"].decode()) for h in arr]

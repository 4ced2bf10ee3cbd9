"""Executed warp instructions of cof_single_kernel by phase (verification, filter, append,
...) from an ncu report's mixed cuda/sass source page; phase boundaries are found by
marker strings in csrc/single.cu, so the map follows edits:  python tools/ncu_phase.py REP"""
import collections
import csv
import io
import os
import subprocess
import sys

SRC = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                   "paper_conf_socc_jinv23_b200", "csrc", "single.cu")
MARKERS = [   # (marker substring, phase starting at that line)
    ("__device__ __forceinline__ uint32_t s_member", "PAM test"),
    ("__device__ __forceinline__ uint32_t lds32", "filter LDS"),
    ("__device__ __forceinline__ void site_bases", "site_bases"),
    ("__device__ __forceinline__ unsigned long long s_key", "other"),
    ("auto flush = [&]", "verify (flush)"),
    ("// per-lane state of the tile being appended", "other"),
    ("// ---------------- compare a batch", "batch start"),
    ("for (uint32_t b = 0;; b += 4", "filter loop + survivor append"),
    ("__syncwarp();\n                // (at most", "survivor rounds mgmt"),
    ("head = (head + SBATCH) & (SQ - 1);", "other"),
    ("// ---------------- append pending sites", "append"),
    ("// ---------------- next chunk", "tile fetch"),
    ("for (uint32_t e = 0; e < a.ne; e++)", "PAM test"),
    ("if (a.count_items) {\n#pragma unroll", "other"),
]


def phase_map():
    text = open(SRC).read()
    starts = []
    for m, ph in MARKERS:
        i = text.find(m)
        if i >= 0:
            starts.append((text.count("\n", 0, i) + 1, ph))
    return sorted(starts)


def main():
    rep = sys.argv[1]
    starts = phase_map()
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    fname, hdr, agg, tot = None, None, collections.Counter(), 0
    for r in rows:
        if len(r) == 2 and r[0] == "File Path":
            fname = r[1].split("/")[-1]
            continue
        if r and r[0] == "Line No":
            hdr = {h: i for i, h in enumerate(r) if h != "Source"}
            continue
        if hdr is None or not r or not r[0]:
            continue
        try:
            ie = int(r[hdr["Instructions Executed"]])
            ln = int(r[0])
        except (ValueError, KeyError, IndexError):
            continue
        tot += ie
        if fname == "filter_circuit.cuh":
            ph = "filter circuit"
        elif fname != "single.cu":
            ph = "intrinsics (" + fname + ")"
        else:
            ph = "other"
            for s, p in starts:
                if ln >= s:
                    ph = p
        agg[ph] += ie
    print(f"total {tot:.4e} warp instructions (source-line attribution)")
    for k, v in agg.most_common():
        print(f"  {k:34s} {v / tot * 100:5.1f}%")


if __name__ == "__main__":
    main()

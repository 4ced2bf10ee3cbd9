"""Debug helper: raw comparer keys of the mma and table comparers on tiny cases."""
import sys
import numpy as np
import torch
sys.path.insert(0, "/root/repo")
from paper_conf_socc_jinv23_b200 import cof


def keys(seq, pat, guides, thr, impl):
    cof.cof_set_comparer(impl)
    L = len(pat)
    plan = cof.cof_plan_create(pat, guides, thr)
    s = torch.cuda.current_stream()
    pd = torch.empty(cof.cof_plan_device_bytes(plan) + 256, dtype=torch.uint8, device="cuda")
    cof.cof_plan_upload(plan, pd, s)
    n = len(seq)
    owned = n - L + 1
    w = cof.cof_plane_words(n)
    host = np.zeros((3, w), np.uint32)
    cof.cof_pack(np.frombuffer(seq, np.uint8).copy(), n, host[0], host[1], host[2])
    d = torch.from_numpy(host.view(np.int32)).cuda()
    dch = cof.make_chunk(0, 0, n, owned, d[0], d[1], d[2])
    items = torch.empty((2, owned), dtype=torch.int32, device="cuda")
    ws = torch.empty(cof.cof_find_workspace_bytes(n), dtype=torch.uint8, device="cuda")
    nf, nr = cof.cof_find_pam(plan, pd, dch, ws, items[0], items[1], owned, s)
    hits = torch.zeros(100000, dtype=torch.int64, device="cuda")
    nh = cof.cof_compare(plan, pd, dch, items[0], nf, items[1], nr, hits, 100000, s)
    k = np.sort(hits[:nh].cpu().numpy().view(np.uint64))
    return [(int(x >> 32), int((x >> 31) & 1), int((x >> 7) & 0xFFFFFF), int(x & 127)) for x in k]


cases = [
    (b"ACGTAGTTCTACGTACGAAG", "NNNNNN", ["ACGTNN"], [6]),
    (b"ACGTAGTTCTACGTACGAAG", "NNNNNN", ["ACGTNN", "TTTTNN"], [6, 6]),
    (b"ACGTAGTTCTACGTACGAAG", "NNNNNN", ["NNNNNN", "ACGTNN", "TTTTNN"], [6, 6, 6]),
    (b"AAAAAAAAAAAAAAAAAAAA", "NNNNNN", ["ACGTNN", "AAAANN"], [6, 6]),
]
for seq, pat, guides, thr in cases:
    a = keys(seq, pat, guides, thr, "table")
    b = keys(seq, pat, guides, thr, "mma")
    print("CASE", pat, guides, thr, "ok" if a == b else "MISMATCH", len(a), len(b))
    sa, sb = set(a), set(b)
    for h in sorted(sa | sb):
        print("  ", "both" if h in sa and h in sb else ("tab " if h in sa else "mma "), h)

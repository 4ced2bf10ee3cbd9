"""torchrun worker of tests/test_gpu_multi.py (not collected by pytest): every rank runs
the multi-process product path search.search_dist on a seeded synthetic workload; rank 0
saves the merged hit list.  Ranks may share one GPU (COF_DIST_BACKEND=gloo)."""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import torch
    import torch.distributed as dist
    from paper_conf_socc_jinv23_b200 import search, synth

    name, scale, chunk, out = sys.argv[1], float(sys.argv[2]), int(sys.argv[3]), sys.argv[4]
    n_guides = int(sys.argv[5]) if len(sys.argv) > 5 else None
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local % torch.cuda.device_count())
    dist.init_process_group(os.environ.get("COF_DIST_BACKEND", "nccl"))
    w = synth.make_workload(name, scale=scale, n_guides=n_guides)
    res = search.search_dist(w.seqs, w.cfg.pattern, w.guides, w.thresholds, chunk_bases=chunk)
    if dist.get_rank() == 0:
        np.save(out, np.asarray(res))
    dist.destroy_process_group()


if __name__ == "__main__":
    main()

"""The bench contract on a small workload: one JSON line with the required keys, and the
multi-rank path (LPT chromosome shards, max-over-ranks timing) on one GPU with two ranks
sharing it over gloo -- the per-rank hit counts must add up to the single-rank count."""
import json
import os
import socket
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
ARGS = ["--config", "C3", "--scale", "0.01", "--steps", "2", "--warmup", "3", "--no-cpu"]


def _port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _last_json(out):
    lines = [ln for ln in out.splitlines() if ln.startswith("{")]
    assert lines, out[-2000:]
    return json.loads(lines[-1])


def test_bench_one_gpu_contract():
    r = subprocess.run([sys.executable, "bench.py", *ARGS], cwd=ROOT, capture_output=True, text=True, timeout=900)
    assert r.returncode == 0, r.stderr[-3000:]
    d = _last_json(r.stdout)
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better",
              "scaling", "vs_baseline", "dtype", "data", "config", "roofline", "finder_roofline",
              "gpu_launches", "clocks", "e2e"):
        assert k in d, k
    assert d["n_gpus"] == 1 and d["value"] > 0 and d["gpu_launches"] > 0
    assert d["roofline"]["bound"] == "alu" and 0 < d["roofline"]["frac"] < 1.2
    assert d["e2e"]["value"] > 0 and d["e2e"]["h2d_bytes_per_step"] > 0
    assert d["config"]["workload"] == "C3"


def test_bench_two_ranks_share_one_gpu():
    one = subprocess.run([sys.executable, "bench.py", *ARGS, "--no-e2e"], cwd=ROOT, capture_output=True,
                         text=True, timeout=900)
    assert one.returncode == 0, one.stderr[-3000:]
    d1 = _last_json(one.stdout)
    env = dict(os.environ, COF_DIST_BACKEND="gloo")
    two = subprocess.run([sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node=2",
                          "--master-addr=127.0.0.1", f"--master-port={_port()}", "bench.py", "--gpus", "2", *ARGS],
                         cwd=ROOT, capture_output=True, text=True, timeout=900, env=env)
    assert two.returncode == 0, two.stderr[-3000:]
    d2 = _last_json(two.stdout)
    assert d2["n_gpus"] == 2 and d2["scaling"] == "strong"
    assert d2["hits_per_step"] == d1["hits_per_step"] and d2["items_per_step"] == d1["items_per_step"]
    # N > 1 e2e: per-rank pipelines + merge_dist; the merged list has every hit
    assert d2["e2e"]["hits"] == d1["hits_per_step"] and d2["e2e"]["value"] > 0
    assert "merge_dist" in d2["e2e"]["path"]

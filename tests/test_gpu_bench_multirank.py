"""bench.py's N > 1 path (the driver's SCALE run) end to end on the one GPU here:
torchrun with 2 ranks, `gloo` over 127.0.0.1, both ranks on cuda:0 (test hooks
VF_BENCH_BACKEND / VF_BENCH_DEVICE; the driver runs NCCL, one GPU per rank).

Covers the weak-scaling config-2 headline (max over ranks, one JSON line from
rank 0) and the per-app block's strong-scaling paths: graph vertex blocks
with bitmap BFS / label / contribution all-gathers, GEN row slabs with halo
rows, N-body / collision id blocks, STUT row slabs, TRAF ring blocks, ray
strips, at code-path test sizes (--app-small). Every app's variants must agree
with each other (cross-variant result equality on all ranks' merged state).
"""
import json
import os
import socket
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def test_bench_two_ranks_one_gpu():
    env = dict(os.environ, VF_BENCH_BACKEND="gloo", VF_BENCH_DEVICE="0")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
           "--master-addr", "127.0.0.1", "--master-port", str(_free_port()), "bench.py", "--gpus", "2",
           "--steps", "5", "--warmup", "3", "--objects", str(1 << 20), "--no-variants", "--no-e2e", "--no-cpu",
           "--app-small", "--app-variants", "cuda_packed,coal,typeptr", "--strong"]
    r = subprocess.run(cmd, cwd=ROOT, env=env, capture_output=True, text=True, timeout=1200)
    assert r.returncode == 0, r.stderr[-4000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, r.stdout[-2000:]  # rank 0 alone prints
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["parity_sample_ok"] and d["value"] > 0 and d["scaling"] == "strong"
    apps = d["apps"]
    assert set(apps) == {"gol", "ray", "nbody", "gen", "traf", "stut", "collide", "graph"}
    for name, row in apps.items():
        assert row["variants_agree"], name
        assert set(row["variants"]) == {"cuda_packed", "coal", "typeptr"}, name  # heap arm skipped at N > 1
        assert all(v["calls_per_s"] > 0 for v in row["variants"].values()), name

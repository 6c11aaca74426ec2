"""The N-rank path of bench.py on one GPU (gloo process group, every rank on cuda:0): self-launch
of the ranks, batch sharding, the bucketed overlapped all-reduce, the weak-scaling line and the
deterministic leaf-tree exchange.  Timings are meaningless here; the point is that the code the
driver's multi-GPU scaling run executes works, and that the tree exchange gives bitwise the same
dW and db with 1 and 2 ranks end to end (bench --dump of the same global batch)."""
import json
import os
import subprocess
import sys

import numpy as np
import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _bench(args, tmp=None):
    env = dict(os.environ)
    for k in ("WORLD_SIZE", "RANK", "LOCAL_RANK", "MASTER_ADDR", "MASTER_PORT"):
        env.pop(k, None)
    cmd = [sys.executable, os.path.join(ROOT, "bench.py"), "--steps", "2", "--warmup", "2",
           "--no-cpu-baseline", "--no-e2e"] + args
    if tmp is not None:
        cmd += ["--dump", str(tmp)]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=600, env=env)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, r.stdout[-2000:]
    return json.loads(lines[0])


def test_two_ranks_bucketed_exchange():
    d = _bench(["--workload", "2", "--gpus", "2", "--dist-backend", "gloo", "--same-device"])
    assert d["n_gpus"] == 2 and d["scaling"] == "strong" and d["config"]["global_batch"] == 64
    assert d["config"]["per_gpu_batch"] == 32 and d["weak_scaling"]["global_batch"] == 128
    assert "buckets" in d["config"]["exchange"]


@pytest.mark.parametrize("math", ["fp32", "tf32"])
def test_tree_exchange_bitwise_one_vs_two_ranks(math, tmp_path):
    """--exchange tree: dW||db of every layer is bitwise the same from 1 and from 2 ranks."""
    base = ["--workload", "2", "--math", math, "--exchange", "tree", "--no-extra-modes"]
    _bench(base + ["--gpus", "1"], tmp_path / "g1")
    _bench(base + ["--gpus", "2", "--dist-backend", "gloo", "--same-device"], tmp_path / "g2")
    meta = json.load(open(tmp_path / "g1" / "meta.json"))
    for i, _ in enumerate(meta["units"]):
        for k in ("dw", "db"):
            a = np.load(tmp_path / "g1" / f"u{i}_{k}.npy")
            b = np.load(tmp_path / "g2" / f"u{i}_{k}.npy")
            np.testing.assert_array_equal(a, b, err_msg=f"unit {i} {k}")

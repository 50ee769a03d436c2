"""bench.py's N > 1 path (the driver's scaling runs) end to end: torchrun with 2 ranks
sharing the GPU(s) over gloo (NCCL when >= 2 GPUs), the reduced bench legs; the rank-0
JSON line must carry the contract keys and the exhaustive count of the whole batch."""
import json
import os
import socket
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


@pytest.mark.parametrize("shard", ["requests", "candidates"])
def test_bench_two_ranks(shard):
    import torch
    backend = "nccl" if torch.cuda.device_count() >= 2 else "gloo"
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node=2",
           "--master-addr", "127.0.0.1", "--master-port", str(_port()), os.path.join(ROOT, "bench.py"),
           "--gpus", "2", "--steps", "3", "--warmup", "3", "--config", "3", "--shard", shard,
           "--no-c4", "--no-cpu-baseline"]
    res = subprocess.run(cmd, capture_output=True, text=True, timeout=900, cwd=ROOT,
                         env={**os.environ, "FFS_DIST_BACKEND": backend})
    out = res.stdout + res.stderr
    assert res.returncode == 0, out[-4000:]
    lines = [json.loads(x) for x in res.stdout.splitlines() if x.startswith("{")]
    assert len(lines) == 1, out[-2000:]
    d = lines[0]
    assert d["n_gpus"] == 2 and d["metric"] == "candidates_scored_per_s" and d["value"] > 0
    assert d["config"]["scored_counter_equals_sum_S"] is True  # summed over both ranks
    assert d["production"]["keys_identical_to_exhaustive"] is True
    assert d["e2e"]["value"] > 0 and d["gpu_launches"] > 0

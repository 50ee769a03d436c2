"""The multi-rank path on real kernels: torchrun with 2 and 4 ranks (gloo) on the
available GPU(s); keys combined by all_reduce(MIN) and decoded slices must equal the
single-rank result bit for bit."""
import os
import socket
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
HERE = os.path.dirname(os.path.abspath(__file__))


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _torchrun(world, backend):
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={world}",
           "--master-addr", "127.0.0.1", "--master-port", str(_port()), os.path.join(HERE, "_dist_run.py")]
    res = subprocess.run(cmd, capture_output=True, text=True, timeout=900,
                         env={**os.environ, "FFS_DIST_BACKEND": backend})
    out = res.stdout + res.stderr
    assert res.returncode == 0, out[-4000:]
    for shard in ("requests", "candidates"):
        assert f"dist-run ok world={world} backend={backend} shard={shard}" in out


@pytest.mark.parametrize("world", [2, 4])
def test_torchrun_sharded_step(world):
    """Several ranks sharing the GPU(s) over gloo (runs on a one-GPU box)."""
    _torchrun(world, "gloo")


def test_torchrun_sharded_step_nccl():
    """The NCCL path (one rank per GPU, all_reduce(MIN) over NVLink for candidate
    shards): needs >= 2 GPUs, so it runs on the driver's multi-GPU box."""
    import torch
    n = torch.cuda.device_count()
    if n < 2:
        pytest.skip("NCCL path needs >= 2 GPUs (one rank per GPU)")
    _torchrun(min(n, 8), "nccl")

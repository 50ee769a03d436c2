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


@pytest.mark.parametrize("world", [2, 4])
def test_torchrun_sharded_step(world):
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={world}",
           "--master-addr", "127.0.0.1", "--master-port", str(_port()), os.path.join(HERE, "_dist_run.py")]
    res = subprocess.run(cmd, capture_output=True, text=True, timeout=900,
                         env={**os.environ, "FFS_DIST_BACKEND": "gloo"})
    out = res.stdout + res.stderr
    assert res.returncode == 0, out[-4000:]
    assert f"dist-run ok world={world}" in out

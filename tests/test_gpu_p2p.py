"""Fused fold + merge over peer memory (include/sassi.h, sassi_add_peer_table): two processes
(torchrun, gloo) fold disjoint parts of a stream into each other's table images through CUDA IPC;
every image then equals the oracle over the whole stream. On a one-GPU node both ranks share the
device (IPC between processes on one device), which exercises the same protocol and kernels."""
import os
import socket
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")
HERE = os.path.dirname(os.path.abspath(__file__))


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


@pytest.mark.parametrize("world", [2, 3])
def test_fused_merge_two_processes(world):
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", str(world),
           "--master-addr", "127.0.0.1", "--master-port", str(_free_port()),
           os.path.join(HERE, "p2p_worker.py")]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stdout[-2000:] + r.stderr[-4000:]
    for k in range(world):
        assert "p2p ok rank %d of %d" % (k, world) in r.stdout

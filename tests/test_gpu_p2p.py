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


def test_bench_two_ranks_sharing_the_gpu_fused_merge():
    """bench.py's N > 1 code path on a one-GPU box: `--gpus 2 --share-gpu --merge p2p` self-launches
    two ranks (gloo), both on cuda:0, each folding its c2 warp shard into both table images; one
    JSON line with n_gpus = 2 (the device-side draws are checked against the host-output draws
    inside bench.py). Not a scaling measurement: the two ranks share one GPU."""
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import json
    root = os.path.dirname(HERE)
    cmd = [sys.executable, os.path.join(root, "bench.py"), "--gpus", "2", "--share-gpu", "--merge", "p2p",
           "--workload", "c2", "--steps", "3", "--warmup", "1", "--no-e2e", "--no-cpu-baseline",
           "--no-slowdown", "--no-injection"]
    env = {k: v for k, v in os.environ.items() if k not in ("RANK", "WORLD_SIZE", "LOCAL_RANK")}
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=900, env=env, cwd=root)
    assert r.returncode == 0, r.stdout[-2000:] + r.stderr[-4000:]
    lines = [json.loads(l) for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1
    d = lines[0]
    assert d["n_gpus"] == 2 and d["value"] > 0 and d["config"]["shared_gpu"] is True
    assert "fused fold + merge over peer memory" in d["config"]["parallelism"]

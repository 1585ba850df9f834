"""Multi-rank path with the CUDA kernels: torchrun with 2 ranks on one GPU
(the box has one), gloo for the tally.  Each rank's kernel outputs on its minibatch shard are
compared with the oracle on that shard (tests/_dist_gpu_worker.py), and the tally with the
single-process count.  bench.py's own N>1 path is exercised end to end with --same-device."""
import json
import os
import socket
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def torchrun(args, timeout=900):
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
           "--master-addr", "127.0.0.1", "--master-port", str(free_port())] + args
    return subprocess.run(cmd, capture_output=True, text=True, timeout=timeout, cwd=ROOT)


def test_two_ranks_kernels_match_oracle_per_shard(gist, cuda):
    r = torchrun([os.path.join(ROOT, "tests", "_dist_gpu_worker.py")])
    assert r.returncode == 0, (r.stdout + r.stderr)[-4000:]
    assert "dist OK" in r.stdout


def test_bench_two_ranks_same_device_strong_c4(gist, cuda):
    r = torchrun([os.path.join(ROOT, "bench.py"), "--gpus", "2", "--config", "C4", "--steps", "3", "--warmup", "3",
                  "--same-device", "--no-e2e", "--cpu-seconds", "1"])
    assert r.returncode == 0, (r.stdout + r.stderr)[-4000:]
    line = json.loads([ln for ln in r.stdout.splitlines() if ln.startswith("{")][-1])
    assert line["n_gpus"] == 2 and line["scaling"] == "strong"
    assert line["config"]["global_batch"] == 64
    assert line["value"] > 0 and line["gpu_launches"] > 0

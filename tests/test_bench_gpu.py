"""bench.py end to end on the GPU: the JSON contract at N = 1, and the N > 1 code
path (torchrun, peer-memory exchange between processes) on one GPU via the
diagnostic ARCV_BENCH_ONE_GPU mode -- parity of the timed result must be "ok"."""
import json
import os
import socket
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
KEYS = {"metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better", "scaling",
        "vs_baseline", "dtype", "data", "config", "parity", "gpu_launches", "roofline", "e2e"}


def _last_json(out):
    lines = [ln for ln in out.splitlines() if ln.startswith("{")]
    assert lines, out[-2000:]
    return json.loads(lines[-1])


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


@pytest.mark.timeout(600)
def test_bench_single_gpu_contract():
    p = subprocess.run([sys.executable, "bench.py", "--n", str(1 << 24), "--steps", "5", "--warmup", "3",
                        "--e2e-steps", "1", "--no-cpu-baseline"], cwd=ROOT, capture_output=True, text=True,
                       timeout=540)
    assert p.returncode == 0, p.stderr[-3000:]
    line = _last_json(p.stdout)
    assert KEYS <= set(line), KEYS - set(line)
    assert line["parity"] == "ok" and line["n_gpus"] == 1
    assert line["gpu_launches"] == 5  # one K1 per step (the report phase runs in its tail)
    assert line["roofline"]["bound"] == "hbm" and line["roofline"]["achieved"] > 0
    assert line["e2e"]["h2d_bytes_per_step"] == 2 * (1 << 24) * 8


@pytest.mark.timeout(600)
def test_bench_two_ranks_peer_exchange_one_gpu():
    env = dict(os.environ, ARCV_BENCH_ONE_GPU="1")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
           "--master-addr", "127.0.0.1", "--master-port", str(_port()), "bench.py", "--gpus", "2",
           "--n-elements", str(1 << 24), "--steps", "5", "--warmup", "3", "--e2e-steps", "1"]
    p = subprocess.run(cmd, cwd=ROOT, env=env, capture_output=True, text=True, timeout=540)
    assert p.returncode == 0, p.stderr[-3000:]
    line = _last_json(p.stdout)
    assert line["n_gpus"] == 2 and line["config"]["exchange"] == "peer"
    assert line["parity"] == "ok"
    assert line["gpu_launches"] == 5  # one K1 per step: the exchange runs in its tail (rank 0)

"""bench.py at N = 2 ranks (torchrun, gloo, both ranks on the one GPU of the box): the
multi-GPU code path of the scaling run -- shard setup, the agreement on the tail
exchange, the timed step, max-over-ranks timing and the per-rank parity check -- with
the NCCL-style exchange (all-gather + mps_apply_tails) and with the fused peer-memory
exchange."""
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


@pytest.mark.parametrize("tails", ["nccl", "p2p"])
def test_bench_two_ranks(tails):
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node=2",
           "--master-addr", "127.0.0.1", "--master-port", str(_port()),
           os.path.join(ROOT, "bench.py"), "--gpus", "2", "--steps", "3", "--warmup", "3",
           "--workload", "pubmed", "--K", "64", "--dist-backend", "gloo", "--tails", tails]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=600, cwd=ROOT)
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-3000:]
    lines = [json.loads(ln) for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, r.stdout          # rank 0 alone prints one line
    d = lines[0]
    assert d["n_gpus"] == 2 and d["steps"] == 3 and d["value"] > 0
    assert d["config"]["tail_exchange"] == tails
    assert d["parity"]["ok"] and d["parity"]["all_ranks_ok"]


@pytest.mark.parametrize("wl,K,extra", [("pubmed", 64, []), ("rmat", 64, []),
                                        ("cora", 16, ["--cuda-graph"])])
def test_bench_single_gpu_all_legs(wl, K, extra):
    """The N = 1 bench line with every leg on (e2e through the host-buffer ABI, the CPU
    baseline, cuSPARSE, L2 probe, gather replay, parity check): one JSON line carrying
    the contract's keys."""
    cmd = [sys.executable, os.path.join(ROOT, "bench.py"), "--workload", wl, "--K", str(K),
           "--steps", "3", "--warmup", "3", "--e2e-steps", "1", "--cpu-seconds", "1"] + extra
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=900, cwd=ROOT)
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-3000:]
    lines = [json.loads(ln) for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1
    d = lines[0]
    for key in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step",
                "higher_is_better", "scaling", "vs_baseline", "dtype", "data", "config",
                "roofline", "cpu_baseline", "e2e", "gpu_launches", "clocks", "parity"):
        assert key in d, key
    assert d["value"] > 0 and d["gpu_launches"] > 0 and d["parity"]["ok"]
    assert d["e2e"]["value"] > 0 and d["e2e"]["h2d_bytes_per_step"] > 0
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] >= 1
    assert {"bound", "achieved", "peak", "unit", "frac"} <= set(d["roofline"])

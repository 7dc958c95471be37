"""The driver's commands on the GPU: bench.py prints one JSON line with the
contract's keys, on one GPU and with ranks launched by bench.py itself
(--gpus 2 without a torchrun environment; the ranks share cuda:0 here)."""
import json
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _bench(*args, timeout=900):
    env = {k: v for k, v in os.environ.items() if k not in ("RANK", "WORLD_SIZE", "LOCAL_RANK", "MASTER_ADDR", "MASTER_PORT")}
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), *args], capture_output=True, text=True,
                       timeout=timeout, env=env)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [l for l in r.stdout.strip().splitlines() if l.startswith("{")]
    assert len(lines) == 1, r.stdout
    return json.loads(lines[0])


def _check_line(j, n):
    import bench

    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better", "scaling",
              "vs_baseline", "dtype", "data", "config", "roofline", "e2e", "gpu_launches", "clocks"):
        assert k in j, k
    assert j["metric"] == bench.METRIC and j["n_gpus"] == n and j["value"] > 0 and j["gpu_launches"] > 0
    r = j["roofline"]
    assert r["bound"] == "hbm" and r["unit"] == "GB/s" and r["achieved"] > 0 and r["peak"] > 0
    assert abs(r["frac"] - r["achieved"] / r["peak"]) < 1e-3
    e = j["e2e"]
    assert e["value"] > 0 and e["h2d_bytes_per_step"] > 0 and e["d2h_bytes_per_step"] > 0


def test_bench_one_gpu_c2():
    j = _bench("--config", "c2", "--steps", "20", "--warmup", "3")
    _check_line(j, 1)
    assert j["config"]["kernel_variant"] == "jit" and j["cpu_baseline"]["kind"] == "oracle"
    assert j["cpu_baseline"]["cores"] >= 1 and "value_1_thread" in j["cpu_baseline"]


def test_bench_self_launched_ranks():
    """--gpus 2 with no WORLD_SIZE: bench.py starts torchrun itself; the two
    ranks (sharing cuda:0, peer-memory transport) print ONE line."""
    j = _bench("--gpus", "2", "--share-gpu", "--transport", "p2p", "--config", "c2", "--steps", "10", "--warmup", "3")
    _check_line(j, 2)
    assert "one-sided puts" in j["config"]["parallelism"]

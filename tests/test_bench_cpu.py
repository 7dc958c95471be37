"""bench.py pieces that run without a GPU: the reference arm (the oracle on
the host cores) prints the driver's JSON line with the SAME metric string,
unit and direction as the CRSD arm, and the row partitions cover the matrix."""
import json
import os
import subprocess
import sys

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402


@pytest.mark.parametrize("cfg", ["c1", "c3"])
def test_reference_arm_line(cfg):
    env = dict(os.environ, CRSD_REF_BUDGET_S="2")
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--config", cfg,
                        "--steps", "3", "--warmup", "3"], capture_output=True, text=True, timeout=600, env=env)
    assert r.returncode == 0, r.stderr[-2000:]
    line = json.loads(r.stdout.strip().splitlines()[-1])
    assert line["impl"] == "reference"
    assert line["metric"] == bench.METRIC and line["unit"] == "GFLOP/s" and line["higher_is_better"] is True
    assert line["value"] > 0 and line["cpu_baseline"]["kind"] == "oracle" and line["cpu_baseline"]["cores"] >= 1
    assert line["e2e"]["h2d_bytes_per_step"] == 0 and line["e2e"]["value"] == line["value"]


def test_reference_arm_other_ranks_exit_quietly():
    env = dict(os.environ, RANK="1", WORLD_SIZE="2")
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--config", "c1",
                        "--gpus", "2", "--steps", "3", "--warmup", "3"], capture_output=True, text=True, timeout=300,
                       env=env)
    assert r.returncode == 0 and r.stdout.strip() == ""


@pytest.mark.parametrize("cfg", ["c5", "c4", "c2"])
@pytest.mark.parametrize("world", [1, 2, 4, 8])
def test_rank_rows_cover_the_matrix(cfg, world):
    blocks = [bench.rank_rows(cfg, world, r) for r in range(world)]
    N = blocks[0][0]
    assert blocks[0][1] == 0 and blocks[-1][2] == N
    for (_, a, b), (_, c, d) in zip(blocks, blocks[1:]):
        assert b == c and a < b and c < d
    if cfg == "c5":  # uniform rows: byte-balanced = equal within one segment
        sizes = np.array([b - a for _, a, b in blocks])
        assert sizes.max() - sizes.min() <= 256


def test_cpu_sample_is_a_prefix_of_the_workload():
    """The reference arm and cpu_baseline generate only rows [0, cut) -- the
    same entries the full C5 generator gives for those rows."""
    import gen

    N, ncols, cut, r, c, v, total = bench.cpu_sample("c5", "f64", 2_000_000)
    assert total == 3_167_354_880 and r.max() < cut <= N
    a = gen.config5(row_begin=0, row_end=cut)
    assert np.array_equal(a.row, r) and np.array_equal(a.col, c) and np.array_equal(a.val, v)

"""bench.py's measurement logic on the CPU: the algorithmic byte models DESIGN.md §6 states, the
committed traffic / L2 evidence it attaches to the roofline object, and the reference arm's JSON line
(the oracle timed on a small slope) with the contract's keys; other ranks of the reference arm exit
without work."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import bench  # noqa: E402


def test_spmv_bytes_per_row():
    # D 288 + u (V 288 + 3 x 4 indices) + 8 (row_ptr, low_ptr) + x 48 + y 48
    assert bench.bytes_per_row_spmv(3.0) == 1292.0
    assert bench.bytes_per_row_spmv(0.0) == 392.0


def test_scaled_solve_bytes_per_iteration():
    """Each further iteration of the scaled engine adds 300u + 448 bytes per block row (DESIGN.md §6:
    phase A 300u + 8 + p_old, p, q, x traffic; phase B 152), each exact test 240."""
    n, nnzb = 1000, 2996
    u = nnzb / n
    f = bench.pcg_launch_bytes_scaled
    assert abs((f(n, nnzb, 11, 0) - f(n, nnzb, 10, 0)) - n * (300.0 * u + 448.0)) < 1e-6
    assert abs((f(n, nnzb, 10, 3) - f(n, nnzb, 10, 2)) - n * 240.0) < 1e-6


def test_committed_roofline_evidence():
    t = bench.traffic_for(1001096, "pcg_scaled_persistent")
    assert t is not None and t["bytes"] > 3e11
    l2 = bench.l2_roofline(1001096, 269, 81.0)
    assert l2 is not None and 0.8 < l2["frac"] < 1.3
    assert bench.traffic_for(12345, "pcg_scaled_persistent") is None


def test_reference_arm_line():
    env = dict(os.environ, RANK="0", WORLD_SIZE="1")
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--blocks", "2000",
                          "--steps", "1", "--warmup", "0"], env=env, capture_output=True, text=True, timeout=600)
    assert out.returncode == 0, out.stderr[-2000:]
    line = json.loads(out.stdout.strip().splitlines()[-1])
    for k in ("impl", "metric", "value", "unit", "higher_is_better", "n_gpus", "steps", "warmup", "ms_per_step",
              "dtype", "config", "cpu_baseline", "e2e"):
        assert k in line, k
    assert line["impl"] == "reference" and line["value"] > 0 and line["higher_is_better"] is False
    assert line["cpu_baseline"]["kind"] == "oracle" and line["cpu_baseline"]["cores"] == 1
    assert line["e2e"]["h2d_bytes_per_step"] == 0 and line["e2e"]["value"] == line["value"]


def test_reference_arm_other_ranks_exit_without_work():
    env = dict(os.environ, RANK="1", WORLD_SIZE="2")
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--gpus", "2",
                          "--steps", "1", "--warmup", "0"], env=env, capture_output=True, text=True, timeout=300)
    assert out.returncode == 0 and out.stdout.strip() == ""

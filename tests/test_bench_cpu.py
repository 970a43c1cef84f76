"""The bench's reference arm (the oracle timed on the host, --impl reference)
runs without a GPU and prints the contract's JSON line."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_reference_arm_json_line():
    r = subprocess.run([sys.executable, "bench.py", "--impl", "reference", "--steps", "2", "--warmup", "1"],
                       cwd=ROOT, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stderr[-2000:]
    line = json.loads(r.stdout.strip().splitlines()[-1])
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better",
              "scaling", "vs_baseline", "dtype", "data", "config", "cpu_baseline", "e2e"):
        assert k in line, k
    assert line["impl"] == "reference" and line["value"] > 0
    assert line["cpu_baseline"]["kind"] == "oracle" and line["cpu_baseline"]["cores"] == 1
    assert line["e2e"]["h2d_bytes_per_step"] == 0 and line["e2e"]["value"] == line["value"]
    assert "workload" in line["config"]


def test_reference_arm_non_zero_rank_is_silent():
    env = dict(os.environ, RANK="1", WORLD_SIZE="2")
    r = subprocess.run([sys.executable, "bench.py", "--impl", "reference", "--steps", "1", "--warmup", "1"],
                       cwd=ROOT, capture_output=True, text=True, timeout=300, env=env)
    assert r.returncode == 0 and r.stdout.strip() == ""


def test_json_line_is_strict_json():
    """NaN / inf never reach the JSON line (a strict parser would reject it)."""
    import importlib.util
    spec = importlib.util.spec_from_file_location("bench_mod", os.path.join(ROOT, "bench.py"))
    b = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(b)
    line = b._finite({"slowdown": float("nan"), "x": [1.5, float("inf")], "y": {"z": float("-inf"), "w": 2}})
    assert line == {"slowdown": None, "x": [1.5, None], "y": {"z": None, "w": 2}}
    json.dumps(line, allow_nan=False)


def _bench():
    import importlib.util
    spec = importlib.util.spec_from_file_location("bench_mod", os.path.join(ROOT, "bench.py"))
    b = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(b)
    return b


def test_value_is_per_source_at_every_n():
    """BASELINE.json's metric is per SOURCE GPU: at N > 1 the line's value is
    one rank's swapped bytes over the max-over-ranks step time (== the
    per_rank_gbs key), and the whole-job sum is all_ranks_gbs = N x value."""
    b = _bench()
    per_step = 2 * 8 * (900 << 20)
    for n in (1, 2, 4, 8):
        value, all_ranks = b.headline_values(n, per_step, 4.5)
        assert value == per_step / 4.5e-3 / 1e9
        assert all_ranks == n * value


def test_bootstrap_ci95():
    b = _bench()
    xs = [0.01 * i for i in range(41)]              # median 0.20
    lo, hi = b.bootstrap_ci95(xs)
    assert lo < 0.20 < hi and 0.10 < lo and hi < 0.30
    assert b.bootstrap_ci95([0.05] * 30) == (0.05, 0.05)
    lo, hi = b.bootstrap_ci95([])
    assert lo != lo and hi != hi                     # NaN when there is nothing to resample

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


def test_north_star_summary():
    """Config 4's target row (BJ:5, BJ:10): N-1 peers, sizes >= 256 MiB, the
    better SM kernel per size, the slower direction, min over sizes, against
    0.8 x 900 GB/s; copy-engine rows and smaller sizes / fewer peers ignored."""
    b = _bench()
    M = 1 << 20

    def row(P, size, path, o, i):
        return {"peers": P, "bytes": size, "path": path, "out_gbs": o, "in_gbs": i}
    rows = [row(7, 256 * M, "direct", 700, 760), row(7, 256 * M, "bulk", 745, 750),
            row(7, 1024 * M, "direct", 790, 780), row(7, 1024 * M, "bulk", 770, 800),
            row(7, 1024 * M, "ce", 890, 890), row(3, 1024 * M, "bulk", 100, 100),
            row(7, 64 * M, "bulk", 10, 10)]
    ns = b.north_star_summary(rows, 8)
    assert ns["sizes"] == [256 * M, 1024 * M]
    assert ns["best_sm_path_per_size"] == {str(256 * M): "bulk", str(1024 * M): "direct"}
    assert ns["min_gbs_over_sizes_and_directions"] == 745
    assert ns["meets_target"] and abs(ns["frac_of_900"] - 745 / 900) < 1e-12
    rows[1] = row(7, 256 * M, "bulk", 719, 750)
    ns = b.north_star_summary(rows, 8)
    assert ns["min_gbs_over_sizes_and_directions"] == 719 and not ns["meets_target"]
    ns4 = b.north_star_summary(rows, 4)                # N = 4: the 3-peer rows only
    assert ns4["sizes"] == [1024 * M] and ns4["min_gbs_over_sizes_and_directions"] == 100
    assert b.north_star_summary(rows, 2) is None       # no 1-peer row >= 256 MiB

"""The committed bench line (profiles/r02/bench.json, written by bench.py on
a B200) satisfies the driver's contract: strict JSON, the required keys and
types, the roofline / cpu_baseline / e2e / clocks objects, and internal
consistency (value from ms_per_step, roofline frac = achieved / peak)."""
import json
import math
import os

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _line():
    with open(os.path.join(ROOT, "profiles", "r02", "bench.json")) as f:
        text = f.read().strip().splitlines()[-1]

    def bad(c):
        raise ValueError("non-finite constant %s in the bench line" % c)
    return json.loads(text, parse_constant=bad)


def test_required_keys_and_types():
    d = _line()
    for k, t in (("metric", str), ("value", float), ("unit", str), ("n_gpus", int), ("steps", int),
                 ("warmup", int), ("ms_per_step", float), ("higher_is_better", bool), ("scaling", str),
                 ("dtype", str), ("data", str), ("config", dict), ("roofline", dict),
                 ("cpu_baseline", dict), ("e2e", dict), ("gpu_launches", int), ("clocks", dict)):
        assert isinstance(d[k], t), k
    assert d["warmup"] >= 3 and d["steps"] >= 1
    assert "workload" in d["config"] and "l2" in d["config"]
    assert d["vs_baseline"] is None          # no published number for this metric
    assert d["gpu_launches"] > 0


def test_internal_consistency():
    d = _line()
    r = d["roofline"]
    assert r["bound"] in ("hbm", "nvlink", "tensor", "alu")
    assert math.isclose(r["frac"], r["achieved"] / r["peak"], rel_tol=1e-9)
    assert 0 < r["frac"] <= 1.05
    assert r["traffic"] is None or r["traffic"] > 0
    # value = swapped bytes (out + in) of all micro-batches per step / step time
    per_step = 2 * d["config"]["micro_batch_bytes"] * d["config"]["micro_batches"]   # per source GPU
    assert math.isclose(d["value"], per_step / (d["ms_per_step"] / 1e3) / 1e9, rel_tol=1e-6)
    c = d["cpu_baseline"]
    assert c["kind"] == "oracle" and c["cores"] >= 1 and c["value"] > 0
    e = d["e2e"]
    assert e["h2d_bytes_per_step"] > 0 and e["d2h_bytes_per_step"] > 0 and e["value"] > 0
    assert d["clocks"]["sm_mhz"] > 0
    bad = {"hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown"}
    assert not bad & set(d["clocks"]["reasons"])


def test_round2_keys():
    """Round-2 additions: the per-source value with the whole-job sum beside
    it, the duplex leg, and the GEMM slowdown as a bootstrap interval over
    >= 30 paired rounds with its regime and the pace of the swap."""
    d = _line()
    assert d["per_rank_gbs"] == d["value"] and math.isclose(d["all_ranks_gbs"], d["n_gpus"] * d["value"])
    assert d["duplex_gbs"] > 0 and d["duplex"]["bit_exact"]
    for key in ("gemm_slowdown", "gemm_slowdown_ce"):
        g = d[key]
        lo, hi = g["slowdown_ci95"]
        assert lo <= g["slowdown"] <= hi and g["rounds"] >= 30
        assert g["regime"] in ("burst", "sustained")
        assert g["meets_10pct"] == (hi < 0.10)
    # the direct (LSU) GEMM-concurrent swaps are paced, the TMA ones are not
    g = d["gemm_slowdown"]
    assert (g["swap_pace_mbps"] > 0) == (g["swap_setting"].split(":")[0] not in ("bulk", "ce"))
    sus = d["gemm_slowdown_sustained"]
    # the power-capped leg: >= 5 paired windows of ~3 s (the verdict's "windows of 3 s or more")
    assert sus["rounds"] >= 5 and sus["slowdown_ci95"][0] <= sus["slowdown"] <= sus["slowdown_ci95"][1]
    assert sus["alone_ms"] * int(sus["gemm"].split("windows of ")[1].split()[0]) >= 2500
    if "fallback" in sus:   # re-measured with --gemm-sus-fallback: the first setting missed the rate
        assert sus["first_setting"]["swap_gbs_during"] < 720 and sus["swap_setting"] != sus["first_setting"]["swap_setting"]

"""NEXT-4: the §III-D decision rule between GPU-CPU swap, recomputation and
D2D swap (reading R26).  CPU only.  Pins: the paper's own worked example --
Table III's six tensors and the choices P:358-364 derives for them
(tests/golden/t3_table_iii.json) -- and, with ample spare memory, exhaustive
search (the rule then reaches the minimum total overhead)."""
import json
import os
import random

import pytest

from oracle import compaction as OC
import paper_conf_hpca_zhouwylbyx23_b200 as mp

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")
NAMES = {"cpu": OC.CPU, "recompute": OC.RECOMPUTE, "d2d": OC.D2D}


def _table3():
    return json.load(open(os.path.join(GOLDEN, "t3_table_iii.json")))


def test_table_iii_choices():
    g = _table3()
    stats = g["tensors"]
    want = [NAMES[c] for c in g["expect_choice"]]
    for cap in (10 ** 12, sum(t["bytes"] for t in stats)):   # spare memory not binding
        ch, ov, tot, used = OC.compaction_plan(stats, cap)
        assert ch == want and ov == g["expect_overhead_ns"]
        assert used == stats[1]["bytes"] + stats[4]["bytes"]
        assert mp.compaction_plan(stats, cap) == (ch, ov, tot, used)


def test_table_iii_spare_binds():
    """Spare memory for only 400 MB: the tensors with the most overhead are
    served first.  Initially t6 costs 14 ms (recompute), t5 8 ms
    (recompute), t3 4 ms, t2 3 ms; t6 (1152 MB) does not fit, t5 (384 MB)
    moves to D2D (0 ms), t3's D2D is not cheaper (4 ms) and t2 (115 MB) no
    longer fits, so it keeps recomputation."""
    stats = _table3()["tensors"]
    ch, ov, tot, used = OC.compaction_plan(stats, 400_000_000)
    assert ch[4] == OC.D2D and ch[1] == OC.RECOMPUTE and used == 384_000_000
    assert mp.compaction_plan(stats, 400_000_000) == (ch, ov, tot, used)


def _rand_stats(rng, n):
    out = []
    for _ in range(n):
        live = rng.randint(0, 100)
        out.append(dict(bytes=rng.randint(1, 10), live_ns=live,
                        recompute_ns=rng.choice([OC.NOT_RECOMPUTABLE, rng.randint(1, 60)]),
                        cpu_swap_ns=rng.randint(1, 200), d2d_swap_ns=rng.randint(1, 40)))
    return out


def test_ample_spare_reaches_the_minimum():
    rng = random.Random(215)
    for _ in range(300):
        stats = _rand_stats(rng, rng.randint(1, 6))
        cap = sum(t["bytes"] for t in stats)
        _, _, tot, _ = OC.compaction_plan(stats, cap)
        assert tot == OC.brute_force_total(stats, cap)


def test_capacity_respected_and_parity_random():
    rng = random.Random(229)
    for _ in range(500):
        stats = _rand_stats(rng, rng.randint(0, 12))
        cap = rng.randint(0, 40)
        o = OC.compaction_plan(stats, cap)
        assert o[3] <= cap
        assert mp.compaction_plan(stats, cap) == o
        # never worse than doing only the initial assignment
        init = OC.compaction_plan(stats, 0)
        assert o[2] <= init[2]

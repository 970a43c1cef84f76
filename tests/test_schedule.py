"""NEXT-2: 1F1B swap schedule with the live-interval check (reading R24).
CPU only.  Pins of the oracle: a hand-derived two-stage timeline
(tests/golden/p1_*.json), the 1F1B closed form (M+S-1)(t_f+t_b) for the
makespan, the fn.2 rule that a swap longer than the live interval
delays the backward, and the memory bound (no swap: stage 0 holds
min(S, M) micro-batches).  The library (a DAG longest-path pass,
csrc/schedule.cpp) must equal the oracle (a resource sweep) exactly."""
import json
import os
import random

import pytest

from oracle import pipeline as P
import paper_conf_hpca_zhouwylbyx23_b200 as mp

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


def test_golden_two_stage_timeline():
    g = json.load(open(os.path.join(GOLDEN, "p1_1f1b_two_stages.json")))
    q = g["params"]
    args = (q["stages"], q["stage"], q["micro_batches"], q["t_fwd_ns"], q["t_bwd_ns"],
            q["t_out_ns"], q["t_in_ns"])
    slots, summ = P.schedule(*args, duplex=bool(q["duplex"]))
    assert slots == g["slots"] and summ == g["summary"]
    assert mp.schedule_1f1b(*args, duplex=bool(q["duplex"])) == (g["slots"], g["summary"])


@pytest.mark.parametrize("case", range(4))
def test_golden_slack(case):
    """The swap-in slack rule (fn.1 P:226, reading R24): hand-derived
    triggers for slack > 0, the fall-back to F(m) itself when no op qualifies,
    and the <= boundary; by the oracle and by the library."""
    g = json.load(open(os.path.join(GOLDEN, "p1_1f1b_slack.json")))["cases"][case]
    q = g["params"]
    args = (q["stages"], q["stage"], q["micro_batches"], q["t_fwd_ns"], q["t_bwd_ns"],
            q["t_out_ns"], q["t_in_ns"])
    assert P.schedule(*args, duplex=bool(q["duplex"]), slack=q["slack_ns"]) == (g["slots"], g["summary"])
    assert mp.schedule_1f1b(*args, duplex=bool(q["duplex"]), slack_ns=q["slack_ns"]) == \
        (g["slots"], g["summary"])


@pytest.mark.parametrize("S,M", [(1, 1), (1, 5), (2, 3), (4, 8), (8, 8), (8, 16), (5, 2)])
def test_1f1b_closed_form_makespan(S, M):
    s, e = P.timeline_noswap(S, M, 7, 13)
    assert max(e.values()) == (M + S - 1) * (7 + 13)


@pytest.mark.parametrize("S,M", [(2, 4), (4, 8), (8, 8), (8, 4)])
def test_stage0_memory_without_swap(S, M):
    """stage 0 keeps up to min(S, M) micro-batches' activations alive."""
    _, summ = P.schedule(S, 0, M, 10, 20, 1, 1)
    assert summ["peak_resident_noswap"] == min(S, M)


def test_slow_swap_is_exposed():
    """fn.2: when out + in exceeds the live interval the backward waits."""
    slots, summ = P.schedule(4, 0, 8, 10, 20, 200, 200)
    assert all(s["hidden"] == 0 for s in slots)
    assert summ["makespan_ns"] > summ["makespan_noswap_ns"]
    slots, summ = P.schedule(4, 0, 8, 10, 20, 1, 1)
    assert all(s["hidden"] == 1 and s["exposed_ns"] == 0 for s in slots)
    assert summ["makespan_ns"] == summ["makespan_noswap_ns"]
    assert summ["peak_resident"] < summ["peak_resident_noswap"]   # the memory D2D saves


def test_library_matches_oracle_random():
    rng = random.Random(236)
    for _ in range(400):
        S = rng.randint(1, 8)
        M = rng.randint(1, 12)
        e = rng.randrange(S)
        args = (S, e, M, rng.randint(1, 50), rng.randint(1, 90), rng.randint(0, 120), rng.randint(0, 120))
        duplex = rng.random() < 0.5
        slack = rng.choice([0, 0, 5, 40])
        assert mp.schedule_1f1b(*args, duplex=duplex, slack_ns=slack) == \
            P.schedule(*args, duplex=duplex, slack=slack), (args, duplex, slack)


def test_bert_stage0_scale():
    """Config 2's stage 0 at the paper's scale (8 stages, 8 micro-batches,
    ms-range ops, 900 MiB micro-batches at ~750 GB/s NVLink)."""
    args = (8, 0, 8, 800_000, 1_600_000, 1_260_000, 1_260_000)
    a = mp.schedule_1f1b(*args)
    assert a == P.schedule(*args)
    slots, summ = a
    assert all(s["hidden"] for s in slots)
    assert summ["peak_resident_noswap"] == 8 and summ["peak_resident"] < 8


def test_errors():
    with pytest.raises(mp.MPressError):
        mp.schedule_1f1b(0, 0, 1, 1, 1, 1, 1)
    with pytest.raises(mp.MPressError):
        mp.schedule_1f1b(2, 2, 1, 1, 1, 1, 1)
    with pytest.raises(mp.MPressError):
        mp.schedule_1f1b(2, 0, 0, 1, 1, 1, 1)
